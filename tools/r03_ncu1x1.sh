python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 400 ncu --set full --clock-control none -k regex:"mac_1x1|gather" -s 0 -c 4 -o gpurun_out/r03_1x1_l3 python tools/hk_one.py 256 256 14 14 1024 1 1 1 0 > gpurun_out/r03_ncu1x1.log 2>&1; echo rc=$?
