python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 400 ncu --set full --clock-control none --import-source on -k regex:mac_1x1 -s 2 -c 1 -o gpurun_out/r03_1x1_l3src python tools/hk_one.py 256 256 14 14 1024 1 1 1 0 > gpurun_out/r03_ncu1x1b.log 2>&1; echo "rc=$?"
timeout 400 ncu --set full --clock-control none --import-source on -k regex:mac_1x1 -s 2 -c 1 -o gpurun_out/r03_1x1_l2dsrc python tools/hk_one.py 256 256 56 56 512 1 1 2 0 >> gpurun_out/r03_ncu1x1b.log 2>&1; echo "rc=$?"
