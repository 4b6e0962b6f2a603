mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null
HK_MATH=fp32 timeout 400 ncu --set full --clock-control none --import-source on -k regex:mac_fp32 -s 2 -c 1 -o gpurun_out/r03_fp32_conv3x python tools/hk_one.py 32 128 28 28 128 3 3 1 1 fp32 > gpurun_out/r03_fp32_ncu.log 2>&1
echo "rc=$?"
