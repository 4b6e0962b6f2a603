python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
POLYCONV_HK_IM2=0 POLYCONV_HK_RESIDENT=1 HK_DBGS="40" timeout 300 python tools/hk_trace.py 256 3 224 224 64 7 7 2 3 > gpurun_out/r03_stemtr.log 2>&1
HK_DBGS="40" timeout 300 python tools/hk_trace.py 256 128 28 28 128 3 3 >> gpurun_out/r03_stemtr.log 2>&1
