python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_gpu.log
L=gpurun_out/r03_planes2.log; rm -f $L
for SHAPE in "256 1024 14 14 256 1 1 1 0" "256 256 14 14 256 3 3" "64 512 14 14 512 3 3" "256 512 7 7 512 3 3" "256 2048 7 7 512 1 1 1 0" "256 1024 7 7 512 1 1 1 0" "256 128 28 28 128 3 3" "32 128 28 28 128 3 3"; do
  for PL in 1 2; do echo "== $SHAPE PL=$PL" >> $L; POLYCONV_HK_PLANES=$PL POLYCONV_HK_VERBOSE=1 HK_DBGS="0" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1; done
done
