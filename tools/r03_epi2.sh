python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_gpu.log
L=gpurun_out/r03_epi2.log; rm -f $L
for SHAPE in "256 3 224 224 64 7 7 2 3" "32 128 28 28 128 3 3" "256 64 56 56 64 3 3" "256 128 28 28 128 3 3" "256 256 14 14 256 3 3" "256 512 7 7 512 3 3"; do
  echo "== $SHAPE" >> $L
  HK_DBGS="0" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1
  HK_DBGS="0" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1
done
