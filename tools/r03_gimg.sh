python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "1x1" > gpurun_out/r03_pytest_1x1.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_1x1.log
L=gpurun_out/r03_gimg.log; rm -f $L
for SHAPE in "256 512 7 7 2048 1 1 1 0" "256 2048 7 7 512 1 1 1 0" "256 1024 14 14 2048 1 1 2 0" "256 512 14 14 512 1 1 1 0" "32 512 7 7 2048 1 1 1 0"; do
  for G in 0 1 0 1; do
    echo "== $SHAPE gimg=$G tc_1x1" >> $L; POLYCONV_1X1_GIMG=$G HK_KERNEL=tc_1x1 HK_DBGS="0" timeout 120 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
  echo "== $SHAPE auto" >> $L; HK_KERNEL=auto HK_DBGS="0" timeout 120 python tools/hk_trace.py $SHAPE >> $L 2>&1
done
