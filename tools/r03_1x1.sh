python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q -k "1x1 or resnet50 or vgg or k1" > gpurun_out/r03_pytest_1x1.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_1x1.log
L=gpurun_out/r03_1x1.log; rm -f $L
for SHAPE in "256 256 14 14 1024 1 1 1 0" "256 512 28 28 128 1 1 1 0" "256 128 28 28 512 1 1 1 0" "256 64 56 56 256 1 1 1 0" "256 512 7 7 2048 1 1 1 0" "256 256 56 56 128 1 1 1 0"; do
  for R in 0 1 0 1; do
    echo "== $SHAPE RESA=$R" >> $L
    POLYCONV_1X1_RESA=$R HK_KERNEL=auto HK_DBGS="0" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
