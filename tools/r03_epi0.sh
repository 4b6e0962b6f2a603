python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_epi0.log; rm -f $L
for SHAPE in "256 256 14 14 1024 1 1 1 0" "256 256 56 56 512 1 1 2 0" "256 512 28 28 1024 1 1 2 0" "256 128 28 28 512 1 1 1 0" "256 64 56 56 256 1 1 1 0" "256 512 28 28 256 1 1 1 0" "256 512 7 7 2048 1 1 1 0" "256 1024 14 14 2048 1 1 2 0"; do
  for E in 1 0 1 0; do
    if [ $E = 1 ]; then unset POLYCONV_1X1_EPI_TMA; else export POLYCONV_1X1_EPI_TMA=0; fi
    echo "== $SHAPE epi_tma_allowed=$E" >> $L; HK_KERNEL=tc_1x1 HK_DBGS="0" timeout 120 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
  unset POLYCONV_1X1_EPI_TMA
done
