python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || { tail -20 gpurun_out/r03_build.log; exit 1; }
L=gpurun_out/r03_q.log; rm -f $L
for SHAPE in "256 256 14 14 256 3 3" "256 512 7 7 512 3 3" "32 128 28 28 128 3 3"; do
  for Q in 1 2 4; do for D in 8 2056; do
    echo "== $SHAPE Q=$Q D=$D" >> $L
    POLYCONV_HK_Q=$Q HK_DBGS="$D" timeout 200 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done; done
done
