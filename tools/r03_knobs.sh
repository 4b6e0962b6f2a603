python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_knobs.log; rm -f $L
for SHAPE in "256 256 14 14 256 3 3" "256 512 7 7 512 3 3" "256 128 28 28 128 3 3"; do
  for V in "X=0" "POLYCONV_HK_T=1" "POLYCONV_HK_FSLOTS=8" "POLYCONV_HK_WSLOTS=2" "POLYCONV_HK_ACC1=0" "X=0"; do
    echo "== $SHAPE $V" >> $L
    env $V HK_DBGS="0" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
