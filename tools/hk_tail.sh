# tail-split check (correctness under each forced split) + timing of the gate layers
L=gpurun_out/hk_tail.log
for TS in 0 1 2 4 8; do
  echo "== TSPLIT=$TS" >> $L
  POLYCONV_HK_TSPLIT=$TS POLYCONV_HK_VERBOSE=1 timeout 300 python tools/hk_check.py tail >> $L 2>&1
done
for SHAPE in "32 128 28 28 128 3 3" "256 64 56 56 64 3 3" "256 128 28 28 128 3 3" "256 256 14 14 256 3 3" "256 512 7 7 512 3 3" "64 512 28 28 512 3 3"; do
  for TS in 0 1 2 4 8; do
    echo "== $SHAPE TSPLIT=$TS" >> $L
    POLYCONV_HK_TSPLIT=$TS POLYCONV_HK_VERBOSE=1 HK_DBGS="0" timeout 120 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
