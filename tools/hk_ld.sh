# window-load cache-policy experiment (POLYCONV_HK_DEBUG bits 6-7)
L=gpurun_out/hk_ld.log
for SHAPE in "256 64 56 56 64 3 3" "256 128 28 28 128 3 3" "64 128 112 112 128 3 3"; do
  echo "== $SHAPE" >> $L
  HK_DBGS="0 64 128 192 4 68 132 196" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1
done
