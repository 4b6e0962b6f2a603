# vector window loader (POLYCONV_HK_VEC=8/4): correctness + timing against the pair loader
L=gpurun_out/hk_vec.log
for V in 8 4; do
  echo "== check VEC=$V" >> $L
  POLYCONV_HK_VEC=$V POLYCONV_HK_VERBOSE=1 timeout 300 python tools/hk_check.py quick >> $L 2>&1
  POLYCONV_HK_VEC=$V timeout 300 python tools/hk_check.py tail >> $L 2>&1
done
for SHAPE in "256 64 56 56 64 3 3" "256 128 28 28 128 3 3" "32 128 28 28 128 3 3" "64 128 112 112 128 3 3" "64 256 56 56 256 3 3" "64 512 28 28 512 3 3"; do
  for V in 0 8 4; do
    echo "== $SHAPE VEC=$V" >> $L
    POLYCONV_HK_VEC=$V POLYCONV_HK_VERBOSE=1 HK_DBGS="0 4" timeout 200 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
