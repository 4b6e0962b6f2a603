# one TMEM accumulator buffer with twice the positions per item (POLYCONV_HK_ACC1=1)
L=gpurun_out/hk_acc1.log
POLYCONV_HK_ACC1=1 POLYCONV_HK_VERBOSE=1 timeout 300 python tools/hk_check.py tail >> $L 2>&1
POLYCONV_HK_ACC1=1 timeout 300 python tools/hk_check.py quick >> $L 2>&1
for SHAPE in "256 512 7 7 512 3 3" "256 256 14 14 256 3 3" "64 512 28 28 512 3 3" "256 128 28 28 128 3 3" "256 64 56 56 64 3 3" "32 128 28 28 128 3 3"; do
  for A in 0 1; do
    echo "== $SHAPE ACC1=$A" >> $L
    POLYCONV_HK_ACC1=$A POLYCONV_HK_VERBOSE=1 HK_DBGS="0 4" timeout 200 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
echo "== l4 ACC1 F=6" >> $L
POLYCONV_HK_ACC1=1 POLYCONV_HK_FSLOTS=6 HK_DBGS="0" timeout 200 python tools/hk_trace.py 256 512 7 7 512 3 3 >> $L 2>&1
echo "== l3 ACC1 F=6" >> $L
POLYCONV_HK_ACC1=1 POLYCONV_HK_FSLOTS=6 HK_DBGS="0" timeout 200 python tools/hk_trace.py 256 256 14 14 256 3 3 >> $L 2>&1
