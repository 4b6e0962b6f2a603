# TC_HANKEL on the ResNet-50 1x1 layers (R = S = 1: one tap, no halo) vs the AUTO kernel
L=gpurun_out/hk_1x1.log
for S in "256 1024 14 14 256 1 1 1 0" "256 256 14 14 1024 1 1 1 0" "256 1024 14 14 512 1 1 1 0" "256 512 28 28 256 1 1 1 0" "256 512 28 28 128 1 1 1 0" "256 128 28 28 512 1 1 1 0" "256 64 56 56 256 1 1 1 0" "256 256 56 56 64 1 1 1 0" "256 256 56 56 128 1 1 1 0" "256 64 56 56 64 1 1 1 0" "256 2048 7 7 512 1 1 1 0" "256 512 7 7 2048 1 1 1 0"; do
  echo "== $S" >> $L
  POLYCONV_HK_VERBOSE=1 HK_DBGS="0" timeout 200 python tools/hk_trace.py $S >> $L 2>&1
  HK_KERNEL=auto HK_DBGS="0" timeout 200 python tools/hk_trace.py $S >> $L 2>&1
done
