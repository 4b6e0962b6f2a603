# Sweep the shared-memory footprint knobs of TC_HANKEL (POLYCONV_HK_T / _WSLOTS / _FSLOTS /
# _STREAM / _RESIDENT): smaller footprints leave more L1 for the window loaders' global loads.
L=gpurun_out/hk_slots3.log
run() { echo "$*" >> $L; env "$@" POLYCONV_HK_VERBOSE=1 HK_DBGS="0" timeout 120 python tools/hk_trace.py $SHAPE >> $L 2>&1; }
for SHAPE in "256 256 14 14 256 3 3" "256 512 7 7 512 3 3" "64 512 28 28 512 3 3"; do
  echo "== $SHAPE" >> $L
  run X=0
  run POLYCONV_HK_FSLOTS=6
done
for SHAPE in "256 128 28 28 128 3 3" "32 128 28 28 128 3 3" "256 64 56 56 64 3 3" "32 64 56 56 64 3 3"; do
  echo "== $SHAPE" >> $L
  run X=0
  run POLYCONV_HK_T=1
  run POLYCONV_HK_T=2
  run POLYCONV_HK_T=1 POLYCONV_HK_STREAM=1
  run POLYCONV_HK_T=2 POLYCONV_HK_STREAM=1
  run POLYCONV_HK_RESIDENT=1 POLYCONV_HK_T=1
  run POLYCONV_HK_RESIDENT=1 POLYCONV_HK_T=2
done
