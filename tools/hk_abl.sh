# ablations (POLYCONV_HK_DEBUG 1 no loads, 2 no stores, 4 no MMAs) of the streamed layers at
# filter ring depths 4 and 8, + the per-window pipeline trace of CTA 0 (dbg 16)
L=gpurun_out/hk_abl.log
for SHAPE in "256 512 7 7 512 3 3" "256 256 14 14 256 3 3" "256 128 28 28 128 3 3"; do
  for F in 4 8; do
    echo "== $SHAPE F=$F" >> $L
    POLYCONV_HK_FSLOTS=$F HK_DBGS="0 1 2 4 3 16" timeout 200 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
