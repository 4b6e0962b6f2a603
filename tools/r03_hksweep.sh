# mac_hankel tiling sweep on the gate layers and conv3x (T, resident/streamed filter, window slots)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_hksweep.log; rm -f $L
for SHAPE in "256 64 56 56 64 3 3" "256 128 28 28 128 3 3" "32 128 28 28 128 3 3" "256 256 14 14 256 3 3" "256 512 7 7 512 3 3"; do
  echo "== $SHAPE default" >> $L; HK_DBGS="0" timeout 60 python tools/hk_trace.py $SHAPE >> $L 2>&1
  for T in 1 2 4; do
    for W in 2 3 4 5 6; do
      echo "== $SHAPE T=$T stream W=$W" >> $L; POLYCONV_HK_T=$T POLYCONV_HK_STREAM=1 POLYCONV_HK_WSLOTS=$W HK_DBGS="0" timeout 60 python tools/hk_trace.py $SHAPE >> $L 2>&1
    done
    echo "== $SHAPE T=$T resident" >> $L; POLYCONV_HK_T=$T POLYCONV_HK_RESIDENT=1 HK_DBGS="0" timeout 60 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
