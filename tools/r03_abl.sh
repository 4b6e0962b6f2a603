# round-2b ablation: per-layer floors of mac_hankel (dbg 1 no loads, 2 no stores, 4 no MMAs, 8 trace)
L=gpurun_out/r03_abl.log
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || { tail -20 gpurun_out/r03_build.log; exit 1; }
for SHAPE in "32 128 28 28 128 3 3" "256 64 56 56 64 3 3" "256 128 28 28 128 3 3" "256 256 14 14 256 3 3" "256 512 7 7 512 3 3"; do
  echo "== $SHAPE" >> $L
  HK_DBGS="8 9 10 11 12 14" timeout 200 python tools/hk_trace.py $SHAPE >> $L 2>&1
done
