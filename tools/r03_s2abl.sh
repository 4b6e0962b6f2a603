python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_s2abl.log; rm -f $L
for SHAPE in "256 128 56 56 128 3 3 2 1" "256 256 28 28 256 3 3 2 1" "256 512 14 14 512 3 3 2 1" "256 3 224 224 64 7 7 2 3"; do
  echo "== $SHAPE" >> $L; HK_DBGS="0 1 2 4 7" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1
done
