# fixed per-forward costs: launch probe + full ablation (dbg 15 = no loads, stores, MMAs) + pack only
./tools/launch_probe > gpurun_out/r03_launch_probe.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || { tail -20 gpurun_out/r03_build.log; exit 1; }
for SHAPE in "32 128 28 28 128 3 3" "256 256 14 14 256 3 3"; do
  echo "== $SHAPE" >> gpurun_out/r03_fixed.log
  HK_DBGS="15 8" timeout 200 python tools/hk_trace.py $SHAPE >> gpurun_out/r03_fixed.log 2>&1
done
