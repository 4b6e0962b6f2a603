python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_gpu.log
L=gpurun_out/r03_rowtile.log; rm -f $L
for SHAPE in "256 3 224 224 64 7 7 2 3" "32 3 224 224 64 7 7 2 3"; do
  for RT in 0 1 0 1; do echo "== $SHAPE RT=$RT" >> $L; POLYCONV_HK_ROWTILE=$RT POLYCONV_HK_VERBOSE=1 HK_DBGS="0" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1; done
done
for RT in 0 1; do POLYCONV_HK_ROWTILE=$RT timeout 600 python bench.py --workload resnet50 --no-cpu-baseline --no-cudnn > /tmp/r50_$RT.json 2>/dev/null; python -c "
import json; r=json.loads(open('/tmp/r50_$RT.json').read().strip().splitlines()[-1]); print('r50 RT=$RT', r['value'], r['ms_per_step'])" >> $L; done
