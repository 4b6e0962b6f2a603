python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_gpu.log
L=gpurun_out/r03_gimg2.log; rm -f $L
for V in v0 new v0 new; do
  if [ $V = v0 ]; then lib=$PWD/ab_tmp/libs/v0.so; else lib=""; fi
  POLYCONV_LIB=$lib timeout 600 python bench.py --workload resnet50 --no-cpu-baseline --no-cudnn > /tmp/r50_$V.json 2>/dev/null; python -c "
import json; r=json.loads(open('/tmp/r50_$V.json').read().strip().splitlines()[-1]); print('r50 $V', r['value'], r['ms_per_step'], r['config'].get('kernels'), r['clocks'])" >> $L
done
timeout 900 python tools/layer_sweep.py resnet50 > gpurun_out/r03_sweep_resnet50_n256.jsonl 2>&1; echo "sweep rc=$?"
