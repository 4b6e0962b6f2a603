python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "host" > gpurun_out/r03_pytest_host.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_host.log
L=gpurun_out/r03_ramp.log; rm -f $L
for R in 0 1 0 1 0 1; do
  POLYCONV_HOST_RAMP=$R timeout 300 python bench.py --no-cpu-baseline --no-cudnn --no-gate --no-by-math --steps 50 > /tmp/c_$R.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/c_$R.json').read().strip().splitlines()[-1]); e=d['e2e']; print('ramp=$R', round(e['value'],2), round(e['ms_per_step']*1e3,1), 'us')" >> $L
done
for G in 6 8; do
  POLYCONV_HOST_CHUNKS=$G timeout 300 python bench.py --no-cpu-baseline --no-cudnn --no-gate --no-by-math --steps 50 > /tmp/c_$G.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/c_$G.json').read().strip().splitlines()[-1]); e=d['e2e']; print('ramp chunks=$G', round(e['value'],2), round(e['ms_per_step']*1e3,1), 'us')" >> $L
done
