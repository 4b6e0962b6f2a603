python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_gpu.log
L=gpurun_out/r03_planes.log; rm -f $L
for round in 1 2; do for PL in 0 1; do
  POLYCONV_HK_PLANES=$PL timeout 600 python bench.py --no-cpu-baseline --no-by-math --no-cudnn --steps 50 > /tmp/pl_$PL.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/pl_$PL.json').read().strip().splitlines()[-1])
print('planes $PL', round(d['value'],1), 'gate', round(d['gate']['gate_frac'],4), [round(l['t_med_ms']*1e3,1) for l in d['gate']['layers']])
" >> $L
done; done
for SHAPE in "256 512 7 7 512 3 3" "128 128 7 7 128 3 3" "256 1024 7 7 256 1 1 1 0"; do
  for PL in 0 1; do echo "== $SHAPE PL=$PL" >> $L; POLYCONV_HK_PLANES=$PL POLYCONV_HK_VERBOSE=1 HK_DBGS="0" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1; done
done
