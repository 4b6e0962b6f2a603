# same-box A/B: a = 53c77ac (before f4) vs HEAD
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_fused_gather.py tests/test_parallel.py -q > gpurun_out/r03_pytest_f4.log 2>&1; echo "f4 rc=$?"; tail -2 gpurun_out/r03_pytest_f4.log
for round in 1 2; do
for v in a head; do
  if [ $v = head ]; then d=.; else d=ab_tmp/$v; fi
  (cd $d && timeout 600 python bench.py --no-cpu-baseline --no-by-math --steps 100 > /tmp/ab_$v.json 2>/dev/null)
  python -c "
import json; d=json.loads(open('/tmp/ab_$v.json').read().strip().splitlines()[-1])
print('$v', round(d['value'],1), 'gate', [round(l['t_med_ms']*1e3,1) for l in d['gate']['layers']], 'cudnn', round(d['cudnn']['value'],1))
" >> gpurun_out/r03_ab.log
done; done
