# same-box A/B of library variants through the same binding (POLYCONV_LIB)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_libab.log; rm -f $L
for round in 1 2; do
for v in head ${VARS:-v2 v3 v4}; do
  if [ $v = head ]; then lib=""; else lib=$PWD/ab_tmp/libs/$v.so; fi
  POLYCONV_LIB=$lib timeout 600 python bench.py --no-cpu-baseline --no-by-math --no-cudnn --steps 100 > /tmp/ab_$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/ab_$v.json').read().strip().splitlines()[-1])
print('$v', round(d['value'],1), 'gate', round(d['gate']['gate_frac'],4), [round(l['t_med_ms']*1e3,1) for l in d['gate']['layers']])
" >> $L
done; done
