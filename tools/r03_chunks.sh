python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_chunks.log; rm -f $L
for G in 1 2 4 8 16 4 8; do
  POLYCONV_HOST_CHUNKS=$G timeout 300 python bench.py --no-cpu-baseline --no-cudnn --no-gate --no-by-math --steps 50 > /tmp/c_$G.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/c_$G.json').read().strip().splitlines()[-1]); e=d['e2e']; print('chunks=$G', round(e['value'],2), round(e['ms_per_step']*1e3,1), 'us')" >> $L
done
