python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_pack.log; rm -f $L
for round in 1 2; do
for T in 128 32 16 64; do
  POLYCONV_PACK_TPB=$T timeout 600 python bench.py --no-cpu-baseline --no-by-math --no-cudnn --no-gate --steps 200 > /tmp/pk_$T.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/pk_$T.json').read().strip().splitlines()[-1])
print('tpb $T', round(d['value'],1), round(d['ms_per_step']*1e3,2), 'kern', round(d['roofline']['kernel_ms']*1e3,2))
" >> $L
done; done
