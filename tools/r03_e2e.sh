python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_e2e.log; rm -f $L
for CH in 1 2 4 8 16; do
  POLYCONV_HOST_CHUNKS=$CH timeout 600 python bench.py --no-cpu-baseline --no-by-math --no-cudnn --no-gate --steps 50 > /tmp/e_$CH.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/e_$CH.json').read().strip().splitlines()[-1])
print('chunks $CH', round(d['e2e']['value'],1), round(d['e2e']['ms_per_step']*1e3,1), 'us')
" >> $L
done
python tools/pcie_probe.py > gpurun_out/r03_pcie.txt 2>&1 || true
