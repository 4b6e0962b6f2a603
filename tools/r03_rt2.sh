# stride-1 row-tile epilogue (pitch 64/128, TMA-stored rows) vs the 2-byte-store epilogue, same box
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_gpu.log
L=gpurun_out/r03_rt2.log; rm -f $L
for SHAPE in "256 64 56 56 64 3 3" "64 64 224 224 64 3 3" "64 128 112 112 128 3 3" "64 256 56 56 256 3 3" "32 64 32 32 64 3 3"; do
  for RT in 0 1 0 1; do echo "== $SHAPE RT=$RT" >> $L; POLYCONV_HK_ROWTILE=$RT HK_DBGS="0" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1; done
done
for RT in 0 1 0 1; do POLYCONV_HK_ROWTILE=$RT timeout 600 python bench.py --no-cpu-baseline --no-by-math --no-cudnn --steps 100 > /tmp/g_$RT.json 2>/dev/null
python -c "
import json; d=json.loads(open('/tmp/g_$RT.json').read().strip().splitlines()[-1])
print('gate RT=$RT', round(d['value'],1), 'gate', round(d['gate']['gate_frac'],4), [round(l['t_med_ms']*1e3,1) for l in d['gate']['layers']])
" >> $L; done
for RT in 0 1; do POLYCONV_HK_ROWTILE=$RT timeout 600 python bench.py --workload resnet50 --no-cpu-baseline --no-cudnn > /tmp/r50_$RT.json 2>/dev/null; python -c "
import json; r=json.loads(open('/tmp/r50_$RT.json').read().strip().splitlines()[-1]); print('r50 RT=$RT', r['value'], r['ms_per_step'])" >> $L; done
