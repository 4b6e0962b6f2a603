python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q -k "fp32 or FP32" > gpurun_out/r03_pytest_f32.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/r03_pytest_f32.log
L=gpurun_out/r03_f32split.log; rm -f $L
for round in 1 2; do for SP in 1 2 3 4; do
  POLYCONV_F32_SPLIT=$SP timeout 600 python bench.py --math fp32 --no-cpu-baseline --no-by-math --no-cudnn --no-gate --steps 30 > /tmp/fs_$SP.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/fs_$SP.json').read().strip().splitlines()[-1])
print('split $SP', round(d['value'],2), round(d['roofline']['frac'],3))
" >> $L
done; done
