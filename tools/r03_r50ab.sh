# same-box A/B of the ResNet-50 N=256 stack (bench --workload resnet50) for library variants
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q -k "1x1 or gather or resnet50 or k1" > gpurun_out/r03_pytest_1x1.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/r03_pytest_1x1.log
L=gpurun_out/r03_r50ab.log; rm -f $L
for round in 1 2; do
for v in ${VARS:-base gather}; do
  POLYCONV_LIB=$PWD/ab_tmp/libs/$v.so timeout 600 python bench.py --workload resnet50 --no-cpu-baseline --no-cudnn > /tmp/r50_$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/r50_$v.json').read().strip().splitlines()[-1])
print('$v', round(d['value'],1), round(d['ms_per_step'],4))
" >> $L
done; done
