python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -m gpu -x -q -k "1x1" > gpurun_out/r03_pytest_1x1.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_1x1.log
L=gpurun_out/r03_epi2ld.log; rm -f $L
for SHAPE in "256 128 28 28 512 1 1 1 0" "256 512 28 28 128 1 1 1 0" "256 64 56 56 256 1 1 1 0" "256 256 56 56 64 1 1 1 0" "256 256 56 56 128 1 1 1 0" "256 64 56 56 64 1 1 1 0"; do
  for V in v1 new v1 new; do
    if [ $V = v1 ]; then lib=$PWD/ab_tmp/libs/v1.so; else lib=""; fi
    echo "== $SHAPE $V" >> $L; POLYCONV_LIB=$lib HK_KERNEL=tc_1x1 HK_DBGS="0" timeout 120 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
for V in v1 new v1 new; do
  if [ $V = v1 ]; then lib=$PWD/ab_tmp/libs/v1.so; else lib=""; fi
  POLYCONV_LIB=$lib timeout 600 python bench.py --workload resnet50 --no-cpu-baseline --no-cudnn > /tmp/r50_$V.json 2>/dev/null; python -c "
import json; r=json.loads(open('/tmp/r50_$V.json').read().strip().splitlines()[-1]); print('r50 $V', r['value'], r['ms_per_step'], r['clocks'])" >> $L
done
