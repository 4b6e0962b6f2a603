# same-box A/B: v0 (4-warp epilogue, element gather) vs the 8-warp epilogue with each gather
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_1x1ab.log; rm -f $L
for SHAPE in "256 256 14 14 1024 1 1 1 0" "256 512 7 7 2048 1 1 1 0" "256 1024 14 14 2048 1 1 2 0" "256 128 28 28 512 1 1 1 0" "256 64 56 56 256 1 1 1 0" "256 256 56 56 64 1 1 1 0" "256 256 56 56 512 1 1 2 0" "256 512 28 28 1024 1 1 2 0"; do
  for V in v0 elem stage v0 elem stage; do
    if [ $V = v0 ]; then lib=$PWD/ab_tmp/libs/v0.so; else lib=""; fi
    echo "== $SHAPE $V" >> $L; POLYCONV_LIB=$lib POLYCONV_1X1_GATHER=$V HK_KERNEL=tc_1x1 HK_DBGS="0" timeout 120 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
for V in v0 new; do
  if [ $V = v0 ]; then lib=$PWD/ab_tmp/libs/v0.so; else lib=""; fi
  POLYCONV_LIB=$lib timeout 600 python bench.py --workload resnet50 --no-cpu-baseline --no-cudnn > /tmp/r50_$V.json 2>/dev/null; python -c "
import json; r=json.loads(open('/tmp/r50_$V.json').read().strip().splitlines()[-1]); print('r50 $V', r['value'], r['ms_per_step'])" >> $L
done
