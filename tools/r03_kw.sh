# FP32 FFMA kernel: 8 vs 4 output channels per warp (KW), same box
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_kw.log; rm -f $L
for V in v0 kw4 v0 kw4; do
  POLYCONV_LIB=$PWD/ab_tmp/libs/$V.so timeout 600 python bench.py --no-cpu-baseline --no-cudnn --no-gate --steps 50 > /tmp/b_$V.json 2>/dev/null
  python -c "
import json; d=json.loads(open('/tmp/b_$V.json').read().strip().splitlines()[-1]); f=d['by_math']['fp32']; print('conv3x fp32 $V', round(f['value'],2), round(f['frac'],4), round(f['t_med_ms']*1e3,1))" >> $L
done
for V in v0 kw4; do POLYCONV_LIB=$PWD/ab_tmp/libs/$V.so POLYCONV_NO_FFT=1 timeout 900 python tools/fp32_cmp.py resnet50 > gpurun_out/r03_kw_$V.jsonl 2>&1; done
