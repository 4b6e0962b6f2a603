python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "tc_pair" 2>&1 | tail -15
timeout 120 python tools/pair_trace.py 2>&1 | tail -12
timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline > gpurun_out/pair_bench.json 2>gpurun_out/pair_bench.err; tail -2 gpurun_out/pair_bench.err
python -c "
import json; d=json.load(open('gpurun_out/pair_bench.json'))
print('value %.1f TF/s step %.4f ms kernel %.4f ms frac %.3f cudnn %.1f e2e %.1f kern %s' % (d['value'], d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d['cudnn']['value'], d['e2e']['value'], d['config']['kernel']))"
