python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1 || { echo build failed; exit 1; }
if [ -n "$TESTS" ]; then python -m pytest tests -m gpu -q -x -k "$TESTS" 2>&1 | tail -2; fi
if [ -n "$MODES" ]; then bash tools/pair_exp.sh | grep -E "win|tile|epi|filter|counter|end|pk_"; fi
timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.load(sys.stdin)
print('value %.1f TF/s step %.4f ms kernel %.4f ms frac %.3f cudnn %.1f e2e %.1f kern %s' % (d['value'], d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d['cudnn']['value'], d['e2e']['value'], d['config']['kernel']))"
