#!/bin/bash
# quick GPU iteration: build, tc parity subset, trace, bench line summary
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo build failed; exit 1; }
timeout 300 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} 2>&1 | tail -3
timeout 120 python tools/tc_trace.py ${MATH:-bf16} 0 2>&1 | grep -v "^{"
for m in ${BENCH_MATHS:-bf16}; do
timeout 300 python bench.py --math $m --steps 200 --warmup 10 --no-cpu-baseline | python -c "
import json,sys; d=json.load(sys.stdin)
print('$m value %.1f TF/s step %.4f ms kernel %.4f ms frac %.3f step_frac %.3f cudnn %.1f e2e %.1f' % (d['value'], d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d['roofline']['step_frac'], d['cudnn']['value'], d['e2e']['value']))"
done
