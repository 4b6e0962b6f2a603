#!/bin/bash
# Ablation timings of the tensor-core MAC (POLYCONV_TC_DEBUG modes), bench workload.
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for m in 0 1 2 4 5; do
  echo -n "dbg=$m "; POLYCONV_TC_DEBUG=$m timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-cudnn ${EXTRA:-} | python -c "import json,sys; d=json.load(sys.stdin); print('kernel_ms=%.4f step_ms=%.4f' % (d['roofline']['kernel_ms'], d['ms_per_step']))"
done
