#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for cs in 1 2 4; do echo "CS=$cs"; POLYCONV_TC_CS=$cs timeout 120 python tools/tc_trace.py bf16 0 2 2>&1 | grep -E "mode|first_B|mma_issued|epi_end|cta_end"; done
