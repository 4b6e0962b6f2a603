#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
python tools/tc_trace.py bf16 0 16 1 17 2>&1 | grep -E "mode|mma_issued|epi_end"
for nt in 128 256 112; do echo "NT=$nt"; POLYCONV_TC_NT=$nt python tools/tc_trace.py bf16 0 1 2>&1 | grep -E "mode|first_B|mma_issued|epi_end|tile_m" | cut -c1-200; done
