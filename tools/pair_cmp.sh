python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
python -m pytest tests -m gpu -q -x -k "tc_pair or shard or conv3x" 2>&1 | tail -1
for rep in ${REPS:-1 8}; do for m in ${MODES:-0}; do echo "== rep $rep dbg $m"; POLYCONV_FILTER_REP=$rep timeout 120 python tools/pair_trace.py $m 2>&1 | grep -E "bands|win0|win1|tile|filter|end|pk_band_w|pk_filter"; done; done
