python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || exit 1
for m in ${MODES:-0 1}; do echo "== dbg $m"; timeout 120 python tools/pair_trace.py $m 2>&1 | tail -18 | grep -v "^{"; done
