python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo build failed; exit 1; }
echo "== tc_fused"; KERN=tc_fused timeout 120 python tools/tc_trace.py bf16 0 2>&1 | grep -v "^{"
echo "== tc"; KERN=tc timeout 120 python tools/tc_trace.py bf16 0 2>&1 | grep -v "^{"
echo "== tc mma cycles"; KERN=tc timeout 120 python tools/tc_trace.py bf16 32 2>&1 | grep -v "^{"
echo "== fused mma cycles"; KERN=tc_fused timeout 120 python tools/tc_trace.py bf16 32 2>&1 | grep -v "^{"
echo "== epi"; KERN=tc_fused timeout 120 python tools/tc_trace.py bf16 128 2>&1 | grep -v "^{"
timeout 200 python tools/phase_time.py bf16 tc tc_fused 2>&1 | tail
