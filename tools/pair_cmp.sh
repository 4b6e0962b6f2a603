python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for f in ${FS:-0 1 2}; do POLYCONV_PAIR_FSMEM=$f python -m pytest tests -m gpu -q -x -k "pair or shard or conv3x" 2>&1 | tail -1; done
for f in ${FS:-0 1 2}; do echo "== fsmem $f"; POLYCONV_PAIR_FSMEM=$f timeout 120 python tools/pair_trace.py 0 2>&1 | grep -E "bands|win0|win1|tile|filter|end|pk_band_w|pk_filter"; done
for f in ${FS:-0 1 2}; do POLYCONV_PAIR_FSMEM=$f timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-cudnn 2>/dev/null | python -c "
import json,sys; d=json.load(sys.stdin)
print('fsmem $f value %.1f TF/s step %.4f ms kernel %.4f ms' % (d['value'], d['ms_per_step'], d['roofline']['kernel_ms']))"; done
