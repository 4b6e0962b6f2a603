"""Packer fine trace (clock64 deltas, first window of a few CTAs)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_cgo_xuzc025_b200 as pc, synth
shape = synth.CONV3X
x, w = synth.make_inputs(shape, 1, "uniform")
x, w = torch.from_numpy(x).cuda().bfloat16(), torch.from_numpy(w).cuda().bfloat16()
plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math="bf16", io_dtype="bf16")
lib = pc.load_library()
buf = (ctypes.c_longlong * (160 * 16))()
os.environ["POLYCONV_TC_DEBUG"] = "16"
flush = torch.empty(64 << 20, device="cuda")
for it in range(3):
    flush.zero_(); plan.forward(x, w); torch.cuda.synchronize()
lib.polyconv_dbg_tc2_ptrace(buf)
a = np.array(buf, dtype=np.int64).reshape(160, 16)
for b in [0, 1, 2, 10, 50, 100]:
    n = int(a[b, 15]); t = a[b, :n + 1]
    print(b, "steps", n, "deltas", list(np.diff(t)))
