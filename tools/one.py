"""Run one conv through the C-ABI and compare with the oracle (debug helper).
usage: python tools/one.py N C H W K R S s p math [io]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_cgo_xuzc025_b200 as pc, synth, oracle
a = sys.argv[1:]
N, C, H, W, K, R, S, st, pd = map(int, a[:9]); math = a[9]; io = a[10] if len(a) > 10 else "f32"
shape = synth.ConvShape("one", N, C, H, W, K, R, S, st, st, pd, pd)
x, w = synth.make_inputs(shape, 3, "int")
dt = torch.bfloat16 if io == "bf16" else torch.float32
plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math=math, io_dtype=io)
print(plan.info(), flush=True)
y = plan.forward(torch.from_numpy(x).cuda().to(dt), torch.from_numpy(w).cuda().to(dt))
torch.cuda.synchronize()
ref = oracle.conv2d(x, w, shape.stride, shape.padding)
yy = y.float().cpu().numpy()
if io == "bf16":
    ref = torch.from_numpy(ref.astype(np.float32)).bfloat16().float().numpy()
bad = np.argwhere(yy != ref)
print("mismatches", len(bad), "of", ref.size, bad[:5])
