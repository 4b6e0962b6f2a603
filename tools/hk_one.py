"""Dev helper: run one layer through the AUTO plan a few times (for ncu captures).
    python tools/hk_one.py N C H W K R S [s p] [kernel]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402
a = sys.argv[1:]
N, C, H, W, K, R, S = [int(v) for v in a[:7]]
s, p = (int(a[7]), int(a[8])) if len(a) > 8 else (1, R // 2)
kern = a[9] if len(a) > 9 else "auto"
math = os.environ.get("HK_MATH", "bf16")  # fp32 / tf32: f32 I/O
dt = torch.bfloat16 if math == "bf16" else torch.float32
x = (torch.rand((N, C, H, W), device="cuda") * 2 - 1).to(dt)
w = (torch.rand((K, C, R, S), device="cuda") * 2 - 1).to(dt)
plan = pc.Plan(x.shape, w.shape, (s, s), (p, p), math=math, io_dtype="bf16" if math == "bf16" else "f32", kernel=kern)
y = torch.empty(plan.output_shape, dtype=dt, device="cuda")
flush = torch.empty(64 << 20, device="cuda")
for _ in range(4):
    flush.zero_()
    plan.forward(x, w, y)
torch.cuda.synchronize()
print(plan.info())
