"""Dev helper: run one layer through the FFT solver (fp32) a few times, for ncu launch lists.
    python tools/fft_one.py N C H W K R S [s p]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402
a = [int(v) for v in sys.argv[1:]]
N, C, H, W, K, R, S = a[:7]
s, p = (a[7], a[8]) if len(a) > 8 else (1, R // 2)
x = torch.rand((N, C, H, W), device="cuda") * 2 - 1
w = torch.rand((K, C, R, S), device="cuda") * 2 - 1
plan = pc.Plan(x.shape, w.shape, (s, s), (p, p), math="fp32", io_dtype="f32", kernel="fft")
y = torch.empty(plan.output_shape, device="cuda")
for _ in range(3):
    plan.forward(x, w, y)
torch.cuda.synchronize()
print(plan.info())
