"""Dev probe: kernel timeline (torch.profiler / CUPTI) of one layer's forward, to see the gaps
between the filter pack, the MAC kernel and the surrounding events.
    python tools/kprof.py N C H W K R S [s p] [kernel]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402
a = sys.argv[1:]
N, C, H, W, K, R, S = [int(v) for v in a[:7]]
s, p = (int(a[7]), int(a[8])) if len(a) > 8 else (1, R // 2)
kern = a[9] if len(a) > 9 else "auto"
math = os.environ.get("KPROF_MATH", "bf16")  # fp32 / tf32: f32 I/O
dt = torch.bfloat16 if math == "bf16" else torch.float32
x = (torch.rand((N, C, H, W), device="cuda") * 2 - 1).to(dt)
w = (torch.rand((K, C, R, S), device="cuda") * 2 - 1).to(dt)
plan = pc.Plan(x.shape, w.shape, (s, s), (p, p), math=math, io_dtype="bf16" if math == "bf16" else "f32", kernel=kern)
y = torch.empty(plan.output_shape, dtype=dt, device="cuda")
flush = torch.empty(64 << 20, device="cuda")
for _ in range(5):
    flush.zero_()
    plan.forward(x, w, y)
torch.cuda.synchronize()
from torch.profiler import profile, ProfilerActivity  # noqa: E402
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for _ in range(4):
        flush.zero_()
        plan.forward(x, w, y)
    torch.cuda.synchronize()
evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
evs.sort(key=lambda e: e.time_range.start)
t0 = evs[0].time_range.start
prev = None
for e in evs:
    st, en = e.time_range.start - t0, e.time_range.end - t0
    gap = (st - prev) if prev is not None else 0
    print("%9.2f %9.2f dur %7.2f gap %6.2f  %s" % (st, en, en - st, gap, e.name[:90]))
    prev = en
