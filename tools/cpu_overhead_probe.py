"""Host (CPU) cost of enqueuing polyconv_forward / polyconv_forward_host on conv3x: wall time
of 200 calls without synchronising (the GPU is kept busy so queue space never blocks), and the
GPU time per call for comparison."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_xuzc025_b200 as pc
N, C, H, W, K = 32, 128, 28, 28, 128
x = (torch.rand((N, C, H, W), device="cuda") * 2 - 1).bfloat16()
w = (torch.rand((K, C, 3, 3), device="cuda") * 2 - 1).bfloat16()
plan = pc.Plan(x.shape, w.shape, (1, 1), (1, 1), math="bf16", io_dtype="bf16")
y = torch.empty(plan.output_shape, dtype=torch.bfloat16, device="cuda")
xh, wh, yh = x.cpu().pin_memory(), w.cpu().pin_memory(), torch.empty(plan.output_shape, dtype=torch.bfloat16).pin_memory()
out = {}
for name, fn, n in (("forward", lambda: plan.forward(x, w, y), 200), ("forward_host", lambda: plan.forward_host(xh, wh, yh), 50)):
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(n):
        fn()
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    out[name] = {"cpu_us_per_call": round((t1 - t0) / n * 1e6, 1), "wall_us_per_call": round((t2 - t0) / n * 1e6, 1)}
print(json.dumps(out))
