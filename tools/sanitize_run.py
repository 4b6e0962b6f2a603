"""Every kernel variant once on small shapes (bf16 / tf32 / fp32 as each supports), for
compute-sanitizer memcheck / racecheck / synccheck runs:
    compute-sanitizer --tool memcheck python tools/sanitize_run.py [kernel ...]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402

CASES = {  # kernel: [(x_shape, w_shape, stride, pad, math, io)]
    "tc_hankel": [((2, 64, 12, 12), (64, 64, 3, 3), 1, 1, "bf16", "bf16"),
                  ((2, 40, 9, 7), (48, 40, 3, 3), 1, 1, "bf16", "bf16"),      # odd width: general loader
                  ((2, 64, 12, 12), (64, 64, 3, 3), 2, 1, "tf32", "f32"),
                  ((3, 128, 14, 14), (320, 128, 3, 3), 1, 1, "bf16", "bf16")],  # 2 n-blocks, streamed filter
    "tc": [((2, 64, 12, 12), (64, 64, 3, 3), 1, 1, "bf16", "bf16"), ((2, 64, 12, 12), (64, 64, 3, 3), 1, 1, "tf32", "f32")],
    "tc_fused": [((2, 64, 16, 16), (128, 64, 3, 3), 1, 1, "bf16", "bf16")],
    "tc_pair": [((2, 64, 16, 16), (64, 64, 3, 3), 1, 1, "bf16", "bf16")],
    "tc_1x1": [((2, 64, 16, 16), (128, 64, 1, 1), 1, 0, "bf16", "bf16")],
    "tc_pertap": [((2, 64, 12, 12), (64, 64, 3, 3), 1, 1, "bf16", "f32")],
    "fp32": [((2, 16, 12, 12), (32, 16, 3, 3), 1, 1, "fp32", "f32"), ((2, 24, 9, 13), (40, 24, 5, 5), 2, 2, "fp32", "f32"),
             ((2, 20, 7, 7), (36, 20, 1, 1), 1, 0, "fp32", "f32")],
    "thin": [((1, 1, 8, 8), (1, 1, 3, 3), 1, 0, "fp32", "f32")],
    "fft": [((2, 16, 12, 12), (32, 16, 3, 3), 1, 1, "fp32", "f32"), ((2, 8, 9, 9), (16, 8, 5, 5), 2, 2, "fp32", "f32")],
}
which = sys.argv[1:] or list(CASES) + ["scatter"]
for kern in which:
    if kern == "scatter":  # f4: the K-shard block stored into three output buffers
        x = (torch.rand((2, 64, 12, 12), device="cuda") * 2 - 1).bfloat16()
        w = (torch.rand((64, 64, 3, 3), device="cuda") * 2 - 1).bfloat16()
        plan = pc.Plan(x.shape, w.shape, (1, 1), (1, 1), math="bf16", io_dtype="bf16", kernel="tc_hankel")
        ys = [torch.zeros((2, 160, 12, 12), dtype=torch.bfloat16, device="cuda") for _ in range(3)]
        plan.forward_scatter(x, w, [t.data_ptr() for t in ys], 160, 64)
        torch.cuda.synchronize()
        print("scatter ok", float(ys[2].float().abs().sum()) > 0, flush=True)
        continue
    for xs, ws, s, p, math, io in CASES[kern]:
        dt = torch.bfloat16 if io == "bf16" else torch.float32
        x = (torch.rand(xs, device="cuda") * 2 - 1).to(dt)
        w = (torch.rand(ws, device="cuda") * 2 - 1).to(dt)
        plan = pc.Plan(x.shape, w.shape, (s, s), (p, p), math=math, io_dtype=io, kernel=kern)
        for _ in range(2):
            y = plan.forward(x, w)
        torch.cuda.synchronize()
        print(kern, xs, ws, math, io, "ok", float(y.float().abs().sum()) > 0, flush=True)
