"""Time every BF16 tensor-core kernel that accepts a layer (forced through set_kernel) next to the
AUTO choice (fresh plans; TFLOP/s), L2 flushed before each call, CUDA events: checks the AUTO
rule per layer.

    python tools/kernel_cmp.py [resnet50|vgg16|all] [reps]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402
import synth  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "all"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
# the unique layers of the synthetic 20-layer nets (torch_integration.SyntheticNet, batch 32, width 64)
SYNTHNET = [synth.ConvShape("syn_%d_%d_%d_r%d" % (H, C, K, R), 32, C, H, H, K, R, R, 1, 1, R // 2, R // 2)
            for H in (4, 8, 14, 28, 56) for (C, K, R) in ((64, 64, 3), (64, 128, 5), (128, 64, 1), (64, 128, 7),
                                                         (128, 64, 3))]
layers = {"resnet50": synth.RESNET50, "vgg16": synth.VGG16, "synthnet": SYNTHNET, "sweep": synth.SWEEP}.get(
    which, synth.RESNET50 + synth.VGG16)
flush = torch.empty(64 << 20, device="cuda")


def timed(fn):
    ts = []
    for it in range(reps + 2):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        if it >= 2:
            ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


for L in layers:
    x = torch.randn(L.N, L.C, L.H, L.W, device="cuda").bfloat16()
    w = (torch.randn(L.K, L.C, L.R, L.S, device="cuda") / (L.C * L.R * L.S) ** 0.5).bfloat16()
    plan = pc.Plan(x.shape, w.shape, L.stride, L.padding, math="bf16", io_dtype="bf16")
    y = torch.empty(plan.output_shape, dtype=torch.bfloat16, device="cuda")
    auto = plan.info()["kernel"]
    rec = {"layer": L.name, "auto": auto}
    rec[auto] = round(L.flops() / timed(lambda: plan.forward(x, w, y)) / 1e9, 1)
    del plan
    for k in ("tc_hankel", "tc_fused", "tc", "tc_pair", "tc_1x1"):
        if k == auto:
            continue
        try:
            pk = pc.Plan(x.shape, w.shape, L.stride, L.padding, math="bf16", io_dtype="bf16", kernel=k)
        except pc.PolyconvError:
            continue
        rec[k] = round(L.flops() / timed(lambda: pk.forward(x, w, y)) / 1e9, 1)
        del pk
    print(json.dumps(rec), flush=True)
