"""Run one ResNet-50 / VGG-16 layer (synth.RESNET50 / synth.VGG16, BF16 in/out, AUTO kernel) a
few times, for an ncu launch list or capture of that layer's launches:

    ncu --metrics gpu__time_duration.sum --clock-control none --csv python tools/layer_probe.py stem7x7
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402
import synth  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "stem7x7"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
L = {l.name: l for l in synth.RESNET50 + synth.VGG16}[name]
x = torch.randn(L.N, L.C, L.H, L.W, device="cuda").bfloat16()
w = (torch.randn(L.K, L.C, L.R, L.S, device="cuda") / (L.C * L.R * L.S) ** 0.5).bfloat16()
plan = pc.Plan(x.shape, w.shape, L.stride, L.padding, math="bf16", io_dtype="bf16")
print(name, plan.info(), flush=True)
y = torch.empty(plan.output_shape, dtype=torch.bfloat16, device="cuda")
for _ in range(reps):
    plan.forward(x, w, y)
torch.cuda.synchronize()
