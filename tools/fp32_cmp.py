"""FP32-math kernel comparison per layer (fresh plans; TFLOP/s, L2 flushed): the FFT solver (f1)
against the FFMA direct path and AUTO.  python tools/fp32_cmp.py [resnet50|vgg16|sweep|all]"""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402
import synth  # noqa: E402
which = sys.argv[1] if len(sys.argv) > 1 else "all"
layers = {"resnet50": synth.RESNET50, "vgg16": synth.VGG16, "sweep": synth.SWEEP}.get(
    which, [synth.CONV3X] + synth.RESNET50 + synth.VGG16 + synth.SWEEP)
flush = torch.empty(64 << 20, device="cuda")


def timed(fn, reps=6):
    ts = []
    for it in range(reps + 2):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        if it >= 2:
            ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


for L in layers:
    x = torch.rand(L.N, L.C, L.H, L.W, device="cuda") * 2 - 1
    w = (torch.rand(L.K, L.C, L.R, L.S, device="cuda") * 2 - 1) / (L.C * L.R * L.S) ** 0.5
    rec = {"layer": L.name}
    for kern in ("auto", "fft", "fp32"):
        try:
            plan = pc.Plan(x.shape, w.shape, L.stride, L.padding, math="fp32", kernel=kern)
        except pc.PolyconvError:
            continue
        y = torch.empty(plan.output_shape, device="cuda")
        t = timed(lambda: plan.forward(x, w, y))
        rec[kern] = round(L.flops() / t / 1e9, 2)
        if kern == "auto":
            rec["auto_kernel"] = plan.info()["kernel"]
        del plan, y
    print(json.dumps(rec), flush=True)
