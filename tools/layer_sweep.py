"""Per-layer sweep (BASELINE.json configs[2] VGG-16 N=64 and configs[4] ResNet-50 N=256 on one
GPU): effective TFLOP/s of this library (AUTO kernel, BF16 in/out and math) next to cuDNN on the
same NCHW tensors and on channels_last input, L2 flushed before every timed call, CUDA events
on the current stream.  Writes one JSON line per layer and a summary to stdout.

    python tools/layer_sweep.py [resnet50|vgg16] [reps]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import torch.nn.functional as Fn  # noqa: E402

import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402
import synth  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "resnet50"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
layers = synth.RESNET50 if which == "resnet50" else synth.VGG16
peaks = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                    "MEASURED_PEAKS.json")))
peak = peaks["bf16_tflops"]
torch.backends.cudnn.benchmark = True
flush = torch.empty(64 << 20, device="cuda")
evict = torch.empty(64 << 20, device="cuda")


def timed(fn):
    ts = []
    for it in range(reps + 3):
        flush.zero_()
        evict.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        if it >= 3:
            ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


tot = {"ours": 0.0, "nchw": 0.0, "cl": 0.0, "flop": 0.0}
for L in layers:
    g = torch.Generator(device="cuda").manual_seed(1)
    x = torch.rand((L.N, L.C, L.H, L.W), device="cuda", generator=g).mul_(2).sub_(1).bfloat16()
    w = (torch.rand((L.K, L.C, L.R, L.S), device="cuda", generator=g).mul_(2).sub_(1) /
         (L.C * L.R * L.S) ** 0.5).bfloat16()
    plan = pc.Plan(x.shape, w.shape, L.stride, L.padding, math="bf16", io_dtype="bf16")
    y = torch.empty(plan.output_shape, dtype=torch.bfloat16, device="cuda")
    t_ours = timed(lambda: plan.forward(x, w, y))
    t_nchw = timed(lambda: Fn.conv2d(x, w, stride=L.stride, padding=L.padding))
    xc, wc = x.contiguous(memory_format=torch.channels_last), w.contiguous(memory_format=torch.channels_last)
    t_cl = timed(lambda: Fn.conv2d(xc, wc, stride=L.stride, padding=L.padding))
    ref = Fn.conv2d(x.float(), w.float(), stride=L.stride, padding=L.padding)
    err = float((y.float() - ref).abs().max() / ref.abs().max())
    F = L.flops()
    rec = {"layer": L.name, "count": L.count, "kernel": plan.info()["kernel"], "ms": t_ours,
           "tflops": F / t_ours / 1e9, "frac_of_peak": F / t_ours / 1e9 / peak,
           "cudnn_nchw_tflops": F / t_nchw / 1e9, "cudnn_cl_tflops": F / t_cl / 1e9,
           "normwise_vs_torch_fp32": err}
    print(json.dumps(rec), flush=True)
    tot["ours"] += L.count * t_ours
    tot["nchw"] += L.count * t_nchw
    tot["cl"] += L.count * t_cl
    tot["flop"] += L.count * F
    del plan
print(json.dumps({"summary": which, "layers": len(layers), "ours_ms": tot["ours"], "cudnn_nchw_ms": tot["nchw"],
                  "cudnn_cl_ms": tot["cl"], "ours_tflops": tot["flop"] / tot["ours"] / 1e9,
                  "cudnn_nchw_tflops": tot["flop"] / tot["nchw"] / 1e9,
                  "cudnn_cl_tflops": tot["flop"] / tot["cl"] / 1e9}))
