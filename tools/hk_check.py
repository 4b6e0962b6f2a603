"""Dev check of the TC_HANKEL kernel (not a test): integer-valued inputs (every product and
partial sum exact in bf16/tf32/fp32) against torch fp64 conv2d on the same GPU, bit-exact,
then random inputs against fp64 normwise; plus timing vs cuDNN (best layout) with L2 flushed.

    python tools/hk_check.py [quick|gate|all]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import torch.nn.functional as Fn  # noqa: E402

import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "quick"
kern = os.environ.get("HK_KERNEL", "tc_hankel")
PEAK = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["bf16_tflops"]
torch.backends.cudnn.benchmark = True
torch.backends.cudnn.allow_tf32 = False
flush = torch.empty(64 << 20, device="cuda")


def timed(fn, reps=10):
    ts = []
    for it in range(reps + 3):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        if it >= 3:
            ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


def run(N, C, H, W, K, R, S, s, p, math="bf16", io="bf16", time_it=False, name=""):
    g = torch.Generator(device="cuda").manual_seed(N * 7 + C + K + H)
    xi = torch.randint(-8, 9, (N, C, H, W), device="cuda", generator=g).double()
    wi = torch.randint(-4, 5, (K, C, R, S), device="cuda", generator=g).double()
    dt = torch.bfloat16 if io == "bf16" else torch.float32
    plan = pc.Plan(xi.shape, wi.shape, (s, s), (p, p), math=math, io_dtype=io, kernel=kern)
    info = plan.info()
    y = plan.forward(xi.to(dt).contiguous(), wi.to(dt).contiguous())
    ref = Fn.conv2d(xi, wi, stride=s, padding=p)
    torch.cuda.synchronize()
    if io == "bf16":
        exact = bool(torch.equal(y.double(), ref.to(torch.bfloat16).double()))
    else:
        exact = bool(torch.equal(y.double(), ref))
    bad = None
    if not exact:
        d = (y.double() - (ref.to(torch.bfloat16).double() if io == "bf16" else ref)).abs()
        idx = (d > 0).nonzero()
        bad = {"n_bad": int(idx.shape[0]), "first": idx[:4].tolist(), "max": float(d.max())}
    xr = (torch.rand((N, C, H, W), device="cuda", generator=g) * 2 - 1)
    wr = (torch.rand((K, C, R, S), device="cuda", generator=g) * 2 - 1) / (C * R * S) ** 0.5
    y2 = plan.forward(xr.to(dt).contiguous(), wr.to(dt).contiguous())
    r2 = Fn.conv2d(xr.double(), wr.double(), stride=s, padding=p)
    nw = float((y2.double() - r2).abs().max() / r2.abs().max())
    rec = {"name": name, "shape": [N, C, H, W, K, R, S, s, p], "math": math, "io": io, "exact_int": exact,
           "normwise": nw, "T": info["tile_m"] // 256, "NN": info["tile_n"], "kernel": info["kernel"]}
    if bad:
        rec["bad"] = bad
    if time_it:
        xb, wb = xr.to(dt).contiguous(), wr.to(dt).contiguous()
        yb = torch.empty(plan.output_shape, dtype=dt, device="cuda")
        t = timed(lambda: plan.forward(xb, wb, yb))
        F = 2.0 * N * K * C * R * S * y.shape[2] * y.shape[3]
        xc, wc = xb.contiguous(memory_format=torch.channels_last), wb.contiguous(memory_format=torch.channels_last)
        tc = min(timed(lambda: Fn.conv2d(xb, wb, stride=s, padding=p)), timed(lambda: Fn.conv2d(xc, wc, stride=s, padding=p)))
        rec.update({"ms": t, "tflops": F / t / 1e9, "frac": F / t / 1e9 / PEAK, "cudnn_tflops": F / tc / 1e9})
    print(json.dumps(rec), flush=True)
    return rec


if which in ("quick", "all"):
    for args in [(1, 64, 8, 8, 64, 3, 3, 1, 1), (2, 64, 14, 14, 128, 3, 3, 1, 1), (3, 128, 28, 28, 128, 3, 3, 1, 1),
                 (2, 80, 13, 11, 48, 3, 3, 1, 1), (2, 64, 7, 7, 512, 3, 3, 1, 1), (2, 256, 14, 14, 256, 3, 3, 1, 1),
                 (1, 3, 16, 16, 16, 3, 3, 1, 1), (2, 64, 20, 20, 64, 5, 5, 1, 2), (2, 32, 17, 17, 64, 3, 3, 2, 1),
                 (2, 64, 9, 9, 64, 1, 1, 1, 0), (2, 64, 12, 12, 64, 3, 3, 1, 0), (4, 512, 7, 7, 512, 3, 3, 1, 1)]:
        run(*args, name="quick")
    for args in [(2, 64, 14, 14, 128, 3, 3, 1, 1), (2, 80, 13, 11, 48, 3, 3, 1, 1)]:
        run(*args, math="bf16", io="f32", name="quick_f32io")
        run(*args, math="tf32", io="f32", name="quick_tf32")
if which in ("tail", "all"):
    # unit counts just past a multiple of the pair count: tail units split into sub-units
    for args in [(40, 128, 28, 28, 128, 3, 3, 1, 1), (100, 256, 14, 14, 256, 3, 3, 1, 1),
                 (90, 512, 7, 7, 512, 3, 3, 1, 1), (70, 64, 28, 28, 96, 3, 3, 1, 1), (33, 96, 20, 21, 192, 3, 3, 1, 1)]:
        run(*args, name="tail")
        run(*args, math="tf32", io="f32", name="tail_tf32")
if which in ("stem", "all"):
    # 7x7 stride 2, C = 3: small-C phase mode, 32-byte window rows
    for args in [(2, 3, 32, 32, 64, 7, 7, 2, 3), (3, 3, 30, 26, 40, 7, 7, 2, 3), (2, 4, 20, 20, 48, 7, 7, 2, 3),
                 (2, 2, 16, 24, 64, 5, 5, 2, 2), (8, 3, 224, 224, 64, 7, 7, 2, 3)]:
        run(*args, name="stem")
    run(256, 3, 224, 224, 64, 7, 7, 2, 3, time_it=True, name="stem7x7")
    # stride 1, C <= 16: 32-byte rows (VGG conv1_1)
    for args in [(2, 3, 32, 32, 64, 3, 3, 1, 1), (3, 5, 18, 20, 40, 3, 3, 1, 1), (2, 16, 16, 16, 48, 3, 3, 1, 1),
                 (2, 3, 20, 24, 32, 5, 5, 1, 2), (4, 3, 224, 224, 64, 3, 3, 1, 1)]:
        run(*args, name="smallc")
    run(64, 3, 224, 224, 64, 3, 3, 1, 1, time_it=True, name="vgg_conv1_1")
if which in ("s2", "all"):
    # stride 2: phase-split mode (reading R19) where W % 4 == 0 and C % 32 == 0
    for args in [(2, 64, 16, 16, 64, 3, 3, 2, 1), (3, 128, 56, 56, 128, 3, 3, 2, 1), (2, 256, 28, 28, 256, 3, 3, 2, 1),
                 (2, 32, 12, 20, 48, 3, 3, 2, 1), (2, 64, 24, 24, 64, 5, 5, 2, 2), (2, 64, 15, 16, 64, 3, 3, 2, 1),
                 (2, 64, 16, 16, 64, 3, 3, 2, 0), (40, 128, 56, 56, 128, 3, 3, 2, 1), (2, 96, 20, 12, 80, 5, 5, 2, 1),
                 (3, 64, 14, 14, 96, 3, 3, 2, 1), (2, 32, 10, 18, 64, 5, 5, 2, 2), (20, 512, 14, 14, 512, 3, 3, 2, 1)]:
        run(*args, name="s2")
    for args, nm in [((256, 128, 56, 56, 128, 3, 3, 2, 1), "l2_3x3_128_s2"), ((256, 256, 28, 28, 256, 3, 3, 2, 1), "l3_3x3_256_s2"),
                     ((256, 512, 14, 14, 512, 3, 3, 2, 1), "l4_3x3_512_s2")]:
        run(*args, time_it=True, name=nm)
if which in ("gate", "all"):
    for args, nm in [((32, 128, 28, 28, 128, 3, 3, 1, 1), "conv3x_n32"), ((256, 64, 56, 56, 64, 3, 3, 1, 1), "l1_3x3_64"),
                     ((256, 128, 28, 28, 128, 3, 3, 1, 1), "l2_3x3_128"), ((256, 256, 14, 14, 256, 3, 3, 1, 1), "l3_3x3_256"),
                     ((256, 512, 7, 7, 512, 3, 3, 1, 1), "l4_3x3_512")]:
        run(*args, time_it=True, name=nm)
