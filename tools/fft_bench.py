"""Dev timing of the FFT solver against the FP32 FFMA path (and the tensor-core paths) on
layers whose padded planes fit L <= 8192.  python tools/fft_bench.py"""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402
import synth  # noqa: E402
flush = torch.empty(64 << 20, device="cuda")


def timed(fn, reps=10):
    ts = []
    for it in range(reps + 3):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        if it >= 3:
            ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


shapes = [synth.CONV3X] + [s for s in synth.SWEEP if s.name in ("A_h14_s1", "A_h28_s1", "A_h56_s1", "B_r3_s1", "B_r5_s1", "B_r7_s1", "C_c64_s2", "C_c128_s2")] + \
         [s for s in synth.RESNET50 if s.name in ("l2_3x3_128", "l3_3x3_256", "l4_3x3_512", "l1_3x3_64")]
for L in shapes:
    x = torch.rand(L.N, L.C, L.H, L.W, device="cuda") * 2 - 1
    w = (torch.rand(L.K, L.C, L.R, L.S, device="cuda") * 2 - 1) / (L.C * L.R * L.S) ** 0.5
    rec = {"layer": L.name}
    for kern in ("fft", "auto"):
        try:
            plan = pc.Plan(x.shape, w.shape, L.stride, L.padding, math="fp32", kernel=kern)
        except pc.PolyconvError:
            continue
        y = torch.empty(plan.output_shape, device="cuda")
        t = timed(lambda: plan.forward(x, w, y))
        rec[kern if kern == "fft" else plan.info()["kernel"]] = round(L.flops() / t / 1e9, 2)
        if kern == "fft":
            rec["L"] = plan.info()["tile_m"]
        del plan
    print(json.dumps(rec), flush=True)
