"""Dev probe of TC_HANKEL: time one layer under each POLYCONV_HK_DEBUG ablation and print the
per-CTA trace (median / max over CTAs, us from the earliest start).

    python tools/hk_trace.py N C H W K R S [s p]
"""
import ctypes
import os
import subprocess
import sys
import json

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

if os.environ.get("HK_CHILD"):
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    a = [int(v) for v in sys.argv[1:]]
    N, C, H, W, K, R, S = a[:7]
    s, p = (a[7], a[8]) if len(a) > 8 else (1, R // 2)
    x = (torch.rand((N, C, H, W), device="cuda") * 2 - 1).bfloat16()
    w = (torch.rand((K, C, R, S), device="cuda") * 2 - 1).bfloat16()
    plan = pc.Plan(x.shape, w.shape, (s, s), (p, p), math="bf16", io_dtype="bf16",
                   kernel=os.environ.get("HK_KERNEL", "tc_hankel"))
    y = torch.empty(plan.output_shape, dtype=torch.bfloat16, device="cuda")
    flush = torch.empty(64 << 20, device="cuda")
    ts = []
    for it in range(13):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        plan.forward(x, w, y)
        e1.record()
        torch.cuda.synchronize()
        if it >= 3:
            ts.append(e0.elapsed_time(e1))
    ts.sort()
    out = {"dbg": os.environ.get("POLYCONV_HK_DEBUG", "0"), "ms": ts[len(ts) // 2], "info": plan.info()}
    F = 2.0 * N * K * C * R * S * plan.output_shape[2] * plan.output_shape[3]
    out["tflops"] = F / out["ms"] / 1e9
    if int(out["dbg"]) & 8:
        lib = pc.load_library()
        buf = (ctypes.c_ulonglong * (160 * 16))()
        lib.polyconv_dbg_hk_trace(buf)
        grid = 2 * out["info"].get("grid", 74) if False else 148
        rows = [[buf[b * 16 + i] for i in range(16)] for b in range(grid)]
        rows = [r for r in rows if r[0]]
        t0 = min(r[0] for r in rows)
        summ = {}
        for i in range(11):
            v = sorted((r[i] - t0) / 1e3 for r in rows if r[i])
            if v:
                summ[i] = [round(v[len(v) // 2], 2), round(v[-1], 2)]
        out["trace_us_med_max"] = summ
    if int(out["dbg"]) & 16:
        lib = pc.load_library()
        buf = (ctypes.c_ulonglong * (64 * 8))()
        lib.polyconv_dbg_hk_wtrace(buf)
        t0 = buf[0]
        out["wtrace_us"] = [[round((buf[i * 8 + j] - t0) / 1e3, 2) if buf[i * 8 + j] else None for j in range(5)]
                            for i in range(64) if buf[i * 8]]
    if int(out["dbg"]) & 32:
        lib = pc.load_library()
        buf = (ctypes.c_ulonglong * (64 * 16))()
        lib.polyconv_dbg_hk_ltrace(buf)
        t0 = min(v for v in buf if v)
        out["ltrace_us"] = [[round((buf[i * 16 + j] - t0) / 1e3, 2) if buf[i * 16 + j] else None for j in range(16)]
                            for i in range(64) if buf[i * 16]]
    print(json.dumps(out), flush=True)
else:
    for dbg in os.environ.get("HK_DBGS", "8 9 10 12 15").split():
        env = dict(os.environ, HK_CHILD="1", POLYCONV_HK_DEBUG=dbg)
        subprocess.run([sys.executable, __file__] + sys.argv[1:], env=env)
