"""Test helpers: seeded inputs (synth/), the CUDA path through the binding, and
the oracle (oracle/), kept side by side but never mixed."""
from __future__ import annotations

import numpy as np

import synth

# Normwise parity gates (BASELINE.json north_star; reading R14):
#   err = max|y - y64| / max|y64| over the whole compared tensor
GATE = {"fp32": 1e-5, "tf32": 2e-2, "bf16": 2e-2}


def normwise(y, ref) -> float:
    y = np.asarray(y, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    den = np.max(np.abs(ref))
    return float(np.max(np.abs(y - ref)) / (den if den > 0 else 1.0))


def bf16_round(a):
    """Round fp64/fp32 values to bf16 (RNE) and back, via torch (a library routine)."""
    import torch
    return torch.from_numpy(np.asarray(a, dtype=np.float32)).bfloat16().float().numpy()


def gpu_forward(shape: synth.ConvShape, x, w, math="bf16", io="f32", kernel="auto", plan=None):
    """Run the CUDA path on numpy inputs; returns (y as fp32 numpy, plan)."""
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    dt = torch.bfloat16 if io == "bf16" else torch.float32
    xt = torch.from_numpy(x).to("cuda").to(dt).contiguous()
    wt = torch.from_numpy(w).to("cuda").to(dt).contiguous()
    if plan is None:
        plan = pc.Plan(xt.shape, wt.shape, shape.stride, shape.padding, math=math, io_dtype=io, kernel=kernel)
    y = plan.forward(xt, wt)
    torch.cuda.synchronize()
    return y.float().cpu().numpy(), plan
