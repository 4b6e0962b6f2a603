"""Host-side cost per convolution call on a tiny layer (the GPU work is a few microseconds, so
back-to-back calls measure the issue path): raw C-ABI forward, Plan.forward, the torch custom op,
PolyConv2d, and torch's conv2d (cuDNN), plus a CUDA-graph replay of the op.
Usage: python tools/op_overhead.py"""
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_xuzc025_b200 as pc  # noqa: E402
from paper_conf_cgo_xuzc025_b200 import torch_integration as ti  # noqa: E402


def per_call_us(fn, n=2000):
    for _ in range(50):
        fn()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(n):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t) / n * 1e6


def main():
    dt = torch.bfloat16
    x = torch.randn(32, 64, 8, 8, device="cuda", dtype=dt)
    w = torch.randn(64, 64, 3, 3, device="cuda", dtype=dt)
    plan = pc.Plan(x.shape, w.shape, (1, 1), (1, 1), math="bf16", io_dtype="bf16")
    y = torch.empty(plan.output_shape, device="cuda", dtype=dt)
    s = torch.cuda.current_stream().cuda_stream
    mod = ti.PolyConv2d(64, 64, 3, padding=1, weight=torch.nn.Parameter(w))
    res = {
        "kernel": plan.info()["kernel"],
        "c_abi_forward_ptr_us": per_call_us(lambda: plan.forward_ptr(x.data_ptr(), w.data_ptr(), y.data_ptr(), s)),
        "plan_forward_us": per_call_us(lambda: plan.forward(x, w, y)),
        "pc_conv2d_us": per_call_us(lambda: pc.conv2d(x, w, (1, 1), (1, 1))),
        "custom_op_us": per_call_us(lambda: torch.ops.polyconv.conv2d(x, w, [1, 1], [1, 1], "bf16")),
        "polyconv2d_module_us": per_call_us(lambda: mod(x)),
        "torch_conv2d_cudnn_us": per_call_us(lambda: torch.nn.functional.conv2d(x, w, padding=1)),
    }
    g = torch.cuda.CUDAGraph()
    try:
        with torch.cuda.graph(g):
            for _ in range(20):
                yg = mod(x)
        res["graph_replay_per_conv_us"] = per_call_us(g.replay, n=200) / 20
    except Exception as e:  # report, do not hide
        res["graph_error"] = repr(e)[:300]
    print(json.dumps(res))


if __name__ == "__main__":
    main()
