"""Forward + backward step time of the synthetic 20-layer nets (f3 + f4): torch conv2d (cuDNN, NCHW,
benchmark mode) against `replace_conv2d` (forward, dgrad and wgrad through libpolyconv.so), bf16,
same weights and input; CUDA events around whole steps (loss = y.float().square().mean()),
median of --iters after --warmup.
Usage: python tools/synthnet_train.py [--batch 32] [--sizes 14,28,56] > out.jsonl"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cgo_xuzc025_b200 import torch_integration as ti  # noqa: E402


def step_ms(net, x, warmup, iters):
    ts = []
    for it in range(warmup + iters):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        net.zero_grad(set_to_none=True)
        xi = x.detach().requires_grad_()
        net(xi).float().square().mean().backward()
        b.record()
        torch.cuda.synchronize()
        if it >= warmup:
            ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=32)
    ap.add_argument("--width", type=int, default=64)
    ap.add_argument("--sizes", default="14,28,56")
    ap.add_argument("--designs", default=",".join(ti.SYNTH_NETS))
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--iters", type=int, default=10)
    a = ap.parse_args()
    torch.backends.cudnn.benchmark = True
    for design in a.designs.split(","):
        for H in (int(s) for s in a.sizes.split(",")):
            net = ti.SyntheticNet(design, in_ch=3, width=a.width, seed=5, device="cuda", dtype=torch.bfloat16)
            x = (torch.rand(a.batch, 3, H, H, generator=torch.Generator().manual_seed(H)) * 2 - 1).to(
                "cuda", torch.bfloat16)
            t_cudnn = step_ms(net, x, a.warmup, a.iters)
            ti.replace_conv2d(net, math="bf16")
            t_poly = step_ms(net, x, a.warmup, a.iters)
            print(json.dumps({"design": design, "input": H, "batch": a.batch, "width": a.width, "dtype": "bf16",
                              "step": "fwd+bwd", "polyconv_ms": t_poly, "cudnn_nchw_ms": t_cudnn,
                              "speedup_vs_cudnn": t_cudnn / t_poly}), flush=True)
            del net, x
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
