"""PAPER.md §4.2 / Fig. 6 methodology on B200: the synthetic 20-layer networks
over input sizes 4–224, "the accumulated time spent on the convolution operator" (P.1970–1972),
with PyTorch's own conv2d (cuDNN, benchmark=True) on NCHW and on channels_last tensors (the
better one is the comparison), and after `replace_conv2d` (every convolution
through libpolyconv.so, AUTO kernel, NCHW). Same weights, same seeded input, bf16.

Per conv layer, CUDA events recorded by forward hooks on the current stream bracket the operator;
the sum over the 20 layers is the median of --iters passes after --warmup passes.
Usage: python tools/synthnet_bench.py [--batch 32] [--width 64] [--sizes 4,8,...] > out.jsonl
"""
from __future__ import annotations

import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cgo_xuzc025_b200 import torch_integration as ti  # noqa: E402


def conv_flops(net, N, H):
    f = 0
    for c in net.convs:
        f += 2 * N * c.out_channels * c.in_channels * c.kernel_size[0] * c.kernel_size[1] * H * H
    return f


def timed_conv_ms(net, x, warmup, iters):
    convs = [m for m in net.modules() if isinstance(m, (torch.nn.Conv2d, ti.PolyConv2d))]
    assert len(convs) == ti.N_LAYERS
    pairs = []

    def pre(mod, inp):
        e = torch.cuda.Event(enable_timing=True)
        e.record()
        pairs.append([e, None])

    def post(mod, inp, out):
        e = torch.cuda.Event(enable_timing=True)
        e.record()
        pairs[-1][1] = e

    hs = [c.register_forward_pre_hook(pre) for c in convs] + [c.register_forward_hook(post) for c in convs]
    with torch.no_grad():
        for _ in range(warmup):
            net(x)
        torch.cuda.synchronize()
        pairs.clear()
        for _ in range(iters):
            net(x)
        torch.cuda.synchronize()
    for h in hs:
        h.remove()
    per_pass = sorted(sum(a.elapsed_time(b) for a, b in pairs[i * ti.N_LAYERS:(i + 1) * ti.N_LAYERS])
                      for i in range(iters))
    return per_pass[iters // 2]  # median pass (host hiccups land in single passes)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=32)
    ap.add_argument("--width", type=int, default=64)
    ap.add_argument("--sizes", default="4,8,14,28,56,112,224")
    ap.add_argument("--designs", default=",".join(ti.SYNTH_NETS))
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--iters", type=int, default=10)
    a = ap.parse_args()
    torch.backends.cudnn.benchmark = True
    dt = torch.bfloat16
    for design in a.designs.split(","):
        for H in (int(s) for s in a.sizes.split(",")):
            net = ti.SyntheticNet(design, in_ch=3, width=a.width, seed=5, device="cuda", dtype=dt)
            g = torch.Generator().manual_seed(H)
            x = (torch.rand(a.batch, 3, H, H, generator=g) * 2 - 1).to("cuda", dt)
            flops = conv_flops(net, a.batch, H)
            t_nchw = timed_conv_ms(net, x, a.warmup, a.iters)
            net_cl = net.to(memory_format=torch.channels_last)
            t_cl = timed_conv_ms(net_cl, x.contiguous(memory_format=torch.channels_last), a.warmup, a.iters)
            net = net.to(memory_format=torch.contiguous_format)
            t_cudnn, layout = (t_nchw, "nchw") if t_nchw <= t_cl else (t_cl, "channels_last")
            ti.replace_conv2d(net, math="bf16")
            t_poly = timed_conv_ms(net, x, a.warmup, a.iters)
            print(json.dumps({"design": design, "input": H, "batch": a.batch, "width": a.width, "dtype": "bf16",
                              "conv_gflop": flops / 1e9, "polyconv_ms": t_poly, "cudnn_nchw_ms": t_nchw,
                              "cudnn_channels_last_ms": t_cl, "cudnn_best_layout": layout,
                              "polyconv_tflops": flops / t_poly / 1e9, "cudnn_tflops": flops / t_cudnn / 1e9,
                              "speedup_vs_cudnn_best": t_cudnn / t_poly,
                              "speedup_vs_cudnn_nchw": t_nchw / t_poly}), flush=True)
            del net, x
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
