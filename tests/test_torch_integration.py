"""the torch custom op / PolyConv2d / replace_conv2d and the paper's
synthetic 20-layer networks (§4.2, P.1833–1853).

CPU tests: shape inference through the op's fake kernel (meta tensors), module swapping, and that
the op refuses CPU tensors (no CPU path). GPU tests: every layer of a synthetic net, run through
the library, against the fp64 oracle on that layer's own input."""
from __future__ import annotations

import numpy as np
import pytest
import torch
from torch import nn

import oracle
from helpers import GATE, normwise

ti = pytest.importorskip("paper_conf_cgo_xuzc025_b200.torch_integration")


def test_fake_kernel_shapes():
    for (N, C, H, W, K, R, s, p) in [(2, 3, 8, 8, 5, 3, 1, 1), (1, 4, 9, 7, 2, 5, 2, 2), (3, 2, 4, 4, 6, 1, 1, 0)]:
        x = torch.empty(N, C, H, W, device="meta")
        w = torch.empty(K, C, R, R, device="meta")
        y = torch.ops.polyconv.conv2d(x, w, [s, s], [p, p], "bf16")
        ref = torch.nn.functional.conv2d(torch.empty(N, C, H, W), torch.empty(K, C, R, R), stride=s, padding=p)
        assert tuple(y.shape) == tuple(ref.shape)


def test_refuses_cpu_tensors():
    with pytest.raises(RuntimeError, match="CUDA"):
        torch.ops.polyconv.conv2d(torch.zeros(1, 1, 4, 4), torch.zeros(1, 1, 3, 3), [1, 1], [0, 0], "fp32")


@pytest.mark.parametrize("design", ti.SYNTH_NETS)
def test_synthetic_net_structure(design):
    net = ti.SyntheticNet(design, in_ch=3, width=8, seed=1)
    convs = [m for m in net.modules() if isinstance(m, nn.Conv2d)]
    assert len(convs) == ti.N_LAYERS
    if design == "mixed_kernels":
        assert {c.kernel_size[0] for c in convs} == {1, 3, 5, 7}
    n = ti.replace_conv2d(net)
    assert n == ti.N_LAYERS
    assert not any(isinstance(m, nn.Conv2d) for m in net.modules())
    assert sum(isinstance(m, ti.PolyConv2d) for m in net.modules()) == ti.N_LAYERS
    # the swapped net keeps spatial size ("same" padding) through all 20 layers (meta tensors)
    net = net.to("meta")
    y = net(torch.empty(2, 3, 12, 12, device="meta"))
    assert tuple(y.shape) == (2, convs[-1].out_channels, 12, 12)


def test_replace_skips_unsupported():
    m = nn.Sequential(nn.Conv2d(4, 4, 3, bias=True), nn.Conv2d(4, 4, 3, groups=2, bias=False),
                      nn.Conv2d(4, 4, 3, dilation=2, bias=False), nn.Conv2d(4, 4, 3, padding=1, bias=False))
    assert ti.replace_conv2d(m) == 1
    assert isinstance(m[3], ti.PolyConv2d) and m[3].weight is not None
    assert [type(c) for c in m[:3]] == [nn.Conv2d] * 3


def test_synthetic_net_weights_seeded():
    a = ti.SyntheticNet("mixed_kernels", width=8, seed=3)
    b = ti.SyntheticNet("mixed_kernels", width=8, seed=3)
    for ca, cb in zip(a.convs, b.convs):
        assert torch.equal(ca.weight, cb.weight)


@pytest.mark.gpu
@pytest.mark.parametrize("design", ti.SYNTH_NETS)
@pytest.mark.parametrize("dtype,math", [(torch.bfloat16, "bf16"), (torch.float32, "fp32")])
def test_synthetic_net_layers_vs_oracle(design, dtype, math):
    """Every layer's output (through the library) against the oracle on the same layer input."""
    net = ti.SyntheticNet(design, in_ch=3, width=16, seed=7, device="cuda", dtype=dtype)
    ti.replace_conv2d(net, math=math)
    records = []

    def hook(mod, inp, out):
        records.append((mod, inp[0].detach().float().cpu().numpy(), out.detach().float().cpu().numpy()))

    hs = [c.register_forward_hook(hook) for c in net.convs]
    g = torch.Generator().manual_seed(11)
    x = (torch.rand(2, 3, 10, 10, generator=g) * 2 - 1).to("cuda", dtype)
    with torch.no_grad():
        net(x)
    torch.cuda.synchronize()
    for h in hs:
        h.remove()
    assert len(records) == ti.N_LAYERS
    for mod, xin, y in records:
        w = mod.weight.detach().float().cpu().numpy().astype(np.float64)
        ref = oracle.conv2d(xin.astype(np.float64), w, mod.stride, mod.padding)
        err = normwise(y, ref)
        assert err <= GATE[math], f"{design} {mod}: normwise {err:.3e}"


@pytest.mark.gpu
def test_custom_op_vs_oracle():
    g = torch.Generator().manual_seed(4)
    x = (torch.rand(3, 5, 11, 9, generator=g) * 2 - 1)
    w = (torch.rand(7, 5, 3, 5, generator=g) * 2 - 1)
    ref = oracle.conv2d(x.double().numpy(), w.double().numpy(), (2, 1), (1, 2))
    y = torch.ops.polyconv.conv2d(x.cuda(), w.cuda(), [2, 1], [1, 2], "fp32")
    assert normwise(y.cpu().numpy(), ref) <= GATE["fp32"]


@pytest.mark.gpu
def test_synthetic_net_cuda_graph_replay_bit_identical():
    """The eager library path captures into a CUDA graph; replay reproduces eager bit for bit."""
    net = ti.SyntheticNet("mixed_kernels", in_ch=3, width=16, seed=2, device="cuda", dtype=torch.bfloat16)
    ti.replace_conv2d(net)
    x = torch.rand(4, 3, 12, 12, device="cuda").bfloat16()
    with torch.no_grad():
        eager = net(x)
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            net(x)  # plans created outside the capture
        torch.cuda.current_stream().wait_stream(s)
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            out = net(x)
        graph.replay()
    torch.cuda.synchronize()
    assert torch.equal(out, eager)


# --- f4: gradients through the forward library (include/polyconv.h, "Gradients") ---------------
@pytest.mark.gpu
@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
def test_flip_and_swap_bit_exact(dtype):
    import paper_conf_cgo_xuzc025_b200 as pc
    w = torch.randn(5, 3, 4, 7).to(dtype)
    wt = pc.flip_filter(w.cuda()).cpu()
    assert torch.equal(wt, w.permute(1, 0, 2, 3).flip(2, 3))  # wt[c][k][R-1-i][S-1-j] = w[k][c][i][j]
    for shape in [(3, 4, 5, 7), (2, 6, 8, 8), (1, 1, 1, 1)]:   # odd rows (element loop) and 16-B rows (vector)
        x = torch.randn(*shape).to(dtype)
        assert torch.equal(pc.swap_nc(x.cuda()).cpu(), x.transpose(0, 1))


@pytest.mark.gpu
@pytest.mark.parametrize("shape", [(2, 5, 9, 11, 7, 3, 3, 1, 1), (3, 4, 8, 8, 6, 5, 3, 2, 0), (2, 3, 6, 7, 4, 1, 1, 0, 0)],
                         ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype,math,gate", [(torch.float32, "fp32", 1e-5), (torch.bfloat16, "bf16", 2e-2)])
def test_polyconv2d_gradients(shape, dtype, math, gate):
    """dx and dw of PolyConv2d against torch's fp64 CPU autograd of the same convolution (a
    library routine, independent of this path), normwise as the forward gates (reading R14)."""
    N, C, H, W, K, R, S, ph, pw = shape
    g = torch.Generator().manual_seed(sum(shape))
    x = (torch.rand(N, C, H, W, generator=g) * 2 - 1).to(dtype)
    w = (torch.rand(K, C, R, S, generator=g) * 2 - 1).to(dtype)
    P, Q = H + 2 * ph - R + 1, W + 2 * pw - S + 1
    dy = (torch.rand(N, K, P, Q, generator=g) * 2 - 1).to(dtype)
    x64, w64 = x.double().requires_grad_(), w.double().requires_grad_()
    torch.nn.functional.conv2d(x64, w64, padding=(ph, pw)).backward(dy.double())
    mod = ti.PolyConv2d(C, K, (R, S), padding=(ph, pw), math=math,
                        weight=torch.nn.Parameter(w.cuda()))
    xc = x.cuda().requires_grad_()
    y = mod(xc)
    assert tuple(y.shape) == (N, K, P, Q)
    y.backward(dy.cuda())
    assert normwise(xc.grad.float().cpu().numpy(), x64.grad.numpy()) <= gate
    assert normwise(mod.weight.grad.float().cpu().numpy(), w64.grad.numpy()) <= gate


@pytest.mark.gpu
def test_polyconv2d_backward_rejects_wide_padding():
    mod = ti.PolyConv2d(2, 2, 3, padding=3, math="fp32", weight=torch.nn.Parameter(torch.randn(2, 2, 3, 3).cuda()))
    y = mod(torch.randn(1, 2, 8, 8, device="cuda", requires_grad=True))
    with pytest.raises(NotImplementedError):
        y.sum().backward()


@pytest.mark.gpu
@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
def test_dilate_bit_exact(dtype):
    import paper_conf_cgo_xuzc025_b200 as pc
    x = torch.randn(2, 3, 5, 4).to(dtype)
    xd = pc.dilate(x.cuda(), (2, 3), (1, 2)).cpu()
    ref = torch.zeros(2, 3, 4 * 2 + 1 + 1, 3 * 3 + 1 + 2, dtype=dtype)
    ref[:, :, 0:9:2, 0:10:3] = x
    assert torch.equal(xd, ref)


@pytest.mark.gpu
@pytest.mark.parametrize("shape", [(2, 5, 9, 11, 7, 3, 3, 1, 1, 2, 2), (3, 4, 10, 9, 6, 1, 1, 0, 0, 2, 2),
                                   (2, 3, 15, 13, 4, 7, 7, 3, 3, 2, 2), (2, 4, 11, 10, 5, 3, 2, 1, 0, 3, 2)],
                         ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype,math,gate", [(torch.float32, "fp32", 1e-5), (torch.bfloat16, "bf16", 2e-2)])
def test_polyconv2d_gradients_strided(shape, dtype, math, gate):
    """Strided layers (ResNet's 3x3 / 1x1 / 7x7 stride-2 shapes, ragged and stride 3): dx and dw
    against torch's fp64 CPU autograd."""
    N, C, H, W, K, R, S, ph, pw, sh, sw = shape
    g = torch.Generator().manual_seed(sum(shape))
    x = (torch.rand(N, C, H, W, generator=g) * 2 - 1).to(dtype)
    w = (torch.rand(K, C, R, S, generator=g) * 2 - 1).to(dtype)
    x64, w64 = x.double().requires_grad_(), w.double().requires_grad_()
    y64 = torch.nn.functional.conv2d(x64, w64, stride=(sh, sw), padding=(ph, pw))
    dy = (torch.rand(y64.shape, generator=g) * 2 - 1).to(dtype)
    y64.backward(dy.double())
    mod = ti.PolyConv2d(C, K, (R, S), stride=(sh, sw), padding=(ph, pw), math=math,
                        weight=torch.nn.Parameter(w.cuda()))
    xc = x.cuda().requires_grad_()
    y = mod(xc)
    assert tuple(y.shape) == tuple(y64.shape)
    y.backward(dy.cuda())
    assert normwise(xc.grad.float().cpu().numpy(), x64.grad.numpy()) <= gate
    assert normwise(mod.weight.grad.float().cpu().numpy(), w64.grad.numpy()) <= gate
