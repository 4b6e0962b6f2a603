"""GPU parity coverage of every BASELINE config in every math, the
gradients against the oracle, and the launch-safety properties (CUDA-graph replay with new
inputs, other work holding SMs).

Full-size launches (the shapes the bench and sweeps time); the output is compared against O1 on
a sample of images and, for the largest layers, of output channels, so that the fp64 oracle's
work stays bounded ("at BASELINE.json's full sizes ... on sampled outputs").
Gates: normwise 1e-5 (FP32_FMA) / 2e-2 (TF32, BF16) (reading R14).
"""
import numpy as np
import pytest

import oracle
import synth
from synth import ConvShape
from helpers import GATE, normwise, bf16_round, gpu_forward

pytestmark = pytest.mark.gpu

ORACLE_GFLOP = 2.0   # fp64 work per comparison


def _full_launch_sampled(shape, math, io, seed):
    """Launch the whole layer; compare images {0, N-1} (or only N-1) and a prefix of the
    output channels sized so the oracle does at most ORACLE_GFLOP of work."""
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    dt = torch.bfloat16 if io == "bf16" else torch.float32
    gen = torch.Generator(device="cuda").manual_seed(seed)
    x = (torch.rand((shape.N, shape.C, shape.H, shape.W), generator=gen, device="cuda") * 2 - 1).to(dt)
    w = ((torch.rand((shape.K, shape.C, shape.R, shape.S), generator=gen, device="cuda") * 2 - 1)
         / np.sqrt(shape.C * shape.R * shape.S)).to(dt)
    plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math=math, io_dtype=io)
    y = plan.forward(x, w)
    torch.cuda.synchronize()
    per_img_ch = 2.0 * shape.C * shape.R * shape.S * shape.P * shape.Q / 1e9   # GFLOP per (image, k)
    images = sorted({0, shape.N - 1})
    if per_img_ch * shape.K * len(images) > ORACLE_GFLOP:
        images = [shape.N - 1]
    kk = int(max(8, min(shape.K, ORACLE_GFLOP / (per_img_ch * len(images)))))
    xs = x[images].float().cpu().numpy()
    ws = w[:kk].float().cpu().numpy()
    ref = oracle.conv2d(xs, ws, shape.stride, shape.padding)
    got = y[images][:, :kk].float().cpu().numpy()
    return normwise(got, ref), plan.info()["kernel"]


# ---- BASELINE configs[4]: ResNet-50 N=256, every unique shape, TF32 / FP32 / BF16 (f32 I/O) ----
@pytest.mark.parametrize("shape", synth.RESNET50, ids=lambda s: s.name)
@pytest.mark.parametrize("math", ["tf32", "fp32", "bf16"])
def test_resnet50_all_maths(shape, math):
    err, kern = _full_launch_sampled(shape, math, "f32", seed=41)
    assert err <= GATE[math], (kern, err)


# ... and BF16 with bf16 I/O, the bench's and the sweeps' configuration: the stride-2 phase
# mode, the stem's 32-byte rows and the wide-input 1x1 routing of mac_hankel are bf16-I/O paths
@pytest.mark.parametrize("shape", synth.RESNET50, ids=lambda s: s.name)
def test_resnet50_bf16_io(shape):
    err, kern = _full_launch_sampled(shape, "bf16", "bf16", seed=44)
    assert err <= GATE["bf16"], (kern, err)


# ---- BASELINE configs[3]: all 34 sweep points, BF16 (bf16 I/O) / TF32 / FP32 ----
@pytest.mark.parametrize("shape", synth.SWEEP, ids=lambda s: s.name)
@pytest.mark.parametrize("math,io", [("bf16", "bf16"), ("tf32", "f32"), ("fp32", "f32")])
def test_sweep_all_points(shape, math, io):
    err, kern = _full_launch_sampled(shape, math, io, seed=42)
    assert err <= GATE[math], (kern, err)


# ---- BASELINE configs[2]: all 13 VGG-16 layers, TF32 / FP32 (bf16 I/O in test_gpu_parity) ----
@pytest.mark.parametrize("shape", synth.VGG16, ids=lambda s: s.name)
@pytest.mark.parametrize("math,io", [("tf32", "f32"), ("fp32", "f32"), ("bf16", "bf16")])
def test_vgg16_all_layers(shape, math, io):
    err, kern = _full_launch_sampled(shape, math, io, seed=43)
    assert err <= GATE[math], (kern, err)


# ---- gradients against the oracle (f4) -------------------------------------------------------
def _dgrad_oracle(dy, w, stride, padding, H, W):
    """dx = conv(dy spread on the stride lattice, flipped w^T) with padding R-1-p, computed by O1
    (the test only rearranges data: zero-spreading and the filter flip/transpose)."""
    N, K, P, Q = dy.shape
    _, C, R, S = w.shape
    (sh, sw), (ph, pw) = stride, padding
    Hd = (P - 1) * sh + 1 + (H + 2 * ph - R) % sh
    Wd = (Q - 1) * sw + 1 + (W + 2 * pw - S) % sw
    dyd = np.zeros((N, K, Hd, Wd))
    dyd[:, :, 0:(P - 1) * sh + 1:sh, 0:(Q - 1) * sw + 1:sw] = dy
    wt = np.ascontiguousarray(np.flip(np.transpose(w, (1, 0, 2, 3)), axis=(2, 3)))
    return oracle.conv2d(dyd, wt, (1, 1), (R - 1 - ph, S - 1 - pw))


def _wgrad_sum(x, dy, R, S, stride, padding):
    """dw[k][c][i][j] = sum_{n,oh,ow} dy[n][k][oh][ow] * xpad[n][c][sh*oh+i][sw*ow+j], fp64."""
    N, C, H, W = x.shape
    _, K, P, Q = dy.shape
    (sh, sw), (ph, pw) = stride, padding
    xp = np.pad(x.astype(np.float64), ((0, 0), (0, 0), (ph, ph), (pw, pw)))
    dw = np.zeros((K, C, R, S))
    for i in range(R):
        for j in range(S):
            win = xp[:, :, i:i + (P - 1) * sh + 1:sh, j:j + (Q - 1) * sw + 1:sw]   # [N][C][P][Q]
            dw[:, :, i, j] = np.einsum("nkpq,ncpq->kc", dy.astype(np.float64), win)
    return dw


@pytest.mark.parametrize("shape", [(2, 5, 9, 11, 7, 3, 3, 1, 1, 1, 1), (3, 4, 8, 8, 6, 5, 3, 2, 0, 1, 1),
                                   (2, 6, 10, 10, 8, 3, 3, 1, 1, 2, 2), (2, 3, 15, 13, 4, 7, 7, 3, 3, 2, 2),
                                   (2, 8, 9, 9, 16, 1, 1, 0, 0, 2, 2)],
                         ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("math,gate", [("fp32", 1e-5), ("bf16", 2e-2)])
def test_gradients_vs_oracle(shape, math, gate):
    """PolyConv2d's dx and dw against O1 (dgrad as an oracle convolution of rearranged data)
    and an explicit fp64 sum (wgrad), on bf16-representable inputs."""
    import torch
    from paper_conf_cgo_xuzc025_b200 import torch_integration as ti
    N, C, H, W, K, R, S, ph, pw, sh, sw = shape
    rng = np.random.default_rng(sum(shape))
    x = bf16_round(rng.uniform(-1, 1, (N, C, H, W)))
    w = bf16_round(rng.uniform(-1, 1, (K, C, R, S)))
    P, Q = oracle.output_dims(H, W, R, S, (sh, sw), (ph, pw))
    dy = bf16_round(rng.uniform(-1, 1, (N, K, P, Q)))
    dt = torch.float32 if math == "fp32" else torch.bfloat16
    mod = ti.PolyConv2d(C, K, (R, S), stride=(sh, sw), padding=(ph, pw), math=math,
                        weight=torch.nn.Parameter(torch.from_numpy(w).to(dt).cuda()))
    xc = torch.from_numpy(x).to(dt).cuda().requires_grad_()
    mod(xc).backward(torch.from_numpy(dy).to(dt).cuda())
    dx_ref = _dgrad_oracle(dy, w, (sh, sw), (ph, pw), H, W)
    dw_ref = _wgrad_sum(x, dy, R, S, (sh, sw), (ph, pw))
    assert normwise(xc.grad.float().cpu().numpy(), dx_ref) <= gate
    assert normwise(mod.weight.grad.float().cpu().numpy(), dw_ref) <= gate


def test_wgrad_propagates_nan():
    """A NaN in dy reaches dw as NaN in bf16 (the output rounding keeps NaN: ADVICE round 1)."""
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    x = torch.rand(2, 4, 8, 8, device="cuda").bfloat16()
    dy = torch.rand(2, 8, 8, 8, device="cuda").bfloat16()
    dy[1, 3, 2, 5] = float("nan")
    dw = pc.wgrad(x, dy, (8, 4, 3, 3), (1, 1), (1, 1))
    torch.cuda.synchronize()
    assert torch.isnan(dw[3].float()).all() and not torch.isnan(dw[:3].float()).any()


def test_wgrad_rejects_mismatched_shapes():
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    x = torch.rand(2, 4, 8, 8, device="cuda")
    with pytest.raises(pc.PolyconvError):
        pc.wgrad(x, torch.rand(2, 8, 7, 8, device="cuda"), (8, 4, 3, 3), (1, 1), (1, 1))   # P != 8
    with pytest.raises(pc.PolyconvError):
        pc.wgrad(x, torch.rand(2, 8, 8, 8, device="cuda"), (8, 5, 3, 3), (1, 1), (1, 1))   # C != 4


def test_double_backward_raises():
    """The backward runs library kernels autograd cannot differentiate: create_graph=True must
    raise rather than return silent zeros (once_differentiable)."""
    import torch
    from paper_conf_cgo_xuzc025_b200 import torch_integration as ti
    mod = ti.PolyConv2d(4, 8, 3, padding=1, math="fp32",
                        weight=torch.nn.Parameter(torch.randn(8, 4, 3, 3, device="cuda")))
    x = torch.randn(2, 4, 8, 8, device="cuda", requires_grad=True)
    y = mod(x).sum()
    (gx,) = torch.autograd.grad(y, x, create_graph=True)
    with pytest.raises(RuntimeError):
        gx.sum().backward()


# ---- launch safety -------------------------------------------------------------------------
GRAPH_CASES = [("auto", ConvShape("g_hankel", 4, 64, 28, 28, 64, 3, 3, 1, 1, 1, 1)),
               ("tc_pair", ConvShape("g_pair", 4, 64, 16, 16, 64, 3, 3, 1, 1, 1, 1)),
               ("tc_fused", ConvShape("g_fused", 4, 64, 16, 16, 128, 3, 3, 1, 1, 1, 1)),
               ("tc", ConvShape("g_tc", 4, 64, 16, 16, 128, 3, 3, 1, 1, 1, 1))]


@pytest.mark.parametrize("kernel,shape", GRAPH_CASES, ids=lambda v: v if isinstance(v, str) else v.name)
def test_cuda_graph_replays_with_new_inputs(kernel, shape):
    """A forward captured into a CUDA graph and replayed three times with new x and w each
    time gives the oracle's result every time (integer data, bit-exact); no kernel keeps state
    between launches that a replay would reuse."""
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    x0, w0 = synth.make_inputs(shape, 31, "int")
    x = torch.from_numpy(x0).bfloat16().cuda()
    w = torch.from_numpy(w0).bfloat16().cuda()
    plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math="bf16", io_dtype="bf16", kernel=kernel)
    y = torch.empty(plan.output_shape, dtype=torch.bfloat16, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        plan.forward(x, w, y)   # warm-up on the capture stream (workspace, tensor maps)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph, stream=s):
        plan.forward(x, w, y, stream=s)
    for it in range(3):
        xi, wi = synth.make_inputs(shape, 100 + it, "int")
        x.copy_(torch.from_numpy(xi).bfloat16())
        w.copy_(torch.from_numpy(wi).bfloat16())
        y.zero_()
        graph.replay()
        torch.cuda.synchronize()
        ref = bf16_round(oracle.conv2d(xi, wi, shape.stride, shape.padding))
        assert np.array_equal(y.float().cpu().numpy(), ref), (kernel, it)


@pytest.mark.parametrize("kernel,shape", GRAPH_CASES, ids=lambda v: v if isinstance(v, str) else v.name)
def test_forward_while_other_work_holds_sms(kernel, shape):
    """A forward enqueued while a long chain of GEMMs on another stream holds the SMs: it
    either runs correctly or fails cleanly, and the context stays usable (no grid-wide barrier
    that needs the whole grid co-resident, no watchdog trap)."""
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    xi, wi = synth.make_inputs(shape, 37, "int")
    x = torch.from_numpy(xi).bfloat16().cuda()
    w = torch.from_numpy(wi).bfloat16().cuda()
    plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math="bf16", io_dtype="bf16", kernel=kernel)
    a = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16)
    other = torch.cuda.Stream()
    torch.cuda.synchronize()
    with torch.cuda.stream(other):
        for _ in range(30):
            a = (a @ a).clamp_(-1, 1)
    y = plan.forward(x, w)
    torch.cuda.synchronize()
    assert np.array_equal(y.float().cpu().numpy(), bf16_round(oracle.conv2d(xi, wi, shape.stride, shape.padding)))
    assert torch.isfinite(a).all()


# ---- f1: the FFT-domain solver (Eq. 13-15), FP32 -------------------------------------------
FFT_SHAPES = [synth.TINY, synth.CONV3X,
              ConvShape("fft_s2", 4, 32, 21, 19, 48, 3, 3, 2, 2, 1, 1),
              ConvShape("fft_5x5", 8, 64, 28, 28, 64, 5, 5, 1, 1, 2, 2),
              ConvShape("fft_7x7_nopad", 4, 16, 30, 26, 24, 7, 7, 1, 1, 0, 0),
              ConvShape("fft_1x1", 4, 64, 14, 14, 96, 1, 1),
              ConvShape("fft_rect", 3, 24, 9, 40, 40, 2, 4, 1, 1, 0, 1)] + \
             [s for s in synth.SWEEP if s.name in ("A_h14_s1", "A_h28_s1", "A_h56_s1", "B_r7_s1", "B_r5_s2")] + \
             [s for s in synth.RESNET50 if s.name in ("l3_3x3_256", "l4_3x3_512", "l4_3x3_512_s2")]


@pytest.mark.parametrize("shape", FFT_SHAPES, ids=lambda s: s.name)
@pytest.mark.parametrize("io", ["f32"])
def test_fft_solver(shape, io):
    """FFT of every A_{n,c}(t) and U_{k,c}(t), per-frequency channel sum, IFFT, Eq. 12
    extraction (math FP32_FMA: fp32 spectra, f32 I/O): within the FP32 gate of O1."""
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    dt = torch.bfloat16 if io == "bf16" else torch.float32
    gen = torch.Generator(device="cuda").manual_seed(51)
    x = (torch.rand((shape.N, shape.C, shape.H, shape.W), generator=gen, device="cuda") * 2 - 1).to(dt)
    w = ((torch.rand((shape.K, shape.C, shape.R, shape.S), generator=gen, device="cuda") * 2 - 1)
         / np.sqrt(shape.C * shape.R * shape.S)).to(dt)
    plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math="fp32", io_dtype=io, kernel="fft")
    y = plan.forward(x, w).float().cpu().numpy()
    images = sorted({0, shape.N - 1})
    ref = oracle.conv2d(x[images].float().cpu().numpy(), w.float().cpu().numpy(), shape.stride, shape.padding)
    gate = GATE["fp32"] if io == "f32" else 2 ** -8
    assert normwise(y[images], ref) <= gate


def test_fft_rejects_large_planes_and_tensor_math():
    import paper_conf_cgo_xuzc025_b200 as pc
    with pytest.raises(pc.PolyconvError):
        pc.Plan((1, 8, 100, 100), (8, 8, 3, 3), padding=(1, 1), math="fp32", kernel="fft")   # L > 8192
    with pytest.raises(pc.PolyconvError):
        pc.Plan((1, 8, 20, 20), (8, 8, 3, 3), padding=(1, 1), math="bf16", kernel="fft")
