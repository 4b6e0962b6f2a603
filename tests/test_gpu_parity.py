"""GPU parity: the CUDA path (through the C-ABI) against the fp64 oracle.

Element-by-element on seeded inputs (synth/), at sizes the oracle finishes in
seconds spanning several tiles and ragged tails, and at BASELINE sizes on
sampled images.  Gates: normwise 1e-5 (FP32_FMA), 2e-2 (TF32/BF16); packing,
extraction and integer-valued inputs bit-exact.
"""
import numpy as np
import pytest

import oracle
from oracle import poly_ref as pr
import synth
from synth import ConvShape
from helpers import GATE, normwise, bf16_round, gpu_forward

pytestmark = pytest.mark.gpu

MATH_KERNELS = [("fp32", "fp32"), ("fp32", "thin"), ("tf32", "tc"), ("bf16", "tc"), ("tf32", "tc_pertap"),
                ("bf16", "tc_pertap"), ("tf32", "tc_fused"), ("bf16", "tc_fused"), ("tf32", "thin"),
                ("bf16", "thin"), ("bf16", "tc_pair"), ("bf16", "tc_hankel"), ("tf32", "tc_hankel"), ("fp32", "fft")]

SHAPES = [
    ConvShape("tiny", 1, 1, 8, 8, 1, 3, 3),                      # BASELINE configs[0]
    ConvShape("ragged", 2, 20, 13, 11, 40, 3, 3, 1, 1, 1, 1),   # C, K, plane all ragged
    ConvShape("multi_tile", 3, 70, 17, 19, 80, 3, 3, 1, 1, 1, 1),
    ConvShape("stride2", 2, 32, 15, 14, 64, 3, 3, 2, 2, 1, 1),
    ConvShape("k5", 2, 16, 12, 12, 48, 5, 5, 1, 1, 2, 2),
    ConvShape("k1", 2, 64, 9, 9, 96, 1, 1, 1, 1, 0, 0),
    ConvShape("k1s2", 2, 48, 10, 10, 64, 1, 1, 2, 2, 0, 0),
    ConvShape("stem", 1, 3, 30, 30, 64, 7, 7, 2, 2, 3, 3),
    ConvShape("wideK", 1, 64, 10, 10, 320, 3, 3, 1, 1, 1, 1),   # 2 n-tiles, ragged last
    ConvShape("rect", 2, 24, 7, 16, 32, 2, 4, 1, 1, 0, 1),
    ConvShape("thinK", 2, 33, 9, 9, 8, 3, 3, 1, 1, 1, 1),
]


def _pair_supported(shape, io):
    """tc_pair takes a shape only with its separate packing grid (TMA views of x: H*W*elem
    a multiple of 16 bytes, K <= 128, an output row within 128 positions)."""
    import paper_conf_cgo_xuzc025_b200 as pc
    try:
        pc.Plan((shape.N, shape.C, shape.H, shape.W), (shape.K, shape.C, shape.R, shape.S), shape.stride,
                shape.padding, math="bf16", io_dtype=io, kernel="tc_pair")
        return True
    except pc.PolyconvError:
        return False


def _skip_unsupported(shape, math, kernel, io="f32"):
    if kernel == "fp32" and max(shape.R, shape.S) > 7:
        pytest.skip("fp32 kernel limited to S<=7")
    if kernel == "tc_pair" and not _pair_supported(shape, io):
        pytest.skip("tc_pair: no split packing grid for this shape")


@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: s.name)
@pytest.mark.parametrize("math,kernel", MATH_KERNELS, ids=lambda v: str(v))
def test_parity_uniform(shape, math, kernel):
    _skip_unsupported(shape, math, kernel)
    x, w = synth.make_inputs(shape, synth.seed_for(9, hash(shape.name) % 997), "uniform")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, plan = gpu_forward(shape, x, w, math=math, kernel=kernel)
    assert plan.info()["kernel"] == kernel
    assert y.shape == ref.shape
    err = normwise(y, ref)
    assert err <= GATE[math], f"normwise {err:.3e} > {GATE[math]} ({math}/{kernel})"


@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: s.name)
@pytest.mark.parametrize("math,kernel", MATH_KERNELS, ids=lambda v: str(v))
def test_integer_exact(shape, math, kernel):
    """|x|<=8, |w|<=4: every product and partial sum is an integer < 2^24, so
    every precision must reproduce the oracle bit for bit.  The FFT solver
    (f1) rounds in its transforms: not an exact method, checked by the normwise gates."""
    if kernel == "fft":
        pytest.skip("FFT solver: fp32 transforms round (normwise gate in test_parity_uniform)")
    _skip_unsupported(shape, math, kernel)
    x, w = synth.make_inputs(shape, synth.seed_for(8, hash(shape.name) % 997), "int")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, _ = gpu_forward(shape, x, w, math=math, kernel=kernel)
    assert np.array_equal(y, ref)


@pytest.mark.parametrize("shape", [SHAPES[1], SHAPES[3], SHAPES[7]], ids=lambda s: s.name)
def test_bf16_io(shape):
    """bf16 in/out (math BF16): integer data -> output equals round_bf16(oracle);
    uniform data within the 2e-2 gate against the fp32-input oracle."""
    x, w = synth.make_inputs(shape, 77, "int")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, _ = gpu_forward(shape, x, w, math="bf16", io="bf16")
    assert np.array_equal(y, bf16_round(ref))
    x, w = synth.make_inputs(shape, 78, "uniform")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, _ = gpu_forward(shape, x, w, math="bf16", io="bf16")
    assert normwise(y, ref) <= GATE["bf16"]


# bf16 in/out shapes with a TMA view of x (H*W*2 % 16 == 0): the fused tensor-core
# kernel takes its ring-staged 8x8-transpose packing mode on these
MX_SHAPES = [
    ConvShape("mx_a", 3, 64, 12, 12, 128, 3, 3, 1, 1, 1, 1),
    ConvShape("mx_partial", 2, 80, 16, 10, 96, 3, 3, 1, 1, 1, 1),   # second channel chunk partial
    ConvShape("mx_s2", 2, 48, 20, 20, 64, 3, 3, 2, 2, 1, 1),        # C < kc, stride 2
    ConvShape("mx_k5", 2, 32, 16, 16, 48, 5, 5, 1, 1, 2, 2),        # kc = 32 (64-byte swizzle)
    ConvShape("mx_k1", 2, 64, 8, 8, 64, 1, 1, 1, 1, 0, 0),
    ConvShape("mx_many", 9, 64, 8, 8, 128, 3, 3, 1, 1, 1, 1),       # windows span several images
    ConvShape("mx_asym", 2, 64, 14, 20, 72, 3, 5, 1, 1, 0, 2),
    # stride 2 with W % 4 == 0, C % 32 == 0: tc_hankel runs the phase-split convolution (R19)
    ConvShape("mx_s2_phase", 2, 64, 16, 20, 96, 3, 3, 2, 2, 1, 1),
    ConvShape("mx_s2_phase_k5", 2, 32, 20, 16, 48, 5, 5, 2, 2, 2, 2),
    ConvShape("mx_s2_phase_oddH", 3, 96, 15, 12, 64, 3, 3, 2, 2, 1, 1),
    ConvShape("mx_s2_phase_p0", 2, 64, 16, 16, 40, 3, 3, 2, 2, 0, 0),
    ConvShape("mx_s2_phase_w14", 3, 64, 14, 14, 96, 3, 3, 2, 2, 1, 1),   # W/2 odd: per-position decode
    ConvShape("mx_k1_wide", 2, 512, 14, 14, 128, 1, 1, 1, 1, 0, 0),  # AUTO: tc_hankel from 24 units
    ConvShape("mx_stem", 2, 3, 32, 32, 64, 7, 7, 2, 2, 3, 3),   # small-C phase mode, 32-byte rows
    ConvShape("mx_stem_c4", 2, 4, 20, 24, 40, 7, 7, 2, 2, 3, 3),
    ConvShape("mx_smallc", 3, 3, 20, 22, 64, 3, 3, 1, 1, 1, 1),     # stride 1, C <= 16: 32-byte rows
    ConvShape("mx_smallc16", 2, 16, 12, 16, 40, 3, 3, 1, 1, 1, 1),
]


@pytest.mark.parametrize("shape", MX_SHAPES, ids=lambda s: s.name)
@pytest.mark.parametrize("kernel", ["tc_fused", "tc", "tc_pair", "tc_hankel"])
def test_bf16_io_fused_packing(shape, kernel):
    """bf16 in/out, BF16 math: integer data bit-exact against round_bf16(O1);
    uniform data within the BF16 gate."""
    _skip_unsupported(shape, "bf16", kernel, "bf16")
    x, w = synth.make_inputs(shape, synth.seed_for(7, hash(shape.name) % 997), "int")
    y, plan = gpu_forward(shape, x, w, math="bf16", io="bf16", kernel=kernel)
    assert plan.info()["kernel"] == kernel
    assert np.array_equal(y, bf16_round(oracle.conv2d(x, w, shape.stride, shape.padding)))
    x, w = synth.make_inputs(shape, synth.seed_for(7, hash(shape.name) % 991), "uniform")
    y, _ = gpu_forward(shape, x, w, math="bf16", io="bf16", kernel=kernel)
    assert normwise(y, oracle.conv2d(x, w, shape.stride, shape.padding)) <= GATE["bf16"]


@pytest.mark.parametrize("kernel", ["tc_fused", "tc_pair", "tc_hankel"])
def test_conv3x_fused_bf16_io(kernel):
    """BASELINE configs[1] in full, bf16 in/out, the one-launch kernels."""
    shape = synth.CONV3X
    xi, wi = synth.make_inputs(shape, synth.seed_for(1), "int")
    y, plan = gpu_forward(shape, xi, wi, math="bf16", io="bf16", kernel=kernel)
    assert np.array_equal(y, bf16_round(oracle.conv2d(xi, wi, shape.stride, shape.padding)))


@pytest.mark.parametrize("math,kernel", [("fp32", "fp32"), ("bf16", "tc"), ("tf32", "tc"), ("fp32", "thin"),
                                         ("bf16", "tc_pertap"), ("bf16", "tc_fused"),
                                         ("bf16", "tc_pair"), ("bf16", "tc_hankel"), ("tf32", "tc_hankel")])
def test_delta_filter_bit_exact(math, kernel):
    """w[k][c][i][j] = [c == k mod C][i == i0][j == j0] -> y = shifted xpad,
    bit-exact for every tap (checks each shift e(i,j) and the padding)."""
    import torch
    shape = ConvShape("delta", 2, 16, 9, 10, 32, 3, 3, 1, 1, 1, 1)
    _skip_unsupported(shape, math, kernel)
    x, _ = synth.make_inputs(shape, 5, "uniform")
    x = bf16_round(x)  # representable in every operand format
    xp = np.pad(x, ((0, 0), (0, 0), (1, 1), (1, 1)))
    for i0 in range(3):
        for j0 in range(3):
            w = np.zeros((32, 16, 3, 3), np.float32)
            for k in range(32):
                w[k, k % 16, i0, j0] = 1.0
            y, _ = gpu_forward(shape, x, w, math=math, kernel=kernel)
            want = xp[:, [k % 16 for k in range(32)], i0:i0 + 9, j0:j0 + 10]
            assert np.array_equal(y, want), (i0, j0)


@pytest.mark.parametrize("math", ["fp32", "tf32", "bf16"])
def test_conv3x_full(math):
    """BASELINE configs[1] (ResNet-50 conv3_x, N=32) in full against O1."""
    shape = synth.CONV3X
    x, w = synth.make_inputs(shape, synth.seed_for(1), "uniform")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, plan = gpu_forward(shape, x, w, math=math)
    assert normwise(y, ref) <= GATE[math]


def test_conv3x_bench_launch_config():
    """The exact launch the bench times (conv3_x, bf16 in/out, math BF16, AUTO)."""
    shape = synth.CONV3X
    x, w = synth.make_inputs(shape, synth.seed_for(1), "uniform")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, plan = gpu_forward(shape, x, w, math="bf16", io="bf16")
    assert plan.info()["kernel"] == "tc_hankel"  # bf16: the persistent pair kernel fed from NCHW x
    assert normwise(y, ref) <= GATE["bf16"]
    xi, wi = synth.make_inputs(shape, synth.seed_for(1), "int")
    y, _ = gpu_forward(shape, xi, wi, math="bf16", io="bf16", plan=plan)
    assert np.array_equal(y, bf16_round(oracle.conv2d(xi, wi, shape.stride, shape.padding)))


# --------------------------------------------------------------- single steps --

PACK_SHAPES = [ConvShape("p1", 2, 5, 7, 6, 9, 3, 2, 1, 1, 1, 2), ConvShape("p2", 1, 70, 5, 5, 33, 3, 3, 1, 1, 1, 1),
               ConvShape("p3", 3, 3, 11, 4, 64, 5, 5, 2, 2, 2, 2),
               # H*W*elem a multiple of 16 bytes: the TMA band pack path
               ConvShape("p4", 2, 70, 8, 12, 16, 3, 3, 1, 1, 1, 1), ConvShape("p5", 3, 130, 16, 16, 8, 3, 3, 1, 1, 2, 1)]


@pytest.mark.parametrize("shape", PACK_SHAPES, ids=lambda s: s.name)
@pytest.mark.parametrize("math", ["fp32", "tf32", "bf16"])
def test_pack_bit_exact(shape, math):
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    x, w = synth.make_inputs(shape, 4, "uniform")
    xt, wt = torch.from_numpy(x).cuda(), torch.from_numpy(w).cuda()
    plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math=math)
    inf = plan.info()
    wdt = np.uint16 if math == "bf16" else np.uint32
    # planar input A_{n,c}(t) (Eq. 10)
    got = plan.pack_input(xt, "planar").cpu().numpy().view(wdt)
    want = pr.pack_input_planar(x, shape.padding, math)
    assert np.array_equal(got, want.reshape(-1))
    # interleaved input [N*L_A][Cp]: the same words, channels innermost, zero channel padding
    got = plan.pack_input(xt, "interleaved").cpu().numpy().view(wdt).reshape(shape.N * inf["L_A"], inf["Cp"])
    wi = np.zeros((shape.N, inf["L_A"], inf["Cp"]), wdt)
    wi[:, :, :shape.C] = want.transpose(0, 2, 1)
    assert np.array_equal(got, wi.reshape(-1, inf["Cp"]))
    # planar filter U_{k,c}(t) (Eq. 6/11, reading R1)
    got = plan.pack_filter(wt, "planar").cpu().numpy().view(wdt)
    wantu = pr.pack_filter_planar(w, inf["Wp"], math)
    assert np.array_equal(got, wantu.reshape(-1))
    # tap-major filter [R*S][Kp][Cp]: the nonzero coefficients of U by degree e(i,j)
    got = plan.pack_filter(wt, "interleaved").cpu().numpy().view(wdt).reshape(shape.R * shape.S, inf["Kp"], inf["Cp"])
    tm = np.zeros_like(got)
    for i in range(shape.R):
        for j in range(shape.S):
            e = pr.kernel_degree(i, j, shape.R, shape.S, inf["Wp"])
            tm[i * shape.S + j, :shape.K, :shape.C] = wantu[:, :, e]
    assert np.array_equal(got, tm)


@pytest.mark.parametrize("shape", PACK_SHAPES + [synth.TINY], ids=lambda s: s.name)
def test_extract_bit_exact(shape):
    """a5 alone: (1) index-valued coefficients -> y holds exactly the Eq. 12
    degrees; (2) the oracle's full product (np.convolve) -> y == O1."""
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    plan = pc.Plan((shape.N, shape.C, shape.H, shape.W), (shape.K, shape.C, shape.R, shape.S), shape.stride,
                   shape.padding, math="fp32")
    inf = plan.info()
    Lp = inf["L_A"] + inf["L_U"] - 1
    idx = np.arange(shape.N * shape.K * Lp, dtype=np.float32).reshape(shape.N, shape.K, Lp)  # exact < 2^24
    y = plan.extract(torch.from_numpy(idx).cuda()).cpu().numpy()
    for n in range(shape.N):
        for k in range(shape.K):
            deg = np.array([[pr.extraction_degree(oh, ow, shape.R, shape.S, inf["Wp"], shape.sh, shape.sw)
                             for ow in range(inf["Q"])] for oh in range(inf["P"])])
            assert np.array_equal(y[n, k], idx[n, k][deg])
    if shape.sh == 1 and shape.sw == 1:
        x, w = synth.make_inputs(shape, 6, "int")
        fp = pr.full_product(x, w, shape.padding).astype(np.float32)
        y = plan.extract(torch.from_numpy(fp).cuda()).cpu().numpy()
        assert np.array_equal(y, oracle.conv2d(x, w, shape.stride, shape.padding))


# ------------------------------------------------------- larger / sampled sizes --

def _sampled(shape, math, io="f32", images=None, seed=0):
    """Full-size launch; compare images {0, N-1} against O1 on those images."""
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    N = shape.N
    images = images or sorted({0, N - 1})
    dt = torch.bfloat16 if io == "bf16" else torch.float32
    gen = torch.Generator(device="cuda").manual_seed(seed)
    x = (torch.rand((N, shape.C, shape.H, shape.W), generator=gen, device="cuda") * 2 - 1)
    w = (torch.rand((shape.K, shape.C, shape.R, shape.S), generator=gen, device="cuda") * 2 - 1) / np.sqrt(
        shape.C * shape.R * shape.S)
    x, w = x.to(dt), w.to(dt)
    plan = pc.Plan(x.shape, w.shape, shape.stride, shape.padding, math=math, io_dtype=io)
    y = plan.forward(x, w)
    torch.cuda.synchronize()
    xs = x[images].float().cpu().numpy()
    ref = oracle.conv2d(xs, w.float().cpu().numpy(), shape.stride, shape.padding)
    return normwise(y[images].float().cpu().numpy(), ref), plan


@pytest.mark.parametrize("shape", [s for s in synth.RESNET50], ids=lambda s: s.name)
def test_resnet50_sampled_bf16(shape):
    err, plan = _sampled(shape, "bf16", io="bf16", seed=11)
    assert err <= GATE["bf16"]


@pytest.mark.parametrize("shape", [synth.VGG16[i] for i in (0, 1, 4, 8, 12)], ids=lambda s: s.name)
@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
def test_vgg16_sampled(shape, math):
    err, plan = _sampled(shape, math, seed=12)
    assert err <= GATE[math]


@pytest.mark.parametrize("shape", [s for s in synth.SWEEP if s.flops() < 4e11][::3], ids=lambda s: s.name)
def test_sweep_sampled_bf16(shape):
    err, plan = _sampled(shape, "bf16", seed=13)
    assert err <= GATE["bf16"]


def test_batch_shard_bit_identical():
    """Per-image results do not depend on the batch they are computed in
    (reading R12): forward(x[a:b]) == forward(x)[a:b] bit for bit -- the basis
    of the batch-sharded multi-GPU path."""
    shape = ConvShape("shard", 8, 64, 14, 14, 128, 3, 3, 1, 1, 1, 1)
    x, w = synth.make_inputs(shape, 21, "uniform")
    for math in ("bf16", "tf32", "fp32"):
        y_all, _ = gpu_forward(shape, x, w, math=math)
        for a, b in [(0, 2), (2, 5), (5, 8)]:
            ys, _ = gpu_forward(shape.with_batch(b - a), x[a:b], w, math=math)
            assert np.array_equal(ys, y_all[a:b]), (math, a, b)


def test_errors_on_device():
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    plan = pc.Plan((1, 4, 8, 8), (8, 4, 3, 3), math="bf16")
    x = torch.zeros(1 * 4 * 8 * 8 + 1, device="cuda")
    w = torch.zeros((8, 4, 3, 3), device="cuda")
    y = torch.zeros((1, 8, 6, 6), device="cuda")
    with pytest.raises(pc.PolyconvError) as e:
        plan.forward_ptr(x.data_ptr() + 4, w.data_ptr(), y.data_ptr())   # misaligned x
    assert e.value.status == pc.NOT_SUPPORTED
    with pytest.raises(pc.PolyconvError) as e:
        plan.forward_ptr(x.data_ptr(), w.data_ptr(), x.data_ptr())       # y aliases x
    assert e.value.status == pc.BAD_PARAM


def test_pair_repeated_launches_one_plan():
    """tc_pair keeps per-plan state across launches (grid counter epochs, band flags,
    cached tensor maps): consecutive forwards on one plan with new inputs and new
    output buffers must each match the oracle bit for bit (integer data)."""
    import torch
    shape = ConvShape("pair_rep", 3, 64, 16, 16, 64, 3, 3, 1, 1, 1, 1)
    plan = None
    for it in range(4):
        x, w = synth.make_inputs(shape, synth.seed_for(11, it), "int")
        ref = bf16_round(oracle.conv2d(x, w, shape.stride, shape.padding))
        y, plan = gpu_forward(shape, x, w, math="bf16", io="bf16", kernel="tc_pair", plan=plan)
        assert plan.info()["kernel"] == "tc_pair"
        assert np.array_equal(y, ref), it


@pytest.mark.parametrize("shape", [ConvShape("pair_rows1", 2, 64, 9, 100, 64, 3, 3, 1, 1, 1, 1),   # tr = 1
                                   ConvShape("pair_s2", 3, 64, 29, 29, 64, 3, 3, 2, 2, 1, 1),       # stride 2, odd P
                                   ConvShape("pair_c192", 2, 192, 10, 10, 48, 3, 3, 1, 1, 1, 1),    # 3 chunks, K % 64
                                   ConvShape("pair_k1", 4, 128, 14, 14, 128, 1, 1, 1, 1, 0, 0)],
                         ids=lambda s: s.name)
@pytest.mark.parametrize("io", ["bf16", "f32"])
def test_pair_shapes(shape, io):
    """tc_pair tilings off the bench shape: one output row per tile, stride 2 with a
    ragged last row block, three channel chunks with K not a multiple of 64, 1x1."""
    _skip_unsupported(shape, "bf16", "tc_pair", io)
    x, w = synth.make_inputs(shape, synth.seed_for(12, hash(shape.name) % 997), "int")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, plan = gpu_forward(shape, x, w, math="bf16", io=io, kernel="tc_pair")
    assert plan.info()["kernel"] == "tc_pair"
    assert np.array_equal(y, bf16_round(ref) if io == "bf16" else ref)


@pytest.mark.parametrize("shape", [ConvShape("pp_3x3s2", 2, 32, 15, 14, 64, 3, 3, 2, 2, 1, 1),
                                   ConvShape("pp_5x5s2", 2, 16, 17, 17, 48, 5, 5, 2, 2, 2, 2),
                                   ConvShape("pp_7x7s2_c3", 2, 3, 30, 30, 64, 7, 7, 2, 2, 3, 3),
                                   ConvShape("pp_3x3s3", 1, 8, 16, 16, 16, 3, 3, 3, 3, 1, 1),
                                   ConvShape("pp_4x2s2", 2, 8, 11, 9, 16, 4, 2, 2, 2, 1, 0)],
                         ids=lambda s: s.name)
@pytest.mark.parametrize("math,io", [("bf16", "bf16"), ("fp32", "f32"), ("tf32", "f32")])
def test_polyphase_stride(shape, math, io, monkeypatch):
    """Stride s as a stride-1 convolution of the s*s input phases (reading R4b), forced on
    for every kernel size: integer data bit-exact against the oracle."""
    monkeypatch.setenv("POLYCONV_POLYPHASE", "1")
    x, w = synth.make_inputs(shape, synth.seed_for(13, hash(shape.name) % 997), "int")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, plan = gpu_forward(shape, x, w, math=math, io=io)
    assert plan.info()["launches"] >= 3  # phase split + the inner plan's launches
    assert np.array_equal(y, bf16_round(ref) if io == "bf16" else ref)


@pytest.mark.parametrize("shape", [ConvShape("k1_a", 2, 64, 8, 8, 96, 1, 1),          # one partial block
                                   ConvShape("k1_b", 3, 130, 16, 16, 200, 1, 1),      # 3 chunks, 2 k-tiles
                                   ConvShape("k1_c", 2, 48, 28, 28, 64, 1, 1),        # ragged last block, C < 64
                                   ConvShape("k1_d", 1, 256, 56, 56, 64, 1, 1)],      # 13 blocks
                         ids=lambda s: s.name)
@pytest.mark.parametrize("epi", ["auto", "direct"])
def test_1x1_planes_as_operand(shape, epi, monkeypatch):
    """1x1 stride-1 layers read the NCHW planes directly as the MN-major operand (mac_1x1):
    integer data bit-exact against round_bf16(oracle); AUTO picks it for bf16 in/out.
    epi: the staged bulk/TMA-stored epilogue (auto) or per-thread stores (direct)."""
    if epi == "direct":
        monkeypatch.setenv("POLYCONV_1X1_EPI_TMA", "0")
    x, w = synth.make_inputs(shape, synth.seed_for(14, hash(shape.name) % 997), "int")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, plan = gpu_forward(shape, x, w, math="bf16", io="bf16")
    assert plan.info()["kernel"] == "tc_1x1"
    assert np.array_equal(y, bf16_round(ref))
    x, w = synth.make_inputs(shape, synth.seed_for(15, hash(shape.name) % 997), "uniform")
    y, _ = gpu_forward(shape, x, w, math="bf16", io="bf16", plan=plan)
    assert normwise(y, oracle.conv2d(x, w, shape.stride, shape.padding)) <= GATE["bf16"]


@pytest.mark.parametrize("shape", [ConvShape("k1g_6x6", 3, 96, 6, 6, 130, 1, 1),              # 36 px: gathered
                                   ConvShape("k1g_14", 2, 72, 14, 14, 64, 1, 1),              # 196 px
                                   ConvShape("k1g_s2", 2, 64, 28, 28, 128, 1, 1, 2, 2, 0, 0),  # stride 2
                                   ConvShape("k1g_s2_odd", 2, 32, 15, 13, 48, 1, 1, 2, 2, 0, 0),
                                   ConvShape("k1g_7", 2, 64, 7, 7, 96, 1, 1),                  # 49 px, odd
                                   ConvShape("k1g_7_k40", 2, 32, 7, 7, 40, 1, 1),              # K % 32 != 0
                                   ConvShape("k1g_s2_14", 3, 64, 14, 14, 64, 1, 1, 2, 2, 0, 0),  # 7x7 out
                                   ConvShape("k1g_10x9", 2, 130, 10, 9, 160, 1, 1),            # 90 px, 3 chunks
                                   ConvShape("k1g_rows", 80, 1024, 7, 7, 32, 1, 1),            # many planes, odd size
                                   ConvShape("k1g_5x5_tail", 1, 3, 5, 5, 16, 1, 1),            # x ends mid-vector
                                   ConvShape("k1g_7_n7", 7, 64, 7, 7, 64, 1, 1),               # 4-image tiles, ragged group
                                   ConvShape("k1g_5x5_c8", 5, 8, 5, 5, 32, 1, 1),              # 4-image tiles, C < 64, 25 px
                                   ConvShape("k1g_s2_8x8", 6, 64, 16, 16, 160, 1, 1, 2, 2, 0, 0),  # 4-image, 2 k-tiles
                                   ConvShape("k1g_s2_56", 2, 64, 56, 56, 96, 1, 1, 2, 2, 0, 0),  # s2, 16-byte groups
                                   ConvShape("k1g_s2_24", 3, 40, 24, 20, 64, 1, 1, 2, 2, 0, 0),  # s2, Q = 10: 8-byte
                                   ConvShape("k1g_big", 1, 2, 160, 160, 32, 1, 1, 2, 2, 0, 0)],  # plane past the stage
                         ids=lambda s: s.name)
def test_1x1_gathered(shape):
    """1x1 layers whose planes cannot be read in place (stride > 1, or a plane size that is
    not a multiple of 8 pixels): the output-lattice pixels are gathered first, then the same
    MN-major GEMM; bit-exact on integer data."""
    x, w = synth.make_inputs(shape, synth.seed_for(16, hash(shape.name) % 997), "int")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    y, plan = gpu_forward(shape, x, w, math="bf16", io="bf16", kernel="tc_1x1")
    assert plan.info()["kernel"] == "tc_1x1" and plan.info()["launches"] == 3
    assert np.array_equal(y, bf16_round(ref))


@pytest.mark.parametrize("shape,math,io", [
    (ConvShape("host_pair", 7, 64, 28, 28, 64, 3, 3, 1, 1, 1, 1), "bf16", "bf16"),   # 4 chunks, tail of 1
    (ConvShape("host_1x1", 6, 64, 16, 16, 128, 1, 1), "bf16", "bf16"),              # 3 chunks of 2
    (ConvShape("host_fp32", 5, 16, 12, 12, 32, 3, 3, 1, 1, 1, 1), "fp32", "f32"),  # 3 chunks, tail 1
    (ConvShape("host_s2", 4, 16, 15, 15, 32, 7, 7, 2, 2, 3, 3), "bf16", "bf16"),    # polyphase: one piece
    (ConvShape("host_n18", 18, 32, 12, 12, 64, 3, 3, 1, 1, 1, 1), "bf16", "bf16")],  # chunks 5,5,5,3
    ids=lambda v: v.name if isinstance(v, ConvShape) else str(v))
@pytest.mark.parametrize("chunks", ["default", "1"])
def test_forward_host_pipeline(shape, math, io, chunks, monkeypatch):
    """polyconv_forward_host (pinned host buffers): the chunked copy/compute pipeline gives the
    bytes of a device forward of the whole batch (same kernel per chunk), repeated calls too,
    and integer data equals round(oracle)."""
    import torch
    import paper_conf_cgo_xuzc025_b200 as pc
    if chunks != "default":
        monkeypatch.setenv("POLYCONV_HOST_CHUNKS", chunks)
    x, w = synth.make_inputs(shape, synth.seed_for(17, hash(shape.name) % 997), "int")
    dt = torch.bfloat16 if io == "bf16" else torch.float32
    xh = torch.from_numpy(x).to(dt).contiguous().pin_memory()
    wh = torch.from_numpy(w).to(dt).contiguous().pin_memory()
    plan = pc.Plan(xh.shape, wh.shape, shape.stride, shape.padding, math=math, io_dtype=io)
    yh = torch.empty(plan.output_shape, dtype=dt).pin_memory()
    for _ in range(3):
        yh.zero_()
        plan.forward_host(xh, wh, yh)
        torch.cuda.synchronize()
        yd = plan.forward(xh.cuda(), wh.cuda())
        torch.cuda.synchronize()
        assert torch.equal(yh, yd.cpu())
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    assert np.array_equal(yh.float().numpy(), bf16_round(ref) if io == "bf16" else ref)
