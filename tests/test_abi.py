"""CPU-side checks of the C-ABI library: it loads without a GPU, exports every
symbol include/polyconv.h declares, and its host logic (argument validation,
a1 size math, kernel selection, status strings) behaves as documented."""
import ctypes
import os
import re

import pytest

import paper_conf_cgo_xuzc025_b200 as pc
import oracle
from oracle import poly_ref as pr

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "polyconv.h")).read()
    declared = set(re.findall(r"\b(polyconv_\w+)\s*\(", hdr))
    assert declared == set(pc.EXPORTS)
    lib = pc.load_library()
    for name in declared:
        assert hasattr(lib, name), name
    assert lib.polyconv_abi_version() == 1


def test_exports_only_the_c_abi():
    """The shared library exports the polyconv_* C-ABI and nothing else: the static CUDA runtime
    and the internal C++ symbols stay local (version script + --exclude-libs)."""
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", pc.LIB_PATH], capture_output=True, text=True).stdout
    names = [l.split()[-1] for l in out.splitlines() if l.strip()]
    assert names and all(n.startswith("polyconv_") for n in names), [n for n in names if not n.startswith("polyconv_")]
    assert "cudaMemcpyAsync" not in names


def test_status_strings():
    for s in range(5):
        assert pc.status_string(s).startswith("POLYCONV_STATUS_")


@pytest.mark.parametrize("args", [
    (0, 1, 8, 8, 1, 3, 3, 1, 1, 0, 0), (1, 1, 8, 8, 1, 3, 3, 0, 1, 0, 0), (1, 1, 8, 8, 1, 3, 3, 1, 1, -1, 0),
    (1, 1, 2, 2, 1, 3, 3, 1, 1, 0, 0), (1, 0, 8, 8, 1, 3, 3, 1, 1, 0, 0), (1, 1, 8, 8, 0, 3, 3, 1, 1, 0, 0)])
def test_plan_rejects_bad_params(args):
    lib = pc.load_library()
    h = ctypes.c_void_p()
    st = lib.polyconv_plan(ctypes.byref(h), *args, 0, 2, 0)
    assert st == pc.BAD_PARAM and not h.value


def test_plan_rejects_bad_combos():
    lib = pc.load_library()
    h = ctypes.c_void_p()
    assert lib.polyconv_plan(ctypes.byref(h), 1, 1, 8, 8, 1, 3, 3, 1, 1, 0, 0, 1, 0, 0) == pc.BAD_PARAM  # bf16 io, fp32 math
    assert lib.polyconv_plan(ctypes.byref(h), 1, 1, 8, 8, 1, 3, 3, 1, 1, 0, 0, 0, 7, 0) == pc.BAD_PARAM  # bad math
    assert lib.polyconv_plan(None, 1, 1, 8, 8, 1, 3, 3, 1, 1, 0, 0, 0, 0, 0) == pc.BAD_PARAM
    # > 2^31 elements
    assert lib.polyconv_plan(ctypes.byref(h), 4096, 512, 224, 224, 64, 3, 3, 1, 1, 1, 1, 0, 2, 0) == pc.NOT_SUPPORTED


@pytest.mark.parametrize("H,W,R,S,s,p", [(8, 8, 3, 3, 1, 0), (28, 28, 3, 3, 1, 1), (224, 224, 7, 7, 2, 3),
                                         (7, 11, 2, 5, 3, 2), (56, 56, 1, 1, 2, 0)])
def test_plan_sizes_match_oracle(H, W, R, S, s, p):
    plan = pc.Plan((2, 8, H, W), (16, 8, R, S), (s, s), (p, p), math="bf16")
    inf = plan.info()
    assert (inf["P"], inf["Q"]) == oracle.output_dims(H, W, R, S, (s, s), (p, p))
    z = pr.sizes(H, W, R, S, s, s, p, p)
    assert (inf["Hp"], inf["Wp"], inf["L_A"], inf["L_U"]) == (z["Hp"], z["Wp"], z["L_A"], z["L_U"])


def test_kernel_selection_and_forcing():
    # bf16 3x3 / 5x5, stride <= 2, even width, C % 8 == 0, >= 24 pair units: mac_hankel
    assert pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="bf16").info()["kernel"] == "tc_hankel"
    # under 24 pair units (10x10, N=1): the single-CTA tensor-core kernel
    assert pc.Plan((1, 64, 10, 10), (320, 64, 3, 3), padding=(1, 1), math="bf16").info()["kernel"] == "tc"
    with pytest.raises(pc.PolyconvError):
        pc.Plan((1, 64, 10, 10), (320, 64, 3, 3), padding=(1, 1), math="bf16", kernel="tc_pair")
    with pytest.raises(pc.PolyconvError):
        pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="tf32", kernel="tc_pair")
    with pytest.raises(pc.PolyconvError):
        pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="fp32", kernel="tc_hankel")
    assert pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="tf32").info()["kernel"] == "tc_hankel"
    assert pc.Plan((1, 64, 10, 10), (320, 64, 3, 3), padding=(1, 1), math="tf32").info()["kernel"] == "tc"
    assert pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="tf32",
                   kernel="tc_hankel").info()["kernel"] == "tc_hankel"
    assert pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="fp32").info()["kernel"] == "fp32"
    assert pc.Plan((1, 1, 8, 8), (1, 1, 3, 3), math="fp32").info()["kernel"] == "thin"
    assert pc.Plan((1, 1, 8, 8), (1, 1, 3, 3), math="bf16").info()["kernel"] == "thin"
    with pytest.raises(pc.PolyconvError):
        pc.Plan((1, 4, 8, 8), (16, 4, 3, 3), math="fp32", kernel="tc")
    with pytest.raises(pc.PolyconvError):
        pc.Plan((1, 4, 8, 8), (16, 4, 3, 3), math="bf16", kernel="fp32")
    p = pc.Plan((1, 4, 8, 8), (16, 4, 3, 3), math="bf16", kernel="thin")
    assert p.info()["kernel"] == "thin"
    # 1x1 (bf16 in/out): in place on 56x56, gathered on 14x14 / strided, mac_tc2 for an
    # expansion layer on 7x7 planes (mac1x1_auto)
    k1 = lambda xs, ws, s=1: pc.Plan(xs, ws, (s, s), math="bf16", io_dtype="bf16").info()
    assert (k1((4, 64, 56, 56), (256, 64, 1, 1))["kernel"], k1((4, 64, 56, 56), (256, 64, 1, 1))["launches"]) == \
        ("tc_1x1", 2)
    assert (k1((4, 1024, 14, 14), (256, 1024, 1, 1))["kernel"], k1((4, 1024, 14, 14), (256, 1024, 1, 1))["launches"]) \
        == ("tc_1x1", 3)
    # ... but wide-input 1x1 layers on planes that need the gather go to mac_hankel from 24
    # pair units (C >= 512, C >= 2K), reading x in place
    assert k1((256, 1024, 14, 14), (256, 1024, 1, 1))["kernel"] == "tc_hankel"
    assert k1((256, 256, 14, 14), (1024, 256, 1, 1))["kernel"] == "tc_1x1"
    assert k1((4, 256, 28, 28), (512, 256, 1, 1), 2)["kernel"] == "tc_1x1"
    assert k1((4, 1024, 7, 7), (512, 1024, 1, 1))["kernel"] == "tc_1x1"
    # planes of <= 64 pixels with K % 32 == 0: four images per mac_1x1 tile, expansions included
    # (ResNet-50 512->2048 7x7 N=256: 63.6 us vs 80.9 for mac_tc2, profiles/r03_1x1_gimg.log)
    assert k1((4, 512, 7, 7), (2048, 512, 1, 1))["kernel"] == "tc_1x1"
    assert k1((1, 512, 7, 7), (2048, 512, 1, 1))["kernel"] == "tc"     # one image: the old rule
    assert k1((4, 512, 7, 7), (2040, 512, 1, 1))["kernel"] == "tc"     # K % 32 != 0
    # bf16 in/out (profiles/r02_kcmp_*.jsonl): mac_hankel for 3x3 / 5x5 from 24 pair
    # units, stride 1 or 2; odd plane widths, 7x7 kernels and sub-round problems keep the
    # earlier rules (pack + mac_tc2 below one round of pair tiles, in-kernel packing for 3x3
    # on narrow planes, a pack launch for 7x7)
    k3 = lambda xs, ws, s=1: pc.Plan(xs, ws, (s, s), (ws[2] // 2, ws[3] // 2), math="bf16",
                                     io_dtype="bf16").info()["kernel"]
    assert k3((32, 128, 28, 28), (128, 128, 3, 3)) == "tc_hankel"
    assert k3((256, 512, 7, 7), (512, 512, 3, 3)) == "tc_hankel"     # odd width, wide layer
    assert k3((256, 128, 7, 7), (128, 128, 3, 3)) == "tc"            # odd width, narrow
    assert k3((256, 128, 56, 56), (128, 128, 3, 3), 2) == "tc_hankel"
    assert k3((32, 64, 8, 8), (64, 64, 3, 3)) == "tc"                # 12 units < 24
    assert k3((32, 128, 14, 14), (64, 128, 3, 3)) == "tc_hankel"
    assert k3((32, 64, 56, 56), (64, 64, 3, 3)) == "tc_hankel"
    assert k3((32, 64, 56, 56), (128, 64, 5, 5)) == "tc_hankel"
    assert k3((32, 64, 56, 56), (128, 64, 7, 7)) == "tc"
    # f32 I/O, bf16 math: the same rule
    assert pc.Plan((32, 64, 8, 8), (64, 64, 3, 3), (1, 1), (1, 1), math="bf16").info()["kernel"] == "tc_pair"
    assert pc.Plan((32, 64, 28, 28), (64, 64, 3, 3), (1, 1), (1, 1), math="bf16").info()["kernel"] == "tc_hankel"


def test_fft_solver_planning():
    """f1: the FFT length is the power of two >= L_A + L_U - 1 (Eq. 14, reading Z9); FP32 math
    only; AUTO takes it for FP32 layers where the measured cost model favours it (fft_pays)."""
    inf = pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="fp32", kernel="fft").info()
    assert inf["kernel"] == "fft" and inf["tile_m"] == 1024 and inf["launches"] == 4   # 900 + 63 - 1 -> 1024
    inf = pc.Plan((2, 8, 7, 7), (8, 8, 3, 3), padding=(1, 1), math="fp32", kernel="fft").info()
    assert inf["tile_m"] == 128                                                          # 81 + 21 - 1 -> 128
    with pytest.raises(pc.PolyconvError):
        pc.Plan((1, 8, 100, 100), (8, 8, 3, 3), padding=(1, 1), math="fp32", kernel="fft")   # L > 8192
    with pytest.raises(pc.PolyconvError):
        pc.Plan((1, 8, 20, 20), (8, 8, 3, 3), padding=(1, 1), math="tf32", kernel="fft")
    auto = lambda xs, ws, s=1: pc.Plan(xs, ws, (s, s), (ws[2] // 2, ws[3] // 2), math="fp32").info()["kernel"]
    # FFT / FFMA TFLOP/s, profiles/r03_fp32_cmp.jsonl
    assert auto((256, 512, 7, 7), (512, 512, 3, 3)) == "fft"      # ResNet-50 l4 3x3 (L = 128): 40 vs 31
    assert auto((256, 256, 28, 28), (256, 256, 3, 3), 2) == "fft"  # l3 3x3 s2 (L = 1024): 12.8 vs 9.7
    assert auto((64, 512, 28, 28), (512, 512, 3, 3)) == "fft"     # VGG-16 conv4_2 (C*K = 256K): 56 vs 38
    assert auto((256, 128, 28, 28), (128, 128, 3, 3)) == "fp32"   # l2 3x3: 31 vs 38
    assert auto((256, 256, 14, 14), (256, 256, 3, 3)) == "fp32"   # l3 3x3 (L = 512): 29 vs 34
    assert auto((256, 64, 56, 56), (64, 64, 3, 3)) == "fp32"      # l1 3x3 (L = 4096): 12 vs 38
    assert auto((32, 128, 28, 28), (128, 128, 3, 3)) == "fp32"    # conv3_x at N=32: 20 vs 32
    assert auto((256, 2048, 7, 7), (512, 2048, 1, 1)) == "fp32"   # l4 1x1 2048->512: 9.4 vs 18.3


def test_tc_tiling_choices():
    # default TC: tile = nt positions x 128 output channels; conv3_x (G = 31*900 + 838
    # positions) -> nt = 208 gives 139 tiles, one wave on 148 SMs
    inf = pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="bf16", kernel="tc").info()
    assert (inf["tile_m"], inf["tile_n"], inf["Cp"], inf["Kp"]) == (208, 128, 128, 128)
    inf = pc.Plan((2, 3, 30, 30), (64, 3, 7, 7), (2, 2), (3, 3), math="bf16", kernel="tc").info()
    assert inf["Cp"] == 16 and inf["Kp"] == 128           # C=3 -> one 32-byte swizzle row
    inf = pc.Plan((2, 3, 30, 30), (64, 3, 7, 7), (2, 2), (3, 3), math="tf32").info()
    assert inf["Cp"] == 8
    inf = pc.Plan((1, 64, 10, 10), (320, 64, 3, 3), (1, 1), (1, 1), math="bf16").info()
    assert inf["tile_n"] == 128 and inf["Kp"] == 384
    # TC_PAIR (bf16 default): pair tile = 256 positions x NN output channels (NN = K
    # rounded up to 64), channels in chunks of 64/32/16; one launch
    inf = pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="bf16", kernel="tc_pair").info()
    assert (inf["tile_m"], inf["tile_n"], inf["Cp"], inf["Kp"], inf["launches"]) == (256, 128, 128, 128, 2)
    # TC_HANKEL: pair item = 256*T positions x NN output channels; NN = K (<= 256) else 256,
    # T*NN <= 256 (two TMEM accumulators), NN = 256 streamed: T = 2 in one accumulator;
    # channels in chunks of 64 (bf16) / 32 (tf32); filter pack + one launch
    hk = lambda xs, ws, m="bf16": pc.Plan(xs, ws, (1, 1), (1, 1), math=m, kernel="tc_hankel").info()
    inf = hk((256, 64, 56, 56), (64, 64, 3, 3))
    assert (inf["tile_m"], inf["tile_n"], inf["Cp"], inf["Kp"], inf["launches"]) == (1024, 64, 64, 64, 2)
    inf = hk((256, 256, 14, 14), (256, 256, 3, 3))
    assert (inf["tile_m"], inf["tile_n"], inf["Kp"]) == (512, 256, 256)
    inf = hk((256, 512, 7, 7), (512, 512, 3, 3))
    assert (inf["tile_m"], inf["tile_n"], inf["Kp"]) == (512, 256, 512)
    inf = hk((2, 40, 9, 9), (72, 40, 3, 3), "tf32")
    assert (inf["tile_n"], inf["Cp"], inf["Kp"]) == (80, 64, 80)
    # TC_PAIR needs its separate packing grid (TMA views of x: H*W*elem % 16 == 0); the
    # one-launch mode with a grid barrier is gone, so other shapes are not supported
    with pytest.raises(pc.PolyconvError):
        pc.Plan((2, 3, 30, 30), (64, 3, 7, 7), (2, 2), (3, 3), math="bf16", io_dtype="bf16", kernel="tc_pair")
    inf = pc.Plan((2, 40, 8, 8), (72, 40, 3, 3), (1, 1), (1, 1), math="bf16", kernel="tc_pair").info()
    assert (inf["kernel"], inf["Cp"], inf["Kp"], inf["launches"]) == ("tc_pair", 64, 128, 2)
    # TC_PERTAP (ablation): tile = 128 positions x bn output channels
    inf = pc.Plan((32, 128, 28, 28), (128, 128, 3, 3), padding=(1, 1), math="bf16", kernel="tc_pertap").info()
    assert (inf["tile_m"], inf["tile_n"], inf["Cp"], inf["Kp"]) == (128, 128, 128, 128)
    inf = pc.Plan((1, 64, 10, 10), (320, 64, 3, 3), (1, 1), (1, 1), math="bf16", kernel="tc_pertap").info()
    assert inf["tile_n"] == 256 and inf["Kp"] == 512


def test_forward_without_gpu_fails_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    plan = pc.Plan((1, 4, 8, 8), (16, 4, 3, 3), math="bf16")
    with pytest.raises(pc.PolyconvError) as e:
        plan.forward_ptr(4096, 8192, 16384)
    assert e.value.status == pc.NOT_SUPPORTED
    assert plan._lib.polyconv_destroy(None) == pc.SUCCESS
