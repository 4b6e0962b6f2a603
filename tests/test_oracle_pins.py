"""Pins for the oracle (oracle/) against what the paper and mathematics fix.

None of these re-types the oracle's own formula: each compares an oracle
function with a paper-printed value (tests/golden/paper_examples.json, cited),
an independent route (im2col GEMM of Eq. 1-3, scipy/torch library routines,
brute force), a closed form or an invariant.  CPU only.
"""
import json
import os

import numpy as np
import pytest

import oracle
from oracle import poly_ref as pr

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_examples.json")))


# ---------------------------------------------------------------- degrees --

def test_eq4_input_degrees():
    g = GOLD["eq4_input_degrees"]["degrees"]
    got = [[pr.input_degree(r, s, 5) for s in range(5)] for r in range(5)]
    assert got == g
    # and A(t) of an index-valued plane puts element k at degree k
    x = np.arange(25, dtype=np.float64).reshape(5, 5) + 100
    a = pr.input_polynomial(x)
    for r in range(5):
        for s in range(5):
            assert a[g[r][s]] == x[r, s]


def test_eq6_kernel_exponents_and_eq11_misprint():
    want = GOLD["eq6_kernel_exponents"]["exponents"]
    got = [pr.kernel_degree(i, j, 3, 3, 5) for i in range(3) for j in range(3)]
    assert got == want
    # reading R1: Eq. 11 as printed contradicts Eq. 6 (u00 -> t^11, not t^12)
    printed = [pr.kernel_degree_as_printed(i, j, 3, 3, 5, Oh=3) for i in range(3) for j in range(3)]
    assert printed != want
    assert printed[0] == 11 and want[0] == 12


def test_first_row_degree_symmetry():
    rd1 = pr.first_row_degrees(3, 3, 5)
    assert list(rd1) == GOLD["rd_first_row"]["degrees"]
    assert set(rd1 + rd1[::-1]) == {GOLD["rd_first_row"]["sum_with_reverse"]}
    rd2 = np.array(GOLD["rd_second_row"]["degrees"])
    assert set(rd2 + rd1[::-1]) == {GOLD["rd_second_row"]["sum_with_reverse_first"]}
    # U^t = U (.) reverse(row_degree) (P.885-900) is the kernel degree map
    assert list(rd1[::-1]) == [pr.kernel_degree(i, j, 3, 3, 5) for i in range(3) for j in range(3)]


def test_eq7_eq12_result_degrees():
    want = GOLD["eq7_result_degrees"]["degrees"]
    got = [pr.extraction_degree(i, j, 3, 3, 5) for i in range(3) for j in range(3)]
    assert got == want
    # Eq. 12 offset (Ow+Kw-1)*Kh - Ow with Ow=3, Kw=Kh=3 -> 15-3 = 12 = L_U - 1
    assert pr.sizes(5, 5, 3, 3)["L_U"] - 1 == 5 * 3 - 3


def test_eq8_eq9_alternative_construction():
    """Any row works (P.901-906): shifting every kernel degree by +7 (Eq. 8)
    moves the result to degrees 19..31 (Eq. 9) with the same coefficients."""
    alt = GOLD["eq8_alternative_kernel_exponents"]["exponents"]
    base = GOLD["eq6_kernel_exponents"]["exponents"]
    shift = alt[0] - base[0]
    assert all(a - b == shift for a, b in zip(alt, base))
    rng = np.random.default_rng(1)
    x = rng.integers(-5, 6, (5, 5)).astype(np.float64)
    w = rng.integers(-5, 6, (3, 3)).astype(np.float64)
    a = pr.input_polynomial(x)
    u_alt = np.zeros(max(alt) + 1)
    for (i, j), e in zip([(i, j) for i in range(3) for j in range(3)], alt):
        u_alt[e] = w[i, j]
    prod = np.convolve(a, u_alt)
    d_alt = prod[GOLD["eq9_alternative_result_degrees"]["degrees"]]
    y = oracle.conv2d(x[None, None], w[None, None])[0, 0].reshape(-1)
    assert np.array_equal(d_alt, y)


def test_fig2_lshaped_map():
    g = GOLD["fig2_map"]
    deg, starred, bold = pr.lshaped_degree_map(g["Oh"], g["Ow"], g["Kh"], g["Kw"])
    assert starred == g["starred"]
    assert bold == g["bold"]
    for b, (bi, bj) in {"00": (0, 0), "01": (0, 1), "02": (0, 2), "12": (1, 2), "22": (2, 2)}.items():
        assert [deg(bi, bj, 0, rj) for rj in range(3)] == g[f"block{b}_first_row"]
        assert [deg(bi, bj, ri, 2) for ri in (1, 2)] == g[f"block{b}_right_column_below"]


@pytest.mark.parametrize("Oh,Ow,Kh,Kw", [(3, 3, 3, 3), (4, 4, 2, 2), (6, 6, 3, 3), (5, 7, 2, 4),
                                        (28, 28, 3, 3), (2, 9, 5, 1)])
def test_lshaped_map_equals_closed_forms(Oh, Ow, Kh, Kw):
    """§3.1: the traversal visits Ih*Iw distinct values; map == Eq. 10 row-major
    degrees, reversed starred == kernel degrees e(i,j), bold == Eq. 12 degrees."""
    Ih, Iw = Oh + Kh - 1, Ow + Kw - 1
    deg, starred, bold = pr.lshaped_degree_map(Oh, Ow, Kh, Kw)
    seen = {deg(bi, bj, ri, rj) for bi in range(Oh) for bj in range(Kh)
            for ri in range(Ow) for rj in range(Kw)}
    assert seen == set(range(Ih * Iw))
    for bi in range(Oh):
        for bj in range(Kh):
            for ri in range(Ow):
                for rj in range(Kw):
                    assert deg(bi, bj, ri, rj) == pr.input_degree(bi + bj, ri + rj, Iw)
    assert starred[::-1] == [pr.kernel_degree(i, j, Kh, Kw, Iw) for i in range(Kh) for j in range(Kw)]
    assert bold == [pr.extraction_degree(i, j, Kh, Kw, Iw) for i in range(Oh) for j in range(Ow)]


def test_kernel_size_and_gap_padding():
    for R, S, Wp in [(3, 3, 5), (2, 2, 5), (5, 3, 13), (1, 1, 7), (7, 7, 230)]:
        z = pr.sizes(Wp, Wp, R, S)  # H=W=Wp, no padding
        assert z["L_U"] == (R - 1) * Wp + S                       # KernelSize, P.1378-1380
        w = np.arange(1, R * S + 1, dtype=np.float64).reshape(R, S)
        u = pr.kernel_polynomial(w, Wp)
        assert len(u) == z["L_U"]
        # reversed kernel rows, each followed by Wp-S zeros except the last (P.1380-1382)
        rows = [u[r * Wp:r * Wp + S] for r in range(R)]
        for r in range(R):
            assert np.array_equal(rows[r], w[R - 1 - r, ::-1])
            if r < R - 1:
                assert not np.any(u[r * Wp + S:(r + 1) * Wp])


def test_skip_pattern_stride1():
    """P.1398-1401: drop the first (Kh-1)*Iw+Kw-1 values, take Ow, skip Kw-1, ..."""
    for H, W, R, S, p in [(8, 8, 3, 3, 0), (28, 28, 3, 3, 1), (7, 11, 2, 5, 2)]:
        z = pr.sizes(H, W, R, S, 1, 1, p, p)
        idx = []
        pos = (R - 1) * z["Wp"] + S - 1
        for _ in range(z["P"]):
            idx += list(range(pos, pos + z["Q"]))
            pos += z["Q"] + S - 1
        got = [pr.extraction_degree(i, j, R, S, z["Wp"]) for i in range(z["P"]) for j in range(z["Q"])]
        assert got == idx
        assert idx[0] == z["L_U"] - 1 and idx[-1] == z["L_A"] - 1


# ---------------------------------------------------------------- results --

def test_fig1_worked_example():
    g = GOLD["fig1"]
    x = np.array(g["input"], dtype=np.float64)
    assert np.array_equal(pr.pad_plane(x, 1, 1), np.array(g["padded"]))
    u = np.array([[1.0, 2.0], [3.0, 4.0]])
    rows = np.array(g["im2col_rows"], dtype=np.float64)      # one row per kernel element
    y_im2col = (rows.T @ u.reshape(-1)).reshape(4, 4)        # Eq. 3 route
    y1 = oracle.conv2d(x[None, None], u[None, None], padding=(1, 1))[0, 0]
    y2 = pr.polyhankel_conv2d(x[None, None], u[None, None], padding=(1, 1))[0, 0]
    assert np.array_equal(y1, y_im2col)
    assert np.array_equal(y2, y_im2col)
    assert list(pr.kernel_polynomial(u, 5)) == [4, 3, 0, 0, 0, 2, 1]


def test_section22_example_index_valued():
    """§2.2: 5x5 A, 3x3 U; product coefficients at Eq. 7 degrees == im2col (Eq. 1-3)."""
    x = np.arange(25, dtype=np.float64).reshape(5, 5)
    u = np.arange(1, 10, dtype=np.float64).reshape(3, 3)
    # Eq. 1: im2col rows = 3x3 patches in output order; Eq. 2: flattened kernel
    A_im2col = np.array([x[i:i + 3, j:j + 3].reshape(-1) for i in range(3) for j in range(3)])
    D = A_im2col @ u.reshape(-1)
    prod = pr.poly_mul_schoolbook(pr.input_polynomial(x), pr.kernel_polynomial(u, 5))
    assert np.array_equal(prod[GOLD["eq7_result_degrees"]["degrees"]], D)
    assert np.array_equal(oracle.conv2d(x[None, None], u[None, None])[0, 0].reshape(-1), D)
    assert list(D) == [366, 411, 456, 591, 636, 681, 816, 861, 906]


def test_o1_vs_scipy_correlate2d():
    from scipy.signal import correlate2d
    rng = np.random.default_rng(7)
    for H, W, R, S in [(8, 8, 3, 3), (13, 9, 5, 3), (6, 11, 1, 4), (3, 3, 3, 3)]:
        x = rng.standard_normal((H, W))
        w = rng.standard_normal((R, S))
        y = oracle.conv2d(x[None, None], w[None, None])[0, 0]
        np.testing.assert_allclose(y, correlate2d(x, w, mode="valid"), rtol=0, atol=1e-12)


@pytest.mark.parametrize("N,C,H,W,K,R,S,s,p", [
    (2, 3, 8, 8, 4, 3, 3, 1, 1), (1, 5, 9, 7, 3, 3, 2, 2, 1), (2, 2, 7, 7, 2, 5, 5, 1, 2),
    (1, 4, 6, 6, 3, 1, 1, 2, 0), (3, 1, 5, 8, 2, 2, 3, 3, 2), (1, 2, 14, 14, 2, 7, 7, 2, 3)])
def test_o1_vs_torch_float64(N, C, H, W, K, R, S, s, p):
    import torch
    rng = np.random.default_rng(N * 100 + C)
    x = rng.standard_normal((N, C, H, W))
    w = rng.standard_normal((K, C, R, S))
    ref = torch.nn.functional.conv2d(torch.from_numpy(x), torch.from_numpy(w), stride=s, padding=p).numpy()
    y = oracle.conv2d(x, w, (s, s), (p, p))
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("N,C,H,W,K,R,S,s,p", [
    (1, 1, 8, 8, 1, 3, 3, 1, 0), (2, 3, 6, 7, 2, 3, 3, 1, 1), (1, 2, 9, 9, 3, 2, 4, 2, 1),
    (1, 3, 5, 5, 2, 5, 5, 1, 2), (2, 2, 7, 6, 2, 1, 1, 3, 0)])
def test_o1_equals_o2_polynomial_bruteforce(N, C, H, W, K, R, S, s, p):
    rng = np.random.default_rng(11 + H)
    xi = rng.integers(-8, 9, (N, C, H, W)).astype(np.float64)
    wi = rng.integers(-4, 5, (K, C, R, S)).astype(np.float64)
    assert np.array_equal(oracle.conv2d(xi, wi, (s, s), (p, p)),
                          pr.polyhankel_conv2d(xi, wi, (s, s), (p, p)))
    xr = rng.standard_normal((N, C, H, W))
    wr = rng.standard_normal((K, C, R, S))
    np.testing.assert_allclose(oracle.conv2d(xr, wr, (s, s), (p, p)),
                               pr.polyhankel_conv2d(xr, wr, (s, s), (p, p)), rtol=0, atol=1e-12)


def test_full_product_valid_identity():
    """np.convolve(A,U,'valid') rows of Wp truncated to Q equal the direct conv
    (SURVEY B.2); full_product at the Eq. 12 degrees equals O1."""
    rng = np.random.default_rng(3)
    for H, W, R, S, p in [(8, 8, 3, 3, 0), (28, 28, 3, 3, 1), (7, 7, 3, 3, 1), (13, 9, 5, 3, 2)]:
        x = rng.integers(-8, 9, (1, 1, H, W)).astype(np.float64)
        w = rng.integers(-4, 5, (1, 1, R, S)).astype(np.float64)
        z = pr.sizes(H, W, R, S, 1, 1, p, p)
        y = oracle.conv2d(x, w, padding=(p, p))[0, 0]
        a = pr.pad_plane(x[0, 0], p, p).reshape(-1)
        v = np.convolve(a, pr.kernel_polynomial(w[0, 0], z["Wp"]), "valid")
        assert len(v) == (z["P"] - 1) * z["Wp"] + z["Q"]
        v = np.concatenate([v, np.zeros(z["Wp"] - z["Q"])]).reshape(z["P"], z["Wp"])[:, :z["Q"]]
        assert np.array_equal(v, y)
        fp = pr.full_product(x, w, (p, p))[0, 0]
        idx = [pr.extraction_degree(i, j, R, S, z["Wp"]) for i in range(z["P"]) for j in range(z["Q"])]
        assert np.array_equal(fp[idx].reshape(z["P"], z["Q"]), y)


def test_im2col_gemm_route_matches_o1():
    """Eq. 1-3 (im2col + MM) on small multi-channel inputs, independent of O1's loops."""
    rng = np.random.default_rng(5)
    N, C, H, W, K, R, S, s, p = 2, 3, 9, 8, 4, 3, 2, 2, 1
    x = rng.standard_normal((N, C, H, W))
    w = rng.standard_normal((K, C, R, S))
    xp = np.pad(x, ((0, 0), (0, 0), (p, p), (p, p)))
    P = (H + 2 * p - R) // s + 1
    Q = (W + 2 * p - S) // s + 1
    cols = np.zeros((N, C * R * S, P * Q))
    for oh in range(P):
        for ow in range(Q):
            cols[:, :, oh * Q + ow] = xp[:, :, s * oh:s * oh + R, s * ow:s * ow + S].reshape(N, -1)
    y = np.einsum("kf,nfp->nkp", w.reshape(K, -1), cols).reshape(N, K, P, Q)
    np.testing.assert_allclose(oracle.conv2d(x, w, (s, s), (p, p)), y, rtol=0, atol=1e-12)


# ------------------------------------------------------------- invariants --

def test_delta_filter_returns_input():
    rng = np.random.default_rng(9)
    N, C, H, W = 2, 3, 7, 6
    x = rng.standard_normal((N, C, H, W))
    for (R, S, p) in [(3, 3, 1), (5, 3, 2), (2, 2, 0)]:
        for i0 in range(R):
            for j0 in range(S):
                w = np.zeros((C, C, R, S))
                for c in range(C):
                    w[c, c, i0, j0] = 1.0
                y = oracle.conv2d(x, w, padding=(p, p))
                xp = np.pad(x, ((0, 0), (0, 0), (p, p), (p, p)))
                P, Q = y.shape[2:]
                assert np.array_equal(y, xp[:, :, i0:i0 + P, j0:j0 + Q])


def test_linearity_additivity_stride():
    rng = np.random.default_rng(10)
    N, C, H, W, K, R, S = 2, 4, 10, 9, 3, 3, 3
    x1, x2 = rng.integers(-8, 9, (2, N, C, H, W)).astype(np.float64)
    w1, w2 = rng.integers(-4, 5, (2, K, C, R, S)).astype(np.float64)
    f = lambda x, w, s=1: oracle.conv2d(x, w, (s, s), (1, 1))
    assert np.array_equal(f(3 * x1 - 2 * x2, w1), 3 * f(x1, w1) - 2 * f(x2, w1))
    assert np.array_equal(f(x1, 2 * w1 + w2), 2 * f(x1, w1) + f(x1, w2))
    # channel additivity (P.1350-1352): y(C) = sum_c y(channel c)
    parts = sum(f(x1[:, c:c + 1], w1[:, c:c + 1]) for c in range(C))
    assert np.array_equal(f(x1, w1), parts)
    # stride reading R4: O_s = O_1[::s, ::s]
    for s in (2, 3):
        assert np.array_equal(f(x1, w1, s), f(x1, w1)[:, :, ::s, ::s])
    # batch permutation equivariance
    perm = [1, 0]
    assert np.array_equal(f(x1[perm], w1), f(x1, w1)[perm])


def test_bad_params_rejected():
    with pytest.raises(ValueError):
        oracle.conv2d(np.zeros((1, 1, 2, 2)), np.zeros((1, 1, 3, 3)))
    with pytest.raises(ValueError):
        oracle.output_dims(8, 8, 3, 3, (0, 1), (0, 0))
    assert oracle.output_dims(8, 8, 3, 3) == (6, 6)
    assert oracle.output_dims(224, 224, 7, 7, (2, 2), (3, 3)) == (112, 112)


# ---------------------------------------------------- rounding references --

def test_bf16_rne_matches_torch():
    import torch
    rng = np.random.default_rng(12)
    v = np.concatenate([rng.standard_normal(200000).astype(np.float32),
                        (rng.standard_normal(20000) * 1e-30).astype(np.float32),
                        np.array([0.0, -0.0, 1.0, 3.4e38, -3.4e38, 1e-45], np.float32)])
    # exact ties: low 16 bits == 0x8000 with both parities of bit 16
    ties = (rng.integers(0x3f000000 >> 16, 0x43000000 >> 16, 5000).astype(np.uint32) << 16) | 0x8000
    v = np.concatenate([v, ties.view(np.float32)])
    ref = torch.from_numpy(v).bfloat16().view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(pr.round_bf16_rne_bits(v), ref)


def test_tf32_rna():
    one = np.float32(1.0)
    bits = lambda f: np.float32(f).view(np.uint32)
    # 1 + 2^-11 is a tie between 1 and 1 + 2^-10: ties AWAY -> 1 + 2^-10
    assert pr.round_tf32_rna_bits(np.float32(1 + 2 ** -11)) == bits(1 + 2 ** -10)
    assert pr.round_tf32_rna_bits(np.float32(-(1 + 2 ** -11))) == bits(-(1 + 2 ** -10))
    assert pr.round_tf32_rna_bits(np.float32(1 + 2 ** -12)) == bits(one)
    rng = np.random.default_rng(13)
    v = rng.standard_normal(100000).astype(np.float32)
    r = pr.round_tf32_rna_bits(v).view(np.float32)
    assert np.all((r.view(np.uint32) & 0x1FFF) == 0)
    assert np.max(np.abs(r - v) / np.abs(v)) <= 2.0 ** -11
    # small integers are exact in both formats (integer-exact parity mode)
    ints = np.arange(-64, 65, dtype=np.float32)
    assert np.array_equal(pr.round_tf32_rna_bits(ints).view(np.float32), ints)
    assert np.array_equal((pr.round_bf16_rne_bits(ints).astype(np.uint32) << 16).view(np.float32), ints)


def test_pack_references_layout():
    """a2/a3 storage references agree with the fp64 polynomials (Eq. 10/11)."""
    rng = np.random.default_rng(14)
    x = rng.integers(-8, 9, (2, 3, 5, 4)).astype(np.float32)
    w = rng.integers(-4, 5, (2, 3, 3, 2)).astype(np.float32)
    pa = pr.pack_input_planar(x, (1, 2), "fp32").view(np.float32)
    for n in range(2):
        for c in range(3):
            assert np.array_equal(pa[n, c], pr.input_polynomial(x[n, c], 1, 2))
    Wp = 4 + 4
    pu = pr.pack_filter_planar(w, Wp, "fp32").view(np.float32)
    for k in range(2):
        for c in range(3):
            assert np.array_equal(pu[k, c], pr.kernel_polynomial(w[k, c], Wp))
