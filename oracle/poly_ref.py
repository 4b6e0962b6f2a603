"""ORACLE (O2 + packing/extraction references) — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg may
import this module.  It shares no code with the CUDA path.

The PolyHankel method written out step by step in the paper's order and
notation (PAPER.md = /root/reference/PAPER.md, cited as P.<lines>):

  1. input polynomial   A(t)  -- Eq. 4 (P.603-613), Eq. 10 (P.941-950)
  2. kernel polynomial  U(t)  -- Eq. 6 (P.768-771), U = U_im2col (.) reverse(row_degree)
                                 (P.885-900); Eq. 11 (P.954-964, misprinted: reading R1)
  3. product            P(t) = A(t) U(t)   -- P.965; naive product §2.3 P.1021-1025
  4. extraction         d_ij = p_{Wp*i + j + Wp*Kh - Ow}  -- Eq. 12 (P.966-972)
  5. channel sum        y = sum_c                         -- P.1336-1352 (§3.2)

Readings of silent / garbled points (listed in DESIGN.md §Readings):
  R1  Eq. 11 as printed gives u00 -> t^11 in the paper's own 5x5/3x3 example,
      contradicting Eq. 6 (t^12).  We use e(i,j) = Wp*(R-1-i) + (S-1-j).
  R2  Iw in Eq. 10-12 and §3.2 is the padded width Wp = W + 2*pw.
  R3  Padding is symmetric zero padding on all sides (Fig. 1, P.380-402).
  R4  Stride (absent from the paper): keep coefficient Wp*sh*oh + sw*ow + L_U-1.
  R11 fp32->bf16 is round-to-nearest-even; fp32->tf32 is round-to-nearest-away
      (low 13 mantissa bits cleared).

Everything here is fp64 numpy unless a function says it emulates a storage
format bit for bit (the packing references).  Pure-Python loops are used
only where the paper describes a traversal (the Fig. 2 degree map) and are
meant for small cases.
"""
from __future__ import annotations

import numpy as np

# --------------------------------------------------------------------------
# a1: sizes and degrees
# --------------------------------------------------------------------------


def sizes(H, W, R, S, sh=1, sw=1, ph=0, pw=0):
    """Plan sizes.  O = I - K + 1 (P.485) on the padded input, generalised by
    stride (R4).  L_A = Hp*Wp (Eq. 10 has (Oh+Kh-1)(Ow+Kw-1) terms);
    L_U = (Kh-1)*Iw + Kw (KernelSize, P.1378-1380) with Iw := Wp (R2)."""
    Hp, Wp = H + 2 * ph, W + 2 * pw
    P = (Hp - R) // sh + 1
    Q = (Wp - S) // sw + 1
    return dict(Hp=Hp, Wp=Wp, P=P, Q=Q, L_A=Hp * Wp, L_U=(R - 1) * Wp + S)


def input_degree(r, s, Wp):
    """Eq. 10: a_{i,j} multiplies t^{(Ow+Kw-1)*i + j}; Ow+Kw-1 = Wp (R2)."""
    return Wp * r + s


def kernel_degree(i, j, R, S, Wp):
    """Corrected Eq. 11 (reading R1): e(i,j) = Wp*(R-1-i) + (S-1-j).
    Equals reverse(first_row_degree) of P.885-900."""
    return Wp * (R - 1 - i) + (S - 1 - j)


def kernel_degree_as_printed(i, j, R, S, Wp, Oh):
    """Eq. 11 exactly as printed (P.954-964): -(Ow+Kw-1)i - j + (Ow+Kw-1)Kh - Oh - 1.
    Kept only so a test can show it contradicts Eq. 6 (reading R1)."""
    return -Wp * i - j + Wp * R - Oh - 1


def extraction_degree(oh, ow, R, S, Wp, sh=1, sw=1):
    """Eq. 12: d_{i,j} = p_{(Ow+Kw-1)i + j + (Ow+Kw-1)Kh - Ow}.  With Iw:=Wp and
    Ow = Wp-S+1 (stride 1), the offset Wp*Kh - Ow = Wp*(R-1) + S - 1 = L_U - 1.
    Stride reading R4 scales the (i,j) lattice."""
    return Wp * sh * oh + sw * ow + Wp * (R - 1) + S - 1


def first_row_degrees(R, S, Wp):
    """RD_1st (P.849-860): degrees of the first im2col row = input_degree(i,j)."""
    return np.array([input_degree(i, j, Wp) for i in range(R) for j in range(S)])


def lshaped_degree_map(Oh, Ow, Kh, Kw):
    """§3.1 / Fig. 2 (P.1098-1118): traverse the doubly blocked Hankel matrix
    A_im2col (Oh x Kh blocks, each Ow x Kw) along an L-shaped path -- first
    block-row left to right, then the right block-column top to bottom; inside
    each block, first row left to right then right column top to bottom --
    numbering each newly met element 0,1,2,...

    Returns (deg, starred, bold):
      deg[(bi,bj,ri,rj)] -> integer, for every element of the matrix (elements
        equal along anti-diagonals share a number);
      starred = the first row of the map (reversed -> kernel degrees, P.1315-1320)
      bold    = the rightmost column of the map (result degrees, P.1322-1328)
    """
    # Identity of an element of A_im2col: block (bi,bj) holds rows bi+bj of the
    # input (block Hankel), element (ri,rj) of a block holds column ri+rj.
    numbering = {}
    nxt = 0

    def visit_block(bi, bj):
        nonlocal nxt
        order = [(0, rj) for rj in range(Kw)] + [(ri, Kw - 1) for ri in range(1, Ow)]
        for ri, rj in order:
            key = (bi + bj, ri + rj)  # the underlying input element
            if key not in numbering:
                numbering[key] = nxt
                nxt += 1

    outer = [(0, bj) for bj in range(Kh)] + [(bi, Kh - 1) for bi in range(1, Oh)]
    for bi, bj in outer:
        visit_block(bi, bj)

    def deg(bi, bj, ri, rj):
        return numbering[(bi + bj, ri + rj)]

    starred = [deg(0, bj, 0, rj) for bj in range(Kh) for rj in range(Kw)]
    bold = [deg(bi, Kh - 1, ri, Kw - 1) for bi in range(Oh) for ri in range(Ow)]
    return deg, starred, bold


# --------------------------------------------------------------------------
# a2/a3: polynomials (fp64 coefficient vectors)
# --------------------------------------------------------------------------


def pad_plane(x2d, ph, pw):
    """Zero padding on all sides (R3, Fig. 1)."""
    H, W = x2d.shape
    out = np.zeros((H + 2 * ph, W + 2 * pw), dtype=np.float64)
    out[ph:ph + H, pw:pw + W] = x2d
    return out


def input_polynomial(x2d, ph=0, pw=0):
    """A(t) coefficient vector (Eq. 10): coefficient Wp*r + s = xpad[r][s]."""
    xp = pad_plane(x2d, ph, pw)
    Hp, Wp = xp.shape
    a = np.zeros(Hp * Wp, dtype=np.float64)
    for r in range(Hp):
        for s in range(Wp):
            a[input_degree(r, s, Wp)] = xp[r, s]
    return a


def kernel_polynomial(w2d, Wp):
    """U(t) coefficient vector: coefficient e(i,j) = u_{i,j}, all others 0.
    Length L_U = (R-1)*Wp + S: the reversed kernel rows with Wp-S zeros between
    rows and none after the last (P.1365-1382)."""
    R, S = w2d.shape
    u = np.zeros((R - 1) * Wp + S, dtype=np.float64)
    for i in range(R):
        for j in range(S):
            u[kernel_degree(i, j, R, S, Wp)] = w2d[i, j]
    return u


def poly_mul_schoolbook(p, q):
    """Naive product (P.1021-1025): every term of P times every term of Q."""
    r = np.zeros(len(p) + len(q) - 1, dtype=np.float64)
    for a in range(len(p)):
        if p[a] != 0.0:
            r[a:a + len(q)] += p[a] * q
    return r


def extract(prod, P, Q, R, S, Wp, sh=1, sw=1):
    """Eq. 12 (+R4): y[oh][ow] = p[Wp*sh*oh + sw*ow + L_U - 1]."""
    y = np.zeros((P, Q), dtype=np.float64)
    for oh in range(P):
        for ow in range(Q):
            y[oh, ow] = prod[extraction_degree(oh, ow, R, S, Wp, sh, sw)]
    return y


def polyhankel_conv2d(x, w, stride=(1, 1), padding=(0, 0), mul=poly_mul_schoolbook):
    """O2: the whole method by brute force (tiny inputs).  x[N][C][H][W],
    w[K][C][R][S] -> y[N][K][P][Q] (fp64).  Per (n,k): sum over c of the
    product A_{n,c}(t) U_{k,c}(t) (channel option 2, P.1347-1352), then Eq. 12."""
    x = np.asarray(x, dtype=np.float64)
    w = np.asarray(w, dtype=np.float64)
    N, C, H, W = x.shape
    K, C2, R, S = w.shape
    assert C == C2
    sh, sw = stride
    ph, pw = padding
    z = sizes(H, W, R, S, sh, sw, ph, pw)
    y = np.zeros((N, K, z["P"], z["Q"]), dtype=np.float64)
    for n in range(N):
        A = [input_polynomial(x[n, c], ph, pw) for c in range(C)]
        for k in range(K):
            prod = np.zeros(z["L_A"] + z["L_U"] - 1, dtype=np.float64)
            for c in range(C):
                prod += mul(A[c], kernel_polynomial(w[k, c], z["Wp"]))
            y[n, k] = extract(prod, z["P"], z["Q"], R, S, z["Wp"], sh, sw)
    return y


def full_product(x, w, padding=(0, 0)):
    """All coefficients p_{n,k}[m] = sum_c (A_{n,c} U_{k,c})[m], m < L_A+L_U-1,
    via np.convolve (a library polynomial multiplication).  fp64."""
    x = np.asarray(x, dtype=np.float64)
    w = np.asarray(w, dtype=np.float64)
    N, C, H, W = x.shape
    K, _, R, S = w.shape
    ph, pw = padding
    Wp = W + 2 * pw
    L = (H + 2 * ph) * Wp + (R - 1) * Wp + S - 1
    out = np.zeros((N, K, L), dtype=np.float64)
    for n in range(N):
        for c in range(C):
            a = pad_plane(x[n, c], ph, pw).reshape(-1)
            for k in range(K):
                out[n, k] += np.convolve(a, kernel_polynomial(w[k, c], Wp))
    return out


# --------------------------------------------------------------------------
# Storage-format references for the bit-exact pack tests (R11)
# --------------------------------------------------------------------------


def round_bf16_rne_bits(x32):
    """fp32 -> bf16 bits, round to nearest even (R11).  Finite inputs only."""
    u = np.asarray(x32, dtype=np.float32).view(np.uint32).astype(np.uint64)
    r = (u + 0x7FFF + ((u >> 16) & 1)) >> 16
    return r.astype(np.uint16)


def round_tf32_rna_bits(x32):
    """fp32 -> tf32 stored in 32 bits, round to nearest, ties away (R11):
    add half an ulp of the 10-bit mantissa, clear the low 13 bits."""
    u = np.asarray(x32, dtype=np.float32).view(np.uint32).astype(np.uint64)
    r = ((u + 0x1000) & 0xFFFFE000) & 0xFFFFFFFF
    return r.astype(np.uint32)


def _as_format(x32, math):
    """Return the storage words of x32 in the math mode's operand format."""
    x32 = np.asarray(x32, dtype=np.float32)
    if math == "fp32":
        return x32.view(np.uint32)
    if math == "tf32":
        return round_tf32_rna_bits(x32)
    if math == "bf16":
        return round_bf16_rne_bits(x32)
    raise ValueError(math)


def pack_input_planar(x, padding, math):
    """a2, layout (i): A_{n,c}(t) coefficient vectors, [N][C][L_A] storage words."""
    x = np.asarray(x, dtype=np.float32)
    N, C, H, W = x.shape
    ph, pw = padding
    xp = np.zeros((N, C, H + 2 * ph, W + 2 * pw), dtype=np.float32)
    xp[:, :, ph:ph + H, pw:pw + W] = x
    return _as_format(xp.reshape(N, C, -1), math)


def pack_filter_planar(w, Wp, math):
    """a3, paper layout: U_{k,c}(t) coefficient vectors, [K][C][L_U] storage words."""
    w = np.asarray(w, dtype=np.float32)
    K, C, R, S = w.shape
    u = np.zeros((K, C, (R - 1) * Wp + S), dtype=np.float32)
    for i in range(R):
        for j in range(S):
            u[:, :, kernel_degree(i, j, R, S, Wp)] = w[:, :, i, j]
    return _as_format(u, math)
