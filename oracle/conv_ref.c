/*
 * ORACLE (O1) — TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct fp64 CPU direct convolution.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load or run this file's library.  It shares no code, header, table or
 * helper with the CUDA path (paper_conf_cgo_xuzc025_b200/csrc) and neither
 * side includes the other.
 *
 * What it computes (the definition the method reaches exactly):
 *   PAPER.md P.138-150 (§1) and P.488-493 (§2.2):
 *     conv2D(I,K)(ih,iw) = sum_{kh<Kh} sum_{kw<Kw} I[ih+kh, iw+kw] * K[kh,kw]
 *   (cross-correlation, no flip; O = I - K + 1, P.485).
 *   Channels are summed (P.1336-1352, §3.2, the option the paper keeps).
 *   Zero padding on all four sides (Fig. 1, P.380-402; P.1353-1356).
 *   Stride is absent from the paper; reading R4:
 *     output (oh,ow) reads xpad[sh*oh + i][sw*ow + j].
 *
 *   y[n][k][oh][ow] = sum_{c<C} sum_{i<R} sum_{j<S}
 *                       xpad[n][c][sh*oh+i][sw*ow+j] * w[k][c][i][j]
 *   P = floor((H+2ph-R)/sh)+1, Q = floor((W+2pw-S)/sw)+1.
 *
 * Precision: inputs are doubles (callers pass fp32 values widened exactly);
 * every fp32*fp32 product is exact in fp64; accumulation in fixed c->i->j
 * order, one double accumulator per output.  No -ffast-math.
 *
 * Parallelism: OpenMP over (n,k) only; each output is computed by exactly one
 * thread in the same order, so the result does not depend on thread count.
 */
#include <stddef.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* Return codes mirror the library's argument validation: 0 ok, 1 bad param. */
int oracle_output_dims(int H, int W, int R, int S, int sh, int sw, int ph, int pw,
                       int *P, int *Q)
{
    if (H < 1 || W < 1 || R < 1 || S < 1 || sh < 1 || sw < 1 || ph < 0 || pw < 0)
        return 1;
    int hp = H + 2 * ph, wp = W + 2 * pw;
    if (hp < R || wp < S) return 1;
    *P = (hp - R) / sh + 1;
    *Q = (wp - S) / sw + 1;
    return 0;
}

int oracle_conv2d_f64(const double *x, const double *w, double *y,
                      int N, int C, int H, int W, int K, int R, int S,
                      int sh, int sw, int ph, int pw, int nthreads)
{
    int P, Q;
    if (N < 1 || C < 1 || K < 1) return 1;
    if (oracle_output_dims(H, W, R, S, sh, sw, ph, pw, &P, &Q)) return 1;
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif
    long long NK = (long long)N * K;
#pragma omp parallel for schedule(dynamic, 1)
    for (long long nk = 0; nk < NK; ++nk) {
        int n = (int)(nk / K), k = (int)(nk % K);
        for (int oh = 0; oh < P; ++oh) {
            for (int ow = 0; ow < Q; ++ow) {
                double acc = 0.0;
                for (int c = 0; c < C; ++c) {
                    for (int i = 0; i < R; ++i) {
                        int h = sh * oh + i - ph;          /* row in unpadded x */
                        if (h < 0 || h >= H) continue;     /* zero padding */
                        for (int j = 0; j < S; ++j) {
                            int ww = sw * ow + j - pw;
                            if (ww < 0 || ww >= W) continue;
                            acc += x[(((size_t)n * C + c) * H + h) * W + ww] *
                                   w[(((size_t)k * C + c) * R + i) * S + j];
                        }
                    }
                }
                y[(((size_t)n * K + k) * P + oh) * Q + ow] = acc;
            }
        }
    }
    return 0;
}

/* Number of OpenMP threads the oracle would use (reported as `cores`). */
int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
