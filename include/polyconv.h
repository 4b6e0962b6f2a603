/*
 * polyconv.h — C-ABI of the B200 (sm_100a) PolyHankel forward convolution.
 *
 * The operation (PAPER.md = Xu et al., CGO'25; cited as P.<lines>):
 *   y[n][k][oh][ow] = sum_c sum_i sum_j xpad[n][c][sh*oh+i][sw*ow+j] * w[k][c][i][j]
 * computed as polynomial multiplication (§2.2):
 *   A_{n,c}(t): the zero-padded input plane flattened row-major with row pitch
 *               Wp = W + 2*pw  (Eq. 4, P.603-613; Eq. 10, P.941-950);
 *   U_{k,c}(t): the reversed, gap-padded filter, coefficient of degree
 *               e(i,j) = Wp*(R-1-i) + (S-1-j)  (Eq. 6, P.768-771; Eq. 11
 *               P.954-964 as corrected in DESIGN.md reading R1; P.1365-1382);
 *   p_{n,k}(t) = sum_c A_{n,c}(t) U_{k,c}(t)  (P.965; channel sum P.1350-1352);
 *   y[n][k][oh][ow] = coefficient Wp*sh*oh + sw*ow + L_U - 1 of p_{n,k}
 *               (Eq. 12, P.966-972; stride: DESIGN.md reading R4),
 *   with L_A = Hp*Wp, L_U = (R-1)*Wp + S (KernelSize, P.1378-1380).
 * Only the coefficients at the extraction degrees are computed.
 *
 * Problem parameters follow the paper's Table 1 (P.259-271): N, C, Ih=H,
 * Iw=W, K, Kh=R, Kw=S, padding; "the same API design ... as cuDNN"
 * (P.1444-1445).  Stride is an extension (reading R4).
 *
 * Conventions for every entry point:
 *  - Tensors are plain device pointers, dense and contiguous:
 *      x: [N][C][H][W]  w: [K][C][R][S]  y: [N][K][P][Q]  (NCHW, row-major),
 *    element type = the plan's io dtype (fp32 or bf16), 16-byte aligned,
 *    owned by the caller, on the plan's device.  y must not alias x or w.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *    All work is enqueued asynchronously on it; no call synchronises except
 *    polyconv_destroy.
 *  - Errors are returned as polyconv_status_t; the library never aborts or
 *    exits.  Argument errors are detected before any allocation or launch.
 *  - A plan owns its device workspace (packed operands, tensor maps).  Calls on
 *    one plan must be stream-ordered (one forward at a time).  Plans are not
 *    thread-safe; different plans are independent.
 */
#ifndef POLYCONV_H_
#define POLYCONV_H_

#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

#define POLYCONV_ABI_VERSION 1

typedef struct polyconv_plan_s *polyconv_plan_t; /* opaque, library-owned */

typedef enum {
    POLYCONV_STATUS_SUCCESS = 0,
    POLYCONV_STATUS_BAD_PARAM = 1,        /* NULL pointer, dim < 1, stride < 1, pad < 0,
                                             P < 1 or Q < 1, bad enum, unsupported combo */
    POLYCONV_STATUS_NOT_SUPPORTED = 2,    /* no sm_100 device, tensor > 2^31 elements,
                                             misaligned pointer, forced kernel cannot run */
    POLYCONV_STATUS_ALLOC_FAILED = 3,     /* workspace cudaMalloc failed */
    POLYCONV_STATUS_EXECUTION_FAILED = 4  /* CUDA launch/runtime error; see polyconv_last_error */
} polyconv_status_t;

/* Element type of x, w and y. */
typedef enum { POLYCONV_F32 = 0, POLYCONV_BF16 = 1 } polyconv_dtype_t;

/* Arithmetic of the coefficient multiply-accumulate (all accumulate in fp32).
 *   FP32_FMA: fp32 operands, SIMT FFMA           (parity gate 1e-5 normwise)
 *   TF32:     operands rounded fp32->tf32 (RNA) in packing, tcgen05 kind::tf32
 *   BF16:     operands rounded fp32->bf16 (RNE) in packing, tcgen05 kind::f16
 * io_dtype BF16 requires math BF16. */
typedef enum {
    POLYCONV_MATH_FP32_FMA = 0,
    POLYCONV_MATH_TF32 = 1,
    POLYCONV_MATH_BF16 = 2
} polyconv_math_t;

/* MAC kernel variant.  AUTO picks by shape and math; the others force one
 * (ablations/tests; polyconv_plan_set_kernel returns POLYCONV_STATUS_BAD_PARAM when the shape or
 * math does not fit the variant).
 *  TC        tcgen05/TMEM contraction, filters as the M=128 operand, one position window per
 *            channel chunk reused by every tap (Hankel shift = descriptor offset), windows by TMA
 *            from a packed input (TF32 default).
 *  TC_FUSED  the same contraction with the input packed inside the kernel (filter packed by its
 *            own launch).
 *  TC_PERTAP positions as M, one TMA window load per tap (ablation).
 *  TC_PAIR   CTA pairs (cta_group::2) with the filter resident in shared memory, fed by a
 *            separate packing grid (bf16 math, K <= 128, H*W*elem a multiple of 16 bytes).
 *  TC_1X1    1x1 layers: the NCHW planes are the MN-major tensor-core operand.
 *  TC_HANKEL the BF16 default for 3x3/5x5 layers: one persistent launch on CTA pairs that builds
 *            the Hankel windows of the input polynomial in shared memory straight from NCHW x (the
 *            batch as one polynomial whose images share padding rows, reading R16) and
 *            runs tcgen05.mma cta_group::2 with the filter resident or streamed by TMA (bf16 or
 *            tf32 math, any stride / padding / kernel size).
 *  FFT       the paper's solver (Eq. 13-15): FFT of every A_{n,c}(t) and U_{k,c}(t), per-frequency
 *            channel contraction, inverse FFT, Eq. 12 extraction (math FP32_FMA; FFT length
 *            L = power of two >= L_A + L_U - 1 <= 8192).
 *  FP32      SIMT register-blocked FFMA.   THIN  warp-per-output with shuffle reduction.
 * No variant synchronises across CTAs outside a cluster: every launch is safe to capture into a
 * CUDA graph and to run while other work holds SMs (it waits for them). */
typedef enum {
    POLYCONV_KERNEL_AUTO = 0,
    POLYCONV_KERNEL_TC = 1,
    POLYCONV_KERNEL_FP32 = 2,
    POLYCONV_KERNEL_THIN = 3,
    POLYCONV_KERNEL_TC_PERTAP = 4,
    POLYCONV_KERNEL_TC_FUSED = 5,
    POLYCONV_KERNEL_TC_PAIR = 6,
    POLYCONV_KERNEL_TC_1X1 = 7,
    POLYCONV_KERNEL_TC_HANKEL = 8,
    POLYCONV_KERNEL_FFT = 9
} polyconv_kernel_t;

/* Packed-operand layouts exposed for bit-exact tests (a2/a3):
 *   PLANAR      input:  [N][C][L_A]      A_{n,c}(t) coefficient vectors (Eq. 10)
 *               filter: [K][C][L_U]      U_{k,c}(t) coefficient vectors (Eq. 11, R1)
 *   INTERLEAVED input:  [N*L_A][Cp]      coefficient-major, channels innermost
 *                                        (the tensor-core B/A operand layout)
 *               filter: [R*S][Kp][Cp]    tap-major, channels innermost
 * Storage words are the math mode's operand format: fp32 words (FP32_FMA),
 * tf32-in-32-bit words with the low 13 bits zero (TF32), or bf16 (BF16).
 * Cp/Kp are C/K rounded up as reported by polyconv_plan_info. */
typedef enum { POLYCONV_LAYOUT_PLANAR = 0, POLYCONV_LAYOUT_INTERLEAVED = 1 } polyconv_layout_t;

typedef struct {
    int N, C, H, W, K, R, S, sh, sw, ph, pw;
    int P, Q;          /* output height/width */
    int Hp, Wp;        /* padded input height/width */
    long long L_A;     /* input polynomial length Hp*Wp */
    long long L_U;     /* kernel polynomial length (R-1)*Wp + S */
    int Cp, Kp;        /* padded channel counts of the INTERLEAVED layouts */
    int kernel;        /* polyconv_kernel_t the forward will run */
    int tile_m, tile_n, stages; /* MAC tiling: positions x output channels, smem stages */
    int launches;      /* kernel launches per polyconv_forward */
    size_t workspace_bytes; /* device workspace the plan allocates at first use */
} polyconv_info_t;

/* Create a plan.  Validates every argument (no CUDA call happens on error).
 * Device resources are allocated lazily at the first call that needs them,
 * so planning works without a GPU (host-side tests).
 *   N,C,H,W: x shape; K,R,S: w shape [K][C][R][S]; sh,sw >= 1; ph,pw >= 0;
 *   io_dtype/math: see above; device: CUDA ordinal the pointers live on. */
polyconv_status_t polyconv_plan(polyconv_plan_t *plan, int N, int C, int H, int W,
                                int K, int R, int S, int stride_h, int stride_w,
                                int pad_h, int pad_w, polyconv_dtype_t io_dtype,
                                polyconv_math_t math, int device);

/* Force a MAC variant (default AUTO).  BAD_PARAM if the variant cannot run
 * this plan's math mode (TC needs TF32/BF16; FP32 needs FP32_FMA). */
polyconv_status_t polyconv_plan_set_kernel(polyconv_plan_t plan, polyconv_kernel_t kernel);

/* Output spatial size: P = (H+2ph-R)/sh + 1, Q = (W+2pw-S)/sw + 1. */
polyconv_status_t polyconv_output_dims(polyconv_plan_t plan, int *P, int *Q);

/* Sizes, chosen kernel and tiling (host only). */
polyconv_status_t polyconv_plan_info(polyconv_plan_t plan, polyconv_info_t *info);

/* The hot path: pack (a2,a3) -> coefficient MAC over channels (a4) with the
 * extraction/strided NCHW store fused in its epilogue (a5).  y: [N][K][P][Q]. */
polyconv_status_t polyconv_forward(polyconv_plan_t plan, const void *x, const void *w,
                                   void *y, void *stream);

/* Output-channel-sharded forward with the all-gather fused into the MAC epilogue (SURVEY
 * §8(e)/(f) f4; the paper is single-GPU, P.1431-1433).  ys[0..n_out-1] are device pointers to
 * outputs [N][k_total][P][Q] in the io dtype -- local buffers, or every rank's buffer mapped
 * over NVLink (e.g. torch symmetric memory); this plan's K output channels (a block of the
 * layer's k_total) are stored at channel offset k_offset of EVERY ys[r] straight from the
 * epilogue: no local copy, no separate collective.  1 <= n_out <= 8, 0 <= k_offset,
 * k_offset + K <= k_total; all pointers 16-byte aligned (else NOT_SUPPORTED).  The caller
 * orders the peers' reads after this forward (stream order plus a cross-rank barrier).  Only
 * the TC_HANKEL kernel of stride-1 plans stores to peers: NOT_SUPPORTED for plans that resolved
 * to another kernel or to its stride-2 phase mode (nothing written to ys).  Other errors as
 * polyconv_forward. */
polyconv_status_t polyconv_forward_scatter(polyconv_plan_t plan, const void *x, const void *w,
                                           void *const *ys, int n_out, int k_total, int k_offset,
                                           void *stream);

/* polyconv_forward from HOST buffers (the end-to-end call): x, w, y are host
 * pointers (pinned for asynchronous copies; pageable works but serialises).
 * Enqueues on `stream`: H2D copy of x and w into plan-owned device buffers
 * (allocated at first use, freed by polyconv_destroy), polyconv_forward, D2H
 * copy of y.  For N >= 2 the batch is pipelined in chunks (environment
 * POLYCONV_HOST_CHUNKS, default 4, 1 = off): chunk copies run on two
 * plan-owned copy streams ordered by events after the work already on
 * `stream`, each chunk's forward (a plan-owned sub-plan with this plan's
 * kernel: the same bytes as one polyconv_forward) on `stream`, and `stream`
 * waits for the last copy.  Not pipelined for stride >= 2 polyphase plans or
 * while timing events are set.  Does not synchronise: x, w, y must stay valid
 * until `stream` is synchronised.  Errors as polyconv_forward (ALLOC_FAILED if the device
 * buffers cannot be allocated). */
polyconv_status_t polyconv_forward_host(polyconv_plan_t plan, const void *x, const void *w,
                                        void *y, void *stream);

/* Measurement hook: if both are non-NULL cudaEvent_t (passed as void*), every
 * later forward records start_event just before and stop_event just after the
 * coefficient-MAC launch (the dominant kernel) on the forward's stream.  NULL,
 * NULL clears the hook.  BAD_PARAM if exactly one is NULL.  The events stay
 * owned by the caller and must outlive their use. */
polyconv_status_t polyconv_plan_set_timing_events(polyconv_plan_t plan, void *start_event,
                                                  void *stop_event);

/* a2 alone: write A_{n,c}(t) of x into dst in `layout` (see above).  dst must
 * hold polyconv_packed_bytes(plan, 0, layout) bytes. */
polyconv_status_t polyconv_pack_input(polyconv_plan_t plan, const void *x, void *dst,
                                      polyconv_layout_t layout, void *stream);

/* a3 alone: write U_{k,c}(t) of w into dst in `layout`. */
polyconv_status_t polyconv_pack_filter(polyconv_plan_t plan, const void *w, void *dst,
                                       polyconv_layout_t layout, void *stream);

/* Bytes of a packed operand: which = 0 input, 1 filter. */
polyconv_status_t polyconv_packed_bytes(polyconv_plan_t plan, int which,
                                        polyconv_layout_t layout, size_t *bytes);

/* a5 alone (standalone extraction, P.1396-1403): coeffs is the fp32 array of
 * full product coefficients [N][K][L_A+L_U-1]; writes y[n][k][oh][ow] =
 * coeffs[n][k][Wp*sh*oh + sw*ow + L_U-1] in the io dtype (bf16: RNE). */
polyconv_status_t polyconv_extract(polyconv_plan_t plan, const float *coeffs, void *y,
                                   void *stream);

/* --- Gradients (an extension, the paper is forward-only) -------------
 * For a stride-1 convolution y = conv(x, w) with padding (ph, pw) both gradients are
 * forward convolutions (cross-correlation, P.138-150) on re-laid-out operands:
 *   dx   = conv(dy, wt),   wt = polyconv_flip_filter(w),  padding (R-1-ph, S-1-pw)
 *   dw^T = conv(x^T, dy^T) with padding (ph, pw),  ^T = polyconv_swap_nc
 * so a forward plan of the transformed shapes computes them.  Stride (sh, sw) >= 2: dy is first
 * spread onto the stride lattice (polyconv_dilate, eh/ew = (H+2ph-R) mod sh, (W+2pw-S) mod sw);
 * dx is then the stride-1 formula on the dilated dy, and dw^T the first R x S outputs of it.  Both calls are plain
 * stream-ordered device copies (bit-exact), allocate nothing, and return BAD_PARAM for
 * NULL/aliased pointers, dims < 1 or a bad dtype, NOT_SUPPORTED past 2^31 (flip) or 2^40 (swap)
 * elements, EXECUTION_FAILED if the launch fails.  Device pointers, caller-owned. */

/* wt[c][k][R-1-i][S-1-j] = w[k][c][i][j]; w is [K][C][R][S], wt is [C][K][R][S]. */
polyconv_status_t polyconv_flip_filter(const void *w, void *wt, int K, int C, int R, int S,
                                       polyconv_dtype_t dtype, void *stream);

/* xd[n][c][sh*h][sw*w] = x[n][c][h][w], every other element 0; x is [N][C][H][W], xd is
 * [N][C][(H-1)*sh+1+eh][(W-1)*sw+1+ew]. */
polyconv_status_t polyconv_dilate(const void *x, void *xd, int N, int C, int H, int W, int sh, int sw,
                                  int eh, int ew, polyconv_dtype_t dtype, void *stream);

/* wgrad as its own split-K contraction (any stride / padding):
 *   dw[k][c][i][j] = sum_n sum_oh sum_ow dy[n][k][oh][ow] * xpad[n][c][sh*oh+i][sw*ow+j]
 * x [N][C][H][W], dy [N][K][P][Q] (P, Q as for the forward), dw [K][C][R][S], all in `dtype`;
 * ws: caller-owned fp32 device workspace of K*C*R*S floats (zeroed and accumulated here with
 * atomics, so the summation order is not fixed).  dw is written from ws (bf16: RNE). */
polyconv_status_t polyconv_wgrad(const void *x, const void *dy, void *dw, float *ws, int N, int C,
                                 int H, int W, int K, int R, int S, int sh, int sw, int ph, int pw,
                                 polyconv_dtype_t dtype, void *stream);

/* xt[c][n][e] = x[n][c][e] for e < HW; x is [N][C][HW], xt is [C][N][HW]. */
polyconv_status_t polyconv_swap_nc(const void *x, void *xt, int N, int C, long long HW,
                                   polyconv_dtype_t dtype, void *stream);

/* Synchronise the last stream used by the plan, free its workspace and the plan.
 * NULL is accepted (no-op). */
polyconv_status_t polyconv_destroy(polyconv_plan_t plan);

/* Static description of a status code. */
const char *polyconv_status_string(polyconv_status_t status);

/* Text of the last failure on this plan ("" if none).  Valid until the next
 * call on the plan. */
const char *polyconv_last_error(polyconv_plan_t plan);

/* POLYCONV_ABI_VERSION of the loaded library. */
int polyconv_abi_version(void);

#ifdef __cplusplus
}
#endif

#endif /* POLYCONV_H_ */
