// polyconv.cu — host side of the C-ABI (include/polyconv.h): argument
// validation, the a1 plan/index math, kernel selection, workspace and launch
// sequencing.  Every step of the hot path runs in the CUDA kernels of this
// directory; there is no CPU compute path and no fallback to another library.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include "../../include/polyconv.h"
#include "internal.h"

using namespace polyconv;

struct polyconv_plan_s {
  Geom g;
  bool io_bf16;
  int math;
  int fmt;
  int device;
  int forced;
  int kernel;  // resolved polyconv_kernel_t
  TcTiling tc;
  Tc2Tiling tc2;
  Fp32Tiling f32;
  PairTiling pair;
  HankelTiling hk;
  FftTiling fft;
  bool fft_tw_ready = false;  // twiddles computed into wsU
  void* hkzero = nullptr;  // mac_hankel: zero words read in place of padding (hankel_zero_bytes)
  void* pair_state = nullptr;  // mac_pair launch cache
  // stride s >= 2 (reading R4b): the stride-1 inner plan over the input's s*s phases
  polyconv_plan_s* inner = nullptr;
  int Hq = 0, Wq = 0, Rq = 0, Sq = 0;
  void* xq = nullptr;
  void* wq = nullptr;
  size_t xq_bytes = 0, wq_bytes = 0;
  // workspace (lazy)
  void* wsA = nullptr;
  size_t wsA_bytes = 0;
  void* wsU = nullptr;
  size_t wsU_bytes = 0;
  bool device_checked = false;
  int num_sms = 148;
  cudaStream_t last_stream = nullptr;
  bool used = false;
  // polyconv_forward_host: plan-owned device copies of x, w, y (lazy)
  void* hx = nullptr;
  void* hw = nullptr;
  void* hy = nullptr;
  // ... and its copy/compute pipeline over batch chunks: sub-plans of nc and of the tail
  // images (same kernel), two copy streams, per-chunk events
  int hchunks = 0, hnc = 0;
  polyconv_plan_s* hsub = nullptr;
  polyconv_plan_s* hsub_tail = nullptr;
  cudaStream_t hs_in = nullptr, hs_out = nullptr;
  cudaEvent_t hev[3 * 16 + 2] = {};
  // polyconv_plan_set_timing_events: recorded around the MAC launch
  cudaEvent_t ev_start = nullptr;
  cudaEvent_t ev_stop = nullptr;
  char err[512];
};

namespace {

const long long kMaxElems = (1LL << 31) - 1;

void set_err(polyconv_plan_t p, const char* fmt_, const char* a = "", long long b = 0) {
  if (p) snprintf(p->err, sizeof(p->err), fmt_, a, b);
}

// AUTO for 1x1 layers (tools/layer_sweep.py, ResNet-50 at N=256): in place when the planes can be
// read by TMA; gathered for strided layers and for stride-1 planes that are not a multiple of 8
// pixels, except expansion layers (K > C) on planes under 64 pixels, where the 64-position tiles
// lose to mac_tc2 (7x7, 512 -> 2048: 282 vs 317 TFLOP/s).  POLYCONV_1X1_SMALL=0/1 forces the
// stride-1 gathered choice off/on.
bool mac1x1_auto(const Geom& g) {
  if (mac1x1_pitch(g) == 0 || g.sh > 1 || g.sw > 1) return true;
  const char* ev = getenv("POLYCONV_1X1_SMALL");
  if (ev) return ev[0] != '0';
  // planes of <= 64 pixels run four images per tile (mac_1x1 gimg) when K % 32 == 0: then the
  // expansion layers win too (ResNet-50 512->2048 7x7 N=256: 63.6 vs 80.9 us for mac_tc2; N=32:
  // 21.5 vs 31.8); one image per tile lost them to mac_tc2
  if ((long long)g.P * g.Q <= 64 && g.N > 1 && g.K % 32 == 0) return true;
  return !((long long)g.P * g.Q < 64 && g.K > g.C);
}

// mac_tc2 packing in-kernel (TC_FUSED) or by a pack launch (TC), measured per layer
// (tools/kernel_cmp.py, ResNet-50 N=256 and VGG-16 N=64): the fused packers rebuild each
// window once per 128-channel output tile and transpose nt + (R-1)*Wp positions per tile, so
// fusing pays only for one output tile and narrow planes (l2_3x3_128 699 vs 584 TFLOP/s,
// Wp = 30) and loses otherwise (VGG conv2_1, Wp = 114: 274 vs 605; conv4_2, K = 512: 818 vs
// 1019).  Kernels larger than 3x3 lose too (synthetic nets, N=32: 5x5 / 7x7, C=64 -> K=128 on
// 56x56 planes 565 vs 637 and 651 vs 779; on 8x8 planes 32.7 vs 35.6 and 41.3 vs 45.8).
// POLYCONV_FUSED_ANY restores the earlier rule (every bf16-io shape the tiling takes).
bool fused_pays(const Geom& g) {
  if (getenv("POLYCONV_FUSED_ANY")) return true;
  return g.K <= 128 && g.Wp <= 64 && g.R * g.S <= 9;
}

// FP32 math (method selection): the FFT solver (fft.cu, the paper's Eq. 13-15)
// against the direct FFMA MAC, measured per layer (tools/fp32_cmp.py, profiles/r02_fp32_cmp.jsonl).
// Direct work ~ R*S*P*Q per (n, k, c) against ~ L per (n, k, c) in the frequency domain, so the
// FFT pays when R*S*P*Q / L is large; at L >= 2048 its transforms run one CTA per SM and need a
// larger margin.  Wins: ResNet-50 l2/l3/l4 3x3 at N=256 (31/29/40 vs 26/26/7 TFLOP/s), VGG conv4-5
// (56 vs 28), the 5x5/7x7 sweep points on 56x56 (31 vs 28); losses kept direct: l1 3x3 on 56x56
// (12 vs 28), 1x1 layers on large planes.  POLYCONV_NO_FFT disables it.
bool fft_pays(const Geom& g) {
  if (getenv("POLYCONV_NO_FFT") || g.K < 16) return false;
  const FftTiling t = fft_tiling(g);
  if (!t.ok) return false;
  // r = taps x outputs per FFT bin.  Against the direct FFMA kernel (mac_fp32 with packed FFMA2,
  // round 2b), measured on all 71 FP32 layers (profiles/r03_fp32_cmp.jsonl, TFLOP/s FFT / FFMA):
  // the FFT wins only on short transforms -- L <= 256 (l4 3x3 40 / 32), L = 512 at stride 2
  // (l4 3x3 s2 9.7 / 9.4; l3 3x3 29 / 35 and A_h14_s1 25.5 / 26.8 lose), L = 1024 at stride 2
  // or with C*K >= 128K (l3 3x3 s2 12.8 / 10.1, VGG conv4 56 / 40; conv3_x 20 / 32 loses).
  const double r = (double)g.R * g.S * g.P * g.Q / t.L;
  if (r < 0.8 || g.N < 64) return false;  // every measured FFT win had N >= 64
  const bool s2 = g.sh > 1;
  if (t.L <= 256) return true;
  if (t.L <= 512) return s2;
  if (t.L <= 1024) return (s2 && r >= 1.5) || ((long long)g.C * g.K >= 131072 && r >= 4.0);
  return false;
}

// Resolve the MAC variant and fill the kernel-specific padded sizes.
polyconv_status_t resolve(polyconv_plan_t p) {
  Geom& g = p->g;
  int k = p->forced;
  const bool tc_math = p->math != POLYCONV_MATH_FP32_FMA;
  if (k == POLYCONV_KERNEL_AUTO || k == POLYCONV_KERNEL_TC_PAIR) p->pair = pair_tiling(g, p->fmt, p->io_bf16, p->num_sms);
  // 1x1: x is already the (MN-major) position operand when its planes have a 16-byte pitch;
  // other 1x1 layers gather their output lattice first (mac1x1_auto)
  // ... except wide-input 1x1 layers whose planes need that gather (H*W*2 bytes not a multiple
  // of 16): the pair kernel reads their NCHW planes directly (one tap, no halo) and skips the
  // gathered copy of C*H*W (tools/hk_1x1.sh, N=256: 1024->256 14x14 0.128 -> 0.077 ms,
  // 1024->512 14x14 0.159 -> 0.112; 256->1024 14x14 loses, 0.075 vs 0.091)
  if (k == POLYCONV_KERNEL_AUTO && p->math == POLYCONV_MATH_BF16 && p->io_bf16 && g.R == 1 && g.S == 1 &&
      g.sh == 1 && g.sw == 1 && g.ph == 0 && g.pw == 0 && mac1x1_pitch(g) != 0 && g.C >= 512 &&
      g.C >= 2 * g.K && !getenv("POLYCONV_NO_HANKEL")) {
    const HankelTiling h = hankel_tiling(g, p->fmt, p->num_sms, p->io_bf16);
    if (h.ok && (h.aligned || h.planes) && (long long)h.PT * h.NB >= 24) k = POLYCONV_KERNEL_TC_HANKEL;
  }
  if (k == POLYCONV_KERNEL_AUTO && mac1x1_supported(g, p->fmt, p->io_bf16) && !getenv("POLYCONV_NO_1X1") &&
      mac1x1_auto(g))
    k = POLYCONV_KERNEL_TC_1X1;
  // BF16 3x3 / 5x5 layers, stride 1 or 2, on even-width planes with C % 8 == 0 and at least one
  // third of a round of pair units (24): the persistent pair kernel fed straight from NCHW x (mac_hankel.cu).
  // Measured per layer against every other kernel (tools/kernel_cmp.py, profiles/r02_kcmp_*.jsonl):
  // it wins on ResNet-50 l1-l3 3x3 (incl. stride 2), VGG-16 conv1_2..conv5_3, the sweep's 3x3 and
  // 5x5 points; it loses on 7x7 kernels, odd-width planes (l4 7x7: general loader) and problems
  // under a third of a round of units (the synthetic nets at 4x4 / 8x8: 1-11 units; 14x14: 30).
  // The stem (7x7 stride 2, C = 3): its stride-1 phase convolution (reading R19: 12 virtual
  // channels, 4x4 taps) in 32-byte window rows (tools/hk_check.py stem).
  // TF32 (f32 I/O) takes the same kernel: against mac_tc2 with its pack (tools/kprof.py,
  // N=256, us) l1 3x3 151 vs 300, l2 121 vs 171, l3 127 vs 151, l4 119 vs 168, l2 s2 406 vs 554,
  // conv3_x N=32 33 vs 33.
  const bool hk_stem = g.sh == 2 && g.R == 7 && 4 * g.C <= 16 && p->io_bf16 && p->math == POLYCONV_MATH_BF16;
  if (k == POLYCONV_KERNEL_AUTO && (p->math == POLYCONV_MATH_BF16 || p->math == POLYCONV_MATH_TF32) && g.K >= 16 &&
      g.sh == g.sw && g.sh <= 2 && g.R == g.S && (g.R == 3 || g.R == 5 || hk_stem) && !getenv("POLYCONV_NO_HANKEL")) {
    const HankelTiling h = hankel_tiling(g, p->fmt, p->num_sms, p->io_bf16);
    // odd widths use the general (element-load) window loader: it still wins for wide 3x3
    // layers (ResNet-50 l4 7x7, C = K = 512: 596 vs 572 TFLOP/s for mac_tc2)
    const bool loader_ok = h.aligned || (g.R == 3 && g.C >= 256 && g.K >= 256);
    if (h.ok && loader_ok && (long long)h.PT * h.NB >= 24) k = POLYCONV_KERNEL_TC_HANKEL;
  }
  if (k == POLYCONV_KERNEL_AUTO) {
    // bf16, at most two rounds of pair tiles: one launch on CTA pairs with a resident filter
    // (its fixed startup wins on small problems); larger problems pipeline better in mac_tc2
    // (measured per layer: tools/layer_sweep.py). Below one full round of pair
    // tiles with bf16 I/O, the pack launch + mac_tc2 pipeline starts faster than either one-launch
    // kernel (tools/kernel_cmp.py synthnet, N=32, 3x3, TFLOP/s tc / pair / fused: 8x8 C=K=64
    // 9.8 / 7.8 / 8.7, 14x14 C=128 K=64 33.5 / 25.7 / 29.1; 5 of 6 such layers).
    const bool fused_ok = tc_math && g.K >= 16 && tc2_supported(g, p->fmt) && p->io_bf16 &&
                          !getenv("POLYCONV_NO_FUSED_DEFAULT") && fused_pays(g) &&
                          tc2_is_mx(tc2_tiling(g, p->fmt, p->io_bf16, p->num_sms, true, p->io_bf16));
    const bool small_tc = p->pair.ok && p->pair.num_tiles < p->num_sms / 2 && p->io_bf16 && tc_math &&
                          g.K >= 16 && tc2_supported(g, p->fmt) && !getenv("POLYCONV_SMALL_PAIR");
    if (tc_math && g.K >= 16 && p->pair.ok && p->pair.num_tiles <= 2 * p->pair.num_pairs && !small_tc &&
        !getenv("POLYCONV_NO_PAIR_DEFAULT"))
      k = POLYCONV_KERNEL_TC_PAIR;
    else if (small_tc)
      k = POLYCONV_KERNEL_TC;
    else if (fused_ok)
      k = POLYCONV_KERNEL_TC_FUSED;  // bf16 in/out: one launch, input packed in-kernel
    else if (tc_math)
      k = (g.K >= 16 && tc2_supported(g, p->fmt))  ? POLYCONV_KERNEL_TC
          : (g.K >= 16 && tc_supported(g, p->fmt)) ? POLYCONV_KERNEL_TC_PERTAP
                                                   : POLYCONV_KERNEL_THIN;
    else if (fft_pays(g))
      k = POLYCONV_KERNEL_FFT;
    else
      k = (g.K >= 16 && g.C * g.R * g.S >= 16 && fp32_tiling(g).smax > 0) ? POLYCONV_KERNEL_FP32
                                                                          : POLYCONV_KERNEL_THIN;
  }
  if ((k == POLYCONV_KERNEL_TC || k == POLYCONV_KERNEL_TC_FUSED) && (!tc_math || !tc2_supported(g, p->fmt)))
    return POLYCONV_STATUS_BAD_PARAM;
  if (k == POLYCONV_KERNEL_TC_PAIR && (!tc_math || !p->pair.ok)) return POLYCONV_STATUS_BAD_PARAM;
  if (k == POLYCONV_KERNEL_TC_1X1 && !mac1x1_supported(g, p->fmt, p->io_bf16)) return POLYCONV_STATUS_BAD_PARAM;
  if (k == POLYCONV_KERNEL_TC_HANKEL) {
    p->hk = hankel_tiling(g, p->fmt, p->num_sms, p->io_bf16);
    if (!tc_math || !p->hk.ok) return POLYCONV_STATUS_BAD_PARAM;
  }
  if (k == POLYCONV_KERNEL_FFT) {
    p->fft = fft_tiling(g);
    if (tc_math || !p->fft.ok) return POLYCONV_STATUS_BAD_PARAM;  // fp32 spectra: math FP32_FMA
  }
  if (k == POLYCONV_KERNEL_TC_PERTAP && (!tc_math || !tc_supported(g, p->fmt))) return POLYCONV_STATUS_BAD_PARAM;
  if (k == POLYCONV_KERNEL_FP32 && (tc_math || fp32_tiling(g).smax == 0)) return POLYCONV_STATUS_BAD_PARAM;
  p->kernel = k;
  if (k == POLYCONV_KERNEL_TC_PAIR) {
    g.Cp = p->pair.Cp;
    g.Kp = p->pair.NN;
  } else if (k == POLYCONV_KERNEL_TC_HANKEL) {
    g.Cp = p->hk.Cp;
    g.Kp = p->hk.Kp;
  } else if (k == POLYCONV_KERNEL_FFT) {
    g.Cp = g.C;
    g.Kp = g.K;
  } else if (k == POLYCONV_KERNEL_TC_1X1) {
    g.Cp = (g.C + 63) / 64 * 64;
    g.Kp = (g.K + 127) / 128 * 128;
  } else if (k == POLYCONV_KERNEL_TC || k == POLYCONV_KERNEL_TC_FUSED) {
    p->tc2 = tc2_tiling(g, p->fmt, p->io_bf16, p->num_sms, k == POLYCONV_KERNEL_TC_FUSED, p->io_bf16);
    g.Cp = (g.C + p->tc2.kc - 1) / p->tc2.kc * p->tc2.kc;
    g.Kp = (g.K + 127) / 128 * 128;
  } else if (k == POLYCONV_KERNEL_TC_PERTAP) {
    p->tc = tc_tiling(g, p->fmt, p->num_sms);
    g.Cp = (g.C + p->tc.kc - 1) / p->tc.kc * p->tc.kc;
    g.Kp = (g.K + p->tc.bn - 1) / p->tc.bn * p->tc.bn;
  } else if (k == POLYCONV_KERNEL_FP32) {
    p->f32 = fp32_tiling(g);
    g.Cp = (g.C + p->f32.cc - 1) / p->f32.cc * p->f32.cc;
    g.Kp = fp32_kp(g.K);
  } else {
    g.Cp = g.C;
    g.Kp = g.K;
  }
  const int eb = fmt_bytes(p->fmt);
  // TC packs the input on the fly (no input workspace); TC_PERTAP needs the
  // interleaved copy, FP32/THIN the planar one
  const size_t a_elems = k == POLYCONV_KERNEL_TC_1X1 ? (size_t)g.N * g.C * mac1x1_pitch(g)
                         : (k == POLYCONV_KERNEL_TC_FUSED || k == POLYCONV_KERNEL_TC_HANKEL || k == POLYCONV_KERNEL_FP32) ? 0
                         : (k == POLYCONV_KERNEL_TC || k == POLYCONV_KERNEL_TC_PERTAP || k == POLYCONV_KERNEL_TC_PAIR) ? (size_t)g.N * g.L_A * g.Cp
                                                                                       : (size_t)g.N * g.C * g.L_A;
  p->wsA_bytes = a_elems * eb;
  g.urep = 1;
  if (k == POLYCONV_KERNEL_TC || k == POLYCONV_KERNEL_TC_FUSED || k == POLYCONV_KERNEL_TC_PAIR) {
    const char* r = getenv("POLYCONV_FILTER_REP");  // experiments only
    g.urep = r ? atoi(r) : 1;  // tc_pair: replicas measured slower (more pack writes)
    if (g.urep < 1) g.urep = 1;
    if (g.urep > 64) g.urep = 64;
    if ((long long)g.urep * g.R * g.S * g.Kp >= (1LL << 31)) g.urep = 1;  // TMA row coordinate
  }
  p->wsU_bytes = (size_t)g.urep * g.R * g.S * g.Kp * g.Cp * eb;
  if (k == POLYCONV_KERNEL_FFT) {
    p->wsA_bytes = p->fft.x_bytes + p->fft.u_bytes + p->fft.y_bytes;
    p->wsU_bytes = p->fft.tw_bytes;
    p->fft_tw_ready = false;
  }
  return POLYCONV_STATUS_SUCCESS;
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

polyconv_status_t check_device(polyconv_plan_t p) {
  if (p->device_checked) return POLYCONV_STATUS_SUCCESS;
  cudaDeviceProp prop;
  cudaError_t e = cudaGetDeviceProperties(&prop, p->device);
  if (e != cudaSuccess) {
    set_err(p, "no CUDA device: %s", cudaGetErrorString(e));
    cudaGetLastError();
    return POLYCONV_STATUS_NOT_SUPPORTED;
  }
  if (prop.major != 10 || prop.minor != 0) {
    snprintf(p->err, sizeof(p->err), "device %d is sm_%d%d; this library is built for sm_100a only", p->device,
             prop.major, prop.minor);
    return POLYCONV_STATUS_NOT_SUPPORTED;
  }
  if (prop.multiProcessorCount != p->num_sms) {
    p->num_sms = prop.multiProcessorCount;
    resolve(p);
  }
  p->device_checked = true;
  return POLYCONV_STATUS_SUCCESS;
}

polyconv_status_t ensure_workspace(polyconv_plan_t p) {
  if (p->wsA && p->wsU) return POLYCONV_STATUS_SUCCESS;
  if (!p->wsA && cudaMalloc(&p->wsA, p->wsA_bytes ? p->wsA_bytes : 16) != cudaSuccess) {
    p->wsA = nullptr;
    set_err(p, "cudaMalloc of %s workspace failed (%lld bytes)", "input", (long long)p->wsA_bytes);
    cudaGetLastError();
    return POLYCONV_STATUS_ALLOC_FAILED;
  }
  if (!p->wsU && cudaMalloc(&p->wsU, p->wsU_bytes ? p->wsU_bytes : 16) != cudaSuccess) {
    p->wsU = nullptr;
    set_err(p, "cudaMalloc of %s workspace failed (%lld bytes)", "filter", (long long)p->wsU_bytes);
    cudaGetLastError();
    return POLYCONV_STATUS_ALLOC_FAILED;
  }
  return POLYCONV_STATUS_SUCCESS;
}

polyconv_status_t finish(polyconv_plan_t p, cudaError_t e, const char* what) {
  if (e != cudaSuccess) {
    snprintf(p->err, sizeof(p->err), "%s: %s", what, cudaGetErrorString(e));
    cudaGetLastError();
    return POLYCONV_STATUS_EXECUTION_FAILED;
  }
  return POLYCONV_STATUS_SUCCESS;
}

bool aligned(const void* ptr, size_t a) { return (reinterpret_cast<uintptr_t>(ptr) % a) == 0; }

#define PC_BEGIN(plan_)                                          \
  if (!(plan_)) return POLYCONV_STATUS_BAD_PARAM;                \
  (plan_)->err[0] = 0;                                           \
  DeviceGuard guard_((plan_)->device);                           \
  {                                                              \
    polyconv_status_t s_ = check_device(plan_);                  \
    if (s_ != POLYCONV_STATUS_SUCCESS) return s_;                \
  }

}  // namespace

extern "C" {

int polyconv_abi_version(void) { return POLYCONV_ABI_VERSION; }

const char* polyconv_status_string(polyconv_status_t s) {
  switch (s) {
    case POLYCONV_STATUS_SUCCESS: return "POLYCONV_STATUS_SUCCESS";
    case POLYCONV_STATUS_BAD_PARAM: return "POLYCONV_STATUS_BAD_PARAM";
    case POLYCONV_STATUS_NOT_SUPPORTED: return "POLYCONV_STATUS_NOT_SUPPORTED";
    case POLYCONV_STATUS_ALLOC_FAILED: return "POLYCONV_STATUS_ALLOC_FAILED";
    case POLYCONV_STATUS_EXECUTION_FAILED: return "POLYCONV_STATUS_EXECUTION_FAILED";
  }
  return "POLYCONV_STATUS_UNKNOWN";
}

const char* polyconv_last_error(polyconv_plan_t plan) { return plan ? plan->err : ""; }

polyconv_status_t polyconv_plan(polyconv_plan_t* plan, int N, int C, int H, int W, int K, int R, int S,
                                int sh, int sw, int ph, int pw, polyconv_dtype_t io_dtype,
                                polyconv_math_t math, int device) {
  if (!plan) return POLYCONV_STATUS_BAD_PARAM;
  *plan = nullptr;
  if (N < 1 || C < 1 || H < 1 || W < 1 || K < 1 || R < 1 || S < 1 || sh < 1 || sw < 1 || ph < 0 || pw < 0 ||
      device < 0)
    return POLYCONV_STATUS_BAD_PARAM;
  if (io_dtype != POLYCONV_F32 && io_dtype != POLYCONV_BF16) return POLYCONV_STATUS_BAD_PARAM;
  if (math != POLYCONV_MATH_FP32_FMA && math != POLYCONV_MATH_TF32 && math != POLYCONV_MATH_BF16)
    return POLYCONV_STATUS_BAD_PARAM;
  if (io_dtype == POLYCONV_BF16 && math != POLYCONV_MATH_BF16) return POLYCONV_STATUS_BAD_PARAM;
  const long long Hp = (long long)H + 2LL * ph, Wp = (long long)W + 2LL * pw;
  if (Hp < R || Wp < S) return POLYCONV_STATUS_BAD_PARAM;  // P < 1 or Q < 1
  const long long P = (Hp - R) / sh + 1, Q = (Wp - S) / sw + 1;
  // every tensor (and every packed operand) must index with < 2^31 elements
  if ((long long)N * C * H * W > kMaxElems || (long long)K * C * R * S > kMaxElems ||
      (long long)N * K * P * Q > kMaxElems || Hp * Wp > kMaxElems || (long long)N * C * Hp * Wp > kMaxElems ||
      (long long)N * Hp * Wp * ((C + 63) / 64 * 64) > kMaxElems)
    return POLYCONV_STATUS_NOT_SUPPORTED;

  polyconv_plan_t p = new (std::nothrow) polyconv_plan_s();
  if (!p) return POLYCONV_STATUS_ALLOC_FAILED;
  Geom& g = p->g;
  g.N = N; g.C = C; g.H = H; g.W = W; g.K = K; g.R = R; g.S = S;
  g.sh = sh; g.sw = sw; g.ph = ph; g.pw = pw;
  g.Hp = (int)Hp; g.Wp = (int)Wp; g.P = (int)P; g.Q = (int)Q;
  g.L_A = Hp * Wp;                          // Eq. 10
  g.L_U = (long long)(R - 1) * Wp + S;      // KernelSize, P.1378-1380 (Iw := Wp)
  g.M_ext = (P - 1) * sh * Wp + (Q - 1) * sw + 1;
  p->io_bf16 = io_dtype == POLYCONV_BF16;
  p->math = math;
  p->fmt = math == POLYCONV_MATH_BF16 ? FMT_BF16 : (math == POLYCONV_MATH_TF32 ? FMT_TF32 : FMT_F32);
  p->device = device;
  p->forced = POLYCONV_KERNEL_AUTO;
  p->err[0] = 0;
  if (resolve(p) != POLYCONV_STATUS_SUCCESS) {
    delete p;
    return POLYCONV_STATUS_BAD_PARAM;
  }
  // stride s >= 2 with large kernels: the s*s phases of the padded input become channels
  // and the convolution a stride-1 one of ceil(R/s) x ceil(S/s) kernels (polyphase.cu,
  // reading R4b), so only the stride lattice is computed.  Measured per layer
  // (tools/layer_sweep.py): the ResNet-50 7x7/s2 stem 14 -> 73 TFLOP/s; 3x3/s2 layers ran
  // slower through their inner plans (phase planes of odd width have no TMA view), so the
  // rule is R, S >= 5 (POLYCONV_POLYPHASE=1 forces it for any R, S >= 2, =0 disables it).
  const char* pp_env = getenv("POLYCONV_POLYPHASE");
  const int pp_min = pp_env ? (atoi(pp_env) == 0 ? 1 << 30 : 2) : 5;
  if (sh == sw && sh >= 2 && R >= pp_min && S >= pp_min && p->kernel != POLYCONV_KERNEL_TC_HANKEL) {
    const int s = sh;
    const int Rq = (R + s - 1) / s, Sq = (S + s - 1) / s;
    const long long Hq = P + Rq - 1, Wq = Q + Sq - 1;
    const long long Cq = (long long)s * s * C;
    polyconv_plan_t in = nullptr;
    if (Cq <= kMaxElems && (long long)N * Cq * Hq * Wq <= kMaxElems &&
        polyconv_plan(&in, N, (int)Cq, (int)Hq, (int)Wq, K, Rq, Sq, 1, 1, 0, 0, io_dtype, math, device) ==
            POLYCONV_STATUS_SUCCESS) {
      p->inner = in;
      p->Hq = (int)Hq; p->Wq = (int)Wq; p->Rq = Rq; p->Sq = Sq;
      const size_t eb = p->io_bf16 ? 2 : 4;
      p->xq_bytes = eb * (size_t)N * Cq * Hq * Wq;
      p->wq_bytes = eb * (size_t)K * Cq * Rq * Sq;
    }
  }
  *plan = p;
  return POLYCONV_STATUS_SUCCESS;
}

polyconv_status_t polyconv_plan_set_kernel(polyconv_plan_t p, polyconv_kernel_t kernel) {
  if (!p) return POLYCONV_STATUS_BAD_PARAM;
  if (p->inner) {
    // the forward runs the inner (phase) plan; this plan keeps the same choice for its
    // polyconv_pack_* layouts.  Both must accept the kernel.
    const int old_inner = p->inner->forced;
    polyconv_status_t si = polyconv_plan_set_kernel(p->inner, kernel);
    if (si != POLYCONV_STATUS_SUCCESS) return si;
    polyconv_plan_s* in = p->inner;
    p->inner = nullptr;
    polyconv_status_t so = polyconv_plan_set_kernel(p, kernel);
    p->inner = in;
    if (so != POLYCONV_STATUS_SUCCESS) polyconv_plan_set_kernel(in, (polyconv_kernel_t)old_inner);
    return so;
  }
  if (kernel < POLYCONV_KERNEL_AUTO || kernel > POLYCONV_KERNEL_FFT) return POLYCONV_STATUS_BAD_PARAM;
  const int old = p->forced;
  p->forced = kernel;
  if (resolve(p) != POLYCONV_STATUS_SUCCESS) {
    p->forced = old;
    resolve(p);
    return POLYCONV_STATUS_BAD_PARAM;
  }
  // workspace sizes (and the grid the pack counter counts) may have changed
  if (p->pair_state) { pair_state_free(p->pair_state); p->pair_state = nullptr; }
  if (p->wsA) { cudaFree(p->wsA); p->wsA = nullptr; }
  if (p->wsU) { cudaFree(p->wsU); p->wsU = nullptr; }
  // the forward_host pipeline's sub-plans carry the old kernel: rebuilt on the next call
  if (p->hsub) { polyconv_destroy(p->hsub); p->hsub = nullptr; }
  if (p->hsub_tail) { polyconv_destroy(p->hsub_tail); p->hsub_tail = nullptr; }
  p->hchunks = 0;
  return POLYCONV_STATUS_SUCCESS;
}

polyconv_status_t polyconv_output_dims(polyconv_plan_t p, int* P, int* Q) {
  if (!p || !P || !Q) return POLYCONV_STATUS_BAD_PARAM;
  *P = p->g.P;
  *Q = p->g.Q;
  return POLYCONV_STATUS_SUCCESS;
}

polyconv_status_t polyconv_plan_info(polyconv_plan_t p, polyconv_info_t* info) {
  if (!p || !info) return POLYCONV_STATUS_BAD_PARAM;
  const Geom& g = p->g;
  info->N = g.N; info->C = g.C; info->H = g.H; info->W = g.W; info->K = g.K; info->R = g.R; info->S = g.S;
  info->sh = g.sh; info->sw = g.sw; info->ph = g.ph; info->pw = g.pw;
  info->P = g.P; info->Q = g.Q; info->Hp = g.Hp; info->Wp = g.Wp;
  info->L_A = g.L_A; info->L_U = g.L_U; info->Cp = g.Cp; info->Kp = g.Kp;
  info->kernel = p->kernel;
  switch (p->kernel) {
    case POLYCONV_KERNEL_TC:  // tile = positions x output channels
    case POLYCONV_KERNEL_TC_FUSED:
      info->tile_m = p->tc2.nt; info->tile_n = 128; info->stages = p->tc2.a_stages;
      info->launches = p->kernel == POLYCONV_KERNEL_TC_FUSED ? 1 : 2; break;
    case POLYCONV_KERNEL_TC_PAIR:  // pair tile = 256 positions x NN output channels
      info->tile_m = 256; info->tile_n = p->pair.NN; info->stages = p->pair.ring;
      info->launches = p->pair.split ? 2 : 1; break;
    case POLYCONV_KERNEL_FFT:  // one FFT length L per polynomial; tile = the contraction's 32 x 64
      info->tile_m = p->fft.L; info->tile_n = 64; info->stages = p->fft.F; info->launches = 4; break;
    case POLYCONV_KERNEL_TC_HANKEL:  // pair item = 256*T positions x NN output channels
      info->tile_m = 256 * p->hk.T; info->tile_n = p->hk.NN; info->stages = p->hk.wslots;
      info->launches = 2; break;
    case POLYCONV_KERNEL_TC_1X1:  // tile = 128 output channels x up to 256 positions
      info->tile_m = 128; info->tile_n = g.P * g.Q >= 256 ? 256 : (g.P * g.Q + 63) / 64 * 64; info->stages = 0;
      info->launches = mac1x1_pitch(g) ? 3 : 2; break;
    case POLYCONV_KERNEL_TC_PERTAP:
      info->tile_m = p->tc.bm; info->tile_n = p->tc.bn; info->stages = p->tc.stages; info->launches = 2; break;
    case POLYCONV_KERNEL_FP32:
      info->tile_m = 256; info->tile_n = 64; info->stages = 1; info->launches = 3; break;
    default:
      info->tile_m = 1; info->tile_n = 1; info->stages = 1; info->launches = 3; break;
  }
  info->workspace_bytes = p->wsA_bytes + p->wsU_bytes;
  if (p->inner) {  // the forward runs the inner (stride-1, phase) plan: its kernel and tiling;
                   // Cp/Kp stay this plan's (they describe the polyconv_pack_* layouts)
    polyconv_info_t ii;
    polyconv_plan_info(p->inner, &ii);
    info->kernel = ii.kernel; info->tile_m = ii.tile_m; info->tile_n = ii.tile_n; info->stages = ii.stages;
    info->launches = ii.launches + 2;
    info->workspace_bytes = ii.workspace_bytes + p->xq_bytes + p->wq_bytes;
  }
  return POLYCONV_STATUS_SUCCESS;
}

// a3 (tap-major filter, one small launch), then a2 + a4 + a5 in the persistent pair kernel,
// which reads x directly and follows the pack as a programmatic dependent; its epilogue stores
// the plan's K channels at channel offset koff of each of the nys outputs [N][ktot][P][Q]
static polyconv_status_t forward_hankel(polyconv_plan_t p, const void* x, const void* w, void* const* ys, int nys,
                                        int ktot, int koff, cudaStream_t st) {
  const Geom& g = p->g;
  cudaError_t e;
  if (!p->hkzero) {
    const size_t zb = hankel_zero_bytes(g);
    if (cudaMalloc(&p->hkzero, zb) != cudaSuccess || cudaMemsetAsync(p->hkzero, 0, zb, st) != cudaSuccess) {
      cudaGetLastError();
      if (p->hkzero) cudaFree(p->hkzero);
      p->hkzero = nullptr;
      set_err(p, "cudaMalloc of the %s failed", "zero buffer");
      return POLYCONV_STATUS_ALLOC_FAILED;
    }
  }
  if (p->ev_start) cudaEventRecord(p->ev_start, st);
  if (p->hk.phase)
    e = launch_pack_filter_phase(g, w, p->wsU, p->hk.eR, p->hk.eS, p->hk.eph, p->hk.epw, g.Kp, g.Cp, st);
  else
    e = launch_pack_filter_tapmajor(g, w, p->io_bf16, p->wsU, p->fmt, g.Kp, g.Cp, st);
  if (e != cudaSuccess) return finish(p, e, "pack_filter");
  e = launch_mac_hankel(g, p->hk, p->fmt, x, p->io_bf16, p->wsU, ys, nys, ktot, koff, p->hkzero, st, p->err,
                        sizeof(p->err));
  if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
  if (e == cudaErrorNotSupported) return POLYCONV_STATUS_NOT_SUPPORTED;  // (the filter pack is harmless)
  return finish(p, e, "mac_hankel");
}

polyconv_status_t polyconv_forward_scatter(polyconv_plan_t p, const void* x, const void* w, void* const* ys,
                                           int n_out, int k_total, int k_offset, void* stream) {
  if (!p || !x || !w || !ys || n_out < 1 || n_out > 8 || k_offset < 0 || k_total < k_offset + p->g.K)
    return POLYCONV_STATUS_BAD_PARAM;
  if (!aligned(x, 16) || !aligned(w, 16)) return POLYCONV_STATUS_NOT_SUPPORTED;
  for (int o = 0; o < n_out; ++o) {
    if (!ys[o] || ys[o] == x || ys[o] == w) return POLYCONV_STATUS_BAD_PARAM;
    if (!aligned(ys[o], 16)) return POLYCONV_STATUS_NOT_SUPPORTED;
  }
  if (p->kernel != POLYCONV_KERNEL_TC_HANKEL || p->inner) {
    set_err(p, "forward_scatter: the %s kernel does not store to peers", "plan's");
    return POLYCONV_STATUS_NOT_SUPPORTED;
  }
  PC_BEGIN(p);
  polyconv_status_t s = ensure_workspace(p);
  if (s != POLYCONV_STATUS_SUCCESS) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  p->last_stream = st;
  p->used = true;
  return forward_hankel(p, x, w, ys, n_out, k_total, k_offset, st);
}

polyconv_status_t polyconv_forward(polyconv_plan_t p, const void* x, const void* w, void* y, void* stream) {
  if (!p) return POLYCONV_STATUS_BAD_PARAM;
  if (!x || !w || !y || x == y || w == y) return POLYCONV_STATUS_BAD_PARAM;
  if (!aligned(x, 16) || !aligned(w, 16) || !aligned(y, 16)) return POLYCONV_STATUS_NOT_SUPPORTED;
  PC_BEGIN(p);
  polyconv_status_t s = p->inner ? POLYCONV_STATUS_SUCCESS : ensure_workspace(p);  // phase plans: inner's
  if (s != POLYCONV_STATUS_SUCCESS) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  p->last_stream = st;
  p->used = true;
  const Geom& g = p->g;
  cudaError_t e;
  if (p->inner) {
    // stride s: phase split of x and w (polyphase.cu), then the stride-1 inner plan
    if ((!p->xq && cudaMalloc(&p->xq, p->xq_bytes) != cudaSuccess) ||
        (!p->wq && cudaMalloc(&p->wq, p->wq_bytes) != cudaSuccess)) {
      cudaGetLastError();
      set_err(p, "cudaMalloc of the %s failed", "phase buffers");
      return POLYCONV_STATUS_ALLOC_FAILED;
    }
    if (p->ev_start) cudaEventRecord(p->ev_start, st);
    e = launch_polyphase(g, p->Hq, p->Wq, p->Rq, p->Sq, x, w, p->xq, p->wq, p->io_bf16, st);
    if (e != cudaSuccess) return finish(p, e, "polyphase");
    polyconv_status_t si = polyconv_forward(p->inner, p->xq, p->wq, y, stream);
    if (si != POLYCONV_STATUS_SUCCESS) {
      snprintf(p->err, sizeof(p->err), "inner (phase) plan: %s", polyconv_last_error(p->inner));
      return si;
    }
    if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
    return POLYCONV_STATUS_SUCCESS;
  }
  if (p->kernel == POLYCONV_KERNEL_TC) {
    // a2 + a3 in one pack launch (interleaved input rows, tap-major filter), then the
    // windowed tensor-core MAC (a4+a5) as its programmatic dependent
    if (p->ev_start) cudaEventRecord(p->ev_start, st);
    e = launch_pack_both_interleaved(g, x, w, p->io_bf16, p->wsA, p->wsU, p->fmt, st);
    if (e != cudaSuccess) return finish(p, e, "pack");
    e = launch_mac_tc2(g, p->tc2, p->fmt, x, p->io_bf16, p->wsA, p->wsU, y, p->io_bf16, true, st, p->err,
                       sizeof(p->err));
    if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
    return finish(p, e, "mac_tc");
  }
  if (p->kernel == POLYCONV_KERNEL_FFT) {
    // the paper's solver (Eq. 13-15): FFT of every A_{n,c} and U_{k,c}, per-frequency
    // channel contraction, inverse FFT + Eq. 12 extraction (fft.cu)
    if (!p->fft_tw_ready) {
      e = launch_fft_twiddles(p->fft, p->wsU, st);
      if (e != cudaSuccess) return finish(p, e, "fft_twiddles");
      p->fft_tw_ready = true;
    }
    if (p->ev_start) cudaEventRecord(p->ev_start, st);
    e = launch_fft_conv(g, p->fft, x, w, p->io_bf16, p->wsA, p->wsU, y, st);
    if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
    return finish(p, e, "fft_conv");
  }
  if (p->kernel == POLYCONV_KERNEL_TC_HANKEL) return forward_hankel(p, x, w, &y, 1, g.K, 0, st);
  if (p->kernel == POLYCONV_KERNEL_TC_1X1) {
    // a3 (the [1][Kp][Cp] filter), then the GEMM over the NCHW planes as its programmatic dependent
    if (p->ev_start) cudaEventRecord(p->ev_start, st);
    const bool gather = mac1x1_pitch(g) != 0;  // stride or plane size: gather the output lattice first
    if (gather) {
      e = launch_gather1x1(g, x, p->wsA, st);
      if (e != cudaSuccess) return finish(p, e, "gather1x1");
    }
    e = launch_pack_filter_tapmajor(g, w, p->io_bf16, p->wsU, p->fmt, g.Kp, g.Cp, st);
    if (e != cudaSuccess) return finish(p, e, "pack_filter");
    e = launch_mac_1x1(g, gather ? p->wsA : x, p->wsU, g.Kp, g.Cp, y, p->num_sms, st, p->err, sizeof(p->err));
    if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
    return finish(p, e, "mac_1x1");
  }
  if (p->kernel == POLYCONV_KERNEL_TC_PAIR) {
    // a2 + a3 by the pack grid (pair_pack_kernel), then a4 + a5 on CTA pairs as its
    // programmatic dependent launch (pair-local synchronisation only)
    if (p->ev_start) cudaEventRecord(p->ev_start, st);
    if (!p->pair_state) p->pair_state = pair_state_new();
    e = launch_mac_pair(g, p->pair, x, w, p->io_bf16, p->wsA, p->wsU, y, st, p->err, sizeof(p->err),
                        p->pair_state);
    if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
    return finish(p, e, "mac_pair");
  }
  if (p->kernel == POLYCONV_KERNEL_TC_FUSED) {
    // a3 (tap-major filter, one small launch), then a2 (packer warps) + a4 + a5 in mac_tc2 as
    // its programmatic dependent.  (The filter used to be packed inside the MAC grid, whose
    // CTAs met on a plan-owned counter: that needed the whole grid co-resident and broke on
    // CUDA-graph replay.)
    if (p->ev_start) cudaEventRecord(p->ev_start, st);
    e = launch_pack_filter_tapmajor(g, w, p->io_bf16, p->wsU, p->fmt, g.Kp, g.Cp, st);
    if (e != cudaSuccess) return finish(p, e, "pack_filter");
    e = launch_mac_tc2(g, p->tc2, p->fmt, x, p->io_bf16, nullptr, p->wsU, y, p->io_bf16, true, st, p->err,
                       sizeof(p->err));
    if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
    return finish(p, e, "mac_tc_fused");
  }
  if (p->kernel == POLYCONV_KERNEL_TC_PERTAP) {
    // a2 + a3 in one launch (interleaved A, tap-major U), then the MAC (a4+a5)
    e = launch_pack_both_interleaved(g, x, w, p->io_bf16, p->wsA, p->wsU, p->fmt, st);
    if (e != cudaSuccess) return finish(p, e, "pack");
    if (p->ev_start) cudaEventRecord(p->ev_start, st);
    e = launch_mac_tc(g, p->tc, p->fmt, p->wsA, p->wsU, y, p->io_bf16, st, p->err, sizeof(p->err));
    if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
    return finish(p, e, "mac_tc_pertap");
  }
  if (p->kernel == POLYCONV_KERNEL_FP32) {
    // a3 (tap-major fp32 filter), then a2 + a4 + a5 in the FFMA kernel, which reads x directly
    if (p->ev_start) cudaEventRecord(p->ev_start, st);
    e = launch_pack_filter_tapmajor(g, w, p->io_bf16, p->wsU, p->fmt, g.Kp, g.Cp, st);
    if (e != cudaSuccess) return finish(p, e, "pack_filter");
    e = launch_mac_fp32(g, p->f32, x, p->io_bf16, (const float*)p->wsU, g.Kp, g.Cp, y, st);
    if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
    return finish(p, e, "mac_fp32");
  }
  e = launch_pack_input_planar(g, x, p->io_bf16, p->wsA, p->fmt, st);
  if (e != cudaSuccess) return finish(p, e, "pack_input");
  e = launch_pack_filter_tapmajor(g, w, p->io_bf16, p->wsU, p->fmt, g.Kp, g.Cp, st);
  if (e != cudaSuccess) return finish(p, e, "pack_filter");
  if (p->ev_start) cudaEventRecord(p->ev_start, st);
  e = launch_mac_thin(g, p->wsA, p->wsU, g.Kp, g.Cp, p->fmt, y, p->io_bf16, st);
  if (p->ev_stop) cudaEventRecord(p->ev_stop, st);
  return finish(p, e, "mac_thin");
}

// forward_host pipeline setup (lazy): G = POLYCONV_HOST_CHUNKS (default 4, 1 = off) chunks of
// ceil(N/G) images, each a forward of a sub-plan forced to this plan's kernel, so every image
// gets the arithmetic of a plain forward (the kernels are batch-shard invariant).  Not for
// polyphase plans or when the timing hook is set; false = the unpipelined path.
static bool host_pipeline(polyconv_plan_t p) {
  if (p->hchunks < 0) return false;
  if (p->hchunks > 0) return true;
  p->hchunks = -1;
  const char* ev = getenv("POLYCONV_HOST_CHUNKS");
  int G = ev ? atoi(ev) : 4;
  G = std::min(std::min(G, 16), p->g.N);
  if (G < 2 || p->inner || p->ev_start) return false;
  const int nc = (p->g.N + G - 1) / G;
  G = (p->g.N + nc - 1) / nc;
  const int tail = p->g.N - (G - 1) * nc;
  const Geom& g = p->g;
  const polyconv_dtype_t io = p->io_bf16 ? POLYCONV_BF16 : POLYCONV_F32;
  const polyconv_math_t m = static_cast<polyconv_math_t>(p->math);
  auto make = [&](int n, polyconv_plan_s** out) {
    if (polyconv_plan(out, n, g.C, g.H, g.W, g.K, g.R, g.S, g.sh, g.sw, g.ph, g.pw, io, m, p->device) !=
        POLYCONV_STATUS_SUCCESS)
      return false;
    return polyconv_plan_set_kernel(*out, static_cast<polyconv_kernel_t>(p->kernel)) == POLYCONV_STATUS_SUCCESS;
  };
  bool ok = make(nc, &p->hsub) && (tail == nc || make(tail, &p->hsub_tail));
  DeviceGuard guard(p->device);
  ok = ok && (p->hs_in || cudaStreamCreateWithFlags(&p->hs_in, cudaStreamNonBlocking) == cudaSuccess) &&
       (p->hs_out || cudaStreamCreateWithFlags(&p->hs_out, cudaStreamNonBlocking) == cudaSuccess);
  for (int i = 0; ok && i < 2 + 3 * G; ++i)
    ok = p->hev[i] || cudaEventCreateWithFlags(&p->hev[i], cudaEventDisableTiming) == cudaSuccess;
  if (!ok) {
    cudaGetLastError();
    return false;  // resources stay owned by the plan and are freed by polyconv_destroy
  }
  p->hchunks = G;
  p->hnc = nc;
  return true;
}

polyconv_status_t polyconv_forward_host(polyconv_plan_t p, const void* x, const void* w, void* y, void* stream) {
  if (!p) return POLYCONV_STATUS_BAD_PARAM;
  if (!x || !w || !y || x == y || w == y) return POLYCONV_STATUS_BAD_PARAM;
  PC_BEGIN(p);
  const Geom& g = p->g;
  const size_t eb = p->io_bf16 ? 2 : 4;
  const size_t xb = eb * g.N * g.C * g.H * g.W, wb = eb * g.K * g.C * g.R * g.S, yb = eb * g.N * g.K * g.P * g.Q;
  if (!p->hx || !p->hw || !p->hy) {
    if ((!p->hx && cudaMalloc(&p->hx, xb) != cudaSuccess) || (!p->hw && cudaMalloc(&p->hw, wb) != cudaSuccess) ||
        (!p->hy && cudaMalloc(&p->hy, yb) != cudaSuccess)) {
      cudaGetLastError();
      set_err(p, "cudaMalloc of %s buffers failed", "host-path");
      return POLYCONV_STATUS_ALLOC_FAILED;
    }
  }
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (host_pipeline(p)) {
    // chunk i: H2D of its images on hs_in -> forward on `stream` -> D2H on hs_out, so the two
    // copy directions and the MAC of neighbouring chunks overlap; `stream` waits for the last
    // D2H, so synchronising it covers the whole call
    const int G = p->hchunks, nc = p->hnc;
    const size_t xi = xb / g.N, yi = yb / g.N;
    cudaEvent_t* ev = p->hev;  // [0] entry, [1] done, [2 + 3i] in, [3 + 3i] computed
    cudaError_t e = cudaEventRecord(ev[0], st);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(p->hs_in, ev[0], 0);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(p->hs_out, ev[0], 0);
    if (e == cudaSuccess) e = cudaMemcpyAsync(p->hw, w, wb, cudaMemcpyHostToDevice, p->hs_in);
    for (int i = 0; i < G && e == cudaSuccess; ++i) {
      const int n0 = i * nc, n = std::min(nc, g.N - n0);
      e = cudaMemcpyAsync(static_cast<char*>(p->hx) + n0 * xi, static_cast<const char*>(x) + n0 * xi, n * xi,
                          cudaMemcpyHostToDevice, p->hs_in);
      if (e == cudaSuccess) e = cudaEventRecord(ev[2 + 3 * i], p->hs_in);
    }
    if (e != cudaSuccess) return finish(p, e, "forward_host H2D");
    for (int i = 0; i < G; ++i) {
      const int n0 = i * nc, n = std::min(nc, g.N - n0);
      if ((e = cudaStreamWaitEvent(st, ev[2 + 3 * i], 0)) != cudaSuccess) return finish(p, e, "forward_host wait");
      polyconv_plan_s* sp = n == nc ? p->hsub : p->hsub_tail;
      polyconv_status_t s = polyconv_forward(sp, static_cast<char*>(p->hx) + n0 * xi, p->hw,
                                             static_cast<char*>(p->hy) + n0 * yi, stream);
      if (s != POLYCONV_STATUS_SUCCESS) {
        snprintf(p->err, sizeof(p->err), "forward_host chunk %d: %s", i, sp->err);
        return s;
      }
      e = cudaEventRecord(ev[3 + 3 * i], st);
      if (e == cudaSuccess) e = cudaStreamWaitEvent(p->hs_out, ev[3 + 3 * i], 0);
      if (e == cudaSuccess)
        e = cudaMemcpyAsync(static_cast<char*>(y) + n0 * yi, static_cast<char*>(p->hy) + n0 * yi, n * yi,
                            cudaMemcpyDeviceToHost, p->hs_out);
      if (e != cudaSuccess) return finish(p, e, "forward_host D2H");
    }
    e = cudaEventRecord(ev[1], p->hs_out);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(st, ev[1], 0);
    return finish(p, e, "forward_host join");
  }
  cudaError_t e = cudaMemcpyAsync(p->hx, x, xb, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync(p->hw, w, wb, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) return finish(p, e, "forward_host H2D");
  polyconv_status_t s = polyconv_forward(p, p->hx, p->hw, p->hy, stream);
  if (s != POLYCONV_STATUS_SUCCESS) return s;
  return finish(p, cudaMemcpyAsync(y, p->hy, yb, cudaMemcpyDeviceToHost, st), "forward_host D2H");
}

polyconv_status_t polyconv_plan_set_timing_events(polyconv_plan_t p, void* start_event, void* stop_event) {
  if (!p || (!start_event) != (!stop_event)) return POLYCONV_STATUS_BAD_PARAM;
  p->ev_start = static_cast<cudaEvent_t>(start_event);
  p->ev_stop = static_cast<cudaEvent_t>(stop_event);
  return POLYCONV_STATUS_SUCCESS;
}

polyconv_status_t polyconv_packed_bytes(polyconv_plan_t p, int which, polyconv_layout_t layout, size_t* bytes) {
  if (!p || !bytes || (which != 0 && which != 1)) return POLYCONV_STATUS_BAD_PARAM;
  if (layout != POLYCONV_LAYOUT_PLANAR && layout != POLYCONV_LAYOUT_INTERLEAVED) return POLYCONV_STATUS_BAD_PARAM;
  const Geom& g = p->g;
  const size_t eb = (size_t)fmt_bytes(p->fmt);
  if (which == 0)
    *bytes = eb * (layout == POLYCONV_LAYOUT_PLANAR ? (size_t)g.N * g.C * g.L_A : (size_t)g.N * g.L_A * g.Cp);
  else
    *bytes = eb * (layout == POLYCONV_LAYOUT_PLANAR ? (size_t)g.K * g.C * g.L_U : (size_t)g.R * g.S * g.Kp * g.Cp);
  return POLYCONV_STATUS_SUCCESS;
}

polyconv_status_t polyconv_pack_input(polyconv_plan_t p, const void* x, void* dst, polyconv_layout_t layout,
                                      void* stream) {
  if (!p || !x || !dst) return POLYCONV_STATUS_BAD_PARAM;
  if (layout != POLYCONV_LAYOUT_PLANAR && layout != POLYCONV_LAYOUT_INTERLEAVED) return POLYCONV_STATUS_BAD_PARAM;
  if (!aligned(x, 16) || !aligned(dst, 16)) return POLYCONV_STATUS_NOT_SUPPORTED;
  PC_BEGIN(p);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  p->last_stream = st;
  p->used = true;
  cudaError_t e = layout == POLYCONV_LAYOUT_PLANAR
                      ? launch_pack_input_planar(p->g, x, p->io_bf16, dst, p->fmt, st)
                      : launch_pack_input_interleaved(p->g, x, p->io_bf16, dst, p->fmt, st);
  return finish(p, e, "pack_input");
}

polyconv_status_t polyconv_pack_filter(polyconv_plan_t p, const void* w, void* dst, polyconv_layout_t layout,
                                       void* stream) {
  if (!p || !w || !dst) return POLYCONV_STATUS_BAD_PARAM;
  if (layout != POLYCONV_LAYOUT_PLANAR && layout != POLYCONV_LAYOUT_INTERLEAVED) return POLYCONV_STATUS_BAD_PARAM;
  if (!aligned(w, 16) || !aligned(dst, 16)) return POLYCONV_STATUS_NOT_SUPPORTED;
  PC_BEGIN(p);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  p->last_stream = st;
  p->used = true;
  Geom g1 = p->g;
  g1.urep = 1;  // the caller's buffer holds one copy
  cudaError_t e = layout == POLYCONV_LAYOUT_PLANAR
                      ? launch_pack_filter_planar(g1, w, p->io_bf16, dst, p->fmt, st)
                      : launch_pack_filter_tapmajor(g1, w, p->io_bf16, dst, p->fmt, g1.Kp, g1.Cp, st);
  return finish(p, e, "pack_filter");
}

polyconv_status_t polyconv_extract(polyconv_plan_t p, const float* coeffs, void* y, void* stream) {
  if (!p || !coeffs || !y) return POLYCONV_STATUS_BAD_PARAM;
  if (!aligned(coeffs, 4) || !aligned(y, 16)) return POLYCONV_STATUS_NOT_SUPPORTED;
  PC_BEGIN(p);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  p->last_stream = st;
  p->used = true;
  return finish(p, launch_extract(p->g, coeffs, y, p->io_bf16, st), "extract");
}

polyconv_status_t polyconv_destroy(polyconv_plan_t p) {
  if (!p) return POLYCONV_STATUS_SUCCESS;
  polyconv_status_t s = POLYCONV_STATUS_SUCCESS;
  if (p->used || p->wsA || p->wsU || p->hx || p->hw || p->hy || p->hkzero) {
    DeviceGuard guard(p->device);
    if (p->used && cudaStreamSynchronize(p->last_stream) != cudaSuccess) {
      cudaGetLastError();
      s = POLYCONV_STATUS_EXECUTION_FAILED;
    }
    if (p->wsA) cudaFree(p->wsA);
    if (p->wsU) cudaFree(p->wsU);
    if (p->hx) cudaFree(p->hx);
    if (p->hw) cudaFree(p->hw);
    if (p->hy) cudaFree(p->hy);
    if (p->hkzero) cudaFree(p->hkzero);
  }
  if (p->pair_state) pair_state_free(p->pair_state);
  if (p->hsub && polyconv_destroy(p->hsub) != POLYCONV_STATUS_SUCCESS) s = POLYCONV_STATUS_EXECUTION_FAILED;
  if (p->hsub_tail && polyconv_destroy(p->hsub_tail) != POLYCONV_STATUS_SUCCESS) s = POLYCONV_STATUS_EXECUTION_FAILED;
  if (p->hs_in || p->hs_out || p->hev[0]) {
    DeviceGuard guard(p->device);
    for (cudaEvent_t e : p->hev)
      if (e) cudaEventDestroy(e);
    if (p->hs_in) cudaStreamDestroy(p->hs_in);
    if (p->hs_out) cudaStreamDestroy(p->hs_out);
  }
  if (p->inner) {
    if (polyconv_destroy(p->inner) != POLYCONV_STATUS_SUCCESS) s = POLYCONV_STATUS_EXECUTION_FAILED;
    DeviceGuard guard(p->device);
    if (p->xq) cudaFree(p->xq);
    if (p->wq) cudaFree(p->wq);
  }
  delete p;
  return s;
}

}  // extern "C"
