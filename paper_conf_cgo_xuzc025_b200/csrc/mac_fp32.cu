// mac_fp32.cu — a2 + a4 + a5 on the FP32 SIMT pipe (math FP32_FMA, the 1e-5 path), fed straight
// from the NCHW input (no packed copy of x).
//
// What it computes: the coefficient MAC
//   p_{n,k}[m] = sum_c sum_{i,j} A_{n,c}[m - e(i,j)] U_{k,c}[e(i,j)]
// (P.965; the naive product of §2.3, P.1021-1025; channel sum P.1350-1352) at the Eq. 12
// extraction degrees, each tap's operand a shifted window of the input polynomial (P.404-437).
// The input polynomial is the concatenated-batch layout of mac_hankel (reading R16):
//   A_c[q] = x[n][c][h][w] at q = (n*HS + ph + h)*pitch + pw + w, zero elsewhere,
// with pitch = W + pw (adjacent rows share their zero columns) and HS = H + ph (adjacent images
// share their zero rows), so only (H + ph)(W + pw) positions per image are computed (conv3_x:
// 841 for 784 outputs; the per-image padded planes of round 1 computed 1024).  Output
// (n, oh, ow) is position (n*HS + sh*oh)*pitch + sw*ow; tap (i, j) of it reads A_c at
// + pitch*i + j (reading R4 for the stride).
//
// Tiling: a CTA computes 256 consecutive positions x 32 output channels (4 warps; warp w owns
// 8 channels, lane l the 8 positions l + 32b), 8 x 8 fp32 accumulators per thread.  Per chunk
// of CC input channels it stages, double-buffered with cp.async, the union window
// A_c[m0, m0 + 256 + (R-1)*pitch + S - 1) of each channel (decoded from x once per position)
// and the CC x R*S x 32 filter coefficients (tap-major pack, a3).  Inner step per (channel,
// tap): 8 conflict-free LDS.32 of the window (32 consecutive positions per instruction), two
// broadcast LDS.128 of the filter, 64 FFMA.  Small tiles (256 x 32) keep the grid at several
// CTAs per SM, so the work per SM is balanced to a few percent (conv3_x: 424 CTAs).
#include <cstdlib>
#include "common.cuh"

namespace polyconv {

namespace {

#ifndef PC_F32_KW
#define PC_F32_KW 8
#endif
constexpr int KW = PC_F32_KW;            // output channels per warp
constexpr int BP = 256, BK = 4 * KW, NT = 128;

struct F32Geo {
  int pitch, HS, WU, CC;
  long long Mtot;  // positions computed: last extraction position + 1
  FastDiv fpitch, fHS, fsh, fsw;
};

F32Geo f32_geo(const Geom& g, int cc) {
  F32Geo f;
  // shared zero rows / columns need ph < R and pw < S (the last output row / column then stays
  // inside its own image / row); otherwise each image keeps its own padding on both sides
  f.pitch = g.pw < g.S ? g.W + g.pw : g.W + 2 * g.pw;
  if (f.pitch < g.S) f.pitch = g.S;
  f.HS = g.ph < g.R ? g.H + g.ph : g.H + 2 * g.ph;
  f.Mtot = ((long long)(g.N - 1) * f.HS + (long long)(g.P - 1) * g.sh) * f.pitch + (long long)(g.Q - 1) * g.sw + 1;
  f.WU = (BP + (g.R - 1) * f.pitch + g.S - 1 + 3) / 4 * 4;
  f.CC = cc;
  f.fpitch.init((uint32_t)f.pitch);
  f.fHS.init((uint32_t)f.HS);
  f.fsh.init((uint32_t)g.sh);
  f.fsw.init((uint32_t)g.sw);
  return f;
}

int smem_bytes_for(const Geom& g, int cc) {
  const F32Geo f = f32_geo(g, cc);
  return 2 * (cc * f.WU + cc * g.R * g.S * BK) * 4;
}

__device__ __forceinline__ void cp_async4(float* dst, const float* src, bool valid) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(d), "l"(src), "r"(valid ? 4 : 0) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// x element offset (n*C*HW + h*W + w, channel 0) of input-polynomial position q, or -1 (zero)
__device__ __forceinline__ long long f32_src(const Geom& g, const F32Geo& f, long long q) {
  if (q >= (1LL << 31)) return -1;
  const uint32_t vr = f.fpitch.div((uint32_t)q);
  const int w = (int)((uint32_t)q - vr * (uint32_t)f.pitch) - g.pw;
  const int vr2 = (int)vr - g.ph;
  if (vr2 < 0 || w < 0 || w >= g.W) return -1;
  const int n = (int)f.fHS.div((uint32_t)vr2);
  const int h = vr2 - n * f.HS;
  if (h >= g.H || n >= g.N) return -1;
  return ((long long)n * g.C) * g.H * g.W + (long long)h * g.W + w;
}

// RT / ST: compile-time kernel size (0 = runtime g.R / g.S)
template <int RT, int ST>
__global__ void __launch_bounds__(NT, 4) mac_fp32_kernel(Geom g, F32Geo f, const float* __restrict__ x,
                                                         const float* __restrict__ U, int Kp, int Cp,
                                                         float* __restrict__ y) {
  extern __shared__ __align__(16) float fsm[];
  const int R = RT ? RT : g.R, S = ST ? ST : g.S, RS = R * S;
  const int CC = f.CC, WU = f.WU;
  float* s_win = fsm;                  // [2][CC][WU]
  float* s_w = fsm + 2 * CC * WU;      // [2][CC][RS][BK]
  const long long m0 = (long long)blockIdx.x * BP;
  const int k0 = blockIdx.y * BK;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long HW = (long long)g.H * g.W;

  // a2 + a3 staging of channel chunk c0 into buffer b (cp.async; zero-filled outside the image)
  auto stage = [&](int c0, int b) {
    float* win = s_win + b * CC * WU;
    for (int q = threadIdx.x; q < WU; q += NT) {
      const long long src = f32_src(g, f, m0 + q);
      for (int cc = 0; cc < CC; ++cc) {
        const int c = c0 + cc;
        const bool ok = src >= 0 && c < g.C;
        cp_async4(win + cc * WU + q, x + (ok ? src + c * HW : 0), ok);
      }
    }
    float* wd = s_w + b * CC * RS * BK;
    const int nw = CC * RS * BK;
    for (int e = threadIdx.x; e < nw; e += NT) {
      const int cc = e % CC, rest = e / CC;
      const int kk = rest % BK, tap = rest / BK;
      cp_async4(wd + (cc * RS + tap) * BK + kk, U + ((long long)tap * Kp + k0 + kk) * Cp + c0 + cc, true);
    }
    cp_async_commit();
  };

  // accumulators as position pairs: one packed FFMA2 (fma.rn.f32x2, sm_100) per channel and
  // pair -- the same round-to-nearest fp32 FMAs as two FFMA, half the issue slots
  float2 acc[KW][4];
#pragma unroll
  for (int a = 0; a < KW; ++a)
#pragma unroll
    for (int b = 0; b < 4; ++b) acc[a][b] = make_float2(0.f, 0.f);

  const int nch = (g.C + CC - 1) / CC;
  stage(0, 0);
  for (int ch = 0; ch < nch; ++ch) {
    const int b = ch & 1;
    if (ch + 1 < nch) {
      stage((ch + 1) * CC, b ^ 1);
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncthreads();
    const int ccn = min(CC, g.C - ch * CC);
    for (int cc = 0; cc < ccn; ++cc) {
      const float* win = s_win + (b * CC + cc) * WU + lane;
      const float* wr = s_w + ((b * CC + cc) * RS) * BK + warp * KW;
#pragma unroll(RT ? RT : 1)
      for (int i = 0; i < R; ++i) {
#pragma unroll(ST ? ST : 1)
        for (int j = 0; j < S; ++j) {
          float wv[KW];
#pragma unroll
          for (int a4 = 0; a4 < KW; a4 += 4) {
            const float4 w4 = *reinterpret_cast<const float4*>(wr + (i * S + j) * BK + a4);
            wv[a4] = w4.x; wv[a4 + 1] = w4.y; wv[a4 + 2] = w4.z; wv[a4 + 3] = w4.w;
          }
          float2 av[4];
#pragma unroll
          for (int bb = 0; bb < 4; ++bb)
            av[bb] = make_float2(win[i * f.pitch + j + 64 * bb], win[i * f.pitch + j + 64 * bb + 32]);
#pragma unroll
          for (int a = 0; a < KW; ++a)
#pragma unroll
            for (int bb = 0; bb < 4; ++bb) acc[a][bb] = __ffma2_rn(make_float2(wv[a], wv[a]), av[bb], acc[a][bb]);
        }
      }
    }
    __syncthreads();  // buffer b is restaged two chunks later
  }

  // a5: position -> (n, oh, ow) (Eq. 12 + R4 + R16), off-lattice / junk positions dropped
#pragma unroll
  for (int bb = 0; bb < 8; ++bb) {
    const long long q = m0 + lane + 32 * bb;
    if (q >= f.Mtot) continue;
    const uint32_t vr = f.fpitch.div((uint32_t)q);
    const uint32_t col = (uint32_t)q - vr * (uint32_t)f.pitch;
    const uint32_t n = f.fHS.div(vr);
    const uint32_t r = vr - n * (uint32_t)f.HS;
    const uint32_t oh = f.fsh.div(r), ow = f.fsw.div(col);
    if (oh * (uint32_t)g.sh != r || ow * (uint32_t)g.sw != col || (int)oh >= g.P || (int)ow >= g.Q || (int)n >= g.N)
      continue;
    const long long PQ = (long long)g.P * g.Q;
    const long long ybase = (long long)n * g.K * PQ + (long long)oh * g.Q + ow;
#pragma unroll
    for (int a = 0; a < KW; ++a) {
      const int k = k0 + warp * KW + a;
      if (k < g.K) y[ybase + (long long)k * PQ] = (bb & 1) ? acc[a][bb >> 1].y : acc[a][bb >> 1].x;
    }
  }
}

}  // namespace

Fp32Tiling fp32_tiling(const Geom& g) {
  Fp32Tiling t{8, 0, 0};
  // channel chunk: 8 (16 for 1x1: the per-position decode and the chunk barrier amortise over
  // more channels, ResNet-50 1x1 layers 21-22 -> 24-25 TFLOP/s; 3x3 layers lose 2-7% with 16),
  // fewer for large kernels (two buffers of CC x R*S x 32 filter words); POLYCONV_F32_CC
  // overrides the starting value (experiments)
  const char* ev = getenv("POLYCONV_F32_CC");
  const int cc0 = ev ? atoi(ev) : (g.R * g.S == 1 ? 16 : 8);
  for (int cc = cc0; cc >= 1; cc >>= 1) {
    t.cc = cc;
    t.smem_bytes = smem_bytes_for(g, cc);
    if (t.smem_bytes <= 100 * 1024) break;
  }
  const F32Geo f = f32_geo(g, t.cc);
  const bool fits = t.smem_bytes <= 200 * 1024 && f.Mtot + f.WU < (1LL << 31) &&
                    (long long)g.N * g.C * g.H * g.W < (1LL << 40);
  t.smax = fits ? 1 : 0;  // 0: the caller falls back to the thin kernel
  return t;
}

cudaError_t launch_mac_fp32(const Geom& g, const Fp32Tiling& t, const void* x, bool io_bf16, const float* U,
                            int Kp, int Cp, void* y, cudaStream_t st) {
  const F32Geo f = f32_geo(g, t.cc);
  dim3 grid((unsigned)((f.Mtot + BP - 1) / BP), (unsigned)((g.K + BK - 1) / BK));
  if (Kp < (int)grid.y * BK || Cp % t.cc) return cudaErrorInvalidValue;
  cudaError_t e = cudaSuccess;
#define PC_FP32(RT, ST)                                                                                \
  {                                                                                                    \
    auto kern = mac_fp32_kernel<RT, ST>;                                                               \
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, t.smem_bytes);         \
    if (e != cudaSuccess) return e;                                                                    \
    kern<<<grid, NT, t.smem_bytes, st>>>(g, f, static_cast<const float*>(x), U, Kp, Cp, static_cast<float*>(y)); \
  }
  if (io_bf16) return cudaErrorInvalidValue;  // FP32_FMA math takes f32 I/O (plan check)
  if (g.R == 3 && g.S == 3) {
    PC_FP32(3, 3)
  } else if (g.R == 1 && g.S == 1) {
    PC_FP32(1, 1)
  } else if (g.R == 5 && g.S == 5) {
    PC_FP32(5, 5)
  } else if (g.R == 7 && g.S == 7) {
    PC_FP32(7, 7)
  } else {
    PC_FP32(0, 0)
  }
#undef PC_FP32
  return cudaGetLastError();
}

}  // namespace polyconv
