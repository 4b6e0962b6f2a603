// grad.cu — SURVEY §8(f) row f4 (an extension: the paper is forward-only).  The two gradients of a
// stride-1 convolution are themselves convolutions, so the forward plan computes them once two
// layouts exist, and this file makes those layouts (bit-exact copies, HBM-bound):
//   dgrad: dx = conv(dy, flip(w)^T) with padding R-1-p   -> polyconv_flip_filter
//          wt[c][k][R-1-i][S-1-j] = w[k][c][i][j]
//   wgrad: dw^T = conv(x^T, dy^T) with padding p          -> polyconv_swap_nc (x, dy, and back)
//          xt[c][n][:] = x[n][c][:]
// Stride s >= 2: dx = conv(dilate(dy), flip(w)^T) and dw^T = conv(x^T, dilate(dy)^T), cropped,
// where dilate puts dy on the stride lattice of a zero plane      -> polyconv_dilate
// swap_nc: one block per destination row (c, n); the row is a contiguous run of HW elements in
// both layouts, copied with 16-byte vectors when both ends are 16-byte aligned.
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <algorithm>
#include <cstdint>
#include "../../include/polyconv.h"

namespace {

template <typename T>
__global__ void __launch_bounds__(256) flip_filter_kernel(const T* __restrict__ w, T* __restrict__ wt, int K,
                                                          int C, int R, int S) {
  const long long total = (long long)K * C * R * S;
  for (long long idx = blockIdx.x * 256LL + threadIdx.x; idx < total; idx += (long long)gridDim.x * 256) {
    // idx enumerates the destination wt[c][k][i'][j']
    const int rs = R * S;
    const long long ck = idx / rs;
    const int t = (int)(idx - ck * rs);
    const int ip = t / S, jp = t - ip * S;
    const int c = (int)(ck / K), k = (int)(ck - (long long)c * K);
    wt[idx] = w[(((long long)k * C + c) * R + (R - 1 - ip)) * S + (S - 1 - jp)];
  }
}

template <typename T>
__global__ void __launch_bounds__(256) swap_nc_kernel(const T* __restrict__ x, T* __restrict__ xt, int N, int C,
                                                      long long HW, bool vec) {
  for (long long row = blockIdx.x; row < (long long)N * C; row += gridDim.x) {
    const int c = (int)(row / N), n = (int)(row - (long long)c * N);
    const T* src = x + ((long long)n * C + c) * HW;
    T* dst = xt + row * HW;
    if (vec) {
      const long long nv = HW * sizeof(T) / 16;
      const uint4* s4 = reinterpret_cast<const uint4*>(src);
      uint4* d4 = reinterpret_cast<uint4*>(dst);
      for (long long v = threadIdx.x; v < nv; v += 256) d4[v] = s4[v];
    } else {
      for (long long e = threadIdx.x; e < HW; e += 256) dst[e] = src[e];
    }
  }
}

template <typename T>
__global__ void __launch_bounds__(256) dilate_kernel(const T* __restrict__ x, T* __restrict__ xd, long long NC, int H,
                                                    int W, int sh, int sw, int Hd, int Wd) {
  const long long total = NC * Hd * Wd;
  for (long long idx = blockIdx.x * 256LL + threadIdx.x; idx < total; idx += (long long)gridDim.x * 256) {
    // idx enumerates the destination xd[nc][hd][wd]: coalesced stores, zeros off the lattice
    const long long nc = idx / ((long long)Hd * Wd);
    const int t = (int)(idx - nc * Hd * Wd);
    const int hd = t / Wd, wd = t - hd * Wd;
    const int h = hd / sh, w = wd / sw;
    T v = T(0);
    if (hd == h * sh && wd == w * sw && h < H && w < W) v = x[(nc * H + h) * W + w];
    xd[idx] = v;
  }
}

int grid_for(long long work, int per_block) {
  long long b = (work + per_block - 1) / per_block;
  return (int)(b < 1 ? 1 : (b > 148 * 16 ? 148 * 16 : b));
}

polyconv_status_t status_of(cudaError_t e) {
  if (e == cudaSuccess) return POLYCONV_STATUS_SUCCESS;
  cudaGetLastError();
  return POLYCONV_STATUS_EXECUTION_FAILED;
}

}  // namespace

extern "C" polyconv_status_t polyconv_flip_filter(const void* w, void* wt, int K, int C, int R, int S,
                                                  polyconv_dtype_t dtype, void* stream) {
  if (!w || !wt || w == wt || K < 1 || C < 1 || R < 1 || S < 1 || (dtype != POLYCONV_F32 && dtype != POLYCONV_BF16))
    return POLYCONV_STATUS_BAD_PARAM;
  const long long total = (long long)K * C * R * S;
  if (total >= (1LL << 31)) return POLYCONV_STATUS_NOT_SUPPORTED;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (dtype == POLYCONV_F32)
    flip_filter_kernel<uint32_t><<<grid_for(total, 256), 256, 0, st>>>(
        static_cast<const uint32_t*>(w), static_cast<uint32_t*>(wt), K, C, R, S);
  else
    flip_filter_kernel<uint16_t><<<grid_for(total, 256), 256, 0, st>>>(
        static_cast<const uint16_t*>(w), static_cast<uint16_t*>(wt), K, C, R, S);
  return status_of(cudaGetLastError());
}

extern "C" polyconv_status_t polyconv_dilate(const void* x, void* xd, int N, int C, int H, int W, int sh, int sw,
                                             int eh, int ew, polyconv_dtype_t dtype, void* stream) {
  if (!x || !xd || x == xd || N < 1 || C < 1 || H < 1 || W < 1 || sh < 1 || sw < 1 || eh < 0 || ew < 0 ||
      (dtype != POLYCONV_F32 && dtype != POLYCONV_BF16))
    return POLYCONV_STATUS_BAD_PARAM;
  const long long Hd = (long long)(H - 1) * sh + 1 + eh, Wd = (long long)(W - 1) * sw + 1 + ew;
  if (Hd * Wd >= (1LL << 31) || (long long)N * C * Hd * Wd >= (1LL << 40)) return POLYCONV_STATUS_NOT_SUPPORTED;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const long long total = (long long)N * C * Hd * Wd;
  if (dtype == POLYCONV_F32)
    dilate_kernel<uint32_t><<<grid_for(total, 256), 256, 0, st>>>(static_cast<const uint32_t*>(x),
                                                                  static_cast<uint32_t*>(xd), (long long)N * C, H, W,
                                                                  sh, sw, (int)Hd, (int)Wd);
  else
    dilate_kernel<uint16_t><<<grid_for(total, 256), 256, 0, st>>>(static_cast<const uint16_t*>(x),
                                                                  static_cast<uint16_t*>(xd), (long long)N * C, H, W,
                                                                  sh, sw, (int)Hd, (int)Wd);
  return status_of(cudaGetLastError());
}

extern "C" polyconv_status_t polyconv_swap_nc(const void* x, void* xt, int N, int C, long long HW,
                                              polyconv_dtype_t dtype, void* stream) {
  if (!x || !xt || x == xt || N < 1 || C < 1 || HW < 1 || (dtype != POLYCONV_F32 && dtype != POLYCONV_BF16))
    return POLYCONV_STATUS_BAD_PARAM;
  if ((long long)N * C * HW >= (1LL << 40)) return POLYCONV_STATUS_NOT_SUPPORTED;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const size_t eb = dtype == POLYCONV_F32 ? 4 : 2;
  const bool vec = (HW * eb) % 16 == 0 && reinterpret_cast<uintptr_t>(x) % 16 == 0 &&
                   reinterpret_cast<uintptr_t>(xt) % 16 == 0;
  const int grid = grid_for((long long)N * C, 1);
  if (eb == 4)
    swap_nc_kernel<uint32_t><<<grid, 256, 0, st>>>(static_cast<const uint32_t*>(x), static_cast<uint32_t*>(xt), N,
                                                   C, HW, vec);
  else
    swap_nc_kernel<uint16_t><<<grid, 256, 0, st>>>(static_cast<const uint16_t*>(x), static_cast<uint16_t*>(xt), N,
                                                   C, HW, vec);
  return status_of(cudaGetLastError());
}

// ---------------------------------------------------------------------------------------------
// wgrad as its own contraction (the forward-conv mapping leaves R*S positions per plane, see
// DESIGN.md "Backward"): per tap (i, j), dw[:, :, i, j] = DY[K x NPQ] . X_ij[NPQ x C], the NPQ
// sum split across blocks.  Block = one tap, a 64 (k) x 64 (c) tile and a slice of the NPQ
// positions; 32-position chunks of dy and of the tap-shifted x are staged in shared memory
// (coalesced along positions), each thread accumulates 4 x 4 outputs in fp32 and adds them
// into an fp32 workspace with atomics; a second pass converts to the io dtype.
namespace {

__device__ __forceinline__ float ld_as_float(const uint32_t* p, long long i) { return __uint_as_float(p[i]); }
__device__ __forceinline__ float ld_as_float(const uint16_t* p, long long i) {
  return __uint_as_float((uint32_t)p[i] << 16);
}

template <typename T>
__global__ void __launch_bounds__(256) wgrad_kernel(const T* __restrict__ x, const T* __restrict__ dy,
                                                    float* __restrict__ ws, int N, int C, int H, int W, int K, int R,
                                                    int S, int sh, int sw, int ph, int pw, int P, int Q, int splits,
                                                    long long per_split) {
  constexpr int TM = 64, TP = 32;  // 64 (k) x 64 (c) tile, 32 positions per staged chunk
  __shared__ __align__(16) float sdy[TP][TM + 4];
  __shared__ __align__(16) float sx[TP][TM + 4];
  const int tap = blockIdx.z / splits, split = blockIdx.z - tap * splits;
  const int ti = tap / S, tj = tap - ti * S;
  const int k0 = blockIdx.x * TM, c0 = blockIdx.y * TM;
  const long long PQ = (long long)P * Q, NPQ = (long long)N * PQ;
  const long long p_begin = split * per_split, p_end = min(NPQ, p_begin + per_split);
  const int tid = threadIdx.x;
  const int tk = (tid / 16) * 4, tc = (tid % 16) * 4;
  float acc[4][4] = {};
  for (long long p0 = p_begin; p0 < p_end; p0 += TP) {
    // stage [position][row] so each thread's 4 consecutive rows are one 16-byte shared load;
    // every element this thread stages has position q = tid % TP (256 is a multiple of TP), so
    // the (n, oh, ow) decode and the tap shift are done once per chunk; consecutive threads read
    // consecutive positions (coalesced)
    const int q = tid % TP;
    const long long p = p0 + q;
    const bool live = p < p_end;
    long long dy_base = 0, x_base = 0;
    bool x_in = false;
    if (live) {
      const long long n = p / PQ;
      const int r = (int)(p - n * PQ);
      const int oh = r / Q, ow = r - oh * Q;
      const int h = sh * oh + ti - ph, w = sw * ow + tj - pw;
      dy_base = (n * K * P + oh) * (long long)Q + ow;      // + k * PQ
      x_in = h >= 0 && h < H && w >= 0 && w < W;
      x_base = (n * C * H + h) * (long long)W + w;          // + c * H * W
    }
    const long long HW = (long long)H * W;
#pragma unroll
    for (int row = tid / TP; row < TM; row += 256 / TP) {
      float vdy = 0.f, vx = 0.f;
      if (live && k0 + row < K) vdy = ld_as_float(dy, dy_base + (long long)(k0 + row) * PQ);
      if (x_in && c0 + row < C) vx = ld_as_float(x, x_base + (long long)(c0 + row) * HW);
      sdy[q][row] = vdy;
      sx[q][row] = vx;
    }
    __syncthreads();
#pragma unroll 4
    for (int q = 0; q < TP; ++q) {
      const float4 a = *reinterpret_cast<const float4*>(&sdy[q][tk]);
      const float4 b = *reinterpret_cast<const float4*>(&sx[q][tc]);
      const float av[4] = {a.x, a.y, a.z, a.w}, bv[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) acc[u][v] = fmaf(av[u], bv[v], acc[u][v]);
    }
    __syncthreads();
  }
  const long long RS = (long long)R * S;
#pragma unroll
  for (int u = 0; u < 4; ++u)
#pragma unroll
    for (int v = 0; v < 4; ++v) {
      const int k = k0 + tk + u, c = c0 + tc + v;
      if (k < K && c < C) atomicAdd(ws + ((long long)k * C + c) * RS + tap, acc[u][v]);
    }
}

__global__ void __launch_bounds__(256) f32_to_out(const float* __restrict__ ws, void* __restrict__ out, long long n,
                                                  bool bf16) {
  for (long long i = blockIdx.x * 256LL + threadIdx.x; i < n; i += (long long)gridDim.x * 256) {
    const float v = ws[i];
    if (bf16) {
      // round to nearest even; NaN stays NaN and Inf stays Inf (the integer
      // rounding trick turned the canonical NaN into -0)
      static_cast<__nv_bfloat16*>(out)[i] = __float2bfloat16_rn(v);
    } else {
      static_cast<float*>(out)[i] = v;
    }
  }
}

}  // namespace

extern "C" polyconv_status_t polyconv_wgrad(const void* x, const void* dy, void* dw, float* ws, int N, int C, int H,
                                            int W, int K, int R, int S, int sh, int sw, int ph, int pw,
                                            polyconv_dtype_t dtype, void* stream) {
  if (!x || !dy || !dw || !ws || N < 1 || C < 1 || H < 1 || W < 1 || K < 1 || R < 1 || S < 1 || sh < 1 || sw < 1 ||
      ph < 0 || pw < 0 || (dtype != POLYCONV_F32 && dtype != POLYCONV_BF16))
    return POLYCONV_STATUS_BAD_PARAM;
  const int P = (H + 2 * ph - R) / sh + 1, Q = (W + 2 * pw - S) / sw + 1;
  if (H + 2 * ph < R || W + 2 * pw < S || P < 1 || Q < 1) return POLYCONV_STATUS_BAD_PARAM;
  const long long NPQ = (long long)N * P * Q, RS = (long long)R * S;
  if ((long long)N * C * H * W >= (1LL << 40) || (long long)K * C * RS >= (1LL << 31) || RS > 65535)
    return POLYCONV_STATUS_NOT_SUPPORTED;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const long long nout = (long long)K * C * RS;
  cudaError_t e = cudaMemsetAsync(ws, 0, nout * sizeof(float), st);
  if (e != cudaSuccess) return status_of(e);
  const int kt = (K + 63) / 64, ct = (C + 63) / 64;
  // about 4 blocks per SM in total, each with at least 256 positions
  long long splits = (148LL * 4 + kt * ct * RS - 1) / (kt * ct * RS);
  splits = std::max(1LL, std::min(splits, (NPQ + 255) / 256));
  while (splits * RS > 65535) --splits;
  const long long per_split = ((NPQ + splits - 1) / splits + 31) / 32 * 32;
  splits = (NPQ + per_split - 1) / per_split;
  dim3 grid(kt, ct, (unsigned)(splits * RS));
  if (dtype == POLYCONV_F32)
    wgrad_kernel<uint32_t><<<grid, 256, 0, st>>>(static_cast<const uint32_t*>(x), static_cast<const uint32_t*>(dy), ws,
                                                 N, C, H, W, K, R, S, sh, sw, ph, pw, P, Q, (int)splits, per_split);
  else
    wgrad_kernel<uint16_t><<<grid, 256, 0, st>>>(static_cast<const uint16_t*>(x), static_cast<const uint16_t*>(dy), ws,
                                                 N, C, H, W, K, R, S, sh, sw, ph, pw, P, Q, (int)splits, per_split);
  if ((e = cudaGetLastError()) != cudaSuccess) return status_of(e);
  f32_to_out<<<grid_for(nout, 256), 256, 0, st>>>(ws, dw, nout, dtype == POLYCONV_BF16);
  return status_of(cudaGetLastError());
}
