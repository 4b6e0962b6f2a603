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
