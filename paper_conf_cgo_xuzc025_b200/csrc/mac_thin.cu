// mac_thin.cu — a4 for thin contractions (tiny C*R*S, e.g. the 1-channel tiny
// config): one lane group per output coefficient, lanes split the C*R*S
// products, __shfl_xor_sync tree reduction, extraction + NCHW store fused.
//
//   p_{n,k}[m] = sum_c sum_{i,j} A_{n,c}[m - e(i,j)] * U_{k,c}[e(i,j)]
// at m = m(oh,ow) = Wp*sh*oh + sw*ow + L_U-1 (Eq. 12 + R4), where
// m - e(i,j) = Wp*sh*oh + sw*ow + Wp*i + j  (the shifted window, §8(a) a4).
// Channel sum as in P.1350-1352.  Accumulation fp32.
#include "common.cuh"

namespace polyconv {

namespace {

template <int F, int G, typename OutT>
__global__ void __launch_bounds__(256) mac_thin_kernel(Geom g, const typename Word<F>::T* __restrict__ A,
                                                       const typename Word<F>::T* __restrict__ U, int Kp,
                                                       int Cp, OutT* __restrict__ y) {
  const int lane_in_group = threadIdx.x & (G - 1);
  const long long group = (blockIdx.x * 256LL + threadIdx.x) / G;
  const long long ngroups = (long long)gridDim.x * 256 / G;
  const long long total = (long long)g.N * g.K * g.P * g.Q;
  const int RS = g.R * g.S;
  const int CRS = g.C * RS;
  // all lanes of a warp iterate the same number of times (uniform shuffles)
  const long long iters = (total + ngroups - 1) / ngroups;
  for (long long it = 0; it < iters; ++it) {
    const long long idx = group + it * ngroups;
    float acc = 0.f;
    if (idx < total) {
      long long nk = idx / ((long long)g.P * g.Q);
      int pq = (int)(idx - nk * g.P * g.Q);
      int n = (int)(nk / g.K), k = (int)(nk - (long long)n * g.K);
      int oh = pq / g.Q, ow = pq - oh * g.Q;
      long long base = (long long)g.Wp * g.sh * oh + (long long)g.sw * ow;  // m(oh,ow) - (L_U-1)
      for (int f = lane_in_group; f < CRS; f += G) {
        int c = f / RS, tap = f - c * RS;
        int i = tap / g.S, j = tap - i * g.S;
        float a = Word<F>::dec(A[((long long)n * g.C + c) * g.L_A + base + (long long)g.Wp * i + j]);
        float u = Word<F>::dec(U[((long long)tap * Kp + k) * Cp + c]);
        acc = fmaf(a, u, acc);
      }
    }
#pragma unroll
    for (int off = G / 2; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
    if (idx < total && lane_in_group == 0) store_out(y, idx, acc);
  }
}

template <int F, typename OutT>
cudaError_t run(const Geom& g, const void* A, const void* U, int Kp, int Cp, void* y, cudaStream_t st) {
  const int CRS = g.C * g.R * g.S;
  const long long total = (long long)g.N * g.K * g.P * g.Q;
  int G = 1;
  while (G < CRS && G < 32) G <<= 1;
  long long threads = total * G;
  long long b = (threads + 255) / 256;
  unsigned grid = (unsigned)(b > 148 * 64 ? 148 * 64 : (b < 1 ? 1 : b));
  using WT = typename Word<F>::T;
#define PC_THIN(GG)                                                                      \
  case GG:                                                                               \
    mac_thin_kernel<F, GG, OutT><<<grid, 256, 0, st>>>(g, (const WT*)A, (const WT*)U, Kp, Cp, \
                                                       (OutT*)y);                        \
    break;
  switch (G) {
    PC_THIN(1) PC_THIN(2) PC_THIN(4) PC_THIN(8) PC_THIN(16) default : PC_THIN(32)
  }
#undef PC_THIN
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_mac_thin(const Geom& g, const void* A, const void* U, int Kp, int Cp, int fmt,
                            void* y, bool y_bf16, cudaStream_t st) {
  if (y_bf16) {
    switch (fmt) {
      case FMT_F32: return run<FMT_F32, __nv_bfloat16>(g, A, U, Kp, Cp, y, st);
      case FMT_TF32: return run<FMT_TF32, __nv_bfloat16>(g, A, U, Kp, Cp, y, st);
      default: return run<FMT_BF16, __nv_bfloat16>(g, A, U, Kp, Cp, y, st);
    }
  }
  switch (fmt) {
    case FMT_F32: return run<FMT_F32, float>(g, A, U, Kp, Cp, y, st);
    case FMT_TF32: return run<FMT_TF32, float>(g, A, U, Kp, Cp, y, st);
    default: return run<FMT_BF16, float>(g, A, U, Kp, Cp, y, st);
  }
}

}  // namespace polyconv
