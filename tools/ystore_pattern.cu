// Probe: NCHW output-store throughput of the mac_hankel epilogue pattern (lanes = consecutive
// positions of one row, 16 channel planes per TMEM load), 2-byte stores per lane vs lane pairs
// packed into 4-byte stores (shfl), 8 store warps per SM as in the kernel.
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/ysp tools/ystore_pattern.cu
#include <cstdio>
#include <cuda_bf16.h>
#include <vector>
#include <algorithm>
__global__ void __launch_bounds__(256) st16(__nv_bfloat16* y, int planes, int PQ, int Q, int pitch, int iters) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int it = 0; it < iters; ++it) {
    const long long pos = ((long long)(blockIdx.x * iters + it) * 8 + w) * 32 + lane;  // padded position
    const int row = (int)(pos / pitch), col = (int)(pos % pitch);
    if (col >= Q) continue;
    const long long base = (long long)row * Q + col;
    for (int c = 0; c < planes; ++c) y[(long long)c * PQ + (base % PQ)] = __float2bfloat16_rn((float)c);
  }
}
__global__ void __launch_bounds__(256) st32(__nv_bfloat16* y, int planes, int PQ, int Q, int pitch, int iters) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int it = 0; it < iters; ++it) {
    const long long pos = ((long long)(blockIdx.x * iters + it) * 8 + w) * 32 + lane;
    const int row = (int)(pos / pitch), col = (int)(pos % pitch);
    const bool ok = col < Q;
    const long long base = (long long)row * Q + col;
    for (int c = 0; c < planes; ++c) {
      const float v = (float)c;
      const float nb = __shfl_down_sync(0xffffffffu, v, 1);
      const bool pair = ok && ((col & 1) == 0) && col + 1 < Q && lane < 31;
      const bool single = ok && !pair && !((col & 1) && lane > 0 && ((col - 1) >= 0));
      __nv_bfloat16* p = y + (long long)c * PQ + (base % PQ);
      if (pair) *reinterpret_cast<__nv_bfloat162*>(p) = __floats2bfloat162_rn(v, nb);
      else if (single) *p = __float2bfloat16_rn(v);
    }
  }
}
int main() {
  const int planes = 64, Q = 56, pitch = 58, PQ = 56 * 56;
  const size_t n = (size_t)planes * PQ * 64;
  __nv_bfloat16* y; cudaMalloc(&y, n * 2 + (1 << 20));
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  const int blocks = 148 * 4, iters = 64;
  for (int k = 0; k < 2; ++k) {
    std::vector<float> ts;
    for (int r = 0; r < 8; ++r) {
      cudaEventRecord(a);
      if (k == 0) st16<<<blocks, 256>>>(y, planes, PQ, Q, pitch, iters);
      else st32<<<blocks, 256>>>(y, planes, PQ, Q, pitch, iters);
      cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b); ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    const double bytes = (double)blocks * iters * 8 * 32 * planes * 2 * Q / pitch;
    printf("%s: %.3f ms, %.1f GB/s of y\n", k ? "pairs (4-byte)" : "2-byte", ts[4], bytes / ts[4] / 1e6);
  }
  return 0;
}
