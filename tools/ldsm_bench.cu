// ldsm_bench.cu — design probe (not product code): throughput of 8x8-matrix
// moves (ldmatrix .trans / stmatrix) and plain 16-byte shared accesses, in
// batches of 8 independent operations per warp, by number of warps per SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ldsm_bench tools/ldsm_bench.cu
#include <cuda_runtime.h>
#include <cstdio>
#include "../paper_conf_cgo_xuzc025_b200/csrc/sm100.cuh"

using namespace polyconv::sm100;

template <int V>
__global__ void bench(int iters, long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 96 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = i;
  __syncthreads();
  const uint32_t base = smem_u32(sm);
  const uint32_t src0 = base + (warp & 3) * 8192, dst0 = base + 32768 + (warp & 7) * 8192;
  const int c = lane;  // staging row
  uint32_t acc = 0;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    uint32_t d[8][4];
    if (V == 0 || V == 1) {
#pragma unroll
      for (int eg = 0; eg < 8; ++eg)
        ldsm_x4_trans(src0 + c * 128u + 16u * (uint32_t)(eg ^ (c & 7)), d[eg][0], d[eg][1], d[eg][2], d[eg][3]);
    } else {
#pragma unroll
      for (int eg = 0; eg < 8; ++eg) { d[eg][0] = it + eg; d[eg][1] = it; d[eg][2] = eg; d[eg][3] = it ^ eg; }
    }
    if (V == 0 || V == 2) {
#pragma unroll
      for (int eg = 0; eg < 8; ++eg) {
        const uint32_t off = (uint32_t)(eg * 8 + (lane & 7)) * 128u + 16u * (uint32_t)(lane >> 3);
        stsm_x4(dst0 + (off ^ (((off >> 7) & 7u) << 4)), d[eg][0], d[eg][1], d[eg][2], d[eg][3]);
      }
    }
    if (V == 3) {  // the same bytes as 8 x stsm.x4, as 32 x st.shared.v4 (each lane one 16 B chunk per op)
#pragma unroll
      for (int k = 0; k < 32; ++k) {
        const uint32_t off = (uint32_t)(k * 2 + (lane >> 4)) * 128u + 16u * (uint32_t)(lane & 7);
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(dst0 + (off & 8191)), "r"(d[k & 7][0]),
                     "r"(d[k & 7][1]), "r"(d[k & 7][2]), "r"(d[k & 7][3]) : "memory");
      }
    }
#pragma unroll
    for (int eg = 0; eg < 8; ++eg) acc ^= d[eg][0] ^ d[eg][3];
  }
  long long t1 = clock64();
  if (lane == 0) out[warp] = t1 - t0;
  if (acc == 0x12345678u) out[0] = 0;
}

int main() {
  long long* out;
  cudaMalloc(&out, 8 * 64);
  const char* names[] = {"8x(ldsm.x4.trans) + 8x(stsm.x4)", "8x ldsm.x4.trans", "8x stsm.x4",
                         "32x st.shared.v4 (same bytes)"};
  const int iters = 2048;
  auto run = [&](auto kern, int v) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 96 * 1024);
    for (int nw : {1, 4, 8}) {
      kern<<<1, 32 * nw, 96 * 1024>>>(iters, out);
      long long h[32];
      cudaDeviceSynchronize();
      cudaMemcpy(h, out, 8 * nw, cudaMemcpyDeviceToHost);
      long long mx = 0;
      for (int i = 0; i < nw; ++i) mx = h[i] > mx ? h[i] : mx;
      printf("%-34s warps %d: %.1f cycles per batch (per warp), SM moves %.1f B/clk\n", names[v], nw,
             (double)mx / iters, (double)nw * 8 * 512 * iters / mx);
    }
  };
  run(bench<0>, 0);
  run(bench<1>, 1);
  run(bench<2>, 2);
  run(bench<3>, 3);
  return 0;
}
