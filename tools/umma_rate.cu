// umma_rate.cu — design probe (not product code): issue rate of tcgen05.mma
// kind::f16 M=128 x N x K=16 with both operands K-major SW128 in shared memory,
// as a function of N, commit frequency and the B descriptor row shift.
// One CTA per SM; thread 0 issues `iters` MMAs into one TMEM accumulator.
#include <cuda.h>
#include <cstdio>
#include <vector>
#include "../paper_conf_cgo_xuzc025_b200/csrc/sm100.cuh"

using namespace polyconv::sm100;

__global__ void rate(int n, int iters, int commit_every, int shift_rows, int kind_tf32, long long* out) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = raw + (((smem_u32(raw) + 1023) & ~1023u) - smem_u32(raw));
  uint8_t* sA = sm;               // 128 rows x 128 B
  uint8_t* sB = sm + 128 * 128;   // up to 384 rows x 128 B
  __shared__ uint64_t bar, bar2;
  __shared__ uint32_t slot;
  for (int i = threadIdx.x; i < (128 + 384) * 128 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); mbar_init(&bar2, 1); fence_barrier_init(); }
  if (threadIdx.x < 32) tmem_alloc(&slot, 256);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before(); __syncthreads(); tc_fence_after();
  uint32_t tm = slot;
  if (threadIdx.x == 0) {
    const uint32_t ab = kind_tf32 ? 2u : 1u;
    const uint32_t idesc = (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(n >> 3) << 17) | ((128u >> 4) << 24);
    const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB) + shift_rows * 128;
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
      const int ks = it & 3;
      uint64_t ad = make_sdesc(a0 + 32 * ks, 128, 0);
      uint64_t bd = make_sdesc(b0 + 32 * ks, 128, 0);
      if (kind_tf32) umma<true>(tm, ad, bd, idesc, it > 0);
      else umma<false>(tm, ad, bd, idesc, it > 0);
      if (commit_every && (it % commit_every) == commit_every - 1) umma_commit(&bar2);
    }
    long long t1 = clock64();
    umma_commit(&bar);
    // wait for all: the last commit completes the phase after all earlier ones
    mbar_wait(&bar, 0);
    long long t2 = clock64();
    out[blockIdx.x * 2] = t1 - t0;
    out[blockIdx.x * 2 + 1] = t2 - t0;
  }
  tc_fence_before(); __syncthreads();
  if (threadIdx.x < 32) { tc_fence_after(); tmem_dealloc(tm, 256); }
}

// warp-wide issue loop, elected lane issues; descriptors advanced by constants
__global__ void rate_warp(int n, int iters, int commit_every, int shift_rows, long long* out) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = raw + (((smem_u32(raw) + 1023) & ~1023u) - smem_u32(raw));
  uint8_t* sA = sm;
  uint8_t* sB = sm + 128 * 128;
  __shared__ uint64_t bar, bar2;
  __shared__ uint32_t slot;
  for (int i = threadIdx.x; i < (128 + 384) * 128 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); mbar_init(&bar2, 1); fence_barrier_init(); }
  if (threadIdx.x < 32) tmem_alloc(&slot, 256);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before(); __syncthreads(); tc_fence_after();
  uint32_t tm = slot;
  if (threadIdx.x < 32) {
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((128u >> 4) << 24);
    const uint64_t ad0 = make_sdesc(smem_u32(sA), 128, 0);
    const uint64_t bd0 = make_sdesc(smem_u32(sB) + shift_rows * 128, 128, 0);
    long long t0 = clock64();
    for (int it = 0; it < iters; it += 4) {
#pragma unroll
      for (int ks = 0; ks < 4; ++ks) {
        if (elect_one()) umma<false>(tm, ad0 + 2 * ks, bd0 + 2 * ks, idesc, (it | ks) != 0);
        __syncwarp();
      }
      if (commit_every) {
        if (elect_one()) umma_commit(&bar2);
        __syncwarp();
      }
    }
    long long t1 = clock64();
    if (elect_one()) umma_commit(&bar);
    __syncwarp();
    mbar_wait(&bar, 0);
    long long t2 = clock64();
    if (threadIdx.x == 0) { out[blockIdx.x * 2] = t1 - t0; out[blockIdx.x * 2 + 1] = t2 - t0; }
  }
  tc_fence_before(); __syncthreads();
  if (threadIdx.x < 32) { tc_fence_after(); tmem_dealloc(tm, 256); }
}

// realistic operand addresses: A cycles through an 8-stage ring of 16 KB tiles,
// B is a 288-row window read at tap shifts Wp*i + j (Wp = 30), as in mac_tc2
__global__ void rate_ring(int n, int stages, int iters, long long* out, int mode, int group = 1) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = raw + (((smem_u32(raw) + 1023) & ~1023u) - smem_u32(raw));
  uint8_t* sA = sm;                          // stages x 16 KB
  uint8_t* sB = sm + stages * 16384;         // 288 rows x 128 B
  __shared__ uint64_t bar, bar2, done;
  __shared__ uint64_t ring_full[8], ring_empty[8];
  __shared__ uint32_t slot;
  for (int i = threadIdx.x; i < (stages * 16384 + 288 * 128) / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = i;
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1); mbar_init(&bar2, 1); mbar_init(&done, 1);
    for (int s = 0; s < 8; ++s) { mbar_init(ring_full + s, 1); mbar_init(ring_empty + s, 1); }
    fence_barrier_init();
  }
  if (threadIdx.x < 32) tmem_alloc(&slot, 256);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before(); __syncthreads(); tc_fence_after();
  uint32_t tm = slot;
  if (mode >= 11 && mode <= 13 && threadIdx.x >= 64) {
    // idle "epilogue" warps polling an mbarrier that completes only at the end
    const uint32_t ns = mode == 11 ? 256u : (mode == 12 ? 2000u : 0u);
    if (mode == 13) {
      mbar_wait(&bar, 0);  // try_wait loop
    } else {
      mbar_wait_sleep(&bar, 0, ns);
    }
  }
  if ((mode == 9 || mode == 10) && threadIdx.x == 32) {
    volatile int* cnt = reinterpret_cast<volatile int*>(&done);
    for (int it = 0; it <= iters; ++it) cnt[0] = it;  // helper: publishes "stage it ready"
  }
  if ((mode == 2 || mode == 5 || mode == 7 || mode == 8 || mode >= 11) && threadIdx.x >= 32 && threadIdx.x < 64) {
    // producer warp: ring protocol like mac_tc2 (no data movement)
    int st = 0; uint32_t ph = 0;
    for (int it = 0; it < iters; ++it) {
      mbar_wait(ring_empty + st, ph ^ 1u);
      if (elect_one()) mbar_arrive(ring_full + st);
      __syncwarp();
      if (++st == stages) { st = 0; ph ^= 1u; }
    }
  }
  if (mode == 14 && (threadIdx.x >> 5) == 2) {
    // second issuer warp: odd stages
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((128u >> 4) << 24);
    int st = 0; uint32_t ph = 0;
    for (int it = 0; it < iters; ++it) {
      if (it & 1) {
        mbar_wait(ring_full + st, ph);
        tc_fence_after();
        const int tap = it % 9, i = tap / 3, j = tap % 3;
        const uint64_t ad = make_sdesc(smem_u32(sA) + st * 16384, 128, 0);
        const uint64_t bd = make_sdesc(smem_u32(sB) + (30 * i + j) * 128, 128, 0);
        if (elect_one()) {
          for (int ks = 0; ks < 4; ++ks) umma<false>(tm, ad + 2 * ks, bd + 2 * ks, idesc, 1);
          umma_commit(ring_empty + st);
        }
        __syncwarp();
      }
      if (++st == stages) { st = 0; ph ^= 1u; }
    }
  }
  if (threadIdx.x < 32) {
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((128u >> 4) << 24);
    long long t0 = clock64();
    int st = 0; uint32_t ph = 0;
    for (int it = 0; it < iters; ++it) {
      if (mode == 14 && (it & 1)) { if (++st == stages) { st = 0; ph ^= 1u; } continue; }
      if (mode == 14) {
        mbar_wait(ring_full + st, ph);
        tc_fence_after();
      } else if (mode == 9 || mode == 10) {  // poll a shared counter published by a helper warp
        const volatile int* cnt = reinterpret_cast<volatile int*>(&done);
        while (cnt[0] < it) {}
        if (mode == 10) tc_fence_after();
      } else if (mode == 8) {  // group stages: wait/fence only at the start of every group
        if (it % group == 0) {
          int s2 = st; uint32_t p2 = ph;
          for (int g = 0; g < group; ++g) { mbar_wait(ring_full + s2, p2); if (++s2 == stages) { s2 = 0; p2 ^= 1u; } }
          tc_fence_after();
        }
      } else if (mode >= 1) {
        if (mode == 2 || mode == 5 || mode >= 11) mbar_wait(ring_full + st, ph);
        else if (mode == 1 || mode == 3) mbar_wait(&done, 1);  // already-complete phase
        else if (mode == 6) mbar_wait_spin(&done, 1);
        else if (mode == 7) mbar_wait_spin(ring_full + st, ph);
        if (mode == 1 || mode == 2 || mode == 4 || mode == 6 || mode == 7 || mode >= 11) tc_fence_after();
      }
      const int tap = it % 9, i = tap / 3, j = tap % 3;
      const uint64_t ad = make_sdesc(smem_u32(sA) + st * 16384, 128, 0);
      const uint64_t bd = make_sdesc(smem_u32(sB) + (30 * i + j) * 128, 128, 0);
      if (elect_one()) {
        for (int ks = 0; ks < 4; ++ks) umma<false>(tm, ad + 2 * ks, bd + 2 * ks, idesc, (it | ks) != 0);
        umma_commit((mode == 2 || mode == 5 || mode == 7 || mode == 8 || mode >= 11) ? ring_empty + st : &bar2);
      }
      __syncwarp();
      if (++st == stages) { st = 0; ph ^= 1u; }
    }
    long long t1 = clock64();
    if (elect_one()) umma_commit(&bar);
    __syncwarp();
    mbar_wait(&bar, 0);
    long long t2 = clock64();
    if (threadIdx.x == 0) { out[blockIdx.x * 2] = t1 - t0; out[blockIdx.x * 2 + 1] = t2 - t0; }
  }
  tc_fence_before(); __syncthreads();
  if (threadIdx.x < 32) { tc_fence_after(); tmem_dealloc(tm, 256); }
}

int main() {
  long long* d;
  cudaMalloc(&d, 148 * 2 * sizeof(long long));
  cudaFuncSetAttribute(rate, cudaFuncAttributeMaxDynamicSharedMemorySize, 80 * 1024);
  std::vector<long long> h(148 * 2);
  struct Cfg { int n, iters, ce, shift, tf32; } cfgs[] = {
      {256, 4096, 0, 0, 0}, {208, 4096, 0, 0, 0}, {128, 4096, 0, 0, 0}, {64, 4096, 0, 0, 0},
      {208, 4096, 4, 0, 0}, {208, 4096, 1, 0, 0}, {208, 4096, 0, 31, 0}, {208, 4096, 4, 31, 0},
      {256, 4096, 0, 0, 1}, {208, 4096, 4, 31, 1}};
  for (auto c : cfgs) {
    for (int grid : {1, 148}) {
      rate<<<grid, 128, 80 * 1024>>>(c.n, c.iters, c.ce, c.shift, c.tf32, d);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
      cudaMemcpy(h.data(), d, grid * 2 * sizeof(long long), cudaMemcpyDeviceToHost);
      double issue = 0, total = 0;
      for (int b = 0; b < grid; ++b) { issue += h[2 * b]; total += h[2 * b + 1]; }
      issue /= grid; total /= grid;
      double ideal = 128.0 * c.n / 256.0 * (c.tf32 ? 2 : 1);
      printf("%s N=%3d commit_every=%d shift=%2d grid=%3d: issue %.1f cyc/mma, total %.1f cyc/mma (ideal %.0f)\n",
             c.tf32 ? "tf32" : "bf16", c.n, c.ce, c.shift, grid, issue / c.iters, total / c.iters, ideal);
    }
  }
  cudaFuncSetAttribute(rate_ring, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int mode : {0, 2, 14})
  for (int n : {208}) {
    for (int stages : {8}) {
      const int grp = mode == 18 ? 4 : (mode == 28 ? 8 : 2);
      rate_ring<<<148, 320, 200 * 1024>>>(n, stages, 1024, d, mode % 10 == 8 ? 8 : mode, grp);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
      cudaMemcpy(h.data(), d, 148 * 2 * sizeof(long long), cudaMemcpyDeviceToHost);
      double total = 0;
      for (int b = 0; b < 148; ++b) total += h[2 * b + 1];
      printf("mode %d ring A stages=%d, B shifted window: N=%3d total %.1f cyc/mma (ideal %.0f)\n", mode, stages, n,
             total / 148 / (1024 * 4), 128.0 * n / 256.0);
    }
  }
  cudaFuncSetAttribute(rate_warp, cudaFuncAttributeMaxDynamicSharedMemorySize, 80 * 1024);
  struct Cfg2 { int n, ce, shift; } c2[] = {{256, 0, 0}, {208, 0, 0}, {128, 0, 0}, {64, 0, 0}, {256, 4, 0},
                                            {208, 4, 31}, {128, 4, 0}};
  for (auto c : c2) {
    rate_warp<<<148, 128, 80 * 1024>>>(c.n, 4096, c.ce, c.shift, d);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
    cudaMemcpy(h.data(), d, 148 * 2 * sizeof(long long), cudaMemcpyDeviceToHost);
    double issue = 0, total = 0;
    for (int b = 0; b < 148; ++b) { issue += h[2 * b]; total += h[2 * b + 1]; }
    printf("warp-issue bf16 N=%3d commit_per_4=%d shift=%2d: issue %.1f, total %.1f cyc/mma (ideal %.0f)\n", c.n, c.ce,
           c.shift, issue / 148 / 4096, total / 148 / 4096, 128.0 * c.n / 256.0);
  }
  return 0;
}
