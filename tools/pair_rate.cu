// pair_rate.cu — design probe (not product code): issue/completion rate of
// tcgen05.mma.cta_group::2.kind::f16 (M = 256 over a CTA pair) x N x K=16,
// both operands K-major SW128, by N, issue style and A-descriptor row shift.
// 74 clusters of 2 CTAs; the leader's warp 1 issues `iters` MMAs.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pair_rate tools/pair_rate.cu
#include <cuda.h>
#include <cstdio>
#include <vector>
#include <algorithm>
#include "../paper_conf_cgo_xuzc025_b200/csrc/sm100.cuh"

using namespace polyconv::sm100;

__device__ __forceinline__ void umma2(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void commit2(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"((uint16_t)3)
      : "memory");
}

// style 0: elect per MMA (uniform loop); style 1: one elected lane runs the whole loop
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ const uint8_t* g_src;

__global__ void __cluster_dims__(2, 1, 1) rate2(int n, int iters, int shift_rows, int style, long long* out,
                                                 int rnd = 0) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = raw + (((smem_u32(raw) + 1023) & ~1023u) - smem_u32(raw));
  uint8_t* sA = sm;              // 256 rows x 128 B (window)
  uint8_t* sB = sm + 256 * 128;  // style < 2: 128 rows x 128 B; style 2: 18 blocks of 64 rows x 128 B
  __shared__ uint64_t bar, sbar;
  __shared__ uint32_t slot;
  for (int i = threadIdx.x; i < (256 + 18 * 64) * 128 / 4; i += blockDim.x) {
    // rnd: random bf16 pairs in [-1, 1) (exponent 0x3F/0xBF), else zeros
    uint32_t h = (uint32_t)i * 2654435761u + blockIdx.x * 40503u;
    h ^= h >> 13; h *= 0x5bd1e995u; h ^= h >> 15;
    const uint32_t v = (h & 0x807F807Fu) | 0x3F003F00u;
    reinterpret_cast<uint32_t*>(sm)[i] = rnd ? v : 0u;
  }
  if (threadIdx.x == 0) { mbar_init(&bar, 1); mbar_init(&sbar, 1); fence_barrier_init(); }
  if (threadIdx.x >= 32 && threadIdx.x < 64) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&slot)), "r"(512)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  cluster_sync();
  tc_fence_after();
  const uint32_t tm = slot;
  const uint32_t rank = cluster_ctarank();
  if (rank == 0 && threadIdx.x >= 32 && threadIdx.x < 64) {
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((256u >> 4) << 24);
    const uint64_t ad0 = make_sdesc(smem_u32(sA) + shift_rows * 128, 128, 0);
    const uint64_t bd0 = make_sdesc(smem_u32(sB), 128, 0);
    long long t0 = clock64();
    if (style >= 2) {
      // as mac_pair: per tap (i,j) A = window shifted by 30*i + j rows, B = its own 8 KB block
      for (int it = 0; it < iters; it += 4) {
        const int blk = (it / 4) % 18, tap = blk % 9;
        const uint64_t ad = make_sdesc(smem_u32(sA) + (30 * (tap / 3) + tap % 3) * 128, 128, 0);
        const uint64_t bd = make_sdesc(smem_u32(sB) + blk * 8192, 128, 0);
        if (elect_one()) {
          for (int ks = 0; ks < 4; ++ks) umma2(tm, ad + 2 * ks, bd + 2 * ks, idesc, (it | ks) != 0);
        }
        __syncwarp();
      }
    } else if (style == 0) {
      for (int it = 0; it < iters; it += 4) {
#pragma unroll
        for (int ks = 0; ks < 4; ++ks) {
          if (elect_one()) umma2(tm, ad0 + 2 * ks, bd0 + 2 * ks, idesc, (it | ks) != 0);
          __syncwarp();
        }
      }
    } else {
      if (elect_one()) {
        for (int it = 0; it < iters; it += 4)
          for (int ks = 0; ks < 4; ++ks) umma2(tm, ad0 + 2 * ks, bd0 + 2 * ks, idesc, (it | ks) != 0);
      }
      __syncwarp();
    }
    long long t1 = clock64();
    if (elect_one()) commit2(&bar);
    __syncwarp();
    mbar_wait(&bar, 0);
    long long t2 = clock64();
    if (threadIdx.x == 32) { out[blockIdx.x * 2] = t1 - t0; out[blockIdx.x * 2 + 1] = t2 - t0; }
  } else if (rank == 1 && threadIdx.x == 32) {
    mbar_wait(&bar, 0);
  }
  if (style == 3 && threadIdx.x == 64) {
    // concurrent stream: 64 x 4 KB bulk copies (256 KB) from global into a 16 KB scratch area
    uint8_t* scratch = sm + (256 + 18 * 64) * 128;
    for (int k = 0; k < 64; ++k) {
      mbar_arrive_expect_tx(&sbar, 4096);
      bulk_g2s(smem_u32(scratch + (k & 3) * 4096), g_src + ((size_t)blockIdx.x * 64 + k) * 4096, 4096, &sbar);
      mbar_wait(&sbar, k & 1);
    }
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync();
  if (threadIdx.x >= 32 && threadIdx.x < 64) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tm), "r"(512) : "memory");
  }
}

int main() {
  long long* d;
  cudaMalloc(&d, 148 * 2 * sizeof(long long));
  const int smem = (256 + 18 * 64) * 128 + 16384 + 2048;
  uint8_t* src; cudaMalloc(&src, 148 * 64 * 4096); cudaMemset(src, 1, 148 * 64 * 4096);
  cudaMemcpyToSymbol(g_src, &src, sizeof(src));
  cudaFuncSetAttribute(rate2, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 4096;
  for (int rnd : {1})
  for (int grid : {148})
    for (int n : {128})
      for (int style : {2, 3})
        for (int shift : {0, 31}) {
          rate2<<<grid, 128, smem>>>(n, iters, shift, style, d, rnd);
          cudaError_t e = cudaDeviceSynchronize();
          if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
          std::vector<long long> h(grid * 2);
          cudaMemcpy(h.data(), d, grid * 2 * sizeof(long long), cudaMemcpyDeviceToHost);
          long long tot = 0;
          for (int i = 0; i < grid; i += 2) tot = std::max(tot, h[i * 2 + 1]);
          printf("rnd %d grid %3d N=%3d style %d shift %2d: %.1f cyc/mma (ideal per SM %d)\n", rnd, grid, n, style, shift,
                 (double)tot / iters, n / 2);
          (void)rnd;
        }
  return 0;
}
