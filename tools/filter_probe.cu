// filter_probe.cu — design probe (not product code): how fast can 148 CTAs
// (one per SM) each pull a 147 KB filter half into shared memory from L2, by
// access pattern.  The conv3_x tap-major filter U[9][128][128] bf16 (295 KB):
// CTA b loads half (b & 1) as 18 blocks of 64 rows x 128 B.
//   mode 0: 2-D tensor TMA boxes (64 ch x 64 rows, SW128) from ONE shared copy
//   mode 1: as 0, but pair p reads replica p % reps (reps copies in memory)
//   mode 2: 1-D bulk copies of 8 KB contiguous blocks (pre-swizzled layout), one copy
//   mode 3: as 2 with replicas
// Each block lands on its own mbarrier; thread 0 waits for all; reports the
// median/max per-CTA time (globaltimer) from launch start.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/filter_probe tools/filter_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include <algorithm>
#include "../paper_conf_cgo_xuzc025_b200/csrc/sm100.cuh"

using namespace polyconv::sm100;

constexpr int NBLK = 18, BLK = 8192;

__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}

__device__ __forceinline__ void tma_pair(uint32_t dst, const void* tmap, uint32_t mbar_cluster, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(tmap)), "r"(mbar_cluster), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ uint32_t mapa0(uint32_t local) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(r) : "r"(local));
  return r;
}

// mode 4: clusters of 2, tensor TMA .cta_group::2 signalling the leader's barriers (as mac_pair)
__global__ void __cluster_dims__(2, 1, 1) probe2(const __grid_constant__ CUtensorMap tm, unsigned long long* out) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = raw + (((smem_u32(raw) + 1023) & ~1023u) - smem_u32(raw));
  __shared__ uint64_t bars[NBLK];
  unsigned long long t0 = global_ns();
  uint32_t rank;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  if (threadIdx.x == 0) {
    for (int b = 0; b < NBLK; ++b) mbar_init(bars + b, 1);
    fence_barrier_init();
  }
  __syncthreads();
  cluster_sync();
  const int pair = blockIdx.x >> 1;
  if (threadIdx.x == 0) {
    prefetch_tmap(&tm);
    const uint32_t lead = mapa0(smem_u32(bars));
    for (int bi = 0; bi < NBLK; ++bi) {
      const int b = (bi + pair) % NBLK;
      const int ch = b / 9, tap = b % 9;
      if (rank == 0) mbar_arrive_expect_tx(bars + b, 2 * BLK);
      tma_pair(smem_u32(sm + b * BLK), &tm, lead + 8 * b, ch * 64, tap * 128 + rank * 64);
    }
    if (rank == 0) {
      for (int b = 0; b < NBLK; ++b) mbar_wait(bars + b, 0);
      out[blockIdx.x] = global_ns() - t0;
      out[blockIdx.x + 1] = global_ns() - t0;
    }
    out[256 + blockIdx.x] = t0;
  }
  __syncthreads();
  cluster_sync();
}

__global__ void probe(const __grid_constant__ CUtensorMap tm, const uint8_t* U, int mode, int reps, int rot,
                      unsigned long long* out) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = raw + (((smem_u32(raw) + 1023) & ~1023u) - smem_u32(raw));
  __shared__ uint64_t bars[NBLK];
  unsigned long long t0 = global_ns();
  if (threadIdx.x == 0) {
    for (int b = 0; b < NBLK; ++b) mbar_init(bars + b, 1);
    fence_barrier_init();
  }
  __syncthreads();
  const int half = blockIdx.x & 1, pair = blockIdx.x >> 1;
  const int rep = (mode & 1) ? pair % reps : 0;
  if (threadIdx.x == 0) {
    prefetch_tmap(&tm);
    for (int bi = 0; bi < NBLK; ++bi) {
      const int b = rot ? (bi + pair) % NBLK : bi;
      const int ch = b / 9, tap = b % 9;
      mbar_arrive_expect_tx(bars + b, BLK);
      if (mode < 2) {
        tma_load_2d(sm + b * BLK, &tm, bars + b, ch * 64, rep * 9 * 128 + tap * 128 + half * 64);
      } else {
        // pre-swizzled contiguous layout [rep][half][ch][tap][64 rows x 128 B]
        const uint8_t* src = U + ((((size_t)rep * 2 + half) * 2 + ch) * 9 + tap) * BLK;
        bulk_g2s(smem_u32(sm + b * BLK), src, BLK, bars + b);
      }
    }
    for (int b = 0; b < NBLK; ++b) mbar_wait(bars + b, 0);
    out[blockIdx.x] = global_ns() - t0;
    out[256 + blockIdx.x] = t0;
  }
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  const int reps = 74;
  const size_t ubytes = (size_t)reps * 9 * 128 * 128 * 2;  // 74 replicas of U[9][128][128] bf16
  uint8_t* U;
  cudaMalloc(&U, ubytes);
  cudaMemset(U, 0, ubytes);
  unsigned long long* d;
  cudaMalloc(&d, 512 * sizeof(unsigned long long));
  void* f = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
  EncFn enc = reinterpret_cast<EncFn>(f);
  CUtensorMap tm;
  cuuint64_t dims[2] = {128, (cuuint64_t)reps * 9 * 128};
  cuuint64_t strides[1] = {256};
  cuuint32_t box[2] = {64, 64};
  cuuint32_t estr[2] = {1, 1};
  if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, U, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
          CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) !=
      CUDA_SUCCESS) {
    printf("encode failed\n");
    return 1;
  }
  const int smem = NBLK * BLK + 1024;
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(probe2, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const char* names[4] = {"tensor TMA, one copy", "tensor TMA, 74 replicas", "bulk 8KB, one copy",
                          "bulk 8KB, 74 replicas"};
  for (int mode = 0; mode < 4; ++mode)
    for (int rot = 0; rot < 2; ++rot) {
      std::vector<double> meds, maxs;
      for (int it = 0; it < 4; ++it) {
        probe<<<148, 128, smem>>>(tm, U, mode, reps, rot, d);
        if (cudaDeviceSynchronize() != cudaSuccess) { printf("error\n"); return 1; }
        unsigned long long h[512];
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        unsigned long long t0 = ~0ull;
        for (int i = 0; i < 148; ++i) t0 = std::min(t0, h[256 + i]);
        std::vector<double> e(148);
        for (int i = 0; i < 148; ++i) e[i] = (double)(h[256 + i] - t0 + h[i]) / 1e3;
        std::sort(e.begin(), e.end());
        if (it > 0) { meds.push_back(e[74]); maxs.push_back(e[147]); }
      }
      std::sort(meds.begin(), meds.end());
      std::sort(maxs.begin(), maxs.end());
      printf("%-26s rot %d: per-CTA done med %.2f us, max %.2f us (147 KB per CTA, 21.8 MB total)\n", names[mode], rot,
             meds[1], maxs[1]);
    }
  {
    std::vector<double> meds, maxs;
    for (int it = 0; it < 4; ++it) {
      probe2<<<148, 128, smem>>>(tm, d);
      if (cudaDeviceSynchronize() != cudaSuccess) { printf("error probe2\n"); return 1; }
      unsigned long long h[512];
      cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
      unsigned long long t0 = ~0ull;
      for (int i = 0; i < 148; ++i) t0 = std::min(t0, h[256 + i]);
      std::vector<double> e(148);
      for (int i = 0; i < 148; ++i) e[i] = (double)(h[256 + i] - t0 + h[i]) / 1e3;
      std::sort(e.begin(), e.end());
      if (it > 0) { meds.push_back(e[74]); maxs.push_back(e[147]); }
    }
    std::sort(meds.begin(), meds.end());
    std::sort(maxs.begin(), maxs.end());
    printf("%-26s rot 1: per-pair done med %.2f us, max %.2f us\n", "2CTA tensor TMA", meds[1], maxs[1]);
  }
  return 0;
}
