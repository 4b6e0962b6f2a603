// mn_probe.cu — design probe (not product code): which shared-memory descriptor
// encoding makes tcgen05.mma read an MN-major B operand (positions contiguous, as
// NCHW planes are) that TMA wrote as SW128 boxes of [64 channels][64 positions].
// D[m][n] = sum_k A[m][k] * B[k][n], M = 128, N = 128 (two 64-position boxes), K = 16..64.
// A: K-major SW128 [128 rows][64 k].  B: MN-major, box b holds positions 64b..64b+63 as
// 64 k-rows of 128 bytes.  Tries (LBO, SBO) pairs and reports which matches the CPU result.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mn tools/mn_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <vector>
#include "../paper_conf_cgo_xuzc025_b200/csrc/sm100.cuh"

using namespace polyconv::sm100;

__device__ __forceinline__ uint64_t desc_raw(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1u << 46;
  d |= (uint64_t)layout << 61;
  return d;
}

__global__ void probe(const __grid_constant__ CUtensorMap tA, const __grid_constant__ CUtensorMap tB, float* D,
                      uint32_t lbo, uint32_t sbo, int ksteps) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = raw + (((smem_u32(raw) + 1023) & ~1023u) - smem_u32(raw));
  uint8_t* sA = sm;              // 128 x 128 B = 16 KB
  uint8_t* sB = sm + 16384;      // 2 boxes x 8 KB
  __shared__ uint64_t bar, mbar;
  __shared__ uint32_t slot;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); mbar_init(&mbar, 1); fence_barrier_init(); }
  if (threadIdx.x < 32) tmem_alloc(&slot, 128);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = slot;
  if (threadIdx.x == 0) {
    mbar_arrive_expect_tx(&bar, 16384 + 16384);
    tma_load_2d(sA, &tA, &bar, 0, 0);
    tma_load_2d(sB, &tB, &bar, 0, 0);        // positions 0..63, channels 0..63
    tma_load_2d(sB + 8192, &tB, &bar, 64, 0);  // positions 64..127
    mbar_wait(&bar, 0);
    // D f32, A bf16 (K-major), B bf16 (MN-major: transpose-B bit 16), N = 128, M = 128
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((128u >> 3) << 17) | ((128u >> 4) << 24);
    for (int ks = 0; ks < ksteps; ++ks) {
      const uint64_t ad = make_sdesc(smem_u32(sA) + 32 * ks, 128, 0);
      // MN-major: a K step of 16 rows = 16 x 128 B
      const uint64_t bd = desc_raw(smem_u32(sB) + 16 * 128 * ks, lbo, sbo, 2);
      umma<false>(tm, ad, bd, idesc, ks > 0);
    }
    umma_commit(&mbar);
    mbar_wait(&mbar, 0);
  }
  __syncthreads();
  tc_fence_after();
  // each warp w < 4 reads lanes 32w..32w+31, 128 columns in 4 chunks
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp < 4) {
    for (int c = 0; c < 128; c += 32) {
      uint32_t v[32];
      tmem_ld32(tm + ((uint32_t)(warp * 32) << 16) + c, v);
      tmem_ld_wait();
      for (int j = 0; j < 32; ++j) D[(warp * 32 + lane) * 128 + c + j] = __uint_as_float(v[j]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) { tc_fence_after(); tmem_dealloc(tm, 128); }
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  const int M = 128, N = 128, K = 64;
  std::vector<__nv_bfloat16> hA(M * K), hB(K * N);  // A[m][k], B stored [k][n] (n contiguous)
  std::vector<float> fA(M * K), fB(K * N);
  srand(1);
  for (int i = 0; i < M * K; ++i) { fA[i] = (float)(rand() % 9 - 4); hA[i] = __float2bfloat16(fA[i]); }
  for (int i = 0; i < K * N; ++i) { fB[i] = (float)(rand() % 9 - 4); hB[i] = __float2bfloat16(fB[i]); }
  __nv_bfloat16 *dA, *dB;
  float* dD;
  cudaMalloc(&dA, M * K * 2); cudaMalloc(&dB, K * N * 2); cudaMalloc(&dD, M * N * 4);
  cudaMemcpy(dA, hA.data(), M * K * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB.data(), K * N * 2, cudaMemcpyHostToDevice);
  void* f = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
  EncFn enc = reinterpret_cast<EncFn>(f);
  CUtensorMap tA, tB;
  cuuint64_t dA2[2] = {(cuuint64_t)K, (cuuint64_t)M}, sA2[1] = {(cuuint64_t)K * 2};
  cuuint32_t bA[2] = {64, 128}, es[2] = {1, 1};
  enc(&tA, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, dA, dA2, sA2, bA, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cuuint64_t dB2[2] = {(cuuint64_t)N, (cuuint64_t)K}, sB2[1] = {(cuuint64_t)N * 2};
  cuuint32_t bB[2] = {64, 64};
  enc(&tB, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, dB, dB2, sB2, bB, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 48 * 1024);
  std::vector<float> ref(M * N, 0.f), got(M * N);
  for (int ksteps : {1, 4}) {
    const int Kd = 16 * ksteps;
    for (int m = 0; m < M; ++m)
      for (int n = 0; n < N; ++n) {
        float s = 0;
        for (int k = 0; k < Kd; ++k) s += fA[m * K + k] * fB[k * N + n];
        ref[m * N + n] = s;
      }
    // found by sweeping {128 .. 16384}^2 at K = 16 (larger values fault): LBO = 8192 (the next
    // 64-position box), SBO = 1024 (the next 8 k-rows); K = 64 checks the +2048-byte K step
    const uint32_t lbos[] = {8192}, sbos[] = {1024};
    for (uint32_t lbo : lbos)
      for (uint32_t sbo : sbos) {
        cudaMemset(dD, 0, M * N * 4);
        probe<<<1, 128, 48 * 1024>>>(tA, tB, dD, lbo, sbo, ksteps);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("lbo %u sbo %u: %s\n", lbo, sbo, cudaGetErrorString(e)); return 1; }
        cudaMemcpy(got.data(), dD, M * N * 4, cudaMemcpyDeviceToHost);
        int bad = 0;
        for (int i = 0; i < M * N; ++i) bad += std::fabs(got[i] - ref[i]) > 0.5f;
        printf("K=%d lbo=%u sbo=%u: %s (%d mismatches)\n", Kd, lbo, sbo, bad ? "WRONG" : "MATCH", bad);
      }
  }
  printf("done\n");
  return 0;
}
