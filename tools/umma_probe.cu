// umma_probe.cu — design probe (not product code): can a tcgen05 K-major SW128
// smem descriptor start at an arbitrary ROW offset inside a TMA-written,
// swizzled tile?  If yes, one TMA load of a [128 + halo] x 64 window serves all
// R*S taps of the Hankel MAC (the shift Wp*i+j becomes a descriptor offset).
// For each row shift r in 0..15 and base_offset mode {0, (addr>>7)&7} it runs
// D = A[r:r+128, 0:64] * B[0:128, 0:64]^T and compares with a CPU GEMM.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include "../paper_conf_cgo_xuzc025_b200/csrc/sm100.cuh"

using namespace polyconv::sm100;

__global__ void probe(const __grid_constant__ CUtensorMap tA, const __grid_constant__ CUtensorMap tB, float* out,
                      int shift, int mode) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = raw + (((smem_u32(raw) + 1023) & ~1023u) - smem_u32(raw));
  uint8_t* sA = sm;               // 256 rows x 128 B
  uint8_t* sB = sm + 256 * 128;   // 128 rows x 128 B
  __shared__ uint64_t bar, mbar;
  __shared__ uint32_t slot;
  int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); mbar_init(&mbar, 1); fence_barrier_init(); }
  if (warp == 0) tmem_alloc(&slot, 128);
  tc_fence_before(); __syncthreads(); tc_fence_after();
  uint32_t tm = slot;
  if (threadIdx.x == 0) {
    mbar_arrive_expect_tx(&bar, 256 * 128 + 128 * 128);
    tma_load_2d(sA, &tA, &bar, 0, 0);
    tma_load_2d(sA + 128 * 128, &tA, &bar, 0, 128);
    tma_load_2d(sB, &tB, &bar, 0, 0);
    mbar_wait(&bar, 0);
    tc_fence_after();
    uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((128u >> 3) << 17) | ((128u >> 4) << 24);
    for (int ks = 0; ks < 4; ++ks) {
      uint32_t aaddr = smem_u32(sA) + shift * 128 + ks * 32;
      uint32_t boff = mode ? ((aaddr >> 7) & 7) : 0;
      uint64_t ad = make_sdesc(aaddr, 128, boff);
      uint64_t bd = make_sdesc(smem_u32(sB) + ks * 32, 128, 0);
      umma<false>(tm, ad, bd, idesc, ks);
    }
    umma_commit(&mbar);
  }
  __syncthreads();
  mbar_wait(&mbar, 0);
  tc_fence_after();
  uint32_t v[32];
  for (int c = 0; c < 128; c += 32) {
    tmem_ld32(tm + ((warp * 32) << 16) + c, v);
    tmem_ld_wait();
    for (int q = 0; q < 32; ++q) out[(warp * 32 + lane) * 128 + c + q] = __uint_as_float(v[q]);
  }
  tc_fence_before(); __syncthreads();
  if (warp == 0) { tc_fence_after(); tmem_dealloc(tm, 128); }
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  const int RA = 256, RB = 128, KD = 64;
  std::vector<__nv_bfloat16> hA(RA * KD), hB(RB * KD);
  std::vector<float> fA(RA * KD), fB(RB * KD);
  srand(1);
  for (int i = 0; i < RA * KD; ++i) { float v = (rand() % 9) - 4; hA[i] = __float2bfloat16(v); fA[i] = v; }
  for (int i = 0; i < RB * KD; ++i) { float v = (rand() % 9) - 4; hB[i] = __float2bfloat16(v); fB[i] = v; }
  void *dA, *dB; float* dO;
  cudaMalloc(&dA, RA * KD * 2); cudaMalloc(&dB, RB * KD * 2); cudaMalloc(&dO, 128 * 128 * 4);
  cudaMemcpy(dA, hA.data(), RA * KD * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB.data(), RB * KD * 2, cudaMemcpyHostToDevice);
  void* f; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
  Enc enc = (Enc)f;
  CUtensorMap tA, tB;
  cuuint64_t dimA[2] = {64, (cuuint64_t)RA}, dimB[2] = {64, (cuuint64_t)RB}, st[1] = {128};
  cuuint32_t box[2] = {64, 128}, es[2] = {1, 1};
  enc(&tA, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, dA, dimA, st, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  enc(&tB, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, dB, dimB, st, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  std::vector<float> o(128 * 128);
  for (int mode = 0; mode < 2; ++mode) {
    printf("base_offset mode %d:", mode);
    for (int shift = 0; shift < 16; ++shift) {
      cudaMemset(dO, 0, 128 * 128 * 4);
      probe<<<1, 128, 200 * 1024>>>(tA, tB, dO, shift, mode);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf(" shift %d: %s\n", shift, cudaGetErrorString(e)); return 1; }
      cudaMemcpy(o.data(), dO, 128 * 128 * 4, cudaMemcpyDeviceToHost);
      int bad = 0;
      for (int m = 0; m < 128; ++m)
        for (int n = 0; n < 128; ++n) {
          float s = 0;
          for (int k = 0; k < KD; ++k) s += fA[(m + shift) * KD + k] * fB[n * KD + k];
          if (s != o[m * 128 + n]) ++bad;
        }
      printf(" %d:%s", shift, bad ? "BAD" : "ok");
    }
    printf("\n");
  }
  return 0;
}
