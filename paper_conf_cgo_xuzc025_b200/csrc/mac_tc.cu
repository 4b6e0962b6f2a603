// mac_tc.cu — a4+a5 on the 5th-gen tensor cores (tcgen05 + TMEM + TMA), the
// TF32 / BF16 hot path.
//
// The coefficient MAC
//   p_{n,k}[m] = sum_c sum_{i,j} A_{n,c}[m - e(i,j)] * U_{k,c}[e(i,j)]   (P.965, P.1350-1352)
// restricted to the extraction degrees m = base + L_U - 1 is, per kernel tap
// (i,j), a GEMM whose B operand is a *contiguous shifted window* of the packed
// input polynomials -- the doubly blocked Hankel structure (P.404-437) made
// concrete:
//   D[base][k] += sum_c Apack[n*L_A + base + Wp*i + j][c] * Utap[(i,j)][k][c]
// The positions of all images are concatenated (g = n*L_A + base); junk
// positions (off the extraction lattice, or past a plane's last output) are
// computed and dropped, windows that run past the tensor are zero-filled by TMA.
//
// Kernel structure (persistent, one CTA per SM, 6 warps):
//   warp 0  TMA producer (one lane): per k-block (tap, channel chunk) loads the
//           shifted A window [128 positions x kc] and the filter tile [bn x kc]
//           into a `stages`-deep smem ring (128B/64B/32B swizzle).
//   warp 1  TMEM allocator + UMMA issuer (one lane): tcgen05.mma M=128 x N=bn
//           x K=32 bytes per instruction, fp32 accumulators in TMEM, two
//           accumulator buffers so the epilogue of tile t overlaps the MMAs of t+1.
//   warps 2-5 epilogue: tcgen05.ld 32 lanes x 32 columns -> registers, fused
//           extraction (Eq. 12 + R4) and the strided NCHW store (a5).
#include <cuda.h>
#include "common.cuh"
#include "sm100.cuh"
#include <cstdio>

namespace polyconv {

namespace {

using namespace sm100;

constexpr int BM = 128;          // positions per tile (UMMA M, TMEM lanes)
constexpr int kThreads = 192;    // 6 warps

struct TcParams {
  long long G;       // position extent: (N-1)*L_A + M_ext
  long long L_A;
  int Wp, P, Q, sh, sw, K, S, RS;
  int num_m, num_n, num_tiles;
  int nchunks, kblocks, kc;
  int bn, row_bytes, stages, tmem_cols, Kp;
  uint32_t idesc;
  uint32_t a_bytes, b_bytes;  // per stage
  void* y;
  int y_bf16;
};

template <bool kTf32>
__global__ void __launch_bounds__(kThreads, 1)
    mac_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                  const TcParams p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);  // 1024B for the swizzle atoms
  uint8_t* sA = smem;
  uint8_t* sB = smem + (size_t)p.stages * p.a_bytes;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + (size_t)p.stages * p.b_bytes);
  uint64_t* empty = full + p.stages;
  uint64_t* tfull = empty + p.stages;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    for (int s = 0; s < p.stages; ++s) {
      mbar_init(full + s, 1);
      mbar_init(empty + s, 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(tfull + a, 1);
      mbar_init(tempty + a, 4);  // one arrive per epilogue warp
    }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc(tmem_slot, (uint32_t)p.tmem_cols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ------------------------------------------------ TMA producer
      int stage = 0;
      uint32_t phase = 0;
      for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
        const int mt = tile / p.num_n, nt = tile - mt * p.num_n;
        const long long g0 = (long long)mt * BM;
        const int brow0 = nt * p.bn;
        for (int tap = 0; tap < p.RS; ++tap) {
          const int i = tap / p.S, j = tap - i * p.S;
          const int arow = (int)(g0 + (long long)p.Wp * i + j);  // shifted window (Hankel)
          const int brow = tap * p.Kp + brow0;
          for (int ch = 0; ch < p.nchunks; ++ch) {
            mbar_wait(empty + stage, phase ^ 1u);
            mbar_arrive_expect_tx(full + stage, p.a_bytes + p.b_bytes);
            tma_load_2d(sA + (size_t)stage * p.a_bytes, &tmA, full + stage, ch * p.kc, arow);
            tma_load_2d(sB + (size_t)stage * p.b_bytes, &tmB, full + stage, ch * p.kc, brow);
            if (++stage == p.stages) { stage = 0; phase ^= 1u; }
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ------------------------------------------------ UMMA issuer
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      const int ksteps = p.row_bytes / 32;
      for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
        mbar_wait(tempty + acc, acc_phase ^ 1u);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + (uint32_t)(acc * p.bn);
        for (int kb = 0; kb < p.kblocks; ++kb) {
          mbar_wait(full + stage, phase);
          tc_fence_after();
          const uint32_t a_addr = smem_u32(sA + (size_t)stage * p.a_bytes);
          const uint32_t b_addr = smem_u32(sB + (size_t)stage * p.b_bytes);
          for (int ks = 0; ks < ksteps; ++ks) {
            const uint64_t ad = make_sdesc(a_addr + 32u * ks, p.row_bytes, 0);
            const uint64_t bd = make_sdesc(b_addr + 32u * ks, p.row_bytes, 0);
            umma<kTf32>(d_tmem, ad, bd, p.idesc, (uint32_t)(kb | ks));
          }
          umma_commit(empty + stage);  // frees the smem slot when these MMAs complete
          if (++stage == p.stages) { stage = 0; phase ^= 1u; }
        }
        umma_commit(tfull + acc);  // accumulator ready for the epilogue
        if (++acc == 2) { acc = 0; acc_phase ^= 1u; }
      }
    }
  } else {
    // ------------------------------------------------ epilogue (warps 2..5)
    const int quad = warp & 3;  // TMEM lane quadrant this warp may access
    const long long PQ = (long long)p.P * p.Q;
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int tile = blockIdx.x; tile < p.num_tiles; tile += gridDim.x) {
      const int mt = tile / p.num_n, nt = tile - mt * p.num_n;
      const long long gpos = (long long)mt * BM + quad * 32 + lane;
      // a5: degree -> (n, oh, ow); valid iff on the extraction lattice
      const long long n = gpos / p.L_A;
      const int m = (int)(gpos - n * p.L_A);
      const int r = m / p.Wp, s = m - r * p.Wp;
      const int oh = r / p.sh, ow = s / p.sw;
      const bool valid = gpos < p.G && (r - oh * p.sh) == 0 && (s - ow * p.sw) == 0 && oh < p.P && ow < p.Q;
      const int k0 = nt * p.bn;
      const long long ybase = (n * p.K + k0) * PQ + (long long)oh * p.Q + ow;
      mbar_wait(tfull + acc, acc_phase);
      tc_fence_after();
      const uint32_t trow = tmem_base + ((uint32_t)(quad * 32) << 16) + (uint32_t)(acc * p.bn);
      for (int c = 0; c < p.bn; c += 32) {
        uint32_t v[32];
        tmem_ld32(trow + (uint32_t)c, v);
        tmem_ld_wait();
        if (valid) {
          const int kmax = min(32, p.K - (k0 + c));
          if (p.y_bf16) {
            __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.y);
#pragma unroll
            for (int q = 0; q < 32; ++q)
              if (q < kmax) y[ybase + (long long)(c + q) * PQ] = __float2bfloat16_rn(__uint_as_float(v[q]));
          } else {
            float* y = reinterpret_cast<float*>(p.y);
#pragma unroll
            for (int q = 0; q < 32; ++q)
              if (q < kmax) y[ybase + (long long)(c + q) * PQ] = __uint_as_float(v[q]);
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(tempty + acc);
      if (++acc == 2) { acc = 0; acc_phase ^= 1u; }
    }
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem_base, (uint32_t)p.tmem_cols);
  }
}

// ---- host side ------------------------------------------------------------------
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(f);
  }
  return fn;
}

bool encode_2d(CUtensorMap* map, const void* base, int fmt, uint64_t cols, uint64_t rows, uint32_t box_cols,
               uint32_t box_rows, int row_bytes) {
  EncodeTiledFn enc = get_encode();
  if (!enc) return false;
  const int eb = fmt_bytes(fmt);
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {cols * (uint64_t)eb};
  cuuint32_t box[2] = {box_cols, box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUtensorMapSwizzle sw = row_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                          : row_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                            : CU_TENSOR_MAP_SWIZZLE_32B;
  CUtensorMapDataType dt = fmt == FMT_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32;
  CUresult r = enc(map, dt, 2, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

}  // namespace

bool tc_supported(const Geom& g, int fmt) {
  if (fmt != FMT_BF16 && fmt != FMT_TF32) return false;
  if ((long long)g.N * g.L_A >= (1LL << 31) - 4096) return false;  // TMA row coordinate is int32
  if ((long long)g.R * g.S * g.Kp >= (1LL << 31)) return false;
  return true;
}

TcTiling tc_tiling(const Geom& g, int fmt, int num_sms) {
  TcTiling t{};
  const int eb = fmt_bytes(fmt);
  t.bm = BM;
  // channels per k-block: one swizzle row of 128/64/32 bytes, the smallest that holds C
  int kc = 128 / eb;
  const int kmin = 32 / eb;
  while (kc > kmin && kc / 2 >= g.C) kc /= 2;
  t.kc = kc;
  t.row_bytes = kc * eb;
  // output channels per tile (UMMA N): K rounded up to 32, at most 256
  const int kp32 = (g.K + 31) / 32 * 32;
  t.bn = kp32 <= 256 ? kp32 : 256;
  const int stage_bytes = (BM + t.bn) * t.row_bytes;
  const int budget = 227 * 1024 - 1024 - 256;
  t.stages = budget / stage_bytes;
  if (t.stages > 8) t.stages = 8;
  t.smem_bytes = t.stages * stage_bytes + 1024 + 256;
  int cols = 32;
  while (cols < 2 * t.bn) cols <<= 1;
  t.tmem_cols = cols;
  const long long G = (long long)(g.N - 1) * g.L_A + g.M_ext;
  t.num_m = (int)((G + BM - 1) / BM);
  t.num_n = ((g.K + t.bn - 1) / t.bn);
  t.kblocks = g.R * g.S * ((g.C + kc - 1) / kc);
  long long tiles = (long long)t.num_m * t.num_n;
  t.grid = (int)(tiles < num_sms ? tiles : num_sms);
  return t;
}

cudaError_t launch_mac_tc(const Geom& g, const TcTiling& t, int fmt, const void* A, const void* U, void* y,
                          bool y_bf16, cudaStream_t st, char* err, size_t errlen) {
  CUtensorMap tmA, tmB;
  if (!encode_2d(&tmA, A, fmt, (uint64_t)g.Cp, (uint64_t)g.N * g.L_A, t.kc, BM, t.row_bytes) ||
      !encode_2d(&tmB, U, fmt, (uint64_t)g.Cp, (uint64_t)g.R * g.S * g.Kp, t.kc, t.bn, t.row_bytes)) {
    snprintf(err, errlen, "cuTensorMapEncodeTiled failed");
    return cudaErrorInvalidValue;
  }
  TcParams p{};
  p.G = (long long)(g.N - 1) * g.L_A + g.M_ext;
  p.L_A = g.L_A;
  p.Wp = g.Wp; p.P = g.P; p.Q = g.Q; p.sh = g.sh; p.sw = g.sw; p.K = g.K; p.S = g.S;
  p.RS = g.R * g.S;
  p.num_m = t.num_m; p.num_n = t.num_n; p.num_tiles = t.num_m * t.num_n;
  p.nchunks = g.Cp / t.kc;
  p.kblocks = p.RS * p.nchunks;
  p.kc = t.kc;
  p.bn = t.bn; p.row_bytes = t.row_bytes; p.stages = t.stages; p.tmem_cols = t.tmem_cols; p.Kp = g.Kp;
  // instruction descriptor: D=f32, A/B = bf16(1) or tf32(2), both K-major, N>>3 @17, M>>4 @24
  const uint32_t ab = fmt == FMT_BF16 ? 1u : 2u;
  p.idesc = (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(t.bn >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
  p.a_bytes = (uint32_t)(BM * t.row_bytes);
  p.b_bytes = (uint32_t)(t.bn * t.row_bytes);
  p.y = y;
  p.y_bf16 = y_bf16 ? 1 : 0;
  cudaError_t e;
  if (fmt == FMT_TF32) {
    e = cudaFuncSetAttribute(mac_tc_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, t.smem_bytes);
    if (e != cudaSuccess) return e;
    mac_tc_kernel<true><<<t.grid, kThreads, t.smem_bytes, st>>>(tmA, tmB, p);
  } else {
    e = cudaFuncSetAttribute(mac_tc_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, t.smem_bytes);
    if (e != cudaSuccess) return e;
    mac_tc_kernel<false><<<t.grid, kThreads, t.smem_bytes, st>>>(tmA, tmB, p);
  }
  return cudaGetLastError();
}

}  // namespace polyconv
