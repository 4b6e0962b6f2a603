// mac_tc2.cu — a4+a5 on the 5th-gen tensor cores with Hankel-window reuse:
// the default TF32 / BF16 hot path.
//
// The coefficient MAC
//   p_{n,k}[m] = sum_c sum_{i,j} A_{n,c}[m - e(i,j)] * U_{k,c}[e(i,j)]   (P.965, P.1350-1352)
// at m = base + L_U - 1 is, per kernel tap (i,j), a GEMM whose position operand
// is the packed input shifted by Wp*i + j coefficients (the doubly blocked
// Hankel structure, P.404-437):
//   D[k][base] += sum_c U_tap(i,j)[k][c] * Apack[base + Wp*i + j][c]
//
// Design ("mac_tc"):
//  * UMMA A operand = filter tile U_tap[k0:k0+128][c-chunk] (M = 128 output
//    channels); B operand = a window of positions of the packed input
//    (N = nt positions, 16 <= nt <= 256, chosen so the tiles fill the 148 SMs
//    in as few waves as possible); both K-major, 128/64/32-byte swizzle.
//  * Window reuse: for one channel chunk the producer loads ONE window of
//    nt + (nr-1)*Wp + S-1 consecutive positions (nr kernel rows per window; all
//    R rows when it fits), and every tap (i,j) of those rows reads it through a
//    shared-memory descriptor whose start is shifted by (Wp*i + j) rows.  The
//    shifted descriptor start inside a TMA-swizzled tile is exact (probe:
//    tools/umma_probe.cu, profiles/r01_umma_probe.txt).  For 3x3 this cuts the
//    position-operand traffic L2->SMEM 9x relative to one load per tap.
//  * Persistent, warp-specialised: warp 0 = TMA producer (one lane), warp 1 =
//    TMEM allocator + UMMA issuer (one lane), warps 2-5 = epilogue.  Two TMEM
//    accumulators (tile t's epilogue overlaps tile t+1's MMAs).
//  * Epilogue (a5, fused): tcgen05.ld 32 channels x 32 positions -> shared
//    transpose -> each lane owns one position, stores 32 channels with
//    consecutive lanes at consecutive output pixels (coalesced NCHW rows);
//    junk positions (off the Eq. 12 / R4 extraction lattice) are dropped.
#include <cuda.h>
#include "common.cuh"
#include "sm100.cuh"
#include <cstdio>
#include <cstdlib>

namespace polyconv {

namespace {

using namespace sm100;

constexpr int BMK = 128;        // output channels per tile (UMMA M, TMEM lanes)
constexpr int kEpiWarps = 8;  // 2 per TMEM lane quadrant
constexpr int kThreads = 64 + 32 * kEpiWarps;
constexpr int kBoxRows = 32;    // rows per TMA box of the position window
constexpr int kBMaxRows = 384;  // max rows of one position window (48 KB at 128 B rows)
constexpr int kTStride = 33;    // epilogue transpose row stride (floats), conflict-free

struct Tc2Params {
  long long G;      // positions with outputs: (N-1)*L_A + M_ext
  long long L_A;
  long long PQ;
  int Wp, P, Q, sh, sw, K, R, S;
  int nt, brows, nr, ngroups;
  int num_mt, num_kt, num_tiles, num_groups;
  int nchunks, kc, Kp;
  int a_stages;
  uint32_t idesc, a_bytes, b_bytes, row_bytes;
  int acc_stride, tmem_cols;
  void* y;
  int y_bf16;
  int dbg;  // measurement ablations (POLYCONV_TC_DEBUG): 1 = no TMA after the first
            // fill (MMA+epilogue only), 2 = no MMA (TMA only), 4 = no output stores
};

// per-CTA phase timestamps (globaltimer ns) for POLYCONV_TC_DEBUG & 8
__device__ unsigned long long g_tc2_trace[160 * 8];
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

template <bool kTf32, int CS>
__global__ void __launch_bounds__(kThreads, 1)
    mac_tc2_kernel(const __grid_constant__ CUtensorMap tmW, const __grid_constant__ CUtensorMap tmX,
                   const Tc2Params p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  uint8_t* sA = smem;                                        // filter tiles  [a_stages][128][row]
  uint8_t* sB = sA + (size_t)p.a_stages * p.a_bytes;         // position windows [2][brows][row]
  float* sT = reinterpret_cast<float*>(sB + 2 * (size_t)p.b_bytes);  // [kEpiWarps][32][33]
  uint64_t* afull = reinterpret_cast<uint64_t*>(sT + kEpiWarps * 32 * kTStride);
  uint64_t* aempty = afull + p.a_stages;
  uint64_t* bfull = aempty + p.a_stages;
  uint64_t* bempty = bfull + 2;
  uint64_t* tfull = bempty + 2;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // clusters of CS CTAs share one output-channel block: the filter tiles are
  // multicast (each CTA loads 128/CS rows into every peer), the position
  // windows are per CTA (rank r takes position tile mg*CS + r)
  const uint32_t rank = CS > 1 ? cluster_ctarank() : 0u;
  const int cl_id = (int)blockIdx.x / CS, cl_num = (int)gridDim.x / CS;
  const bool trace = (p.dbg & 8) && blockIdx.x < 160;
  unsigned long long* tr = g_tc2_trace + blockIdx.x * 8;
  if (trace && threadIdx.x == 0) tr[0] = gtimer();

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmW);
    prefetch_tmap(&tmX);
    for (int s = 0; s < p.a_stages; ++s) {
      mbar_init(afull + s, 1);
      mbar_init(aempty + s, CS);  // every CTA of the cluster reads the multicast filter tile
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(bfull + s, 1);
      mbar_init(bempty + s, 1);
      mbar_init(tfull + s, 1);
      mbar_init(tempty + s, kEpiWarps);
    }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc(tmem_slot, (uint32_t)p.tmem_cols);
  tc_fence_before();
  __syncthreads();
  if constexpr (CS > 1) cluster_sync();  // peers' barriers are initialised before any multicast
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  if (trace && threadIdx.x == 0) tr[1] = gtimer();

  if (warp == 0) {
    // -------------------------------------------------------------- TMA producer
    // The whole warp runs the loop (uniform control values); one elected lane issues.
    int as = 0, bs = 0, na = 0, nb = 0;
    uint32_t aph = 0, bph = 0;
    for (int grp = cl_id; grp < p.num_groups; grp += cl_num) {
      const int mg = grp / p.num_kt, kt = grp - mg * p.num_kt;
      const long long g0 = (long long)(mg * CS + (int)rank) * p.nt;  // may lie past G: dummy tile
      const int krow0 = kt * BMK;
      for (int ch = 0; ch < p.nchunks; ++ch) {
        for (int rg = 0; rg < p.ngroups; ++rg) {
          const int i0 = rg * p.nr, i1 = min(p.R, i0 + p.nr);
          // one window of positions serves every tap of kernel rows [i0, i1)
          mbar_wait(bempty + bs, bph ^ 1u);
          if (elect_one()) {
            if ((p.dbg & 1) && nb >= 2) {
              mbar_arrive(bfull + bs);
            } else {
              mbar_arrive_expect_tx(bfull + bs, p.b_bytes);
              const int wrow = (int)(g0 + (long long)p.Wp * i0);
              uint8_t* dst = sB + (size_t)bs * p.b_bytes;
              for (int r = 0; r < p.brows; r += kBoxRows)
                tma_load_2d(dst + (size_t)r * p.row_bytes, &tmX, bfull + bs, ch * p.kc, wrow + r);
            }
          }
          __syncwarp();
          ++nb;
          if (++bs == 2) { bs = 0; bph ^= 1u; }
          for (int i = i0; i < i1; ++i) {
            for (int j = 0; j < p.S; ++j) {
              mbar_wait(aempty + as, aph ^ 1u);
              if (elect_one()) {
                if ((p.dbg & 1) && na >= p.a_stages) {
                  mbar_arrive(afull + as);
                } else {
                  mbar_arrive_expect_tx(afull + as, p.a_bytes);
                  if constexpr (CS == 1) {
                    tma_load_2d(sA + (size_t)as * p.a_bytes, &tmW, afull + as, ch * p.kc,
                                (i * p.S + j) * p.Kp + krow0);
                  } else {
                    constexpr int kSub = BMK / CS;  // filter rows this CTA loads for the cluster
                    tma_load_2d_mc(sA + (size_t)as * p.a_bytes + (size_t)rank * kSub * p.row_bytes, &tmW,
                                   afull + as, ch * p.kc, (i * p.S + j) * p.Kp + krow0 + (int)rank * kSub,
                                   (uint16_t)((1u << CS) - 1));
                  }
                }
              }
              __syncwarp();
              ++na;
              if (++as == p.a_stages) { as = 0; aph ^= 1u; }
            }
          }
        }
      }
    }
  } else if (warp == 1) {
    // -------------------------------------------------------------- UMMA issuer
    int as = 0, bs = 0, acc = 0;
    uint32_t aph = 0, bph = 0, accph = 0;
    const int ksteps = (int)p.row_bytes / 32;
    const uint32_t sA0 = smem_u32(sA), sB0 = smem_u32(sB);
    for (int grp = cl_id; grp < p.num_groups; grp += cl_num) {
      mbar_wait(tempty + acc, accph ^ 1u);
      tc_fence_after();
      const uint32_t d_tmem = tmem_base + (uint32_t)(acc * p.acc_stride);
      uint32_t accumulate = 0;
      for (int ch = 0; ch < p.nchunks; ++ch) {
        for (int rg = 0; rg < p.ngroups; ++rg) {
          const int i0 = rg * p.nr, i1 = min(p.R, i0 + p.nr);
          mbar_wait(bfull + bs, bph);
          tc_fence_after();
          if (trace && lane == 0 && ch == 0 && rg == 0 && grp == cl_id) tr[2] = gtimer();
          const uint32_t b_addr = sB0 + (uint32_t)bs * p.b_bytes;
          for (int i = i0; i < i1; ++i) {
            for (int j = 0; j < p.S; ++j) {
              mbar_wait(afull + as, aph);
              tc_fence_after();
              // Hankel shift of tap (i,j) inside the window: Wp*(i-i0) + j rows
              const uint32_t b_shift = (p.dbg & 16) ? 0u : (uint32_t)(p.Wp * (i - i0) + j) * p.row_bytes;
              const uint64_t ad = make_sdesc(sA0 + (uint32_t)as * p.a_bytes, p.row_bytes, 0);
              const uint64_t bd = make_sdesc(b_addr + b_shift, p.row_bytes, 0);
              if (elect_one()) {
                if (p.dbg & 2) {
                  if constexpr (CS == 1) mbar_arrive(aempty + as);
                  else umma_commit_mc(aempty + as, (uint16_t)((1u << CS) - 1));
                } else {
                  // K step = 32 bytes = +2 in the descriptor's start-address field
                  for (int ks = 0; ks < ksteps; ++ks) {
                    umma<kTf32>(d_tmem, ad + 2 * ks, bd + 2 * ks, p.idesc, accumulate);
                    accumulate = 1;
                  }
                  // filter slot free (in every CTA of the cluster) when these MMAs finish
                  if constexpr (CS == 1) umma_commit(aempty + as);
                  else umma_commit_mc(aempty + as, (uint16_t)((1u << CS) - 1));
                }
              }
              __syncwarp();
              accumulate = 1;
              if (++as == p.a_stages) { as = 0; aph ^= 1u; }
            }
          }
          if (elect_one()) {
            if (p.dbg & 2) mbar_arrive(bempty + bs);
            else umma_commit(bempty + bs);  // window free when every tap using it finished
          }
          __syncwarp();
          if (++bs == 2) { bs = 0; bph ^= 1u; }
        }
      }
      if (trace && lane == 0) tr[3] = gtimer();
      if (elect_one()) {
        if (p.dbg & 2) mbar_arrive(tfull + acc);
        else umma_commit(tfull + acc);
      }
      __syncwarp();
      if (++acc == 2) { acc = 0; accph ^= 1u; }
    }
  } else {
    // -------------------------------------------------------------- epilogue
    // kEpiWarps warps; warp w reads TMEM lane quadrant (w % 4) and every
    // (kEpiWarps/4)-th 32-column block of the accumulator.
    const int ew = warp - 2;
    const int quad = warp & 3;
    const int csub = ew >> 2, cstep = kEpiWarps / 4;
    float* T = sT + ew * 32 * kTStride;
    int acc = 0;
    uint32_t accph = 0;
    for (int grp = cl_id; grp < p.num_groups; grp += cl_num) {
      const int mg = grp / p.num_kt, kt = grp - mg * p.num_kt;
      const long long g0 = (long long)(mg * CS + (int)rank) * p.nt;
      const int kq = kt * BMK + quad * 32;  // first output channel of this warp's lanes
      const int kmax = min(32, p.K - kq);
      // decode the tile's first position once: g0 = n0 * L_A + m0
      const long long n0 = g0 / p.L_A;
      const int m0 = (int)(g0 - n0 * p.L_A);
      mbar_wait(tfull + acc, accph);
      tc_fence_after();
      if (trace && ew == 0 && lane == 0) tr[4] = gtimer();
      const uint32_t taddr = tmem_base + ((uint32_t)(quad * 32) << 16) + (uint32_t)(acc * p.acc_stride);
      for (int cb = csub * 32; cb < p.nt; cb += 32 * cstep) {
        uint32_t v[32];
        tmem_ld32(taddr + (uint32_t)cb, v);
        tmem_ld_wait();
#pragma unroll
        for (int q = 0; q < 32; ++q) T[lane * kTStride + q] = __uint_as_float(v[q]);
        __syncwarp();
        // lane -> position g0 + cb + lane; a5: keep it iff on the extraction lattice
        const int c = cb + lane;
        long long n = n0;
        int m = m0 + c;
        while (m >= p.L_A) { m -= (int)p.L_A; ++n; }
        const int r = m / p.Wp, s = m - r * p.Wp;
        const int oh = r / p.sh, ow = s / p.sw;
        const bool valid = c < p.nt && g0 + c < p.G && (r - oh * p.sh) == 0 && (s - ow * p.sw) == 0 &&
                           oh < p.P && ow < p.Q;
        if (valid && !(p.dbg & 4)) {
          const long long ybase = (n * p.K + kq) * p.PQ + (long long)oh * p.Q + ow;
          if (p.y_bf16) {
            __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.y) + ybase;
#pragma unroll 8
            for (int q = 0; q < kmax; ++q) y[(long long)q * p.PQ] = __float2bfloat16_rn(T[q * kTStride + lane]);
          } else {
            float* y = reinterpret_cast<float*>(p.y) + ybase;
#pragma unroll 8
            for (int q = 0; q < kmax; ++q) y[(long long)q * p.PQ] = T[q * kTStride + lane];
          }
        }
        __syncwarp();
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(tempty + acc);
      if (trace && ew == 0 && lane == 0) tr[5] = gtimer();
      if (++acc == 2) { acc = 0; accph ^= 1u; }
    }
  }
  if (trace && warp == 0 && lane == 0) tr[6] = gtimer();
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if constexpr (CS > 1) cluster_sync();  // no CTA exits while peers may still signal it
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem_base, (uint32_t)p.tmem_cols);
  }
  if (trace && threadIdx.x == 0) tr[7] = gtimer();
}

// ---- host side ------------------------------------------------------------------
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode2() {
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

bool encode(CUtensorMap* map, const void* base, int fmt, uint64_t cols, uint64_t rows, uint32_t box_cols,
            uint32_t box_rows, int row_bytes) {
  EncodeTiledFn enc = get_encode2();
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
  return enc(map, dt, 2, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
             CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

inline long long cdiv(long long a, long long b) { return (a + b - 1) / b; }

}  // namespace

bool tc2_supported(const Geom& g, int fmt) {
  if (fmt != FMT_BF16 && fmt != FMT_TF32) return false;
  if ((long long)g.N * g.L_A + 4096 >= (1LL << 31)) return false;  // TMA row coordinate is int32
  if ((long long)g.R * g.S * ((g.K + 127) / 128 * 128) >= (1LL << 31)) return false;
  if (g.S - 1 + 16 > kBMaxRows) return false;  // one kernel row must fit a window
  return true;
}

Tc2Tiling tc2_tiling(const Geom& g, int fmt, int num_sms) {
  Tc2Tiling t{};
  const int eb = fmt_bytes(fmt);
  int kc = 128 / eb;
  const int kmin = 32 / eb;
  while (kc > kmin && kc / 2 >= g.C) kc /= 2;
  t.kc = kc;
  t.row_bytes = kc * eb;
  t.num_kt = (g.K + BMK - 1) / BMK;
  const long long G = (long long)(g.N - 1) * g.L_A + g.M_ext;
  // positions per tile: fewest waves over the SMs, then the largest tile
  long long best_cost = -1;
  const char* force_nt = getenv("POLYCONV_TC_NT");  // experiments only
  // clusters of 2 CTAs share (multicast) the filter tiles; 148 SMs = 74 pairs
  const char* force_cs = getenv("POLYCONV_TC_CS");  // experiments only
  t.cs = force_cs ? atoi(force_cs) : 2;
  if (t.cs != 1 && t.cs != 2 && t.cs != 4) t.cs = 2;
  if (cdiv(G, 16) < 2) t.cs = 1;
  for (int nt = 16; nt <= 256; nt += 16) {
    if (force_nt && nt != atoi(force_nt)) continue;
    if (nt + g.S - 1 > kBMaxRows) break;
    const long long groups = cdiv(cdiv(G, nt), t.cs) * t.num_kt;
    const long long waves = cdiv(groups, num_sms / t.cs);
    const long long cost = waves * (nt + 32);  // +32: per-tile fixed cost in position units
    if (best_cost < 0 || cost <= best_cost) {
      best_cost = cost;
      t.nt = nt;
    }
  }
  // kernel rows per position window: as many as fit kBMaxRows
  int nr = g.R;
  while (nr > 1 && (long long)t.nt + (long long)(nr - 1) * g.Wp + g.S - 1 > kBMaxRows) --nr;
  t.nr = nr;
  t.ngroups = (g.R + nr - 1) / nr;
  t.brows = (int)cdiv((long long)t.nt + (long long)(nr - 1) * g.Wp + g.S - 1, kBoxRows) * kBoxRows;
  t.num_mt = (int)cdiv(G, t.nt);
  t.num_tiles = t.num_mt * t.num_kt;
  t.num_groups = (int)cdiv(t.num_mt, t.cs) * t.num_kt;
  t.nchunks = (g.C + kc - 1) / kc;
  const int a_bytes = BMK * t.row_bytes;
  const int b_bytes = t.brows * t.row_bytes;
  const int fixed = 1024 + 2 * b_bytes + kEpiWarps * 32 * kTStride * 4 + 512;
  int st = (227 * 1024 - fixed) / a_bytes;
  if (st > 8) st = 8;
  t.a_stages = st;
  t.smem_bytes = fixed + st * a_bytes;
  t.acc_stride = t.nt <= 128 ? 128 : 256;
  t.tmem_cols = 2 * t.acc_stride;
  const int max_clusters = num_sms / t.cs;
  t.grid = (t.num_groups < max_clusters ? t.num_groups : max_clusters) * t.cs;
  return t;
}

cudaError_t launch_mac_tc2(const Geom& g, const Tc2Tiling& t, int fmt, const void* A, const void* U, void* y,
                           bool y_bf16, cudaStream_t st, char* err, size_t errlen) {
  if (t.a_stages < 2) {
    snprintf(err, errlen, "mac_tc2: shared memory too small for the window");
    return cudaErrorInvalidValue;
  }
  CUtensorMap tmW, tmX;
  // filter box = the 128/cs rows one CTA loads and multicasts to its cluster
  if (!encode(&tmW, U, fmt, (uint64_t)g.Cp, (uint64_t)g.R * g.S * g.Kp, t.kc, BMK / t.cs, t.row_bytes) ||
      !encode(&tmX, A, fmt, (uint64_t)g.Cp, (uint64_t)g.N * g.L_A, t.kc, kBoxRows, t.row_bytes)) {
    snprintf(err, errlen, "cuTensorMapEncodeTiled failed");
    return cudaErrorInvalidValue;
  }
  Tc2Params p{};
  p.G = (long long)(g.N - 1) * g.L_A + g.M_ext;
  p.L_A = g.L_A;
  p.PQ = (long long)g.P * g.Q;
  p.Wp = g.Wp; p.P = g.P; p.Q = g.Q; p.sh = g.sh; p.sw = g.sw; p.K = g.K; p.R = g.R; p.S = g.S;
  p.nt = t.nt; p.brows = t.brows; p.nr = t.nr; p.ngroups = t.ngroups;
  p.num_mt = t.num_mt; p.num_kt = t.num_kt; p.num_tiles = t.num_tiles; p.num_groups = t.num_groups;
  p.nchunks = t.nchunks; p.kc = t.kc; p.Kp = g.Kp;
  p.a_stages = t.a_stages;
  const uint32_t ab = fmt == FMT_BF16 ? 1u : 2u;
  // instruction descriptor: D=f32 @4, A/B format @7/@10, both K-major, N>>3 @17, M>>4 @24
  p.idesc = (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(t.nt >> 3) << 17) | ((uint32_t)(BMK >> 4) << 24);
  p.row_bytes = (uint32_t)t.row_bytes;
  p.a_bytes = (uint32_t)(BMK * t.row_bytes);
  p.b_bytes = (uint32_t)(t.brows * t.row_bytes);
  p.acc_stride = t.acc_stride; p.tmem_cols = t.tmem_cols;
  p.y = y;
  p.y_bf16 = y_bf16 ? 1 : 0;
  const char* dbg = getenv("POLYCONV_TC_DEBUG");
  p.dbg = dbg ? atoi(dbg) : 0;
  cudaError_t e = cudaSuccess;
#define PC_TC2(TF, CSV)                                                                                  \
  if ((fmt == FMT_TF32) == TF && t.cs == CSV) {                                                         \
    auto kern = mac_tc2_kernel<TF, CSV>;                                                                \
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, t.smem_bytes);          \
    if (e != cudaSuccess) return e;                                                                     \
    cudaLaunchConfig_t cfg = {};                                                                        \
    cfg.gridDim = dim3((unsigned)t.grid);                                                               \
    cfg.blockDim = dim3(kThreads);                                                                      \
    cfg.dynamicSmemBytes = (size_t)t.smem_bytes;                                                        \
    cfg.stream = st;                                                                                    \
    cudaLaunchAttribute attr[1];                                                                        \
    attr[0].id = cudaLaunchAttributeClusterDimension;                                                   \
    attr[0].val.clusterDim.x = CSV;                                                                     \
    attr[0].val.clusterDim.y = 1;                                                                       \
    attr[0].val.clusterDim.z = 1;                                                                       \
    cfg.attrs = attr;                                                                                   \
    cfg.numAttrs = 1;                                                                                   \
    e = cudaLaunchKernelEx(&cfg, kern, tmW, tmX, p);                                                    \
    if (e != cudaSuccess) return e;                                                                     \
  }
  PC_TC2(false, 1) PC_TC2(false, 2) PC_TC2(false, 4) PC_TC2(true, 1) PC_TC2(true, 2) PC_TC2(true, 4)
#undef PC_TC2
  return cudaGetLastError();
}

}  // namespace polyconv

// Debug only (not part of include/polyconv.h): copy the per-CTA phase trace of
// the last POLYCONV_TC_DEBUG&8 launch to host (160 x 8 u64).
extern "C" int polyconv_dbg_tc2_trace(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_tc2_trace, sizeof(unsigned long long) * 160 * 8);
}
