// mac_tc2.cu — a2 (fused input packing) + a4 + a5 on the 5th-gen tensor cores
// with Hankel-window reuse: the default TF32 / BF16 hot path.
//
// The coefficient MAC
//   p_{n,k}[m] = sum_c sum_{i,j} A_{n,c}[m - e(i,j)] * U_{k,c}[e(i,j)]   (P.965, P.1350-1352)
// at m = base + L_U - 1 is, per kernel tap (i,j), a GEMM whose position operand
// is the input polynomial shifted by Wp*i + j coefficients (the doubly blocked
// Hankel structure, P.404-437):
//   D[k][base] += sum_c U_tap(i,j)[k][c] * A[base + Wp*i + j][c]
//
// Design ("mac_tc"):
//  * UMMA A operand = filter tile U_tap[k0:k0+128][c-chunk] (M = 128 output
//    channels), loaded by TMA from the tap-major packed filter (a3, packed by a
//    small kernel that this one overlaps through programmatic dependent launch);
//    UMMA B operand = a window of positions of the input polynomials
//    (N = nt positions, 16 <= nt <= 256, chosen so the tiles fill the SMs in as
//    few waves as possible).  Both K-major, 128/64/32-byte swizzle.
//  * Fused packing (a2): eight "packer" warps build each window straight from
//    the NCHW input -- coefficient r*Wp + s of A_{n,c}(t) is x[n][c][r-ph][s-pw]
//    or 0 (Eq. 10, zero padding P.1353-1356) -- converting to the operand
//    format (BF16 RNE / TF32 RNA, reading R11) and writing the swizzled
//    K-major layout.  No packed copy of the input ever goes to HBM.
//  * Window reuse: one window of nt + (nr-1)*Wp + S-1 positions per channel
//    chunk serves every tap (i,j) of nr kernel rows (all R when it fits): the
//    tap's MMA reads it through a descriptor whose start is shifted by
//    (Wp*i + j) rows (probe: tools/umma_probe.cu, profiles/r01_umma_probe.txt).
//  * Clusters of CS CTAs (default 2) process CS position tiles of the same
//    output-channel block; each CTA loads 128/CS rows of every filter tile and
//    multicasts them to the cluster.
//  * Warp roles (persistent CTA per SM): warp 0 = filter TMA producer (one
//    elected lane), warp 1 = TMEM allocator + UMMA issuer (one elected lane;
//    the loops run warp-wide so their control values stay in uniform
//    registers -- issuing from a divergent lane-0 branch halved the MMA rate,
//    tools/umma_rate.cu), warps 2-9 = packers, warps 10-17 = epilogue.
//  * Epilogue (a5, fused): tcgen05.ld 32 channels x 64 positions -> shared
//    transpose -> each lane owns two adjacent positions and stores them as one
//    bf16x2 / float2 word per channel when they are adjacent output pixels;
//    junk positions (off the Eq. 12 / R4 extraction lattice) are dropped.
#include <cuda.h>
#include <type_traits>
#include "common.cuh"
#include "sm100.cuh"
#include <cstdio>
#include <cstdlib>

namespace polyconv {

namespace {

using namespace sm100;

constexpr int BMK = 128;                 // output channels per tile (UMMA M, TMEM lanes)
constexpr int kPackWarps = 8;
constexpr int kEpiWarps = 8;             // 2 per TMEM lane quadrant
constexpr int kPackWarp0 = 2;
constexpr int kEpiWarp0 = kPackWarp0 + kPackWarps;
constexpr int kThreads = 32 * (kEpiWarp0 + kEpiWarps);
constexpr int kBMaxRows = 384;           // max rows of one position window (48 KB at 128 B rows)
constexpr int kTStride = 68;             // epilogue transpose row stride in floats (64 + 4 pad)

struct Tc2Params {
  const void* x;    // NCHW input, io dtype
  long long G;      // positions with outputs: (N-1)*L_A + M_ext
  long long NLA;    // N*L_A: positions that exist
  long long L_A, PQ, HW;
  int N, C, H, W, ph, pw, Hp;
  int Wp, P, Q, sh, sw, K, R, S;
  int nt, brows, nr, ngroups;
  int num_mt, num_kt, num_tiles, num_groups;
  int nchunks, kc, Kp;
  int a_stages;
  uint32_t idesc, a_bytes, b_bytes, row_bytes;
  int acc_stride, tmem_cols;
  void* y;          // NCHW output, io dtype (= the input's)
  int dbg;          // POLYCONV_TC_DEBUG: 8 = per-CTA phase trace (g_tc2_trace)
};

// per-CTA phase timestamps (globaltimer ns) for POLYCONV_TC_DEBUG & 8
__device__ unsigned long long g_tc2_trace[160 * 8];
// packer fine trace (POLYCONV_TC_DEBUG & 16): clock64 per step of the first window, packer thread 0
__device__ long long g_tc2_ptrace[160 * 16];

// Input element -> operand word (reading R11: BF16 = RNE, TF32 = RNA).
template <typename InT, bool kTf32>
struct ToWord;
template <>
struct ToWord<float, false> {
  __device__ __forceinline__ static uint32_t cvt(float v) {
    return (uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(v));
  }
};
template <>
struct ToWord<__nv_bfloat16, false> {
  __device__ __forceinline__ static uint32_t cvt(__nv_bfloat16 v) { return (uint32_t)__bfloat16_as_ushort(v); }
};
template <>
struct ToWord<float, true> {
  __device__ __forceinline__ static uint32_t cvt(float v) { return to_tf32_rna(v); }
};

template <typename InT, bool kTf32, int CS, bool kVec>
__global__ void __launch_bounds__(kThreads, 1)
    mac_tc2_kernel(const __grid_constant__ CUtensorMap tmW, const Tc2Params p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  uint8_t* sA = smem;                                        // filter tiles  [a_stages][128][row]
  uint8_t* sB = sA + (size_t)p.a_stages * p.a_bytes;         // position windows [2][brows][row]
  float* sT = reinterpret_cast<float*>(sB + 2 * (size_t)p.b_bytes);  // [kEpiWarps][32][kTStride]
  uint64_t* afull = reinterpret_cast<uint64_t*>(sT + kEpiWarps * 32 * kTStride);
  uint64_t* aempty = afull + p.a_stages;
  uint64_t* bfull = aempty + p.a_stages;
  uint64_t* bempty = bfull + 2;
  uint64_t* tfull = bempty + 2;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // clusters of CS CTAs share one output-channel block: the filter tiles are
  // multicast (each CTA loads 128/CS rows into every peer); rank r of cluster
  // work item grp takes position tile (grp / num_kt) * CS + r (a tile past G is
  // a dummy whose outputs are all dropped)
  const uint32_t rank = CS > 1 ? cluster_ctarank() : 0u;
  const int cl_id = (int)blockIdx.x / CS, cl_num = (int)gridDim.x / CS;
  const bool trace = (p.dbg & 8) && blockIdx.x < 160;
  unsigned long long* tr = g_tc2_trace + blockIdx.x * 8;
  if (trace && threadIdx.x == 0) tr[0] = global_ns();

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmW);
    for (int s = 0; s < p.a_stages; ++s) {
      mbar_init(afull + s, 1);
      mbar_init(aempty + s, CS);  // every CTA of the cluster reads the multicast filter tile
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(bfull + s, kPackWarps);
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
  if (trace && threadIdx.x == 0) tr[1] = global_ns();

  if (warp == 0) {
    // ------------------------------------------------------- filter TMA producer
    // The whole warp runs the loop (uniform control values); one elected lane issues.
    // The packed filter comes from the preceding kernel (programmatic dependent launch).
    asm volatile("griddepcontrol.wait;" ::: "memory");
    int as = 0;
    uint32_t aph = 0;
    for (int grp = cl_id; grp < p.num_groups; grp += cl_num) {
      const int kt = grp % p.num_kt;
      const int krow0 = kt * BMK;
      for (int ch = 0; ch < p.nchunks; ++ch) {
        for (int i = 0; i < p.R; ++i) {
          for (int j = 0; j < p.S; ++j) {
            mbar_wait(aempty + as, aph ^ 1u);
            if (elect_one()) {
              {
                mbar_arrive_expect_tx(afull + as, p.a_bytes);
                if constexpr (CS == 1) {
                  tma_load_2d(sA + (size_t)as * p.a_bytes, &tmW, afull + as, ch * p.kc, (i * p.S + j) * p.Kp + krow0);
                } else {
                  constexpr int kSub = BMK / CS;  // filter rows this CTA loads for the cluster
                  tma_load_2d_mc(sA + (size_t)as * p.a_bytes + (size_t)rank * kSub * p.row_bytes, &tmW, afull + as,
                                 ch * p.kc, (i * p.S + j) * p.Kp + krow0 + (int)rank * kSub,
                                 (uint16_t)((1u << CS) - 1));
                }
              }
            }
            __syncwarp();
            if (++as == p.a_stages) { as = 0; aph ^= 1u; }
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
    const uint16_t cl_mask = (uint16_t)((1u << CS) - 1);
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
          if (trace && lane == 0 && ch == 0 && rg == 0 && grp == cl_id) tr[2] = global_ns();
          const uint32_t b_addr = sB0 + (uint32_t)bs * p.b_bytes;
          for (int i = i0; i < i1; ++i) {
            for (int j = 0; j < p.S; ++j) {
              mbar_wait(afull + as, aph);
              tc_fence_after();
              // Hankel shift of tap (i,j) inside the window: Wp*(i-i0) + j rows
              const uint32_t b_shift = (uint32_t)(p.Wp * (i - i0) + j) * p.row_bytes;
              const uint64_t ad = make_sdesc(sA0 + (uint32_t)as * p.a_bytes, p.row_bytes, 0);
              const uint64_t bd = make_sdesc(b_addr + b_shift, p.row_bytes, 0);
              if (elect_one()) {
                // K step = 32 bytes = +2 in the descriptor's start-address field
                for (int ks = 0; ks < ksteps; ++ks) {
                  umma<kTf32>(d_tmem, ad + 2 * ks, bd + 2 * ks, p.idesc, accumulate);
                  accumulate = 1;
                }
                // filter slot free (in every CTA of the cluster) when these MMAs finish
                if constexpr (CS == 1) umma_commit(aempty + as);
                else umma_commit_mc(aempty + as, cl_mask);
              }
              __syncwarp();
              accumulate = 1;
              if (++as == p.a_stages) { as = 0; aph ^= 1u; }
            }
          }
          if (elect_one()) umma_commit(bempty + bs);  // window free when every tap using it finished
          __syncwarp();
          if (++bs == 2) { bs = 0; bph ^= 1u; }
        }
      }
      if (trace && lane == 0) tr[3] = global_ns();
      if (elect_one()) umma_commit(tfull + acc);
      __syncwarp();
      if (++acc == 2) { acc = 0; accph ^= 1u; }
    }
  } else if (warp < kEpiWarp0) {
    // ------------------------------------------- packers: fused a2 (Eq. 10 + padding)
    // Window rows are coefficients gp = wrow + r of the concatenated input
    // polynomials; coefficient pr*Wp + ps of A_{n,c} is x[n][c][pr-ph][ps-pw] or 0.
    // Step 1 zeroes the window (padding coefficients, past N*L_A).  Step 2
    // walks the x elements that land in it in units of EPC channels x V
    // consecutive plane elements: EPC loads (one 16-byte vector per channel
    // plane when kVec), a register transpose, and V 16-byte shared stores --
    // one swizzled chunk (EPC channels of one coefficient) per element.  The 8
    // lanes that share a segment cover the 8 chunks of one 128-byte row.
    const int ptid = (warp - kPackWarp0) * 32 + lane;
    constexpr int kEB = kTf32 ? 4 : 2;                          // operand word bytes
    constexpr int EPC = 16 / kEB;                               // channels per 16-byte chunk
    constexpr int V = kVec ? 16 / (int)sizeof(InT) : 1;         // plane elements per unit
    const uint32_t swmask = p.row_bytes / 16u - 1u;  // 128/64/32-byte swizzle: chunk ^= (addr>>7) & swmask
    const int ncg = (int)p.row_bytes / 16;                      // chunks (channel groups) per row
    const InT* __restrict__ x = reinterpret_cast<const InT*>(p.x);
    int bs = 0;
    uint32_t bph = 0;
    for (int grp = cl_id; grp < p.num_groups; grp += cl_num) {
      const long long g0 = (long long)((grp / p.num_kt) * CS + (int)rank) * p.nt;
      for (int ch = 0; ch < p.nchunks; ++ch) {
        const int cbase = ch * p.kc;
        for (int rg = 0; rg < p.ngroups; ++rg) {
          const long long wrow = g0 + (long long)p.Wp * (rg * p.nr);
          const bool pt = (p.dbg & 16) && ptid == 0 && blockIdx.x < 160 && grp == cl_id && ch == 0 && rg == 0;
          long long* ptr = g_tc2_ptrace + blockIdx.x * 16;
          int npt = 0;
          if (pt) ptr[npt++] = clock64();
          mbar_wait_sleep(bempty + bs, bph ^ 1u, 64);
          if (pt) ptr[npt++] = clock64();
          uint8_t* dst = sB + (size_t)bs * p.b_bytes;
          for (int i = ptid; i < (int)(p.b_bytes >> 4); i += kPackWarps * 32)
            reinterpret_cast<uint4*>(dst)[i] = make_uint4(0u, 0u, 0u, 0u);
          if (pt) ptr[npt++] = clock64();
          asm volatile("bar.sync 1, %0;" ::"n"(kPackWarps * 32) : "memory");
          if (pt) ptr[npt++] = clock64();
          if (wrow < p.NLA) {
            const int n_lo = (int)(wrow / p.L_A);
            const int n_hi = (int)min((long long)p.N - 1, (wrow + p.brows - 1) / p.L_A);
            for (int n = n_lo; n <= n_hi; ++n) {
              const int base = (int)((long long)n * p.L_A - wrow);  // window row of coefficient 0 of image n
              const int pr_lo = base >= 0 ? 0 : (-base) / p.Wp;
              const int pr_hi = min(p.Hp - 1, (p.brows - 1 - base) / p.Wp);
              const int h_lo = max(0, pr_lo - p.ph), h_hi = min(p.H - 1, pr_hi - p.ph);
              if (h_lo > h_hi) continue;
              const int e_lo = (h_lo * p.W) / V * V;
              const int e_hi = min((int)p.HW, ((h_hi + 1) * p.W + V - 1) / V * V);
              const int units = (e_hi - e_lo) / V * ncg;
              const InT* xn = x + ((long long)n * p.C + cbase) * p.HW;
              // kU units per thread per round, all loads issued before any use:
              // the window's x bytes are in flight at once (memory-level parallelism)
              constexpr int kU = 2;
#pragma unroll 1
              for (int u0 = ptid; u0 < units; u0 += kU * kPackWarps * 32) {
                uint32_t L[kU][EPC][V];
#pragma unroll
                for (int t = 0; t < kU; ++t) {
                  const int u = u0 + t * kPackWarps * 32;
                  const int seg = u / ncg, cg = u - seg * ncg;
                  const int e0 = e_lo + seg * V;
#pragma unroll
                  for (int e = 0; e < EPC; ++e) {
                    const int c = cbase + cg * EPC + e;
                    const InT* src = xn + (long long)(cg * EPC + e) * p.HW + e0;
                    const bool ok = u < units && c < p.C;
                    if constexpr (kVec) {
                      const uint4 q = ok ? __ldg(reinterpret_cast<const uint4*>(src)) : make_uint4(0u, 0u, 0u, 0u);
                      const uint32_t r4[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
                      for (int k = 0; k < V; ++k) {
                        if constexpr (sizeof(InT) == 2) L[t][e][k] = (r4[k >> 1] >> ((k & 1) * 16)) & 0xFFFFu;
                        else L[t][e][k] = ToWord<InT, kTf32>::cvt(__uint_as_float(r4[k]));
                      }
                    } else {
                      L[t][e][0] = ok ? ToWord<InT, kTf32>::cvt(__ldg(src)) : 0u;
                    }
                  }
                }
                if (pt && npt < 14) ptr[npt++] = clock64();
#pragma unroll
                for (int t = 0; t < kU; ++t) {
                  const int u = u0 + t * kPackWarps * 32;
                  if (u < units) {
                    const int seg = u / ncg, cg = u - seg * ncg;
                    const int e0 = e_lo + seg * V;
                    // element e0 + k lands in window row base + (h+ph)*Wp + w+pw
                    const int h0 = e0 / p.W;
                    int w = e0 - h0 * p.W;
                    int row = base + (h0 + p.ph) * p.Wp + (w + p.pw);
#pragma unroll
                    for (int k = 0; k < V; ++k) {
                      if (row >= 0 && row < p.brows) {
                        uint4 o;
                        if constexpr (kEB == 2)
                          o = make_uint4(L[t][0][k] | (L[t][1][k] << 16), L[t][2][k] | (L[t][3][k] << 16),
                                         L[t][4][k] | (L[t][5][k] << 16), L[t][6][k] | (L[t][7][k] << 16));
                        else
                          o = make_uint4(L[t][0][k], L[t][1][k], L[t][2][k], L[t][3][k]);
                        const uint32_t off = (uint32_t)row * p.row_bytes + 16u * cg;
                        *reinterpret_cast<uint4*>(dst + (off ^ (((off >> 7) & swmask) << 4))) = o;
                      }
                      // next plane element: next column, or the next row (skipping the padding)
                      if (++w == p.W) { w = 0; row += p.Wp - p.W + 1; } else { ++row; }
                    }
                  }
                }
                if (pt && npt < 14) ptr[npt++] = clock64();
              }
            }
          }
          if (pt) { ptr[npt < 15 ? npt : 15] = clock64(); ptr[15] = npt; }
          // generic-proxy smem writes -> visible to the tensor core (async proxy)
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          __syncwarp();
          if (trace && ptid == 0 && grp == cl_id && ch == 0 && rg == 0) tr[6] = global_ns();
          if (lane == 0) mbar_arrive(bfull + bs);
          if (++bs == 2) { bs = 0; bph ^= 1u; }
        }
      }
    }
  } else {
    // -------------------------------------------------------------- epilogue
    // warp w reads TMEM lane quadrant (w % 4); the two warps of a quadrant take
    // alternate 64-column blocks of the accumulator.
    const int ew = warp - kEpiWarp0;
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
      const long long n0 = g0 / p.L_A;      // decode the tile's first position once
      const int m0 = (int)(g0 - n0 * p.L_A);
      mbar_wait_sleep(tfull + acc, accph, 256);
      tc_fence_after();
      if (trace && ew == 0 && lane == 0) tr[4] = global_ns();
      const uint32_t taddr = tmem_base + ((uint32_t)(quad * 32) << 16) + (uint32_t)(acc * p.acc_stride);
      for (int cb = csub * 64; cb < p.nt; cb += 64 * cstep) {
        uint32_t v0[32], v1[32];
        tmem_ld32(taddr + (uint32_t)cb, v0);
        tmem_ld32(taddr + (uint32_t)cb + 32u, v1);
        tmem_ld_wait();
        // T[channel lane][position 0..63]
        float4* Trow = reinterpret_cast<float4*>(T + lane * kTStride);
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          Trow[q] = make_float4(__uint_as_float(v0[4 * q]), __uint_as_float(v0[4 * q + 1]),
                                __uint_as_float(v0[4 * q + 2]), __uint_as_float(v0[4 * q + 3]));
          Trow[8 + q] = make_float4(__uint_as_float(v1[4 * q]), __uint_as_float(v1[4 * q + 1]),
                                    __uint_as_float(v1[4 * q + 2]), __uint_as_float(v1[4 * q + 3]));
        }
        __syncwarp();
        // lane -> positions c, c+1 of the tile; a5: keep those on the extraction lattice
        const int c = cb + 2 * lane;
        long long n = n0;
        int m = m0 + c;
        while (m >= p.L_A) { m -= (int)p.L_A; ++n; }
        const int r = m / p.Wp, s = m - r * p.Wp;
        const int oh = r / p.sh, ow = s / p.sw;
        const bool v0ok = c < p.nt && g0 + c < p.G && (r - oh * p.sh) == 0 && (s - ow * p.sw) == 0 &&
                          oh < p.P && ow < p.Q;
        int m1 = m + 1;
        long long n1 = n;
        if (m1 >= p.L_A) { m1 -= (int)p.L_A; ++n1; }
        const int r1 = m1 / p.Wp, s1 = m1 - r1 * p.Wp;
        const int oh1 = r1 / p.sh, ow1 = s1 / p.sw;
        const bool v1ok = c + 1 < p.nt && g0 + c + 1 < p.G && (r1 - oh1 * p.sh) == 0 &&
                          (s1 - ow1 * p.sw) == 0 && oh1 < p.P && ow1 < p.Q;
        const long long y0 = (n * p.K + kq) * p.PQ + (long long)oh * p.Q + ow;
        const long long y1 = (n1 * p.K + kq) * p.PQ + (long long)oh1 * p.Q + ow1;
        // adjacent output pixels, even element offset -> one 2-element store per channel
        const bool pair = v0ok && v1ok && y1 == y0 + 1 && (y0 & 1) == 0 && (p.PQ & 1) == 0;
        if (v0ok || v1ok) {
          const float2* Tcol = reinterpret_cast<const float2*>(T + 2 * lane);
          InT* y = reinterpret_cast<InT*>(p.y);
          if (pair) {
            using Pair = typename std::conditional<sizeof(InT) == 2, __nv_bfloat162, float2>::type;
            Pair* yp = reinterpret_cast<Pair*>(y + y0);
            const long long st = p.PQ / 2;
#pragma unroll 4
            for (int q = 0; q < kmax; ++q) {
              const float2 t = Tcol[q * (kTStride / 2)];
              if constexpr (sizeof(InT) == 2) yp[q * st] = __float22bfloat162_rn(t);
              else yp[q * st] = t;
            }
          } else {
#pragma unroll 1
            for (int q = 0; q < kmax; ++q) {
              const float2 t = Tcol[q * (kTStride / 2)];
              if constexpr (sizeof(InT) == 2) {
                if (v0ok) y[y0 + q * p.PQ] = __float2bfloat16_rn(t.x);
                if (v1ok) y[y1 + q * p.PQ] = __float2bfloat16_rn(t.y);
              } else {
                if (v0ok) y[y0 + q * p.PQ] = t.x;
                if (v1ok) y[y1 + q * p.PQ] = t.y;
              }
            }
          }
        }
        __syncwarp();
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(tempty + acc);
      if (trace && ew == 0 && lane == 0) tr[5] = global_ns();
      if (++acc == 2) { acc = 0; accph ^= 1u; }
    }
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if constexpr (CS > 1) cluster_sync();  // no CTA exits while peers may still signal it
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem_base, (uint32_t)p.tmem_cols);
  }
  if (trace && threadIdx.x == 0) tr[7] = global_ns();
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

template <typename InT, bool kTf32, int CS>
cudaError_t launch_one(const Tc2Tiling& t, const CUtensorMap& tmW, const Tc2Params& p, bool vec, bool pdl,
                       cudaStream_t st) {
  auto kern = vec ? mac_tc2_kernel<InT, kTf32, CS, true> : mac_tc2_kernel<InT, kTf32, CS, false>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, t.smem_bytes);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)t.grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = (size_t)t.smem_bytes;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CS;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, tmW, p);
}

}  // namespace

bool tc2_supported(const Geom& g, int fmt) {
  if (fmt != FMT_BF16 && fmt != FMT_TF32) return false;
  if ((long long)g.R * g.S * ((g.K + 127) / 128 * 128) >= (1LL << 31)) return false;  // TMA row coordinate
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
  // clusters of 2 CTAs share (multicast) the filter tiles; 148 SMs = 74 pairs
  const char* force_cs = getenv("POLYCONV_TC_CS");  // experiments only
  t.cs = force_cs ? atoi(force_cs) : 2;
  if (t.cs != 1 && t.cs != 2) t.cs = 2;
  if (cdiv(G, 16) < 2) t.cs = 1;
  // positions per tile: fewest waves over the SMs, then the largest tile
  long long best_cost = -1;
  const char* force_nt = getenv("POLYCONV_TC_NT");  // experiments only
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
  t.brows = (int)cdiv((long long)t.nt + (long long)(nr - 1) * g.Wp + g.S - 1, 8) * 8;
  t.num_mt = (int)cdiv(G, t.nt);
  t.num_tiles = t.num_mt * t.num_kt;
  t.num_groups = (int)cdiv(t.num_mt, t.cs) * t.num_kt;
  t.nchunks = (g.C + kc - 1) / kc;
  const int a_bytes = BMK * t.row_bytes;
  const int b_bytes = (int)cdiv((long long)t.brows * t.row_bytes, 1024) * 1024;
  const int fixed = 1024 + 2 * b_bytes + kEpiWarps * 32 * kTStride * 4 + 512;
  int st = (227 * 1024 - fixed) / a_bytes;
  if (st > 12) st = 12;
  t.a_stages = st;
  t.smem_bytes = fixed + st * a_bytes;
  t.acc_stride = t.nt <= 128 ? 128 : 256;
  t.tmem_cols = 2 * t.acc_stride;
  const int max_clusters = num_sms / t.cs;
  t.grid = (t.num_groups < max_clusters ? t.num_groups : max_clusters) * t.cs;
  return t;
}

cudaError_t launch_mac_tc2(const Geom& g, const Tc2Tiling& t, int fmt, const void* x, bool x_bf16, const void* U,
                           void* y, bool y_bf16, bool pdl, cudaStream_t st, char* err, size_t errlen) {
  if (t.a_stages < 2) {
    snprintf(err, errlen, "mac_tc2: shared memory too small for the window");
    return cudaErrorInvalidValue;
  }
  CUtensorMap tmW;
  // filter box = the 128/cs rows one CTA loads and multicasts to its cluster
  if (!encode(&tmW, U, fmt, (uint64_t)g.Cp, (uint64_t)g.R * g.S * g.Kp, t.kc, BMK / t.cs, t.row_bytes)) {
    snprintf(err, errlen, "cuTensorMapEncodeTiled failed");
    return cudaErrorInvalidValue;
  }
  Tc2Params p{};
  p.x = x;
  p.G = (long long)(g.N - 1) * g.L_A + g.M_ext;
  p.NLA = (long long)g.N * g.L_A;
  p.L_A = g.L_A;
  p.PQ = (long long)g.P * g.Q;
  p.HW = (long long)g.H * g.W;
  p.N = g.N; p.C = g.C; p.H = g.H; p.W = g.W; p.ph = g.ph; p.pw = g.pw; p.Hp = g.Hp;
  // packers load 16-byte vectors when every plane starts 16-byte aligned
  const int eb_in = x_bf16 ? 2 : 4;
  const bool vec = (p.HW % (16 / eb_in)) == 0 && (reinterpret_cast<uintptr_t>(x) % 16) == 0;
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
  p.b_bytes = (uint32_t)(cdiv((long long)t.brows * t.row_bytes, 1024) * 1024);
  p.acc_stride = t.acc_stride; p.tmem_cols = t.tmem_cols;
  p.y = y;
  if (y_bf16 != x_bf16) return cudaErrorInvalidValue;  // y has the io dtype of x
  const char* dbg = getenv("POLYCONV_TC_DEBUG");
  p.dbg = dbg ? atoi(dbg) : 0;
  if (fmt == FMT_TF32) {
    if (x_bf16) return cudaErrorInvalidValue;
    return t.cs == 1 ? launch_one<float, true, 1>(t, tmW, p, vec, pdl, st)
                     : launch_one<float, true, 2>(t, tmW, p, vec, pdl, st);
  }
  if (x_bf16)
    return t.cs == 1 ? launch_one<__nv_bfloat16, false, 1>(t, tmW, p, vec, pdl, st)
                     : launch_one<__nv_bfloat16, false, 2>(t, tmW, p, vec, pdl, st);
  return t.cs == 1 ? launch_one<float, false, 1>(t, tmW, p, vec, pdl, st)
                   : launch_one<float, false, 2>(t, tmW, p, vec, pdl, st);
}

}  // namespace polyconv

// Debug only (not part of include/polyconv.h): copy the per-CTA phase trace of
// the last POLYCONV_TC_DEBUG&8 launch to host (160 x 8 u64).
extern "C" int polyconv_dbg_tc2_ptrace(long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_tc2_ptrace, sizeof(long long) * 160 * 16);
}
extern "C" int polyconv_dbg_tc2_trace(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_tc2_trace, sizeof(unsigned long long) * 160 * 8);
}
