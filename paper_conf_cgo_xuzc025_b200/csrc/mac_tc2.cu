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
//    K-major layout.  No packed copy of the input ever goes to HBM.  The raw
//    input rows are brought in by TMA (boxes of 64 plane elements x kc channel
//    planes, x viewed as [N*C][H*W]) into a staging buffer one window ahead,
//    and transposed shared->shared; when H*W*elem is not a multiple of 16
//    bytes (no TMA view) the packers load x directly (slow path).
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
//  * Epilogue (a5, fused): tcgen05.ld.16x256b gives each lane two adjacent
//    positions of four output channels; each pair is stored as one bf16x2 /
//    float2 word per channel when it is two adjacent output pixels (8 lanes
//    cover 16 consecutive pixels of a channel row); junk positions (off the
//    Eq. 12 / R4 extraction lattice) are dropped.
#include <cuda.h>
#include <type_traits>
#include "common.cuh"
#include "sm100.cuh"
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <algorithm>

namespace polyconv {

namespace {

using namespace sm100;

constexpr int BMK = 128;                 // output channels per tile (UMMA M, TMEM lanes)
constexpr int kPackWarps = 8;
constexpr int kEpiWarps = 8;             // 2 per TMEM lane quadrant
constexpr int kPackWarp0 = 2;
// kernel modes: windows by TMA from the packed input (kModeTma), or built in
// the kernel by packer warps from NCHW x via TMA staging (kModeFusedTma) or
// direct loads (kModeFusedLd)
// kModeFusedMx: packer warps transpose TMA-staged boxes of x with 8x8 matrix
// moves (ldmatrix.trans -> stmatrix) fed by a ring of kRing staged boxes and a
// dedicated staging-producer warp (bf16 input and math)
constexpr int kModeTma = 0, kModeFusedTma = 1, kModeFusedLd = 2, kModeFusedMx = 3;
#ifndef MX_PACK_WARPS
#define MX_PACK_WARPS 6
#endif
constexpr int kMxPackWarps = MX_PACK_WARPS;
// staged x boxes in flight (kModeFusedMx).  Box gb lives in slot gb % kRing and is
// transposed by packer warp gb % kRing: every slot has one consumer that takes its
// boxes in order, so no waiter can be a whole ring cycle ahead of the slot (an
// mbarrier parity wait would then pass on the previous phase)
constexpr int kRing = MX_PACK_WARPS;                 // staged x boxes in flight (kModeFusedMx)
__host__ __device__ constexpr int pack_warps(int mode) {
  return mode == kModeTma ? 0 : (mode == kModeFusedMx ? kMxPackWarps : kPackWarps);
}
__host__ __device__ constexpr int epi_warp0(int mode) { return kPackWarp0 + pack_warps(mode); }
// kModeTma issues the MMAs from two warps (warp 1 and the last warp), alternating
// filter stages: an mbarrier wait in the issuing thread stalls it until its own
// earlier MMAs drain, so one issuer leaves the tensor pipe idle at every stage
// boundary; with two, one issues while the other waits (tools/umma_rate.cu:
// 235 -> 113 cycles per 128x208x16 MMA, ideal 104)
__host__ __device__ constexpr int n_issuers(int mode) { return mode == kModeTma || mode == kModeFusedMx ? 2 : 1; }
// kModeFusedMx: the staging producer is the warp after the epilogue / second issuer
__host__ __device__ constexpr int xld_warp(int mode) { return epi_warp0(mode) + kEpiWarps + n_issuers(mode) - 1; }
__host__ __device__ constexpr int threads_for(int mode) {
  return 32 * (xld_warp(mode) + (mode == kModeFusedMx ? 1 : 0));
}
constexpr int kBMaxRows = 384;           // max rows of one position window (48 KB at 128 B rows)
constexpr int kBoxRows = 32;             // rows per TMA box of a position window (kModeTma)
constexpr int kBoxE = 64;                // plane elements per staging TMA box
constexpr int kMaxSeg = 4;               // images one window may span on the TMA staging path

struct Tc2Params {
  const void* x;    // NCHW input, io dtype
  long long G;      // positions with outputs: (N-1)*L_A + M_ext
  long long NLA;    // N*L_A: positions that exist
  long long L_A, PQ, HW;
  int N, C, H, W, ph, pw, Hp;
  int ealign;       // 16 / sizeof(input element): staging boxes start on this element multiple
  int Wp, P, Q, sh, sw, K, R, S;
  int nt, brows, nr, ngroups;
  int num_mt, num_kt, num_tiles, num_groups;
  int nchunks, kc, Kp, Cp;
  int a_stages;
  uint32_t box_bytes;  // staging TMA box: kBoxE elements x kc planes
  uint32_t stg_bytes;  // staging buffer (max boxes of any window)
  uint32_t idesc, a_bytes, b_bytes, row_bytes;
  uint32_t b_bytes_tx;  // bytes the window TMA boxes deliver (brows * row_bytes), kModeTma
  int tps;              // filter taps per pipeline stage
  int urep;             // filter copies; cluster c reads copy c % urep
  int stages_per_tile;  // filter stages per tile (all chunks and row groups)
  uint32_t tap_bytes;   // one filter tile: 128 x kc words
  int acc_stride, tmem_cols;
  int ecols;            // epilogue columns (positions) staged per pass
  uint32_t stage_bytes, stage_pitch;
  int big_stage;        // the last tile may stage all nt columns in the operand buffers
  // in-kernel a3 (fused modes): every CTA packs a slice of the tap-major filter
  // from w (KCRS) into U, then counts itself in *fcount; the filter producers
  // start when *fcount reaches ftarget (all CTAs are co-resident: grid <= SMs)
  const void* w;
  void* U;
  unsigned long long* fcount;
  unsigned long long ftarget;
  int fpack;
  FastDiv fQ;           // output index -> (oh, ow)
  void* y;          // NCHW output, io dtype (= the input's)
  int dbg;          // POLYCONV_TC_DEBUG: 8 = per-CTA phase trace (g_tc2_trace), 16 = packer
                    // trace; ablations 1 = no filter TMA after the first ring fill,
                    // 2 = no window TMA after the first two (kModeTma, wrong results)
  FastDiv fLA, fWp, fsh, fsw;  // position decode: coefficient -> (n, r, s) -> (oh, ow)
  FastDiv fW;                  // plane element -> (h, w) (kModeFusedMx)
};

// per-CTA phase timestamps (globaltimer ns) for POLYCONV_TC_DEBUG & 8
__device__ unsigned long long g_tc2_trace[160 * 8];
// packer sub-phases of the first two windows (POLYCONV_TC_DEBUG & 16), globaltimer ns
__device__ unsigned long long g_tc2_pk[160 * 8];
// epilogue sub-phase cycles of warp 0 (POLYCONV_TC_DEBUG & 128): tmem ld, staging stores,
// barrier 1, offset table, copy-out, barrier 2
__device__ unsigned long long g_tc2_epi[160 * 8];

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

// ---- packer helpers (fused a2) ---------------------------------------------------
struct Seg {
  int n, e_lo, box0;  // image, first plane element staged, first staging box
};

// Position window wi of this CTA (in the MMA's order): first coefficient, first channel.
template <int CS>
__device__ __forceinline__ void tc2_window(const Tc2Params& p, int cl_id, int cl_num, uint32_t rank, int wi,
                                           long long& wrow, int& cbase) {
  const int wpg = p.nchunks * p.ngroups;
  const int grp = cl_id + (wi / wpg) * cl_num, inner = wi % wpg;
  const int ch = inner / p.ngroups, rg = inner - ch * p.ngroups;
  const long long g0 = (long long)((grp / p.num_kt) * CS + (int)rank) * p.nt;
  wrow = g0 + (long long)p.Wp * (rg * p.nr);
  cbase = ch * p.kc;
}

// The x elements window wrow needs: per image segment q, plane elements
// [e_lo, e_lo + boxes*kBoxE) of image sg[q].n (sg[q].n = -1: no rows of that
// image).  Returns (segments) | (total boxes << 8).
__device__ __forceinline__ int tc2_segments(const Tc2Params& p, long long wrow, Seg (&sg)[kMaxSeg]) {
  int ns = 0, boxes = 0;
#pragma unroll
  for (int q = 0; q < kMaxSeg; ++q) sg[q].n = -1;
  if (wrow >= p.NLA) return 0;
  const int n_lo = (int)p.fLA.div((uint32_t)wrow);
  const int n_hi = min(p.N - 1, (int)p.fLA.div((uint32_t)(wrow + p.brows - 1)));
#pragma unroll
  for (int q = 0; q < kMaxSeg; ++q) {  // unrolled: the segment table stays in registers
    const int n = n_lo + q;
    if (n > n_hi) continue;
    const int base = (int)((long long)n * p.L_A - wrow);  // window row of coefficient 0 of image n
    const int pr_lo = base >= 0 ? 0 : (int)p.fWp.div((uint32_t)(-base));
    const int pr_hi = min(p.Hp - 1, (int)p.fWp.div((uint32_t)(p.brows - 1 - base)));
    const int h_lo = max(0, pr_lo - p.ph), h_hi = min(p.H - 1, pr_hi - p.ph);
    if (h_lo > h_hi) continue;
    // a TMA box must start 16-byte aligned in global memory: round the first
    // element down to a multiple of 16/sizeof(elem) (planes start aligned)
    const int e_lo = (h_lo * p.W) & ~(p.ealign - 1);
    sg[q].n = n;
    sg[q].e_lo = e_lo;
    sg[q].box0 = boxes;
    boxes += ((h_hi + 1) * p.W - e_lo + kBoxE - 1) / kBoxE;
    ns = q + 1;
  }
  return ns | (boxes << 8);
}

// Staging TMA of window (wrow, cbase): boxes of kBoxE plane elements x kc planes.
__device__ __forceinline__ void tc2_issue_staging(const Tc2Params& p, const CUtensorMap* tmX, uint8_t* sX,
                                                  uint64_t* sfull, long long wrow, int cbase) {
  Seg sg[kMaxSeg];
  const int r = tc2_segments(p, wrow, sg);
  const int boxes = r >> 8;
  mbar_arrive_expect_tx(sfull, (uint32_t)boxes * p.box_bytes);
#pragma unroll
  for (int q = 0; q < kMaxSeg; ++q) {
    if (sg[q].n < 0) continue;
    int nxt = boxes;
#pragma unroll
    for (int q2 = kMaxSeg - 1; q2 > q; --q2)
      if (sg[q2].n >= 0) nxt = sg[q2].box0;
    for (int b = sg[q].box0; b < nxt; ++b)
      tma_load_2d(sX + (size_t)b * p.box_bytes, tmX, sfull, sg[q].e_lo + (b - sg[q].box0) * kBoxE,
                  sg[q].n * p.C + cbase);
  }
}

template <typename InT, bool kTf32, int CS, int kMode>
__global__ void __launch_bounds__(threads_for(kMode), 1)
    mac_tc2_kernel(const __grid_constant__ CUtensorMap tmW, const __grid_constant__ CUtensorMap tmX,
                   const Tc2Params p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  uint8_t* sA = smem;                                        // filter tiles  [a_stages][128][row]
  uint8_t* sB = sA + (size_t)p.a_stages * p.a_bytes;         // position windows [2][brows][row]
  uint8_t* sX = sB + 2 * (size_t)p.b_bytes;                  // raw-input staging (TMA path)
  constexpr bool kTmaX = kMode == kModeFusedTma;  // fused packers stage x by TMA
  constexpr bool kStage = kTmaX || kMode == kModeFusedMx;
  constexpr int kEpiWarp0 = epi_warp0(kMode);
  uint8_t* sStage = sX + (kStage ? (size_t)p.stg_bytes : 0);  // epilogue staging [128][ecols] (+16 B pitch pad)
  int* sPos = reinterpret_cast<int*>(sStage + p.stage_bytes);  // [256] output offsets of the tile's positions
  uint8_t* sDummy = reinterpret_cast<uint8_t*>(sPos + 256);  // 128 B sink for dropped stmatrix rows
  uint64_t* afull = reinterpret_cast<uint64_t*>(sDummy + 128);
  uint64_t* aempty = afull + p.a_stages;
  uint64_t* bfull = aempty + p.a_stages;
  uint64_t* bempty = bfull + 2;
  uint64_t* tfull = bempty + 2;
  uint64_t* tempty = tfull + 2;
  uint64_t* sfull = tempty + 2;
  uint64_t* rfull = sfull + 1;       // [kRing] staged box landed (kModeFusedMx)
  uint64_t* rempty = rfull + kRing;  // [kRing] staged box transposed
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(rempty + kRing);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // clusters of CS CTAs share one output-channel block: the filter tiles are
  // multicast (each CTA loads 128/CS rows into every peer); rank r of cluster
  // work item grp takes position tile (grp / num_kt) * CS + r (a tile past G is
  // a dummy whose outputs are all dropped)
  const uint32_t rank = CS > 1 ? cluster_ctarank() : 0u;
  const int cl_id = (int)blockIdx.x / CS, cl_num = (int)gridDim.x / CS;
  const bool trace = (p.dbg & 8) && blockIdx.x < 160;
  unsigned long long* tr = g_tc2_trace + blockIdx.x * 8;
  const bool ptrace = (p.dbg & 16) && blockIdx.x < 160;  // MX sub-phases (g_tc2_pk)
  unsigned long long* pk = g_tc2_pk + blockIdx.x * 8;
  if (trace && threadIdx.x == 0) tr[0] = global_ns();

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmW);
    if constexpr (kMode != kModeFusedLd) prefetch_tmap(&tmX);
    for (int s = 0; s < p.a_stages; ++s) {
      mbar_init(afull + s, 1);
      mbar_init(aempty + s, CS);  // every CTA of the cluster reads the multicast filter tile
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(bfull + s, kMode == kModeTma ? 1 : pack_warps(kMode));
      mbar_init(bempty + s, n_issuers(kMode));  // every issuer commits its share of a window
      mbar_init(tfull + s, n_issuers(kMode));   // and of an accumulator
      mbar_init(tempty + s, kEpiWarps);
    }
    mbar_init(sfull, 1);
    for (int s = 0; s < kRing; ++s) {
      mbar_init(rfull + s, 1);
      mbar_init(rempty + s, 1);
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
    if (p.fpack) {
      // every CTA's slice of the packed filter is in global memory
      if (lane == 0) {
        unsigned long long v;
        uint64_t t0 = 0;
        for (;;) {
          asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p.fcount) : "memory");
          if (v >= p.ftarget) break;
          const uint64_t t = global_ns();
          if (t0 == 0) t0 = t;
          __nanosleep(32);
        }
        asm volatile("fence.proxy.async.global;" ::: "memory");  // generic writes -> TMA reads
      }
      __syncwarp();
    } else {
      asm volatile("griddepcontrol.wait;" ::: "memory");
    }
    int as = 0, bs = 0, na = 0, nb = 0;
    uint32_t aph = 0, bph = 0;
    for (int grp = cl_id; grp < p.num_groups; grp += cl_num) {
      const int kt = grp % p.num_kt;
      const int krow0 = kt * BMK + (cl_id % p.urep) * p.R * p.S * p.Kp;  // this cluster's filter copy
      const long long g0 = (long long)((grp / p.num_kt) * CS + (int)rank) * p.nt;
      for (int ch = 0; ch < p.nchunks; ++ch) {
        for (int rg = 0; rg < p.ngroups; ++rg) {
          const int i0 = rg * p.nr, i1 = min(p.R, i0 + p.nr);
          if constexpr (kMode == kModeTma) {
            // the position window (packed input rows [wrow, wrow+brows), channel chunk ch);
            // rows past N*L_A are zero-filled by TMA
            mbar_wait(bempty + bs, bph ^ 1u);
            if (elect_one()) {
              if ((p.dbg & 2) && nb >= 2) {  // ablation: no window traffic after the first two
                mbar_arrive(bfull + bs);
              } else {
                mbar_arrive_expect_tx(bfull + bs, p.b_bytes_tx);
                const int wrow = (int)(g0 + (long long)p.Wp * i0);
                uint8_t* dst = sB + (size_t)bs * p.b_bytes;
                for (int r = 0; r < p.brows; r += kBoxRows)
                  tma_load_2d(dst + (size_t)r * p.row_bytes, &tmX, bfull + bs, ch * p.kc, wrow + r);
              }
            }
            __syncwarp();
            ++nb;
            if (++bs == 2) { bs = 0; bph ^= 1u; }
          }
          // filter stages: `tps` consecutive taps of this window's kernel rows per stage
          const int ntap = (i1 - i0) * p.S;
          for (int t0 = 0; t0 < ntap; t0 += p.tps) {
            const int nt_st = min(p.tps, ntap - t0);
            mbar_wait(aempty + as, aph ^ 1u);
            if (elect_one()) {
              if ((p.dbg & 1) && na >= p.a_stages) {  // ablation: no filter traffic
                mbar_arrive(afull + as);
              } else {
                mbar_arrive_expect_tx(afull + as, (uint32_t)nt_st * p.tap_bytes);
                for (int t = 0; t < nt_st; ++t) {
                  const int tap = i0 * p.S + t0 + t;  // (i, j) with i*S + j = tap
                  uint8_t* dst = sA + (size_t)as * p.a_bytes + (size_t)t * p.tap_bytes;
                  if constexpr (CS == 1) {
                    tma_load_2d(dst, &tmW, afull + as, ch * p.kc, tap * p.Kp + krow0);
                  } else {
                    constexpr int kSub = BMK / CS;  // filter rows this CTA loads for the cluster
                    tma_load_2d_mc(dst + (size_t)rank * kSub * p.row_bytes, &tmW, afull + as, ch * p.kc,
                                   tap * p.Kp + krow0 + (int)rank * kSub, (uint16_t)((1u << CS) - 1));
                  }
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
  } else if (warp == 1 || (n_issuers(kMode) == 2 && warp == kEpiWarp0 + kEpiWarps)) {
    // -------------------------------------------------------------- UMMA issuer(s)
    // issuer q (0: warp 1, 1: the extra warp) issues the CTA's filter stages g
    // with g % n_issuers == q, in strict alternation: before issuing stage g it
    // waits on named barrier 3 + (g-1)%2 for "stage g-1 issued", and after
    // issuing it arrives on 3 + g%2.  The tensor pipe thus receives the MMAs in
    // one fixed order (deterministic accumulation, reading R12) while each
    // issuer's barrier checks overlap the other's MMAs.
    constexpr int NI = n_issuers(kMode);
    const int q = warp == 1 ? 0 : 1;
    long long gs = 0;  // global stage counter of this CTA
    const long long gs_total =
        (long long)(p.num_groups > cl_id ? (p.num_groups - cl_id + cl_num - 1) / cl_num : 0) * p.stages_per_tile;
    int as = 0, bs = 0, acc = 0;
    uint32_t aph = 0, bph = 0, accph = 0;
    const int ksteps = (int)p.row_bytes / 32;
    const uint32_t sA0 = smem_u32(sA), sB0 = smem_u32(sB);
    const uint16_t cl_mask = (uint16_t)((1u << CS) - 1);
    for (int grp = cl_id; grp < p.num_groups; grp += cl_num) {
      mbar_wait(tempty + acc, accph ^ 1u);
      tc_fence_after();
      const uint32_t d_tmem = tmem_base + (uint32_t)(acc * p.acc_stride);
      int k = 0;  // filter stage index within the tile
      for (int ch = 0; ch < p.nchunks; ++ch) {
        for (int rg = 0; rg < p.ngroups; ++rg) {
          const int i0 = rg * p.nr, i1 = min(p.R, i0 + p.nr);
          mbar_wait(bfull + bs, bph);
          tc_fence_after();
          if (trace && q == 0 && lane == 0 && ch == 0 && rg == 0 && grp == cl_id)
            tr[2] = (p.dbg & 32) ? clock64() : global_ns();
          const uint32_t b_addr = sB0 + (uint32_t)bs * p.b_bytes;
          const int ntap = (i1 - i0) * p.S;
          for (int t0 = 0; t0 < ntap; t0 += p.tps, ++k, ++gs) {
            if (gs % NI == q) {
              const int nt_st = min(p.tps, ntap - t0);
              mbar_wait(afull + as, aph);
              if (NI == 2 && gs > 0) {  // stage gs-1 (the other issuer's) is in the pipe
                if ((gs - 1) & 1) asm volatile("bar.sync 4, 64;" ::: "memory");
                else asm volatile("bar.sync 3, 64;" ::: "memory");
              }
              tc_fence_after();
              const uint32_t a_stage = sA0 + (uint32_t)as * p.a_bytes;
              if (elect_one()) {
                for (int t = 0; t < nt_st; ++t) {
                  const int tl = t0 + t, i = i0 + tl / p.S, j = tl - (tl / p.S) * p.S;
                  // Hankel shift of tap (i,j) inside the window: Wp*(i-i0) + j rows
                  const uint32_t b_shift = (uint32_t)(p.Wp * (i - i0) + j) * p.row_bytes;
                  const uint64_t ad = make_sdesc(a_stage + (uint32_t)t * p.tap_bytes, p.row_bytes, 0);
                  const uint64_t bd = make_sdesc(b_addr + b_shift, p.row_bytes, 0);
                  // K step = 32 bytes = +2 in the descriptor's start-address field
                  for (int ks = 0; ks < ksteps; ++ks)
                    umma<kTf32>(d_tmem, ad + 2 * ks, bd + 2 * ks, p.idesc, (k | t | ks) != 0 ? 1u : 0u);
                }
                // filter slot free (in every CTA of the cluster) when these MMAs finish
                if constexpr (CS == 1) umma_commit(aempty + as);
                else umma_commit_mc(aempty + as, cl_mask);
              }
              __syncwarp();
              if (NI == 2 && gs + 1 < gs_total) {
                if (gs & 1) asm volatile("bar.arrive 4, 64;" ::: "memory");
                else asm volatile("bar.arrive 3, 64;" ::: "memory");
              }
            }
            if (++as == p.a_stages) { as = 0; aph ^= 1u; }
          }
          if (elect_one()) umma_commit(bempty + bs);  // window free when every tap using it finished
          __syncwarp();
          if (++bs == 2) { bs = 0; bph ^= 1u; }
        }
      }
      if (trace && q == 0 && lane == 0) tr[3] = (p.dbg & 32) ? clock64() : global_ns();
      if (elect_one()) umma_commit(tfull + acc);
      __syncwarp();
      if (++acc == 2) { acc = 0; accph ^= 1u; }
    }
  } else if (kMode == kModeFusedMx && warp == xld_warp(kMode)) {
    // ------------------------------------------- staging producer (kModeFusedMx)
    // Boxes of kBoxE plane elements x kc channel planes of x (viewed as
    // [N*C][H*W], 128-byte swizzle) for every window, in window order, into a
    // ring of kRing slots.  x is the caller's input, not produced by the
    // preceding (PDL primary) kernel, so this starts without griddepcontrol.wait.
    const int my_groups = p.num_groups > cl_id ? (p.num_groups - cl_id + cl_num - 1) / cl_num : 0;
    const int nwin = my_groups * p.nchunks * p.ngroups;
    long long gb = 0;
    for (int wi = 0; wi < nwin; ++wi) {
      long long wrow;
      int cbase;
      tc2_window<CS>(p, cl_id, cl_num, rank, wi, wrow, cbase);
      Seg sg[kMaxSeg];
      const int r = tc2_segments(p, wrow, sg);
      const int nbox = r >> 8;
#pragma unroll
      for (int q = 0; q < kMaxSeg; ++q) {
        if (sg[q].n < 0) continue;
        int nxt = nbox;
#pragma unroll
        for (int q2 = kMaxSeg - 1; q2 > q; --q2)
          if (sg[q2].n >= 0) nxt = sg[q2].box0;
        for (int b = sg[q].box0; b < nxt; ++b, ++gb) {
          const int slot = (int)(gb % kRing);
          mbar_wait(rempty + slot, (uint32_t)((gb / kRing) & 1) ^ 1u);
          if (elect_one()) {
            mbar_arrive_expect_tx(rfull + slot, p.box_bytes);
            tma_load_2d(sX + (size_t)slot * p.box_bytes, &tmX, rfull + slot,
                        sg[q].e_lo + (b - sg[q].box0) * kBoxE, sg[q].n * p.C + cbase);
          }
          __syncwarp();
        }
      }
      if (ptrace && lane == 0 && wi == 0) pk[7] = global_ns();
    }
  } else if (kMode == kModeFusedMx && warp < kEpiWarp0) {
    // ------------------------------ packers (kModeFusedMx): fused a2, Eq. 10 + padding
    // Each staged box holds kBoxE consecutive plane elements of kc channels
    // (rows = channels, 128-byte swizzled).  One warp transposes a box as 8x8
    // blocks: ldmatrix.trans reads 8 channels x 8 elements, stmatrix writes 8
    // window rows (the elements' coefficients r*Wp + s of A_{n,c}(t), Eq. 10)
    // of 8 channel words each into the swizzled K-major window.  Elements
    // outside the window go to a dummy row.  Window rows that are padding
    // (reading R3) or past N*L_A are written as zeros.  Boxes of a window are
    // dealt round-robin to the packer warps.
    constexpr int NPW = pack_warps(kMode);
    const int pw = warp - kPackWarp0;
    const uint32_t swmask = p.row_bytes / 16u - 1u;
    const int ncg = (int)p.row_bytes / 16;  // 8-channel groups per window row
    const uint32_t sB0 = smem_u32(sB), sX0 = smem_u32(sX), sD = smem_u32(sDummy);
    const int my_groups = p.num_groups > cl_id ? (p.num_groups - cl_id + cl_num - 1) / cl_num : 0;
    const int nwin = my_groups * p.nchunks * p.ngroups;
    int bs = 0;
    uint32_t bph = 0;
    long long gb0 = 0;  // ring index of the window's first box
    for (int wi = 0; wi < nwin; ++wi) {
      long long wrow;
      int cbase;
      tc2_window<CS>(p, cl_id, cl_num, rank, wi, wrow, cbase);
      Seg sg[kMaxSeg];
      const int r = tc2_segments(p, wrow, sg);
      const int nbox = r >> 8;
      const bool trace0 = trace && pw == 0 && lane == 0 && wi == 0;
      mbar_wait(bempty + bs, bph ^ 1u);
      const uint32_t wbase = sB0 + (uint32_t)bs * p.b_bytes;
      const int cvalid = p.C - cbase;  // channels of this chunk that exist
      for (int j = (int)(((long long)pw - gb0 % NPW + NPW) % NPW); j < nbox; j += NPW) {  // boxes gb0+j = pw mod NPW
        int n = 0, e0 = 0;
#pragma unroll
        for (int q = 0; q < kMaxSeg; ++q)
          if (sg[q].n >= 0 && j >= sg[q].box0) { n = sg[q].n; e0 = sg[q].e_lo + (j - sg[q].box0) * kBoxE; }
        const long long gb = gb0 + j;
        const int slot = (int)(gb % kRing);
        mbar_wait(rfull + slot, (uint32_t)((gb / kRing) & 1));
        if (ptrace && wi == 0 && j < 4 && lane == 0) pk[j] = global_ns();  // box j of window 0 landed
        const uint32_t sbase = sX0 + (uint32_t)slot * p.box_bytes;
        const long long nbase = (long long)n * p.L_A - wrow;  // window row of coefficient 0 of image n
        const long long c_t0 = clock64();
        // this lane's stmatrix rows: element e0 + 8 eg + (lane & 7) -> window row (or -1)
        int prow[kBoxE / 8];
#pragma unroll
        for (int eg = 0; eg < kBoxE / 8; ++eg) {
          const int e = e0 + 8 * eg + (lane & 7);
          prow[eg] = -1;
          if (e < (int)p.HW) {
            const int h = (int)p.fW.div((uint32_t)e), w = e - h * p.W;
            const long long pos = nbase + (long long)(h + p.ph) * p.Wp + (w + p.pw);
            if (pos >= 0 && pos < p.brows) prow[eg] = (int)pos;
          }
        }
        for (int cq = 0; cq < ncg; cq += 4) {
          // 8 independent 8x8 loads in flight, then 8 stores (a single warp is latency-bound otherwise)
          const int c = (cq + (lane >> 3)) * 8 + (lane & 7);  // staging row (channel) this lane addresses
          const uint32_t srow = sbase + (uint32_t)c * 128u;
          uint32_t d[kBoxE / 8][4];
#pragma unroll
          for (int eg = 0; eg < kBoxE / 8; ++eg)
            ldsm_x4_trans(srow + 16u * (uint32_t)(eg ^ (c & 7)), d[eg][0], d[eg][1], d[eg][2], d[eg][3]);
          if (cvalid < p.kc) {  // partial chunk: channels >= C are zero
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int c2 = (cq + q) * 8 + 2 * (lane & 3);
              const uint32_t m = (c2 >= cvalid ? 0u : 0x0000FFFFu) | (c2 + 1 >= cvalid ? 0u : 0xFFFF0000u);
#pragma unroll
              for (int eg = 0; eg < kBoxE / 8; ++eg) d[eg][q] &= m;
            }
          }
          const uint32_t cgoff = 16u * (uint32_t)(cq + (lane >> 3));
#pragma unroll
          for (int eg = 0; eg < kBoxE / 8; ++eg) {
            uint32_t dst = sD + 16u * (uint32_t)(lane & 7);
            if (prow[eg] >= 0) {
              const uint32_t off = (uint32_t)prow[eg] * p.row_bytes + cgoff;
              dst = wbase + (off ^ (((off >> 7) & swmask) << 4));
            }
            stsm_x4(dst, d[eg][0], d[eg][1], d[eg][2], d[eg][3]);
          }
        }
        __syncwarp();
        if (ptrace && wi == 0 && j == 0 && lane == 0) pk[5] = (unsigned long long)(clock64() - c_t0);
        if (ptrace && wi == 1 && j == 0 && lane == 0) pk[4] = (unsigned long long)(clock64() - c_t0);
        if (lane == 0) mbar_arrive(rempty + slot);
      }
      // zero rows: padding coefficients (Eq. 10, reading R3) and rows past N*L_A
      for (int pp = pw * 32 + lane; pp < p.brows; pp += NPW * 32) {
        const long long gp = wrow + pp;
        bool pad = gp >= p.NLA;
        if (!pad) {
          const int n = (int)p.fLA.div((uint32_t)gp);
          const int m = (int)(gp - (long long)n * p.L_A);
          const int pr = (int)p.fWp.div((uint32_t)m), ps = m - pr * p.Wp;
          const int h = pr - p.ph, w = ps - p.pw;
          pad = h < 0 || h >= p.H || w < 0 || w >= p.W;
        }
        if (pad)
          for (int cg = 0; cg < ncg; ++cg) {
            const uint32_t off = (uint32_t)pp * p.row_bytes + 16u * (uint32_t)cg;
            sts128_zero(wbase + (off ^ (((off >> 7) & swmask) << 4)));
          }
      }
      // generic-proxy smem writes -> visible to the tensor core (async proxy)
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (trace0) tr[6] = global_ns();
      if (ptrace && wi == 0 && pw == 0 && lane == 0) pk[6] = global_ns();
      if (lane == 0) mbar_arrive(bfull + bs);
      gb0 += nbox;
      if (++bs == 2) { bs = 0; bph ^= 1u; }
    }
  } else if ((kMode == kModeFusedTma || kMode == kModeFusedLd) && warp < kEpiWarp0) {
    // ------------------------------------------- packers: fused a2 (Eq. 10 + padding)
    // Window row r is coefficient gp = wrow + r of the concatenated input
    // polynomials; coefficient pr*Wp + ps of A_{n,c} is x[n][c][pr-ph][ps-pw],
    // or 0 in the padding / past N*L_A.  Each packer thread builds whole rows:
    // the kc channel words of one coefficient, as row_bytes/16 swizzled
    // 16-byte chunks.  Consecutive lanes take consecutive rows.
    const int ptid = (warp - kPackWarp0) * 32 + lane;
    constexpr int kNP = pack_warps(kMode) * 32;
    constexpr int kEB = kTf32 ? 4 : 2;               // operand word bytes
    constexpr int EPC = 16 / kEB;                    // channels per 16-byte chunk
    const uint32_t swmask = p.row_bytes / 16u - 1u;  // 128/64/32-byte swizzle: chunk ^= (addr>>7) & swmask
    const int ncg = (int)p.row_bytes / 16;           // chunks per row
    const InT* __restrict__ x = reinterpret_cast<const InT*>(p.x);
    const InT* stg = reinterpret_cast<const InT*>(sX);
    const int my_groups = p.num_groups > cl_id ? (p.num_groups - cl_id + cl_num - 1) / cl_num : 0;
    const int nwin = my_groups * p.nchunks * p.ngroups;  // position windows this CTA packs
    if constexpr (kTmaX) {
      if (ptid == 0 && nwin > 0) {
        long long wrow;
        int cbase;
        tc2_window<CS>(p, cl_id, cl_num, rank, 0, wrow, cbase);
        tc2_issue_staging(p, &tmX, sX, sfull, wrow, cbase);
      }
    }
    int bs = 0;
    uint32_t bph = 0, sph = 0;
    for (int wi = 0; wi < nwin; ++wi) {
      long long wrow;
      int cbase;
      tc2_window<CS>(p, cl_id, cl_num, rank, wi, wrow, cbase);
      Seg sg[kMaxSeg];
      int ns = 0;
      if constexpr (kTmaX) ns = tc2_segments(p, wrow, sg) & 0xFF;
      const bool pkt = (p.dbg & 16) && ptid == 0 && wi < 2 && blockIdx.x < 160;
      unsigned long long* pk = g_tc2_pk + blockIdx.x * 8 + wi * 4;
      if (pkt) pk[0] = global_ns();
      mbar_wait_sleep(bempty + bs, bph ^ 1u, 64);
      if constexpr (kTmaX) {
        mbar_wait(sfull, sph);
        sph ^= 1u;
      }
      if (pkt) pk[1] = global_ns();
      uint8_t* dst = sB + (size_t)bs * p.b_bytes;
      // Row r -> (valid, src): src = element index of channel cbase of that
      // coefficient in the staging buffer (TMA path) or in x (direct path).
      // Rows go in pairs (r, r+1); when both come from consecutive staging
      // elements at an even index (the common case for even W, Wp), one 32-bit
      // shared load per channel fetches both rows' values (bf16 fast path).
      const bool full_chunk = cbase + p.kc <= p.C;
      const int rstart = (int)(((p.pw - wrow) % 2 + 2) % 2);
      const long long cstride = kTmaX ? (long long)kBoxE : p.HW;
      const int npairs = (p.brows - rstart) / 2;
      const int nitems = npairs + 2;  // pairs, then the unpaired first / last row
      for (int it = ptid; it < nitems; it += kNP) {
        int ra, nrows;
        if (it < npairs) { ra = rstart + 2 * it; nrows = 2; }
        else if (it == npairs) { ra = 0; nrows = rstart; }  // row 0 when the pairs start at 1
        else { ra = rstart + 2 * npairs; nrows = p.brows - ra; }  // trailing row
        if (nrows <= 0) continue;
        bool valid[2] = {false, false};
        long long src[2] = {0, 0};
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          if (q >= nrows) continue;
          const long long gp = wrow + ra + q;
          if (gp >= p.NLA) continue;
          const int n = (int)p.fLA.div((uint32_t)gp);
          const int m = (int)(gp - (long long)n * p.L_A);
          const int pr = (int)p.fWp.div((uint32_t)m), ps = m - pr * p.Wp;
          const int h = pr - p.ph, w = ps - p.pw;
          if (h < 0 || h >= p.H || w < 0 || w >= p.W) continue;
          valid[q] = true;
          const int e = h * p.W + w;
          if constexpr (kTmaX) {
            int e_lo = 0, box0 = 0;
#pragma unroll
            for (int g = 0; g < kMaxSeg; ++g)  // unrolled: the segment table stays in registers
              if (g < ns && sg[g].n == n) { e_lo = sg[g].e_lo; box0 = sg[g].box0; }
            const int de = e - e_lo;
            src[q] = (long long)(box0 + de / kBoxE) * p.kc * kBoxE + (de % kBoxE);
          } else {
            src[q] = ((long long)n * p.C + cbase) * p.HW + e;
          }
        }
        constexpr bool kPairPath = kTmaX && sizeof(InT) == 2 && !kTf32;
        if (kPairPath && nrows == 2 && full_chunk && valid[0] && valid[1] && src[1] == src[0] + 1 &&
            (src[0] & 1) == 0) {
          const uint32_t* s32 = reinterpret_cast<const uint32_t*>(stg + src[0]);  // 4-byte aligned
          const uint32_t off0 = (uint32_t)ra * p.row_bytes, off1 = off0 + p.row_bytes;
          for (int j = 0; j < ncg; ++j) {
            uint32_t v[8];
#pragma unroll
            for (int t = 0; t < 8; ++t) v[t] = s32[(j * 8 + t) * (kBoxE / 2)];  // channel j*8+t, rows ra, ra+1
            const uint4 o0 = make_uint4(__byte_perm(v[0], v[1], 0x5410), __byte_perm(v[2], v[3], 0x5410),
                                        __byte_perm(v[4], v[5], 0x5410), __byte_perm(v[6], v[7], 0x5410));
            const uint4 o1 = make_uint4(__byte_perm(v[0], v[1], 0x7632), __byte_perm(v[2], v[3], 0x7632),
                                        __byte_perm(v[4], v[5], 0x7632), __byte_perm(v[6], v[7], 0x7632));
            const uint32_t a0 = off0 + 16u * j, a1 = off1 + 16u * j;
            *reinterpret_cast<uint4*>(dst + (a0 ^ (((a0 >> 7) & swmask) << 4))) = o0;
            *reinterpret_cast<uint4*>(dst + (a1 ^ (((a1 >> 7) & swmask) << 4))) = o1;
          }
          continue;
        }
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          if (q >= nrows) continue;
          const uint32_t rowoff = (uint32_t)(ra + q) * p.row_bytes;
          for (int j = 0; j < ncg; ++j) {
            uint32_t wv[EPC];
#pragma unroll
            for (int t = 0; t < EPC; ++t) {
              const int c = j * EPC + t;
              wv[t] = 0u;
              if (valid[q] && (full_chunk || cbase + c < p.C)) {
                const InT v = kTmaX ? stg[src[q] + c * cstride] : __ldg(x + src[q] + c * cstride);
                wv[t] = ToWord<InT, kTf32>::cvt(v);
              }
            }
            uint4 o;
            if constexpr (kEB == 2)
              o = make_uint4(wv[0] | (wv[1] << 16), wv[2] | (wv[3] << 16), wv[4] | (wv[5] << 16), wv[6] | (wv[7] << 16));
            else
              o = make_uint4(wv[0], wv[1], wv[2], wv[3]);
            const uint32_t off = rowoff + 16u * j;
            *reinterpret_cast<uint4*>(dst + (off ^ (((off >> 7) & swmask) << 4))) = o;
          }
        }
      }
      // generic-proxy smem writes -> visible to the tensor core (async proxy); every
      // packer is done with the staging buffer before it is refilled for the next window
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      if (pkt) pk[2] = global_ns();
      asm volatile("bar.sync 1, %0;" ::"n"(kNP) : "memory");
      if (pkt) pk[3] = global_ns();
      if constexpr (kTmaX) {
        if (ptid == 0 && wi + 1 < nwin) {
          long long wrow1;
          int cbase1;
          tc2_window<CS>(p, cl_id, cl_num, rank, wi + 1, wrow1, cbase1);
          tc2_issue_staging(p, &tmX, sX, sfull, wrow1, cbase1);
        }
      }
      if (trace && ptid == 0 && wi == 0) tr[6] = global_ns();
      if (lane == 0) mbar_arrive(bfull + bs);
      if (++bs == 2) { bs = 0; bph ^= 1u; }
    }
  } else {
    // -------------------------------------------------------------- epilogue
    // a5 (Eq. 12 extraction + strided NCHW store), in passes of ecols positions:
    //  A. warp w reads TMEM lane quadrant (w % 4) = output channels kq..kq+31
    //     with tcgen05.ld.32x32b (thread = channel, 32 consecutive positions),
    //     converts to the output type and stores the row segment into the
    //     staging buffer sStage[channel][position - pass start];
    //  B. the warps copy the pass out channel by channel: the pass's
    //     extraction degrees of one image are one contiguous run of output
    //     indices o = oh*Q + ow of y[n][k] (Eq. 12 is monotone in m), so lanes
    //     take consecutive o and the stores are coalesced; coefficient m of o
    //     is Wp*sh*oh + sw*ow (the degree m(oh,ow) minus L_U - 1).
    const int ew = warp - kEpiWarp0;
    const int quad = warp & 3;
    const int hh = ew >> 2;  // which 32-column half of a 64-column step
    if (p.fpack) {
      // a3 (Eq. 6, reversed + gap-padded kernel; MMA view: tap-major [R*S][Kp][Cp],
      // reading R11 conversion): this CTA's slice of the packed filter
      using WT = typename std::conditional<kTf32, uint32_t, uint16_t>::type;
      const InT* __restrict__ wk = reinterpret_cast<const InT*>(p.w);
      WT* __restrict__ U = reinterpret_cast<WT*>(p.U);
      const int RS = p.R * p.S;
      const long long plane = (long long)p.Kp * p.Cp, total = plane * RS;
      const long long per = (total + gridDim.x - 1) / gridDim.x;
      const long long i0 = per * blockIdx.x, i1 = min(total, i0 + per);
      for (long long idx = i0 + ew * 32 + lane; idx < i1; idx += kEpiWarps * 32) {
        const int tap = (int)(idx / plane);
        const int rem = (int)(idx - (long long)tap * plane);
        const int k = rem / p.Cp, c = rem - k * p.Cp;
        uint32_t word = 0;
        if (k < p.K && c < p.C) word = ToWord<InT, kTf32>::cvt(wk[((long long)k * p.C + c) * RS + tap]);
        U[idx] = (WT)word;
      }
      asm volatile("fence.proxy.async.global;" ::: "memory");
      __threadfence();
      asm volatile("bar.sync 2, %0;" ::"n"(kEpiWarps * 32) : "memory");
      if (ew == 0 && lane == 0) atomicAdd(p.fcount, 1ull);
    }
    constexpr int EB = (int)sizeof(InT);
    InT* __restrict__ y = reinterpret_cast<InT*>(p.y);
    const uint32_t st0 = smem_u32(sStage);
    int acc = 0;
    uint32_t accph = 0;
    for (int grp = cl_id; grp < p.num_groups; grp += cl_num) {
      const int mg = grp / p.num_kt, kt = grp - mg * p.num_kt;
      const long long g0 = (long long)(mg * CS + (int)rank) * p.nt;
      mbar_wait_sleep(tfull + acc, accph, 64);
      tc_fence_after();
      if (trace && ew == 0 && lane == 0) tr[4] = global_ns();
      const uint32_t taddr = tmem_base + ((uint32_t)(quad * 32) << 16) + (uint32_t)(acc * p.acc_stride);
      // a5 index math once per tile: sPos[c] = element offset of output (n, k=0, oh, ow)
      // of position g0+c in y when it lies on the Eq. 12 / R4 lattice, else -1
      asm volatile("bar.sync 2, %0;" ::"n"(kEpiWarps * 32) : "memory");  // previous tile's table unused
      for (int c = ew * 32 + lane; c < p.nt; c += kEpiWarps * 32) {
        int off = -1;
        const long long gp = g0 + c;
        if (gp < p.G) {
          const int n = (int)p.fLA.div((uint32_t)gp);
          const int m = (int)gp - n * (int)p.L_A;
          const int r = (int)p.fWp.div((uint32_t)m), sc = m - r * p.Wp;
          const int oh = (int)p.fsh.div((uint32_t)r), ow = (int)p.fsw.div((uint32_t)sc);
          if (r == oh * p.sh && sc == ow * p.sw && oh < p.P && ow < p.Q) off = (n * p.K) * (int)p.PQ + oh * p.Q + ow;
        }
        sPos[c] = off;
      }
      const bool etr = (p.dbg & 128) && ew == 0 && lane == 0 && blockIdx.x < 160;
      unsigned long long ecyc[6] = {0, 0, 0, 0, 0, 0};
      long long et = clock64();
      auto tick = [&](int i) { const long long t = clock64(); ecyc[i] += (unsigned long long)(t - et); et = t; };
      // the CTA's last tile: every MMA is complete and no more operand loads will
      // land, so the whole tile is staged at once in the operand buffers (one
      // pass: no global stores queued in front of later passes' shared stores)
      const bool big = p.big_stage && grp + cl_num >= p.num_groups;
      const int ecols = big ? (p.nt + 31) / 32 * 32 : p.ecols;
      const uint32_t pitch = big ? (uint32_t)(ecols * EB + 16) : p.stage_pitch;
      const uint32_t stb = big ? smem_u32(sA) : st0;
      for (int c0 = 0; c0 < p.nt; c0 += ecols) {
        const int c1 = min(p.nt, c0 + ecols);
        // ---- A: TMEM -> staging (row = channel quad*32 + lane)
        for (int cb = c0 + 32 * hh; cb < c1; cb += 64) {
          uint32_t v[32];
          tmem_ld32(taddr + (uint32_t)cb, v);
          tmem_ld_wait();
          tick(0);
          const uint32_t row = stb + (uint32_t)(quad * 32 + lane) * pitch + (uint32_t)(cb - c0) * EB;
          if constexpr (EB == 2) {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              uint32_t w4[4];
#pragma unroll
              for (int t = 0; t < 4; ++t) {
                const __nv_bfloat162 h2 =
                    __floats2bfloat162_rn(__uint_as_float(v[8 * q + 2 * t]), __uint_as_float(v[8 * q + 2 * t + 1]));
                w4[t] = *reinterpret_cast<const uint32_t*>(&h2);
              }
              asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(row + 16u * q), "r"(w4[0]), "r"(w4[1]),
                           "r"(w4[2]), "r"(w4[3]) : "memory");
            }
          } else {
#pragma unroll
            for (int q = 0; q < 8; ++q)
              asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(row + 16u * q), "r"(v[4 * q]),
                           "r"(v[4 * q + 1]), "r"(v[4 * q + 2]), "r"(v[4 * q + 3]) : "memory");
          }
          tick(1);
        }
        tick(3);
        asm volatile("bar.sync 2, %0;" ::"n"(kEpiWarps * 32) : "memory");
        tick(2);
        // ---- B: staging -> y.  Lane l copies column cs+l of the warp's 16 channels
        // (consecutive lanes -> consecutive output pixels: coalesced; junk columns,
        // off the Eq. 12 / R4 lattice, are predicated off); the 16 shared loads are
        // issued before the 16 stores.
        for (int cs = c0; cs < c1; cs += 32) {
          const int cc = cs + lane;
          const int off = cc < c1 ? sPos[cc] : -1;
          constexpr int KPW = BMK / kEpiWarps;  // channels per warp
          const int kw = kt * BMK + ew;         // the warp's first channel
          const uint32_t sa0 = stb + (uint32_t)ew * pitch + (uint32_t)(cc - c0) * EB;
          InT* yp = y + (long long)kw * p.PQ + (off >= 0 ? off : 0);
          const long long ystep = (long long)kEpiWarps * p.PQ;
          if constexpr (EB == 2) {
            unsigned short b[KPW];
#pragma unroll
            for (int i = 0; i < KPW; ++i)
              asm volatile("ld.shared.u16 %0, [%1];" : "=h"(b[i]) : "r"(sa0 + (uint32_t)(i * kEpiWarps) * pitch));
            if (off >= 0 && !(p.dbg & 64)) {
#pragma unroll
              for (int i = 0; i < KPW; ++i) {
                if (kw + i * kEpiWarps < p.K) *reinterpret_cast<unsigned short*>(yp) = b[i];
                yp += ystep;
              }
            }
          } else {
            float f[KPW];
#pragma unroll
            for (int i = 0; i < KPW; ++i)
              asm volatile("ld.shared.f32 %0, [%1];" : "=f"(f[i]) : "r"(sa0 + (uint32_t)(i * kEpiWarps) * pitch));
            if (off >= 0 && !(p.dbg & 64)) {
#pragma unroll
              for (int i = 0; i < KPW; ++i) {
                if (kw + i * kEpiWarps < p.K) *yp = f[i];
                yp += ystep;
              }
            }
          }
        }
        tick(4);
        asm volatile("bar.sync 2, %0;" ::"n"(kEpiWarps * 32) : "memory");  // staging reused by the next pass
        tick(5);
      }
      if (etr)
        for (int i = 0; i < 6; ++i) g_tc2_epi[blockIdx.x * 8 + i] = ecyc[i];
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
cudaError_t launch_one(const Tc2Tiling& t, const CUtensorMap& tmW, const CUtensorMap& tmX, const Tc2Params& p,
                       bool pdl, cudaStream_t st) {
  auto kern = t.mode == kModeTma        ? mac_tc2_kernel<InT, kTf32, CS, kModeTma>
              : t.mode == kModeFusedTma ? mac_tc2_kernel<InT, kTf32, CS, kModeFusedTma>
                                        : mac_tc2_kernel<InT, kTf32, CS, kModeFusedLd>;
  if constexpr (std::is_same<InT, __nv_bfloat16>::value && !kTf32)
    if (t.mode == kModeFusedMx) kern = mac_tc2_kernel<InT, kTf32, CS, kModeFusedMx>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, t.smem_bytes);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)t.grid);
  cfg.blockDim = dim3(threads_for(t.mode));
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
  return cudaLaunchKernelEx(&cfg, kern, tmW, tmX, p);
}

// Staging demand of the TMA input path: the most boxes (and image segments)
// any position window needs -- the same walk the packers do.
void staging_demand(const Geom& g, const Tc2Tiling& t, int eb_in, int& max_boxes, int& max_segs) {
  max_boxes = 0;
  max_segs = 0;
  const long long NLA = (long long)g.N * g.L_A;
  for (long long mt = 0; mt < (long long)t.num_groups / t.num_kt * t.cs; ++mt) {  // incl. dummy tiles
    for (int rg = 0; rg < t.ngroups; ++rg) {
      const long long wrow = mt * t.nt + (long long)g.Wp * (rg * t.nr);
      if (wrow >= NLA) continue;
      const int n_lo = (int)(wrow / g.L_A);
      const int n_hi = (int)std::min((long long)g.N - 1, (wrow + t.brows - 1) / g.L_A);
      int boxes = 0, segs = 0;
      for (int n = n_lo; n <= n_hi; ++n) {
        const int base = (int)((long long)n * g.L_A - wrow);
        const int pr_lo = base >= 0 ? 0 : (-base) / g.Wp;
        const int pr_hi = std::min(g.Hp - 1, (t.brows - 1 - base) / g.Wp);
        const int h_lo = std::max(0, pr_lo - g.ph), h_hi = std::min(g.H - 1, pr_hi - g.ph);
        if (h_lo > h_hi) continue;
        const int e_lo = (h_lo * g.W) & ~(16 / eb_in - 1);
        boxes += ((h_hi + 1) * g.W - e_lo + kBoxE - 1) / kBoxE;
        ++segs;
      }
      max_boxes = std::max(max_boxes, boxes);
      max_segs = std::max(max_segs, segs);
    }
  }
}

}  // namespace

bool tc2_is_mx(const Tc2Tiling& t) { return t.mode == kModeFusedMx; }

bool tc2_supported(const Geom& g, int fmt) {
  if (fmt != FMT_BF16 && fmt != FMT_TF32) return false;
  if ((long long)g.R * g.S * ((g.K + 127) / 128 * 128) >= (1LL << 31)) return false;  // TMA row coordinate
  if (g.S - 1 + 16 > kBMaxRows) return false;  // one kernel row must fit a window
  if ((long long)g.N * g.L_A + 2 * kBMaxRows + 256 >= (1LL << 31)) return false;  // 32-bit position decode
  return true;
}

Tc2Tiling tc2_tiling(const Geom& g, int fmt, bool x_bf16, int num_sms, bool fused, bool y_bf16) {
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
  // window rows: whole TMA boxes (kModeTma) / swizzle atoms of 8 rows (fused)
  t.brows = (int)cdiv((long long)t.nt + (long long)(nr - 1) * g.Wp + g.S - 1, fused ? 8 : kBoxRows) *
            (fused ? 8 : kBoxRows);
  t.num_mt = (int)cdiv(G, t.nt);
  t.num_tiles = t.num_mt * t.num_kt;
  t.num_groups = (int)cdiv(t.num_mt, t.cs) * t.num_kt;
  t.nchunks = (g.C + kc - 1) / kc;
  const int a_bytes = BMK * t.row_bytes;
  const int b_bytes = (int)cdiv((long long)t.brows * t.row_bytes, 1024) * 1024;
  // input staging for the TMA path: x viewed as [N*C][H*W] needs a 16-byte row pitch
  const int eb_in = x_bf16 ? 2 : 4;
  t.box_bytes = kBoxE * kc * eb_in;
  t.tma_x = fused && ((long long)g.H * g.W * eb_in) % 16 == 0;
  if (t.tma_x) {
    int max_boxes, max_segs;
    staging_demand(g, t, eb_in, max_boxes, max_segs);
    t.stg_bytes = (int)cdiv((long long)std::max(1, max_boxes) * t.box_bytes, 1024) * 1024;
    if (max_segs > kMaxSeg || 1024 + 2 * b_bytes + t.stg_bytes + 18 * 1024 + 512 + 3 * a_bytes > 227 * 1024)
      t.tma_x = false;
  }
  if (!t.tma_x) t.stg_bytes = 0;
  t.mode = !fused ? kModeTma : (t.tma_x ? kModeFusedTma : kModeFusedLd);
  // bf16 input and math with a TMA view: ring-staged 8x8-transpose packers
  if (fused && t.tma_x && x_bf16 && fmt == FMT_BF16 && kc >= 32 && !getenv("POLYCONV_TC_NO_MX")) {
    t.mode = kModeFusedMx;
    t.stg_bytes = kRing * t.box_bytes;
  }
  // epilogue staging: 128 channels x ecols positions of the output type (+16 B per row)
  t.ecols = y_bf16 ? 64 : 32;  // a multiple of the 32 columns one tcgen05.ld.32x32b.x32 returns
  t.stage_pitch = t.ecols * (y_bf16 ? 2 : 4) + 16;
  t.stage_bytes = BMK * t.stage_pitch;  // + the pass's output-offset table (ecols x 8 B)
  const int fixed = 1024 + 2 * b_bytes + t.stg_bytes + t.stage_bytes + 256 * 4 + 128 + 768;
  // taps per filter stage: as many as leave room for a 3-deep ring (fewer, larger
  // stages amortise the per-stage barrier check of the MMA issuer)
  const int budget = 227 * 1024 - fixed;
  int tps = g.R * g.S;
  while (tps > 1 && 3 * tps * a_bytes > budget) --tps;
  if (fused) tps = 1;
  if (const char* f = getenv("POLYCONV_TC_TPS")) tps = std::max(1, std::min(tps, atoi(f)));  // experiments only
  t.tps = tps;
  int st = budget / (tps * a_bytes);
  if (st > 12) st = 12;
  t.a_stages = st;
  t.smem_bytes = fixed + st * tps * a_bytes;
  t.acc_stride = t.nt <= 128 ? 128 : 256;
  t.tmem_cols = 2 * t.acc_stride;
  const int max_clusters = num_sms / t.cs;
  t.grid = (t.num_groups < max_clusters ? t.num_groups : max_clusters) * t.cs;
  return t;
}

cudaError_t launch_mac_tc2(const Geom& g, const Tc2Tiling& t, int fmt, const void* x, bool x_bf16, const void* A,
                           const void* U, void* y, bool y_bf16, bool pdl, cudaStream_t st, char* err, size_t errlen,
                           const void* w, unsigned long long* fcount, unsigned long long ftarget) {
  if (t.a_stages < 2) {
    snprintf(err, errlen, "mac_tc2: shared memory too small for the window");
    return cudaErrorInvalidValue;
  }
  CUtensorMap tmW;
  // filter box = the 128/cs rows one CTA loads and multicasts to its cluster
  if (!encode(&tmW, U, fmt, (uint64_t)g.Cp, (uint64_t)g.urep * g.R * g.S * g.Kp, t.kc, BMK / t.cs, t.row_bytes)) {
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
  // staging TMA map over x as [N*C][H*W] (TMA path); its base must be 16-byte aligned
  CUtensorMap tmX;
  memset(&tmX, 0, sizeof(tmX));
  if (t.mode == kModeTma) {
    // position windows from the packed input [N*L_A][Cp] (a2 done by pack_both), 32-row boxes
    if (!encode(&tmX, A, fmt, (uint64_t)g.Cp, (uint64_t)g.N * g.L_A, t.kc, kBoxRows, t.row_bytes)) {
      snprintf(err, errlen, "cuTensorMapEncodeTiled (packed input) failed");
      return cudaErrorInvalidValue;
    }
  } else if (t.mode == kModeFusedMx) {
    // staging boxes of kBoxE elements x kc planes of x viewed as [N*C][H*W], 128-byte swizzle
    if ((reinterpret_cast<uintptr_t>(x) % 16) != 0) {
      snprintf(err, errlen, "mac_tc2: x must be 16-byte aligned");
      return cudaErrorInvalidValue;
    }
    EncodeTiledFn enc = get_encode2();
    cuuint64_t dims[2] = {(cuuint64_t)p.HW, (cuuint64_t)g.N * g.C};
    cuuint64_t strides[1] = {(cuuint64_t)p.HW * 2};
    cuuint32_t box[2] = {(cuuint32_t)kBoxE, (cuuint32_t)t.kc};
    cuuint32_t estr[2] = {1, 1};
    if (!enc || enc(&tmX, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(x), dims, strides, box, estr,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      snprintf(err, errlen, "cuTensorMapEncodeTiled (input staging, swizzled) failed");
      return cudaErrorInvalidValue;
    }
  } else if (t.tma_x) {
    if ((reinterpret_cast<uintptr_t>(x) % 16) != 0) {
      snprintf(err, errlen, "mac_tc2: x must be 16-byte aligned");
      return cudaErrorInvalidValue;
    }
    EncodeTiledFn enc = get_encode2();
    const int eb_in = x_bf16 ? 2 : 4;
    cuuint64_t dims[2] = {(cuuint64_t)p.HW, (cuuint64_t)g.N * g.C};
    cuuint64_t strides[1] = {(cuuint64_t)p.HW * eb_in};
    cuuint32_t box[2] = {(cuuint32_t)kBoxE, (cuuint32_t)t.kc};
    cuuint32_t estr[2] = {1, 1};
    if (!enc || enc(&tmX, x_bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2,
                    const_cast<void*>(x), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      snprintf(err, errlen, "cuTensorMapEncodeTiled (input staging) failed");
      return cudaErrorInvalidValue;
    }
  }
  p.box_bytes = (uint32_t)t.box_bytes;
  p.ealign = x_bf16 ? 8 : 4;
  p.fLA.init((uint32_t)g.L_A);
  p.fWp.init((uint32_t)g.Wp);
  p.fsh.init((uint32_t)g.sh);
  p.fsw.init((uint32_t)g.sw);
  p.fW.init((uint32_t)g.W);
  p.stg_bytes = (uint32_t)t.stg_bytes;
  p.Wp = g.Wp; p.P = g.P; p.Q = g.Q; p.sh = g.sh; p.sw = g.sw; p.K = g.K; p.R = g.R; p.S = g.S;
  p.nt = t.nt; p.brows = t.brows; p.nr = t.nr; p.ngroups = t.ngroups;
  p.num_mt = t.num_mt; p.num_kt = t.num_kt; p.num_tiles = t.num_tiles; p.num_groups = t.num_groups;
  p.nchunks = t.nchunks; p.kc = t.kc; p.Kp = g.Kp; p.Cp = g.Cp;
  p.a_stages = t.a_stages;
  const uint32_t ab = fmt == FMT_BF16 ? 1u : 2u;
  // instruction descriptor: D=f32 @4, A/B format @7/@10, both K-major, N>>3 @17, M>>4 @24
  p.idesc = (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(t.nt >> 3) << 17) | ((uint32_t)(BMK >> 4) << 24);
  p.row_bytes = (uint32_t)t.row_bytes;
  p.tap_bytes = (uint32_t)(BMK * t.row_bytes);
  p.tps = t.tps;
  p.urep = g.urep;
  p.stages_per_tile = 0;
  for (int rg = 0; rg < t.ngroups; ++rg) {
    const int ntap = (std::min(g.R, (rg + 1) * t.nr) - rg * t.nr) * g.S;
    p.stages_per_tile += (ntap + t.tps - 1) / t.tps;
  }
  p.stages_per_tile *= t.nchunks;
  p.a_bytes = p.tap_bytes * (uint32_t)t.tps;
  p.b_bytes = (uint32_t)(cdiv((long long)t.brows * t.row_bytes, 1024) * 1024);
  p.b_bytes_tx = (uint32_t)(t.brows * t.row_bytes);
  p.acc_stride = t.acc_stride; p.tmem_cols = t.tmem_cols;
  p.ecols = t.ecols;
  p.stage_pitch = (uint32_t)t.stage_pitch;
  p.stage_bytes = (uint32_t)t.stage_bytes;
  p.fQ.init((uint32_t)g.Q);
  {
    const int eb_y = y_bf16 ? 2 : 4;
    const long long need = (long long)BMK * (((t.nt + 31) / 32 * 32) * eb_y + 16);
    p.big_stage = need <= (long long)t.a_stages * BMK * t.row_bytes * t.tps && !getenv("POLYCONV_TC_NO_BIGSTAGE");
  }
  p.y = y;
  if (y_bf16 != x_bf16) return cudaErrorInvalidValue;  // y has the io dtype of x
  p.w = w;
  p.U = const_cast<void*>(U);
  p.fcount = fcount;
  p.ftarget = ftarget;
  p.fpack = (w != nullptr && fcount != nullptr && t.mode != kModeTma) ? 1 : 0;
  if (p.fpack) pdl = false;  // no primary kernel: the filter is packed in this grid
  const char* dbg = getenv("POLYCONV_TC_DEBUG");
  p.dbg = dbg ? atoi(dbg) : 0;
  if (fmt == FMT_TF32) {
    if (x_bf16) return cudaErrorInvalidValue;
    return t.cs == 1 ? launch_one<float, true, 1>(t, tmW, tmX, p, pdl, st)
                     : launch_one<float, true, 2>(t, tmW, tmX, p, pdl, st);
  }
  if (x_bf16)
    return t.cs == 1 ? launch_one<__nv_bfloat16, false, 1>(t, tmW, tmX, p, pdl, st)
                     : launch_one<__nv_bfloat16, false, 2>(t, tmW, tmX, p, pdl, st);
  return t.cs == 1 ? launch_one<float, false, 1>(t, tmW, tmX, p, pdl, st)
                   : launch_one<float, false, 2>(t, tmW, tmX, p, pdl, st);
}

}  // namespace polyconv

// Debug only (not part of include/polyconv.h): copy the per-CTA phase trace of
// the last POLYCONV_TC_DEBUG&8 launch to host (160 x 8 u64).
extern "C" int polyconv_dbg_tc2_pk(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_tc2_pk, sizeof(unsigned long long) * 160 * 8);
}
extern "C" int polyconv_dbg_tc2_epi(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_tc2_epi, sizeof(unsigned long long) * 160 * 8);
}
extern "C" int polyconv_dbg_tc2_trace(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_tc2_trace, sizeof(unsigned long long) * 160 * 8);
}
