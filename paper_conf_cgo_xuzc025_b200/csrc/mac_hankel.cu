// mac_hankel.cu — a2 + a4 + a5 in one persistent, warp-specialised tcgen05
// kernel on CTA pairs, fed straight from the NCHW input (no packed copy of x).
//
// What it computes: per output position q and channel k,
//   p_k[q] = sum_c sum_{i,j} A_c[q + pitch*i + j] * w[k][c][i][j]
// i.e. the coefficient MAC p_{n,k}[m] = sum_c sum_{i,j} A_{n,c}[m - e(i,j)] U_{k,c}[e(i,j)]
// (P.965; schoolbook product P.1021-1025; channel sum P.1350-1352) at the Eq. 12
// extraction degrees, with every tap's operand a *shifted window* of the same input
// polynomial (the Hankel structure, P.404-437).
//
// Input polynomial layout (reading R16).  All images' padded planes are
// concatenated into one long polynomial (the paper's segment concatenation with
// padding between segments, P.1356-1360):
//   A_c[q] = x[n][c][h][w]  at  q = (n*HS + ph + h)*pitch + pw + w + delta,
//   zero everywhere else,
// with row pitch `pitch` = W + 2*pw (the paper's Iw = Wp, Eq. 10) or W + pw, and image
// stride HS = H + ph rows: consecutive images share their ph zero rows (the bottom
// padding of image n is the top padding of image n+1), and with pitch W + pw each row
// shares its pw zero columns with the next row.  delta (0/1) aligns position pairs with
// 4-byte input pairs.  Output (n, oh, ow) is the coefficient at
//   q = (n*HS + sh*oh)*pitch + sw*ow + delta
// (Eq. 12 with L_U - 1 absorbed into the window origin; stride: reading R4).
//
// Design (DESIGN.md §4 "mac_hankel"):
//  * Pair MMA (tcgen05.mma.cta_group::2, kind::f16 / kind::tf32): M = 256 positions
//    (128 per CTA = the TMEM lanes), N = NN output channels (each CTA holds NN/2 filter
//    rows), K-step 16 bf16 / 8 tf32 channels.  A = the position window (K-major, 128-B
//    swizzled rows of 64 bf16 / 32 tf32 channels); each tap's MMA reads it through a
//    descriptor shifted by pitch*i + j rows.  B = the tap-major packed filter (a3).
//  * A work item is T in {1,2,4} 128-position tiles per CTA (a window of 128*T +
//    (R-1)*pitch + S-1 rows) x one block of NN output channels; the T accumulators
//    share every filter block, so the filter bytes per MAC fall by T.  Each pair takes a
//    contiguous range of 256-position units (balanced to +-1 unit), grouped into items.
//  * Filter resident in shared memory when the pair's half fits (loaded once per
//    launch), else streamed through a ring of (chunk, tap) blocks by TMA.
//  * Warp roles per CTA: warp 0 filter producer (TMA), warp 1 TMEM allocator + MMA
//    issuer (leader CTA), warps 2-9 window loaders, warps 10-17 epilogue.
//  * Loaders (a2): each lane converts two consecutive positions x 8 (bf16) / 4 (tf32)
//    channels: one 4-/8-byte load per channel when the pair is an aligned input pair,
//    else two element loads; zeros for padding (Eq. 10, reading R3), for channels past
//    C and past the last image; bf16 RNE / tf32 RNA (reading R11); 16-byte swizzled
//    stores.  No HBM copy of the packed input exists.
//  * Epilogue (a5): tcgen05.ld of 16 columns, position -> (n, oh, ow) decode per lane,
//    off-lattice / junk positions dropped, NCHW stores (lanes = consecutive pixels).
//  * Synchronisation is pair-local (mbarriers, cluster scope); no grid-wide
//    barrier, no counters in global memory, so the launch needs no co-residency of
//    the whole grid and is safe to capture into CUDA graphs and replay.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <algorithm>
#include "common.cuh"
#include "sm100.cuh"

namespace polyconv {

namespace {

using namespace sm100;

constexpr int kHkLoadWarps = 16;   // 8 16-byte channel groups x 2 halves of the window rows
constexpr int kHkEpiWarps = 8;     // two per TMEM lane quadrant
constexpr int kHkThreads = 32 * 28;  // 28 warps, 7 per scheduler sub-partition
// Warp roles.  Warp w issues from sub-partition w % 4 and may read TMEM lanes 32*(w % 4)..+31.
// The MMA issuer (warp 1) shares its sub-partition only with the filter producer, the
// forwarders and one epilogue warp, which mostly wait: with loaders beside it the issuer got a
// fraction of the issue slots and the tensor pipe idled between MMAs (measured, tools/hk_trace.py).
// Loaders: the window loads are latency-bound (ncu: long-scoreboard stalls), so 16 warps
// split every window's rows in two halves to halve the round trips per window.
enum HkRole { kRoleIdle = 0, kRoleMma, kRoleProducer, kRoleLoader, kRoleEpi, kRoleFwdW, kRoleFwdE };
__device__ __forceinline__ int hk_role(int warp, int& idx) {
  constexpr int kLoad[16] = {0, 8, 12, 16, 20, 2, 10, 14, 18, 22, 3, 11, 15, 19, 23, 25};
  constexpr int kEpi[8] = {4, 24, 9, 21, 6, 26, 7, 27};  // quadrant = w % 4, column half = order
  if (warp == 1) return kRoleMma;
  if (warp == 5) return kRoleProducer;
  if (warp == 13) return kRoleFwdE;   // epilogue drained -> leader (one cluster arrive per CTA)
  if (warp == 17) return kRoleFwdW;   // window stored -> leader
#pragma unroll
  for (int i = 0; i < 16; ++i)
    if (warp == kLoad[i]) { idx = i; return kRoleLoader; }
#pragma unroll
  for (int i = 0; i < 8; ++i)
    if (warp == kEpi[i]) { idx = i; return kRoleEpi; }
  return kRoleIdle;
}
constexpr int kHkSmemMax = 232448;                         // 227 KB dynamic
constexpr int kHkMaxFBlk = 64;                             // filter ring slots (max)
constexpr int kHkMaxWSlots = 4;

constexpr int kHkMaxOut = 8;  // output buffers of one forward (polyconv_forward_scatter)

struct HkParams {
  const void* x;
  const void* zero;     // plan-owned zero words (>= 8 planes of float2), read for zero pairs
  void* ys[kHkMaxOut];  // outputs [N][Ktot][P][Q]: y, or every rank's (peer-mapped) buffer
  int nys, Ktot, koff;  // number of outputs; their channel count and this plan's channel offset
  int N, C, H, W, K, P, Q, sh, sw, ph, pw;
  int HW, CHW;          // plane size, image size (elements)
  int pitch, HS, delta; // input polynomial layout (reading R16)
  int T;                // max 128-position tiles per CTA per item
  int NN, NB;           // output channels per block (MMA N), blocks
  int Kp, Cp, nchunks, RS, S;
  int PT;               // 256-position units
  int npairs;
  int wrows;            // rows per window slot (128*T + (R-1)*pitch + S-1, rounded to 8)
  int wslots;           // window ring depth
  int fslots;           // filter ring depth (blocks); resident: = nchunks*RS
  int resident;         // filter loaded once
  uint32_t wslot_bytes, fblk_bytes;
  uint32_t idesc;
  int tmem_cols;
  int nacc;             // accumulator buffers in TMEM (2: the epilogue overlaps the next item's MMAs)
  FastDiv fpitch, fHS, fsh, fsw;
  // stride-2 phase mode (reading R19): the kernel runs the stride-1 convolution of the
  // phase-split input; N, C, H, W, ph, pw, sh, sw above are that convolution's, these are x's
  int phase;            // 0 / 1
  int xC, xH, xW;       // x dims (phase mode)
  uint32_t rt_stage;    // kRowTile: bytes of one staged output tile (NN channels x Q pixels, bf16)
  // plane-staged loader (kHW2 == kHkPlanes): whole (image, 64-channel) blocks of x, bulk-copied
  uint32_t pimg_bytes;  // 64 * H * W * 2: one image's 64-channel block (16-byte multiple)
  int pimg_max;         // images a window can touch (staging buffer = pimg_max blocks)
  int psbufs;           // staging buffers (2: the copies run one window ahead; 1 when smem is short)
  int dbg;  // POLYCONV_HK_DEBUG (timing ablations, results wrong): 1 loaders store zeros without
            // loading, 2 epilogue skips stores, 4 no MMAs (commits only), 8 per-CTA trace
};

// per-CTA trace (dbg & 8), globaltimer ns: 0 start, 1 setup done, 2 first window stored (loader
// warp 0), 3 filter resident / first block (MMA), 4 first item's MMAs issued, 5 first item drained
// (epilogue warp 0), 6 last item's MMAs issued, 7 last item drained, 8 end, 9 / 10 first / last
// item's accumulator ready (epilogue warp 0)
__device__ unsigned long long g_hk_trace[160 * 16];
// dbg & 16: CTA 0 pipeline trace (globaltimer ns) of its first 64 windows: [w][0] loader warp 0
// starts waiting for the slot, [1] slot free, [2] window stored, [3] MMA saw it full, [4] MMAs issued
__device__ unsigned long long g_hk_wtrace[64 * 8];
// dbg & 32: per loader warp (16 = 2 CTAs x 8) store-complete time of the first 64 windows of pair 0
__device__ unsigned long long g_hk_ltrace[64 * 16];

// ---- pair PTX (cta_group::2) ------------------------------------------------------
__device__ __forceinline__ uint32_t hk_mapa0(uint32_t local) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(r) : "r"(local));
  return r;
}
__device__ __forceinline__ void hk_tma_pair(uint32_t dst, const void* tmap, uint32_t mbar_cluster, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(tmap)), "r"(mbar_cluster), "r"(c0), "r"(c1)
      : "memory");
}
template <bool kTf32>
__device__ __forceinline__ void hk_mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  if constexpr (kTf32) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
  } else {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
  }
}
__device__ __forceinline__ void hk_commit_both(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"((uint16_t)3)
      : "memory");
}
__device__ __forceinline__ void hk_arrive_cluster(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
// plain parity wait (no watchdog: every wait is on work of the same CTA pair, which the
// hardware co-schedules).  No __nanosleep back-off: try_wait already suspends in hardware, and
// a 32 / 64 ns sleep in the loaders' slot wait and the epilogue's waits cost 3% on 128->128
// 28x28 (838 -> 862 TFLOP/s; 15 us of 71 with the MMAs ablated).
__device__ __forceinline__ void hk_wait(uint64_t* bar, uint32_t parity) {
  const uint32_t a = smem_u32(bar);
  uint32_t done;
  for (;;) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
    if (done) return;
  }
}
__device__ __forceinline__ void hk_tmem_alloc2(uint32_t* slot, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(slot)),
               "r"(ncols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void hk_tmem_dealloc2(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
// 32 lanes x 16 consecutive 32-bit columns
__device__ __forceinline__ void hk_tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
      "{%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
        "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr)
      : "memory");
}

// ---- work decomposition (identical in every role) ---------------------------------
// Pair `pair` owns units [u_lo, u_hi) of the (n-block major, 256-position minor) unit
// space; an item is T consecutive units of one n-block (T = the largest of the plan's
// T, 2, 1 that fits the rest of the range and the block).
struct HkItem {
  int nb, pt, T;
};
__device__ __forceinline__ bool hk_next(const HkParams& p, long long& u, long long u_hi, HkItem& it) {
  if (u >= u_hi) return false;
  it.nb = (int)(u / p.PT);
  it.pt = (int)(u - (long long)it.nb * p.PT);
  const long long room = min(u_hi - u, (long long)(p.PT - it.pt));
  int T = p.T;
  while (T > 1 && room < T) T >>= 1;
  it.T = T;
  u += T;
  return true;
}

// ---- a2: one window of the input polynomial into a shared-memory slot ---------------
// element offset of (n, channel 0, h, w) for position q, or -1 for a zero coefficient
// (branch-free; every position of a launch is < 2^31, checked by the plan)
__device__ __forceinline__ bool hk_pos(const HkParams& p, long long q, int& n, int& h, int& w) {
  const int qq = (int)q - p.delta;
  const uint32_t u = (uint32_t)max(qq, 0);
  const uint32_t vr = p.fpitch.div(u);
  w = (int)(u - vr * (uint32_t)p.pitch) - p.pw;
  const int vr2 = (int)vr - p.ph;
  n = (int)p.fHS.div((uint32_t)max(vr2, 0));
  h = vr2 - n * p.HS;
  return qq >= 0 && w >= 0 && w < p.W && vr2 >= 0 && h < p.H && n < p.N;
}
__device__ __forceinline__ int hk_src(const HkParams& p, long long q) {
  int n, h, w;
  const bool ok = hk_pos(p, q, n, h, w);
  return ok ? n * p.CHW + h * p.W + w : -1;
}

template <typename IoT>
__device__ __forceinline__ uint32_t hk_bf16(uint32_t raw) {
  if constexpr (sizeof(IoT) == 2) return raw;
  else return (uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(__uint_as_float(raw)));  // R11: RNE
}

// The window of this CTA: positions [q0, q0 + wrows) of channels [c0, c0 + 128 B of words).
// Loader warp lw owns 16-byte column group lw of every row (8 bf16 / 4 tf32 channels); its
// lanes take consecutive position pairs, so each load instruction reads a contiguous run of
// one channel plane.  Branch-free: every load is issued (a masked one reads x[0]) before any
// is consumed, B position pairs per lane in flight.  bf16 input is read as the aligned 32-bit
// word holding the element.  The two rows of a pair are stored in the order (lane >> 2) & 1,
// so the 8 lanes of each store phase hit 8 different 16-byte bank groups of the swizzle.
template <typename IoT, bool kTf32>
__device__ __forceinline__ void hk_load_window(const HkParams& p, uint32_t slot, long long q0, int c0, int lw,
                                               int lane, int rp_lo, int rp_hi) {
  const uint32_t* xw = static_cast<const uint32_t*>(p.x);  // 32-bit words of x
  constexpr bool kBf16In = sizeof(IoT) == 2;
  constexpr int CPG = kTf32 ? 4 : 8;  // channels per 16-byte group
  const int cg = c0 + lw * CPG;
  const int nrp = rp_hi;
  const int odd_hw = p.HW & 1;
  const uint32_t sel = (uint32_t)(lane >> 2) & 1u;
  constexpr int B = 2;
  for (int rp0 = rp_lo; rp0 < nrp; rp0 += 32 * B) {
    uint32_t w0[B][CPG], w1[B][CPG];
    int s0[B], s1[B];
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const int rp = rp0 + b * 32 + lane;
      const long long q = q0 + 2 * rp;
      const bool in = rp < nrp && !(p.dbg & 1);
      s0[b] = in ? hk_src(p, q) : -1;
      s1[b] = in ? hk_src(p, q + 1) : -1;
#pragma unroll
      for (int c = 0; c < CPG; ++c) {
        const int coff = (cg + c) * p.HW;
        const bool chok = cg + c < p.C;
        const int e0 = (chok && s0[b] >= 0) ? s0[b] + coff : 0;
        const int e1 = (chok && s1[b] >= 0) ? s1[b] + coff : 0;
        w0[b][c] = __ldg(xw + (kBf16In ? (e0 >> 1) : e0));
        w1[b][c] = __ldg(xw + (kBf16In ? (e1 >> 1) : e1));
      }
    }
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const int rp = rp0 + b * 32 + lane;
      uint32_t r0[4], r1[4];
      uint32_t v0[CPG], v1[CPG];
#pragma unroll
      for (int c = 0; c < CPG; ++c) {
        const bool chok = cg + c < p.C;
        const bool ok0 = chok && s0[b] >= 0, ok1 = chok && s1[b] >= 0;
        if constexpr (kBf16In) {
          const uint32_t h0 = (uint32_t)(s0[b] + odd_hw * (cg + c)) & 1u;
          const uint32_t h1 = (uint32_t)(s1[b] + odd_hw * (cg + c)) & 1u;
          v0[c] = ok0 ? (w0[b][c] >> (16u * h0)) & 0xFFFFu : 0u;
          v1[c] = ok1 ? (w1[b][c] >> (16u * h1)) & 0xFFFFu : 0u;
        } else {
          v0[c] = ok0 ? w0[b][c] : 0u;
          v1[c] = ok1 ? w1[b][c] : 0u;
        }
      }
      if constexpr (kTf32) {
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          r0[c] = to_tf32_rna(__uint_as_float(v0[c]));  // reading R11: RNA
          r1[c] = to_tf32_rna(__uint_as_float(v1[c]));
        }
      } else {
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          r0[c] = hk_bf16<IoT>(v0[2 * c]) | (hk_bf16<IoT>(v0[2 * c + 1]) << 16);
          r1[c] = hk_bf16<IoT>(v1[2 * c]) | (hk_bf16<IoT>(v1[2 * c + 1]) << 16);
        }
      }
      if (rp < nrp) {
        const uint32_t ra = 2u * (uint32_t)rp + sel, rb = 2u * (uint32_t)rp + (sel ^ 1u);
        const uint32_t* da = sel ? r1 : r0;
        const uint32_t* db = sel ? r0 : r1;
        const uint32_t aa = slot + ra * 128u + (((uint32_t)lw ^ (ra & 7u)) << 4);
        const uint32_t ab = slot + rb * 128u + (((uint32_t)lw ^ (rb & 7u)) << 4);
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(aa), "r"(da[0]), "r"(da[1]), "r"(da[2]),
                     "r"(da[3])
                     : "memory");
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(ab), "r"(db[0]), "r"(db[1]), "r"(db[2]),
                     "r"(db[3])
                     : "memory");
      }
    }
  }
}

// Pair-aligned layout (W even, pitch = W + 2pw even, delta = pw & 1): every position pair
// (q, q+1), q even, is either two adjacent input elements (w, w+1) with w even or two zero
// coefficients, so a lane reads one aligned 4-byte (bf16) / 8-byte (fp32) word per channel,
// decodes its pair once, and repacks with byte permutes.  A zero pair (padding, separator
// rows, channels past C) reads the plan's zero buffer through the same channel stride, so no
// load is predicated and no value masked; kHW2 (the plane size in words, 0 = runtime) makes
// the eight channel loads one base register plus immediate offsets.
template <typename IoT, bool kTf32, int kHW2, uint32_t kRowB = 128>
__device__ __forceinline__ void hk_load_window_pairs(const HkParams& p, uint32_t slot, long long q0, int c0, int lw,
                                                     int lane, int rp_lo, int rp_hi) {
  constexpr bool kBf16In = sizeof(IoT) == 2;
  constexpr int CPG = kTf32 ? 4 : 8;          // channels per 16-byte group
  constexpr int B = kBf16In ? 4 : 2;          // position pairs per lane in flight
  const uint32_t hw2 = kHW2 ? (uint32_t)kHW2 : (uint32_t)p.HW >> 1;  // plane size in words / float2
  const int cg = c0 + lw * CPG;
  const int nrp = rp_hi;
  const uint32_t sel = (uint32_t)(lane >> 2) & 1u;
  const bool gz = cg >= p.C;  // group past C (warp-uniform); C % CPG == 0 for this loader
  const uint32_t cgo = gz ? 0u : (uint32_t)cg * hw2;
  for (int rp0 = rp_lo; rp0 < nrp; rp0 += 32 * B) {
    uint32_t lo[B][CPG], hi[B][kBf16In ? 1 : CPG];
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const int rp = rp0 + b * 32 + lane;
      const int e = (rp < nrp && !gz && !(p.dbg & 1)) ? hk_src(p, q0 + 2 * rp) : -1;
      if constexpr (kBf16In) {
        const uint32_t* base = e >= 0 ? static_cast<const uint32_t*>(p.x) + (((uint32_t)e >> 1) + cgo)
                                      : static_cast<const uint32_t*>(p.zero);
        if constexpr (kRowB == 32) {
          // small C (32-byte rows of 16 channels): channels past C read zeros, not x
#pragma unroll
          for (int c = 0; c < CPG; ++c) lo[b][c] = cg + c < p.C ? base[c * hw2] : 0u;
        } else {
#pragma unroll
          for (int c = 0; c < CPG; ++c) lo[b][c] = base[c * hw2];
        }
      } else {
        const float2* base = e >= 0 ? static_cast<const float2*>(p.x) + (((uint32_t)e >> 1) + cgo)
                                    : static_cast<const float2*>(p.zero);
#pragma unroll
        for (int c = 0; c < CPG; ++c) {
          const float2 v = __ldg(base + c * hw2);
          lo[b][c] = __float_as_uint(v.x);
          hi[b][c] = __float_as_uint(v.y);
        }
      }
    }
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const int rp = rp0 + b * 32 + lane;
      uint32_t r0[4], r1[4];
      if constexpr (kTf32) {
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          r0[c] = to_tf32_rna(__uint_as_float(lo[b][c]));  // reading R11: RNA
          r1[c] = to_tf32_rna(__uint_as_float(hi[b][c]));
        }
      } else if constexpr (kBf16In) {
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          r0[c] = __byte_perm(lo[b][2 * c], lo[b][2 * c + 1], 0x5410);
          r1[c] = __byte_perm(lo[b][2 * c], lo[b][2 * c + 1], 0x7632);
        }
      } else {
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const __nv_bfloat162 v0 = __floats2bfloat162_rn(__uint_as_float(lo[b][2 * c]),
                                                          __uint_as_float(lo[b][2 * c + 1]));  // R11: RNE
          const __nv_bfloat162 v1 = __floats2bfloat162_rn(__uint_as_float(hi[b][2 * c]),
                                                          __uint_as_float(hi[b][2 * c + 1]));
          r0[c] = *reinterpret_cast<const uint32_t*>(&v0);
          r1[c] = *reinterpret_cast<const uint32_t*>(&v1);
        }
      }
      if (rp < nrp) {
        const uint32_t ra = 2u * (uint32_t)rp + sel, rb = 2u * (uint32_t)rp + (sel ^ 1u);
        const uint32_t* da = sel ? r1 : r0;
        const uint32_t* db = sel ? r0 : r1;
        const uint32_t xa = kRowB == 128 ? (ra & 7u) : ((ra >> 2) & 1u);  // SW128 / SW32 chunk swizzle
        const uint32_t xb = kRowB == 128 ? (rb & 7u) : ((rb >> 2) & 1u);
        const uint32_t aa = slot + ra * kRowB + (((uint32_t)lw ^ xa) << 4);
        const uint32_t ab = slot + rb * kRowB + (((uint32_t)lw ^ xb) << 4);
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(aa), "r"(da[0]), "r"(da[1]), "r"(da[2]),
                     "r"(da[3])
                     : "memory");
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(ab), "r"(db[0]), "r"(db[1]), "r"(db[2]),
                     "r"(db[3])
                     : "memory");
      }
    }
  }
}

// Phase-split window (reading R19, stride 2, bf16 in and math, x width % 4 == 0, C % 32 == 0).
// The stride-2 convolution is the stride-1 convolution, with R' x S' taps, of the phase planes
// X_{a,c,b}[u][v] = x[c][2u + a][2v + b] (virtual channel (a*C + c)*2 + b); the window holds
// those planes' positions.  One aligned 4-byte word x[c][2u + a][2v .. 2v + 1] is virtual
// channels (a, c, 0) and (a, c, 1) of position (u, v), already in operand order, so a 16-byte
// row group (4 channels x 2 column phases) is 4 loads, no permutes.  Each position of a lane's
// pair is decoded on its own (any W' = W/2); rows 2u + a past x's last row read the zero buffer.
template <bool kAligned, uint32_t kRowB>
__device__ __forceinline__ void hk_load_window_phase(const HkParams& p, uint32_t slot, long long q0, int vc0, int lw,
                                                     int lane, int rp_lo, int rp_hi) {
  constexpr int B = 4;  // position pairs per lane in flight
  const uint32_t hw2 = (uint32_t)(p.xH * p.xW) >> 1, w2 = (uint32_t)p.xW >> 1;
  // this group's 4 (a, c) slots: virtual channels vc0 + 8 lw + 2k + {0, 1}; C % 32 == 0 keeps
  // a (and so the row offset) one per chunk, else (the stem, 4C <= 16) per slot, a >= 2 zero
  int sa[4], sc[4];
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int s2 = vc0 / 2 + lw * 4 + k;
    sa[k] = s2 / p.xC;
    sc[k] = s2 - sa[k] * p.xC;
  }
  const bool small_c = p.xC % 32 != 0;
  const int a = sa[0], c = sc[0];
  const int nrp = rp_hi;
  const uint32_t sel = (uint32_t)(lane >> 2) & 1u;
  for (int rp0 = rp_lo; rp0 < nrp; rp0 += 32 * B) {
    uint32_t lo[B][4], hi[B][4];
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const int rp = rp0 + b * 32 + lane;
      // (n, u, v) of the pair's first position in the phase planes, as hk_src
      // kAligned (W' even, pitch W' + 2pw', delta pw' & 1): both positions of a pair are data of
      // one row or both zero, one decode; else each position is decoded on its own
      const uint32_t* base[2];
      if (small_c) {
        // (the stem) every slot its own row phase and channel; W' even (aligned) assumed
        int n, u, v;
        const bool in = hk_pos(p, q0 + 2 * rp, n, u, v) && rp < nrp && !(p.dbg & 1);
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int r = 2 * u + sa[k];
          const uint32_t* bk = (in && sa[k] < 2 && r < p.xH)
                                   ? static_cast<const uint32_t*>(p.x) + (((uint32_t)n * p.xC + (uint32_t)sc[k]) * hw2 +
                                                                          (uint32_t)r * w2 + (uint32_t)v)
                                   : static_cast<const uint32_t*>(p.zero);
          lo[b][k] = bk[0];
          hi[b][k] = bk[1];
        }
        continue;
      }
#pragma unroll
      for (int s2 = 0; s2 < (kAligned ? 1 : 2); ++s2) {
        int n, u, v;
        const bool in = hk_pos(p, q0 + 2 * rp + s2, n, u, v) && rp < nrp && !(p.dbg & 1);
        const int r = 2 * u + a;
        base[s2] = (in && r < p.xH) ? static_cast<const uint32_t*>(p.x) +
                                          (((uint32_t)n * p.xC + (uint32_t)c) * hw2 + (uint32_t)r * w2 + (uint32_t)v)
                                    : static_cast<const uint32_t*>(p.zero);
      }
      if (kAligned) base[1] = base[0] + 1;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        lo[b][k] = base[0][k * hw2];
        hi[b][k] = base[1][k * hw2];
      }
    }
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const int rp = rp0 + b * 32 + lane;
      if (rp < nrp) {
        const uint32_t ra = 2u * (uint32_t)rp + sel, rb = 2u * (uint32_t)rp + (sel ^ 1u);
        const uint32_t* da = sel ? hi[b] : lo[b];
        const uint32_t* db = sel ? lo[b] : hi[b];
        // 16-B chunk ^= byte-address bits [7, 10) of the row: SW128 row & 7, SW64 (row >> 1) & 3,
        // SW32 (row >> 2) & 1
        const uint32_t xa = kRowB == 128 ? (ra & 7u) : kRowB == 64 ? ((ra >> 1) & 3u) : ((ra >> 2) & 1u);
        const uint32_t xb = kRowB == 128 ? (rb & 7u) : kRowB == 64 ? ((rb >> 1) & 3u) : ((rb >> 2) & 1u);
        const uint32_t aa = slot + ra * kRowB + (((uint32_t)lw ^ xa) << 4);
        const uint32_t ab = slot + rb * kRowB + (((uint32_t)lw ^ xb) << 4);
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(aa), "r"(da[0]), "r"(da[1]), "r"(da[2]),
                     "r"(da[3])
                     : "memory");
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(ab), "r"(db[0]), "r"(db[1]), "r"(db[2]),
                     "r"(db[3])
                     : "memory");
      }
    }
  }
}

// Plane-staged window (bf16 in and math, stride 1, C % 64 == 0; small planes such as 7x7,
// where the element loader above does two 4-byte loads per element): each window touches a few
// whole images, and one image's block of 64 channel planes is one contiguous, 16-byte aligned
// run of x (64*H*W*2 bytes), so the window forwarder bulk-copies those blocks into a staging
// buffer (two buffers, one window ahead) and the loader warps transpose from shared memory:
// 8 two-byte reads (one per channel of the warp's 16-byte group) per position, one 16-byte
// swizzled store per window row (zeros for padding rows / columns).
constexpr int kHkPlanes = -9;
// first image of the window at origin q0 (images before it hold no element of the window)
__device__ __forceinline__ int hk_window_img0(const HkParams& p, long long q0) {
  const long long qq = max(q0 - p.delta, 0LL);
  const int vr = (int)p.fpitch.div((uint32_t)qq) - p.ph;
  return vr < 0 ? 0 : (int)p.fHS.div((uint32_t)vr);
}
__device__ __forceinline__ void hk_planes_issue(const HkParams& p, long long q0, int c0, uint32_t stg, uint64_t* bar) {
  const int n0 = hk_window_img0(p, q0);
  const int nimg = max(0, min(p.pimg_max, p.N - n0));
  mbar_arrive_expect_tx(bar, (uint32_t)nimg * p.pimg_bytes);
  for (int i = 0; i < nimg; ++i) {
    const char* src = static_cast<const char*>(p.x) + ((long long)(n0 + i) * p.C + c0) * p.HW * 2;
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     stg + (uint32_t)i * p.pimg_bytes),
                 "l"(src), "r"(p.pimg_bytes), "r"(smem_u32(bar))
                 : "memory");
  }
}
__device__ __forceinline__ void hk_planes_transpose(const HkParams& p, long long q0, uint32_t stg, uint32_t slot,
                                                    int lw, int lane, int r_lo, int r_hi) {
  const int n0 = hk_window_img0(p, q0);
  for (int r = r_lo + lane; r < r_hi; r += 32) {
    int n, h, w;
    uint32_t d[4] = {0u, 0u, 0u, 0u};
    if (hk_pos(p, q0 + r, n, h, w) && n - n0 < p.pimg_max) {
      const uint32_t e = stg + (((uint32_t)(n - n0) * 64u + (uint32_t)lw * 8u) * (uint32_t)p.HW + (uint32_t)(h * p.W + w)) * 2u;
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        uint16_t lo, hi;
        asm volatile("ld.shared.u16 %0, [%1];" : "=h"(lo) : "r"(e + (uint32_t)(2 * c) * (uint32_t)p.HW * 2u));
        asm volatile("ld.shared.u16 %0, [%1];" : "=h"(hi) : "r"(e + (uint32_t)(2 * c + 1) * (uint32_t)p.HW * 2u));
        d[c] = (uint32_t)lo | ((uint32_t)hi << 16);
      }
    }
    const uint32_t a = slot + (uint32_t)r * 128u + ((((uint32_t)lw) ^ ((uint32_t)r & 7u)) << 4);
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(d[0]), "r"(d[1]), "r"(d[2]), "r"(d[3])
                 : "memory");
  }
}

// ---- a5: one accumulator tile to NCHW y -------------------------------------------------
template <typename IoT>
__device__ __forceinline__ void hk_store(IoT* y, long long i, float v);
template <>
__device__ __forceinline__ void hk_store<float>(float* y, long long i, float v) {
  y[i] = v;
}
template <>
__device__ __forceinline__ void hk_store<__nv_bfloat16>(__nv_bfloat16* y, long long i, float v) {
  y[i] = __float2bfloat16_rn(v);
}

// kScatter: the epilogue stores to every buffer of p.ys at channel offset p.koff of p.Ktot
// (polyconv_forward_scatter); the plain forward (one output, its own channels) keeps the single
// store path (a runtime output loop there cost up to 4 us per ResNet-50 layer, same-box A/B)
// kRowTile (the stem): pitch 128 makes every 128-position tile one output row; the epilogue
// stages the tile's NN channel rows (Q pixels each) in shared memory and one thread writes them
// with a TMA tensor store (y as [N*K][P][Q]) instead of 2-byte stores (the stem was bound by
// its epilogue stores)
template <typename IoT, bool kTf32, int kHW2, int kKC = (kTf32 ? 32 : 64), bool kScatter = false,
          bool kRowTile = false>
__global__ void __launch_bounds__(kHkThreads, 1)
    mac_hankel_kernel(const __grid_constant__ CUtensorMap tmU, const __grid_constant__ CUtensorMap tmY,
                      const HkParams p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  const uint32_t sF = smem_u32(smem);                                   // filter blocks
  const uint32_t sW = sF + (uint32_t)p.fslots * p.fblk_bytes;           // window ring (1 KB aligned)
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + (size_t)p.fslots * p.fblk_bytes +
                                               (size_t)p.wslots * p.wslot_bytes +
                                               (kHW2 == kHkPlanes ? (size_t)p.psbufs * p.pimg_max * p.pimg_bytes : 0) +
                                               (kRowTile ? 2 * (size_t)p.rt_stage : 0));
  const uint32_t sY = sW + (uint32_t)p.wslots * p.wslot_bytes;  // kRowTile: two staged output tiles
  uint64_t* ffull = bars;                    // [kHkMaxFBlk] leader: both halves landed
  uint64_t* fempty = ffull + kHkMaxFBlk;     // [kHkMaxFBlk] both: MMAs done with the block
  uint64_t* wfull = fempty + kHkMaxFBlk;     // [kHkMaxWSlots] leader: both CTAs' loaders done
  uint64_t* wempty = wfull + kHkMaxWSlots;   // [kHkMaxWSlots] both: MMAs done with the window
  uint64_t* tfull = wempty + kHkMaxWSlots;   // [2] both: accumulator ready
  uint64_t* tempty = tfull + 2;              // [2] leader: both CTAs' epilogues drained it
  // The 8 loader (epilogue) warps of a CTA arrive on a local barrier (CTA-scope release), and
  // one forwarder warp per CTA passes it on to the leader with a single cluster-scope arrive:
  // sixteen cluster-scope releases per window stalled every loader warp on a memory barrier
  // (ncu: ERRBAR / membar was the loaders' largest stall after the loads themselves).
  uint64_t* wloc = tempty + 2;               // [kHkMaxWSlots] this CTA's loaders done
  uint64_t* eloc = wloc + kHkMaxWSlots;      // [2] this CTA's epilogue warps drained
  uint64_t* sfull = eloc + 2;                // [2] plane-staged loader: a window's blocks landed
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(sfull + 2);
  const uint32_t sS = sW + (uint32_t)p.wslots * p.wslot_bytes;  // plane-staged loader: 2 staging buffers

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // window / filter rows: kKC channels of 128 B (SW128) or, for the small-C phase convolution
  // (the stem, 4C <= 16 virtual channels), 16 bf16 channels of 32 B (SW32)
  constexpr uint32_t kRowB = kTf32 ? 4u * kKC : 2u * kKC;
  constexpr uint32_t kRow16 = kRowB / 16u;  // 16-byte units per row
  constexpr int kKSteps = (int)kRowB / 32;   // MMA K steps (32 bytes each) per row
  const uint32_t rank = cluster_ctarank();
  const int pair = (int)(blockIdx.x >> 1);
  const long long U = (long long)p.PT * p.NB;
  const long long u_lo = U * pair / p.npairs, u_hi = U * (pair + 1) / p.npairs;

  const bool trace = (p.dbg & 8) && blockIdx.x < 160;
  unsigned long long* tr = g_hk_trace + blockIdx.x * 16;
  if (trace && threadIdx.x == 0) tr[0] = global_ns();
  if (threadIdx.x == 0) {
    prefetch_tmap(&tmU);
    for (int i = 0; i < kHkMaxFBlk; ++i) {
      mbar_init(ffull + i, 1);
      mbar_init(fempty + i, 1);
    }
    for (int i = 0; i < kHkMaxWSlots; ++i) {
      mbar_init(wfull + i, 2);
      mbar_init(wempty + i, 1);
      mbar_init(wloc + i, kHkLoadWarps);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(tfull + i, 1);
      mbar_init(tempty + i, 2);
      mbar_init(eloc + i, kHkEpiWarps);
      mbar_init(sfull + i, 1);
    }
    fence_barrier_init();
  }
  int ridx = 0;
  const int role = hk_role(warp, ridx);
  if (role == kRoleMma) hk_tmem_alloc2(tmem_slot, (uint32_t)p.tmem_cols);
  tc_fence_before();
  cluster_sync();  // barriers of both CTAs initialised, TMEM allocated in both
  tc_fence_after();
  if (trace && threadIdx.x == 0) tr[1] = global_ns();

  if (role == kRoleProducer) {
    // ---- filter producer (a3 output, packed by the preceding launch) ----
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const uint32_t ffull0 = hk_mapa0(smem_u32(ffull));
    long long u = u_lo;
    HkItem it;
    int fs = 0, fuse = 0;  // ring slot, ring lap
    bool first = true;
    while (hk_next(p, u, u_hi, it)) {
      if (!(p.resident && !first)) {
        for (int ch = 0; ch < p.nchunks; ++ch)
          for (int tap = 0; tap < p.RS; ++tap) {
            if (!p.resident) hk_wait(fempty + fs, (uint32_t)(fuse & 1) ^ 1u);
            if (elect_one()) {
              const uint32_t bar = ffull0 + (uint32_t)fs * 8u;
              if (rank == 0) mbar_arrive_expect_tx(ffull + fs, 2u * p.fblk_bytes);
              const int row = tap * p.Kp + it.nb * p.NN + (int)rank * (p.NN / 2);
              hk_tma_pair(sF + (uint32_t)fs * p.fblk_bytes, &tmU, bar, ch * kKC, row);
            }
            __syncwarp();
            if (++fs == p.fslots) { fs = 0; ++fuse; }
          }
      }
      first = false;
    }
  } else if (role == kRoleMma) {
    // ---- MMA issuer (leader CTA; the whole warp runs the loop, one lane issues) ----
    if (rank == 0) {
      const uint32_t tbase = *tmem_slot;
      long long u = u_lo;
      HkItem it;
      int fs = 0, fuse = 0, ws = 0, wuse = 0, item = 0;
      bool first = true;
      const uint32_t row16 = (uint32_t)p.pitch * kRow16;  // one kernel row of taps = pitch window rows, 16-B units
      while (hk_next(p, u, u_hi, it)) {
        const int a = p.nacc == 2 ? (item & 1) : 0;
        hk_wait(tempty + a, (uint32_t)((item / p.nacc) & 1) ^ 1u);
        tc_fence_after();
        const uint32_t dacc = tbase + (uint32_t)(a * p.T * p.NN);
        int fb = 0;  // resident: block index
        for (int ch = 0; ch < p.nchunks; ++ch) {
          hk_wait(wfull + ws, (uint32_t)(wuse & 1));
          tc_fence_after();
          const int wi = (int)(wuse * p.wslots + ws);
          const bool wt = (p.dbg & 16) && blockIdx.x == 0 && lane == 0 && wi < 64;
          if (wt) g_hk_wtrace[wi * 8 + 3] = global_ns();
          // descriptors: window row r of tap (i, j) = t*128 + pitch*i + j (the Hankel shift);
          // +1024 16-B units per 128-row tile, +2 per 32-byte K step
          const uint64_t awin = make_sdesc(sW + (uint32_t)ws * p.wslot_bytes, kRowB, 0);
          uint32_t rowoff = 0;
          int j = 0;
          for (int tap = 0; tap < p.RS; ++tap) {
            const int slot = p.resident ? fb : fs;
            if (!p.resident || first) {
              hk_wait(ffull + slot, p.resident ? 0u : (uint32_t)(fuse & 1));
              tc_fence_after();
              if (trace && lane == 0 && item == 0 && ch == 0 && tap == 0) tr[3] = global_ns();
            }
            const uint64_t bd = make_sdesc(sF + (uint32_t)slot * p.fblk_bytes, kRowB, 0);
            const uint64_t ad = awin + rowoff + (uint32_t)j * kRow16;
            const uint32_t acc0 = (ch | tap) != 0 ? 1u : 0u;
            if (!(p.dbg & 4) && elect_one()) {
              for (int t = 0; t < it.T; ++t) {
                const uint64_t at = ad + (uint64_t)(t * 128 * kRow16);
                const uint32_t d = dacc + (uint32_t)(t * p.NN);
                hk_mma<kTf32>(d, at, bd, p.idesc, acc0);
#pragma unroll
                for (int k = 1; k < kKSteps; ++k) hk_mma<kTf32>(d, at + 2 * k, bd + 2 * k, p.idesc, 1u);
              }
            }
            __syncwarp();
            if (++j == p.S) { j = 0; rowoff += row16; }
            if (!p.resident) {
              if (elect_one()) hk_commit_both(fempty + fs);
              __syncwarp();
              if (++fs == p.fslots) { fs = 0; ++fuse; }
            } else {
              ++fb;
            }
          }
          if (elect_one()) hk_commit_both(wempty + ws);
          __syncwarp();
          if (wt) g_hk_wtrace[wi * 8 + 4] = global_ns();
          if (++ws == p.wslots) { ws = 0; ++wuse; }
        }
        if (elect_one()) hk_commit_both(tfull + a);
        __syncwarp();
        if (trace && lane == 0) tr[item == 0 ? 4 : 6] = global_ns();
        first = false;
        ++item;
      }
    }
  } else if (role == kRoleLoader) {
    // ---- window loaders (a2) ----
    // 16-byte column group of every row this warp converts, and its slice of the row pairs
    // (128-B rows: 8 groups x 2 halves; 32-B rows: 2 groups x 8 slices; split on 32 pairs)
    constexpr int kGroups = (int)kRow16;
    constexpr int kSlices = kHkLoadWarps / kGroups;
    const int lw = ridx % kGroups, sl = ridx / kGroups;
    const int nrp_all = p.wrows >> 1;
    const int per = ((nrp_all + kSlices - 1) / kSlices + 31) / 32 * 32;
    const int rp_lo = min(sl * per, nrp_all), rp_hi = min((sl + 1) * per, nrp_all);
    if constexpr (kHW2 == kHkPlanes) {
      long long u = u_lo;
      HkItem it;
      int ws = 0, wuse = 0, sb = 0, suse = 0;
      while (hk_next(p, u, u_hi, it)) {
        const long long q0 = (long long)it.pt * 256 + (long long)rank * 128 * it.T;
        for (int ch = 0; ch < p.nchunks; ++ch) {
          hk_wait(wempty + ws, (uint32_t)(wuse & 1) ^ 1u);
          hk_wait(sfull + sb, (uint32_t)(suse & 1));
          if (!(p.dbg & 1))
            hk_planes_transpose(p, q0, sS + (uint32_t)sb * (uint32_t)p.pimg_max * p.pimg_bytes,
                                sW + (uint32_t)ws * p.wslot_bytes, lw, lane, 2 * rp_lo, 2 * rp_hi);
          if (++sb == p.psbufs) { sb = 0; ++suse; }
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> MMA reads
          __syncwarp();
          if (lane == 0) mbar_arrive(wloc + ws);
          if (++ws == p.wslots) { ws = 0; ++wuse; }
        }
      }
    } else {
      long long u = u_lo;
      HkItem it;
      int ws = 0, wuse = 0;
      while (hk_next(p, u, u_hi, it)) {
        const long long q0 = (long long)it.pt * 256 + (long long)rank * 128 * it.T;
        for (int ch = 0; ch < p.nchunks; ++ch) {
          const int wi = (int)(wuse * p.wslots + ws);
          const bool wt = (p.dbg & 16) && blockIdx.x == 0 && ridx == 0 && lane == 0 && wi < 64;
          if (wt) g_hk_wtrace[wi * 8 + 0] = global_ns();
          hk_wait(wempty + ws, (uint32_t)(wuse & 1) ^ 1u);
          if (wt) g_hk_wtrace[wi * 8 + 1] = global_ns();
          if constexpr (kHW2 == -2 || kHW2 == -4)
            hk_load_window_phase<kHW2 == -2, kRowB>(p, sW + (uint32_t)ws * p.wslot_bytes, q0, ch * kKC, lw, lane,
                                                    rp_lo, rp_hi);
          else if constexpr (kHW2 >= 0)
            hk_load_window_pairs<IoT, kTf32, kHW2, kRowB>(p, sW + (uint32_t)ws * p.wslot_bytes, q0, ch * kKC, lw,
                                                   lane, rp_lo, rp_hi);
          else
            hk_load_window<IoT, kTf32>(p, sW + (uint32_t)ws * p.wslot_bytes, q0, ch * (kTf32 ? 32 : 64), lw, lane,
                                       rp_lo, rp_hi);
          if (trace && lw == 0 && lane == 0 && u == u_lo + it.T && ch == 0) tr[2] = global_ns();
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> MMA reads
          __syncwarp();
          if (wt) g_hk_wtrace[wi * 8 + 2] = global_ns();
          if ((p.dbg & 32) && blockIdx.x < 2 && lane == 0 && wi < 64) g_hk_ltrace[wi * 16 + rank * 8 + lw] = global_ns();
          if (lane == 0) mbar_arrive(wloc + ws);
          if (++ws == p.wslots) { ws = 0; ++wuse; }
        }
      }
    }
  } else if (role == kRoleFwdW) {
    // ---- forwarder: this CTA's window stored -> the leader's wfull ----
    const uint32_t wfull0 = hk_mapa0(smem_u32(wfull));
    long long u = u_lo;
    HkItem it;
    int ws = 0, wuse = 0;
    if constexpr (kHW2 == kHkPlanes) {
      // plane-staged loader: window w's blocks go to staging buffer w % psbufs; window
      // w + psbufs's are fetched once the loaders are done with window w (= this window stored)
      long long ua = u_lo;
      HkItem ita;
      bool hava = hk_next(p, ua, u_hi, ita);
      int cha = 0, sb = 0;
      auto issue = [&]() {
        if (lane == 0)
          hk_planes_issue(p, (long long)ita.pt * 256 + (long long)rank * 128 * ita.T, cha * kKC,
                          sS + (uint32_t)sb * (uint32_t)p.pimg_max * p.pimg_bytes, sfull + sb);
        __syncwarp();
        if (++sb == p.psbufs) sb = 0;
        if (++cha == p.nchunks) { cha = 0; hava = hk_next(p, ua, u_hi, ita); }
      };
      for (int k = 0; k < p.psbufs && hava; ++k) issue();
      while (hk_next(p, u, u_hi, it)) {
        for (int ch = 0; ch < p.nchunks; ++ch) {
          hk_wait(wloc + ws, (uint32_t)(wuse & 1));
          if (lane == 0) hk_arrive_cluster(wfull0 + (uint32_t)ws * 8u);
          __syncwarp();
          if (++ws == p.wslots) { ws = 0; ++wuse; }
          if (hava) issue();
        }
      }
    } else {
      while (hk_next(p, u, u_hi, it)) {
        for (int ch = 0; ch < p.nchunks; ++ch) {
          hk_wait(wloc + ws, (uint32_t)(wuse & 1));
          if (lane == 0) hk_arrive_cluster(wfull0 + (uint32_t)ws * 8u);
          __syncwarp();
          if (++ws == p.wslots) { ws = 0; ++wuse; }
        }
      }
    }
  } else if (role == kRoleFwdE) {
    // ---- forwarder: this CTA's epilogue drained an accumulator -> the leader's tempty ----
    const uint32_t tempty0 = hk_mapa0(smem_u32(tempty));
    long long u = u_lo;
    HkItem it;
    int item = 0;
    while (hk_next(p, u, u_hi, it)) {
      const int a = p.nacc == 2 ? (item & 1) : 0;
      hk_wait(eloc + a, (uint32_t)((item / p.nacc) & 1));
      if (lane == 0) hk_arrive_cluster(tempty0 + (uint32_t)a * 8u);
      __syncwarp();
      ++item;
    }
  } else if (role == kRoleEpi) {
    // ---- epilogue (a5) ----
    const int e = ridx;
    const int quad = warp & 3;      // TMEM lane quadrant this warp may access
    const int half = e & 1;         // column groups half, half + 2, ...
    const uint32_t tbase = *tmem_slot;
    IoT* y = static_cast<IoT*>(p.ys[0]);
    const long long PQ = (long long)p.P * p.Q;
    // plane size of y as a compile-time constant when the output has the input's size
    const bool pq_const = kHW2 > 0 && PQ == 2LL * kHW2;
    long long u = u_lo;
    HkItem it;
    int item = 0, rt_buf = 0;
    while (hk_next(p, u, u_hi, it)) {
      const int a = p.nacc == 2 ? (item & 1) : 0;
      hk_wait(tfull + a, (uint32_t)((item / p.nacc) & 1));
      tc_fence_after();
      if (trace && e == 0 && lane == 0) tr[item == 0 ? 9 : 10] = global_ns();
      if constexpr (kRowTile) {
        // tile t = output row (n, oh) of the item's block of NN channels; lanes = pixels ow
        for (int t = 0; t < it.T; ++t) {
          const long long qt = (long long)it.pt * 256 + (long long)rank * 128 * it.T + t * 128;
          const uint32_t vr = (uint32_t)(qt >> 7);
          const uint32_t n = p.fHS.div(vr), oh = vr - n * (uint32_t)p.HS;
          const bool row_ok = (int)n < p.N && (int)oh < p.P;
          const uint32_t stg = sY + (uint32_t)(rt_buf & 1) * p.rt_stage;
          if (e == 0 && lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");  // buffer free
          asm volatile("bar.sync 1, %0;" ::"n"(32 * kHkEpiWarps) : "memory");
          const int ow = quad * 32 + lane;
          const uint32_t trow = tbase + ((uint32_t)(quad * 32) << 16) + (uint32_t)(a * p.T * p.NN + t * p.NN);
          for (int g = half; g * 16 < p.NN; g += 2) {
            uint32_t v[16];
            hk_tmem_ld16(trow + (uint32_t)(g * 16), v);
            tmem_ld_wait();
            if (row_ok && ow < p.Q && !(p.dbg & 2)) {
#pragma unroll
              for (int c = 0; c < 16; ++c) {
                const uint32_t ad = stg + ((uint32_t)(g * 16 + c) * (uint32_t)p.Q + (uint32_t)ow) * 2u;
                const unsigned short h = __bfloat16_as_ushort(__float2bfloat16_rn(__uint_as_float(v[c])));
                asm volatile("st.shared.u16 [%0], %1;" ::"r"(ad), "h"(h) : "memory");
              }
            }
          }
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          asm volatile("bar.sync 1, %0;" ::"n"(32 * kHkEpiWarps) : "memory");
          if (e == 0 && lane == 0 && row_ok && !(p.dbg & 2)) {
            const int c2 = (int)n * p.K + it.nb * p.NN;
            asm volatile(
                "cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                    reinterpret_cast<uint64_t>(&tmY)),
                "r"(stg), "r"(0), "r"((int)oh), "r"(c2)
                : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
          }
          ++rt_buf;
        }
      } else
      for (int t = 0; t < it.T; ++t) {
        // position of this lane -> output pixel (Eq. 12 / reading R4 / R16)
        const long long q = (long long)it.pt * 256 + (long long)rank * 128 * it.T + t * 128 + quad * 32 + lane;
        const long long qq = q - p.delta;
        long long ybase = -1;
        if (qq >= 0 && qq < (1LL << 31)) {
          const uint32_t uq = (uint32_t)qq;
          const uint32_t vr = p.fpitch.div(uq);
          const uint32_t col = uq - vr * (uint32_t)p.pitch;
          const uint32_t n = p.fHS.div(vr);
          const uint32_t ohs = vr - n * (uint32_t)p.HS;
          const uint32_t oh = p.fsh.div(ohs), ow = p.fsw.div(col);
          if ((int)n < p.N && oh * (uint32_t)p.sh == ohs && ow * (uint32_t)p.sw == col && (int)oh < p.P &&
              (int)ow < p.Q)
            ybase = kScatter ? ((long long)n * p.Ktot + p.koff + it.nb * p.NN) * PQ + (long long)oh * p.Q + ow
                             : ((long long)n * p.K + it.nb * p.NN) * PQ + (long long)oh * p.Q + ow;
        }
        const uint32_t trow = tbase + ((uint32_t)(quad * 32) << 16) + (uint32_t)(a * p.T * p.NN + t * p.NN);
        for (int g = half; g * 16 < p.NN; g += 2) {
          uint32_t v[16];
          if (!(p.dbg & 512)) {
            hk_tmem_ld16(trow + (uint32_t)(g * 16), v);
            tmem_ld_wait();
          } else {
#pragma unroll
            for (int c = 0; c < 16; ++c) v[c] = 0u;
          }
          if (ybase >= 0 && !(p.dbg & 2)) {
            const int kleft = p.K - (it.nb * p.NN + g * 16);  // output channels left (warp-uniform)
            if constexpr (kScatter) {
              // every output buffer (f4: the K-shard all-gather as peer stores over NVLink)
              for (int o = 0; o < p.nys; ++o) {
                IoT* yp = static_cast<IoT*>(p.ys[o]) + ybase + (long long)(g * 16) * PQ;
#pragma unroll
                for (int c = 0; c < 16; ++c)
                  if (c < kleft) hk_store<IoT>(yp, (long long)c * PQ, __uint_as_float(v[c]));
              }
            } else {
              IoT* yp = y + ybase + (long long)(g * 16) * PQ;
              if (kHW2 > 0 && pq_const && kleft >= 16) {
                // same-size output with a baked-in plane size: one base register, immediate offsets
#pragma unroll
                for (int c = 0; c < 16; ++c)
                  hk_store<IoT>(yp, (long long)c * (2 * (kHW2 > 0 ? kHW2 : 1)), __uint_as_float(v[c]));
              } else {
#pragma unroll
                for (int c = 0; c < 16; ++c)
                  if (c < kleft) hk_store<IoT>(yp, (long long)c * PQ, __uint_as_float(v[c]));
              }
            }
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(eloc + a);
      if (trace && e == 0 && lane == 0) tr[item == 0 ? 5 : 7] = global_ns();
      ++item;
    }
    (void)rt_buf;
    if (kRowTile && e == 0 && lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  // teardown: every role done in both CTAs (remote arrivals land before the peer exits)
  tc_fence_before();
  __syncthreads();
  cluster_sync();
  if (role == kRoleMma) {
    tc_fence_after();
    hk_tmem_dealloc2(*tmem_slot, (uint32_t)p.tmem_cols);
  }
  if (trace && threadIdx.x == 0) tr[8] = global_ns();
}

// ---- host side ----------------------------------------------------------------------
typedef CUresult (*EncodeTiledFnHk)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFnHk get_encode_hk() {
  static EncodeTiledFnHk fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFnHk>(f);
  }
  return fn;
}

int env_int(const char* name, int dflt) {
  const char* v = getenv(name);
  return v ? atoi(v) : dflt;
}

}  // namespace

size_t hankel_zero_bytes(const Geom& g) { return (size_t)32 * g.H * g.W + 256; }

// Tiling.  NN (MMA N) = all output channels when K <= 256 (every window built once), else
// blocks of 256; T = the most 128-position tiles per CTA whose accumulators fit TMEM twice
// (T*NN <= 256): the T tiles share each filter block and each window's halo rows.  Measured at
// N=256 (tools/hk_trace.py with POLYCONV_HK_NN / POLYCONV_HK_T; TFLOP/s): 256->256 14x14
// NN=256/T=1 750 vs NN=128/T=2 713; 512->512 7x7 NN=256/T=1 596 vs NN=128/T=2 416 (fewer
// window rebuilds per output-channel block); 128->128 28x28 NN=128/T=2 862.
// The filter is resident in shared memory when its (single) block fits beside two windows,
// else streamed by TMA through a ring of (chunk, tap) blocks.
// kc16: 32-byte rows of 16 bf16 channels (SW32) for the small-C phase convolution (the stem)
static HankelTiling hankel_tiling_core(const Geom& g, int fmt, int num_sms, int kc_small = 0, int planes = 0,
                                       int force_pitch = 0, uint32_t extra_smem = 0, bool force_res = false) {
  HankelTiling t{};
  t.ok = false;
  if (fmt == FMT_F32) return t;
  const bool tf32 = fmt == FMT_TF32;
  if (kc_small && tf32) return t;
  const int eb = tf32 ? 4 : 2, kc = kc_small ? kc_small : 128 / eb;
  const uint32_t rowb = (uint32_t)(kc * eb);
  // row pitch: the paper's Wp = W + 2pw (even for even W, so position pairs are input
  // pairs), or W + pw (shared column padding, reading R16) for odd W;
  // POLYCONV_HK_PITCH=1 / 2 forces W + pw / W + 2pw
  const int mode = env_int("POLYCONV_HK_PITCH", 0);
  const bool shared_cols = mode == 1 || (mode == 0 && (g.W & 1));
  const int pitch = force_pitch ? force_pitch : std::max(shared_cols ? g.W + g.pw : g.W + 2 * g.pw, g.S);
  const int HS = g.H + g.ph;
  const int delta = (!(pitch & 1) && (g.pw & 1)) ? 1 : 0;
  const long long q_last = ((long long)(g.N - 1) * HS + (long long)g.sh * (g.P - 1)) * pitch +
                           (long long)g.sw * (g.Q - 1) + delta;
  const long long extent = q_last + 1 + 256LL * 8 + (long long)(g.R - 1) * pitch + g.S;
  if (extent >= (1LL << 31) || (long long)g.N * g.C * g.H * g.W >= (1LL << 31) ||
      (long long)g.N * g.K * g.P * g.Q >= (1LL << 31))
    return t;
  const int PT = (int)((q_last + 1 + 255) / 256);
  const int Cp = (g.C + kc - 1) / kc * kc, nchunks = Cp / kc, RS = g.R * g.S;
  const int K16 = (g.K + 15) / 16 * 16;
  const int forceT = env_int("POLYCONV_HK_T", 0), forceNN = env_int("POLYCONV_HK_NN", 0);
  const bool no_res = env_int("POLYCONV_HK_STREAM", 0) != 0;
  const int acc1_mode = env_int("POLYCONV_HK_ACC1", -1);
  const int max_pairs = std::max(1, num_sms / 2);
  const uint32_t fixed0 = 3072 + extra_smem;  // alignment + barriers (+ kRowTile staging)
  int NN = forceNN ? forceNN : (K16 <= 256 ? K16 : 256);
  bool found = false;
  for (int T = 4; T >= 1 && !found; T >>= 1) {
    // T*NN <= 256: two accumulator buffers, the epilogue overlapping the next item's MMAs.
    // NN = 256 with a streamed filter: T = 2 in one buffer (all 512 TMEM columns) halves the
    // filter blocks streamed per MAC, worth more than the overlap (256->256 14x14: 731 -> 792
    // TFLOP/s; VGG 512->512 28x28 N=64: 1139 -> 1306; 512->512 7x7: 635 -> 649; tools/hk_acc1.sh).
    // POLYCONV_HK_ACC1 = 0 / 1 forces it off / on.
    const bool acc1 = acc1_mode == 1 || (acc1_mode < 0 && NN == 256);
    if ((forceT && T != forceT) || T * NN > (acc1 ? 512 : 256)) continue;
    const int NB = (g.K + NN - 1) / NN;
    if ((long long)RS * NB * NN >= (1LL << 31)) break;
    const uint32_t fblk = (uint32_t)(NN / 2) * rowb;
    const int nblk = nchunks * RS;
    const int wrows = (128 * T + (g.R - 1) * pitch + g.S - 1 + 7) / 8 * 8;
    const uint32_t wslot = (uint32_t)wrows * rowb;
    // plane-staged loader: two staging buffers of the images a window touches
    const int pimg_max = planes ? (wrows + HS * pitch - 1) / (HS * pitch) + 1 : 0;
    const uint32_t pimg_bytes = (uint32_t)(64 * g.H * g.W * 2);
    const uint32_t fixed = fixed0 + (uint32_t)planes * (uint32_t)pimg_max * pimg_bytes;  // planes = staging buffers
    bool resident = false;
    int wslots = 0, fslots = 0;
    // Resident only when streaming would re-read more filter bytes per window than the window
    // itself holds: otherwise a short filter ring leaves shared memory to L1, which the window
    // loaders' global loads hit (tools/hk_slots.sh: 64->64 56x56 resident 583 vs streamed 650
    // TFLOP/s; 128->128 28x28 resident 862 vs streamed 838).
    const bool want_res = (size_t)nblk * fblk > wslot || force_res || env_int("POLYCONV_HK_RESIDENT", 0) != 0;
    if (NB == 1 && nblk <= kHkMaxFBlk && !no_res && want_res &&
        (size_t)nblk * fblk + 2 * wslot + fixed <= (size_t)kHkSmemMax) {
      resident = true;
      fslots = nblk;
      wslots = (int)std::min<size_t>(kHkMaxWSlots, (kHkSmemMax - fixed - (size_t)nblk * fblk) / wslot);
    } else {
      if (2 * wslot + fixed + (size_t)4 * fblk > (size_t)kHkSmemMax) continue;
      // three window slots and a four-block filter ring (512->512 7x7: 596 -> 649 TFLOP/s,
      // 256->256 14x14: 731 -> 770); POLYCONV_HK_WSLOTS / _FSLOTS override
      wslots = std::max(2, std::min(kHkMaxWSlots, env_int("POLYCONV_HK_WSLOTS", 3)));
      while (wslots > 2 && (size_t)wslots * wslot + fixed + (size_t)4 * fblk > (size_t)kHkSmemMax) --wslots;
      fslots = (int)std::min<size_t>(kHkMaxFBlk, (kHkSmemMax - fixed - (size_t)wslots * wslot) / fblk);
      fslots = std::min(fslots, nblk);
      const int fcap = env_int("POLYCONV_HK_FSLOTS", 4);
      if (fcap > 0) fslots = std::max(std::min(4, fslots), std::min(fslots, fcap));
    }
    if (wslots < 2) continue;
    found = true;
    t.NN = NN; t.NB = NB; t.T = T; t.wrows = wrows; t.wslot_bytes = wslot; t.wslots = wslots;
    t.planes = planes; t.pimg_max = pimg_max; t.pimg_bytes = pimg_bytes;
    t.resident = resident ? 1 : 0; t.fslots = fslots; t.fblk_bytes = fblk;
    t.npairs = (int)std::min<long long>(max_pairs, (long long)PT * NB);
  }
  if (!found) return t;
  t.pitch = pitch; t.HS = HS; t.delta = delta; t.PT = PT; t.Cp = Cp; t.nchunks = nchunks; t.kc = kc;
  // pair-aligned loader: every position pair is one aligned input pair or zeros
  t.aligned = (!(g.W & 1) && pitch == g.W + 2 * g.pw && delta == (g.pw & 1) && g.C % (tf32 ? 4 : 8) == 0 &&
               env_int("POLYCONV_HK_GENERAL", 0) == 0) ? 1 : 0;
  t.Kp = t.NB * t.NN;
  t.smem_bytes = (int)((size_t)t.fslots * t.fblk_bytes + (size_t)t.wslots * t.wslot_bytes + fixed0 +
                       (size_t)t.planes * t.pimg_max * t.pimg_bytes);
  t.nacc = t.T * t.NN > 256 ? 1 : 2;
  const int tc = t.nacc * t.T * t.NN;
  t.tmem_cols = tc <= 32 ? 32 : tc <= 64 ? 64 : tc <= 128 ? 128 : tc <= 256 ? 256 : 512;
  t.grid = 2 * t.npairs;
  t.ok = true;
  if (env_int("POLYCONV_HK_VERBOSE", 0))
    fprintf(stderr, "mac_hankel tiling: NN=%d NB=%d T=%d wrows=%d wslots=%d fslots=%d resident=%d smem=%d\n", t.NN,
            t.NB, t.T, t.wrows, t.wslots, t.fslots, t.resident, t.smem_bytes);
  return t;
}

// Stride-2 phase split (reading R19): y = the stride-1 convolution of the phase planes
// X_{a,c,b}[u][v] = x[c][2u + a][2v + b] (4C channels, ceil(H/2) x W/2) with R' x S' taps,
// R' = (R - 1 - ph)/2 + ceil(ph/2) + 1, top / left padding ceil(ph/2); same P x Q outputs.
static Geom hk_phase_geom(const Geom& g) {
  Geom e = g;
  e.C = 4 * g.C;
  e.H = (g.H + 1) / 2;
  e.W = g.W / 2;
  e.ph = (g.ph + 1) / 2;
  e.pw = (g.pw + 1) / 2;
  e.R = (g.R - 1 - g.ph) / 2 + e.ph + 1;
  e.S = (g.S - 1 - g.pw) / 2 + e.pw + 1;
  e.sh = e.sw = 1;
  return e;
}

// Every output position computed by the stride-1 window is kept in phase mode; without it a
// stride-2 layer computes all stride-1 positions and keeps a quarter.  Phase mode: bf16 in and
// math, even x width (x[2v], x[2v+1] one aligned word), C % 32 == 0 (a 64-channel chunk never
// straddles the row phase a), R - 1 >= ph; POLYCONV_HK_PHASE=0 turns it off.
HankelTiling hankel_tiling(const Geom& g, int fmt, int num_sms, bool io_bf16) {
  if (g.sh == 2 && g.sw == 2 && fmt == FMT_BF16 && io_bf16 && g.W % 2 == 0 && (g.C % 32 == 0 || g.C <= 4) &&
      g.R - 1 >= g.ph && g.S - 1 >= g.pw && env_int("POLYCONV_HK_PHASE", 1) != 0) {
    const Geom e = hk_phase_geom(g);
    if (e.C <= 16 && e.W + 2 * e.pw <= 128 && e.pw % 2 == 0 && (g.Q * 2) % 16 == 0 && g.K <= 256 &&
        env_int("POLYCONV_HK_ROWTILE", 1) != 0) {
      // the stem: one output row per 128-position tile, TMA-stored epilogue (kRowTile)
      const int NNr = (g.K + 15) / 16 * 16;
      HankelTiling t = hankel_tiling_core(e, fmt, num_sms, 16, 0, 128, 2u * (uint32_t)(NNr * g.Q * 2), true);
      if (t.ok && t.NN == g.K && t.delta == 0) {
        t.phase = 1;
        t.rowtile = 1;
        t.aligned = (e.W % 2 == 0 && t.delta == (e.pw & 1)) ? 1 : 0;
        t.eC = e.C; t.eH = e.H; t.eW = e.W; t.eR = e.R; t.eS = e.S; t.eph = e.ph; t.epw = e.pw;
        if (t.aligned) return t;
      }
    }
    HankelTiling t = hankel_tiling_core(e, fmt, num_sms, e.C <= 16 ? env_int("POLYCONV_HK_KC", 16) : 0);
    if (t.ok) {
      t.phase = 1;
      // position pairs of the phase planes are both data of one row or both zero
      t.aligned = (e.W % 2 == 0 && t.pitch == e.W + 2 * e.pw && t.delta == (e.pw & 1)) ? 1 : 0;
      t.eC = e.C; t.eH = e.H; t.eW = e.W; t.eR = e.R; t.eS = e.S; t.eph = e.ph; t.epw = e.pw;
      return t;
    }
  }
  if (g.sh == 1 && g.sw == 1 && fmt == FMT_BF16 && io_bf16 && g.C <= 16 && env_int("POLYCONV_HK_SMALLC", 1) != 0) {
    // small C at stride 1 (VGG conv1_1, C = 3): 32-byte window rows of 16 channels instead of
    // 128-byte rows of 64 (4x less window and MMA K padding); the pair loader masks channels >= C
    HankelTiling t = hankel_tiling_core(g, fmt, num_sms, 16);
    if (t.ok) {
      t.phase = 0;
      t.aligned = (!(g.W & 1) && t.pitch == g.W + 2 * g.pw && t.delta == (g.pw & 1)) ? 1 : 0;
      if (t.aligned) return t;
    }
  }
  HankelTiling t = hankel_tiling_core(g, fmt, num_sms);
  t.phase = 0;
  const int pl_mode = env_int("POLYCONV_HK_PLANES", 1);  // 0 off, 1 odd widths, 2 also even widths
  if (t.ok && (!t.aligned || pl_mode >= 2) && fmt == FMT_BF16 && io_bf16 && g.C % 64 == 0 && pl_mode != 0) {
    // small planes (7x7): whole (image, 64-channel) blocks by bulk copy instead of the element
    // loader's two 4-byte loads per element; two staging buffers, else one
    for (int nb = 2; nb >= 1; --nb) {
      HankelTiling tp = hankel_tiling_core(g, fmt, num_sms, 0, nb);
      if (tp.ok && tp.T == t.T && tp.NN == t.NN) {
        tp.phase = 0;
        tp.aligned = 0;
        return tp;
      }
    }
  }
  return t;
}

cudaError_t launch_mac_hankel(const Geom& g0, const HankelTiling& t, int fmt, const void* x, bool io_bf16,
                              const void* U, void* const* ys, int nys, int ktot, int koff, const void* zero,
                              cudaStream_t st, char* err, size_t errlen) {
  if (nys < 1 || nys > kHkMaxOut || koff < 0 || koff + g0.K > ktot) {
    snprintf(err, errlen, "mac_hankel: bad output list");
    return cudaErrorInvalidValue;
  }
  if (!t.ok) {
    snprintf(err, errlen, "mac_hankel: shape not supported");
    return cudaErrorInvalidValue;
  }
  const bool tf32 = fmt == FMT_TF32;
  Geom g = g0;  // the geometry the kernel runs (phase mode: the phase-split one)
  if (t.phase) {
    g.C = t.eC; g.H = t.eH; g.W = t.eW; g.R = t.eR; g.S = t.eS; g.ph = t.eph; g.pw = t.epw;
    g.sh = g.sw = 1;
  }
  EncodeTiledFnHk enc = get_encode_hk();
  CUtensorMap tmU;
  {
    const uint32_t eb = tf32 ? 4 : 2;
    cuuint64_t dims[2] = {(cuuint64_t)t.Cp, (cuuint64_t)g.R * g.S * t.Kp};
    cuuint64_t strides[1] = {(cuuint64_t)t.Cp * eb};
    cuuint32_t box[2] = {(cuuint32_t)t.kc, (cuuint32_t)(t.NN / 2)};
    cuuint32_t estr[2] = {1, 1};
    if (!enc || enc(&tmU, tf32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2,
                    const_cast<void*>(U), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    t.kc * eb == 32 ? CU_TENSOR_MAP_SWIZZLE_32B
                    : t.kc * eb == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B,
                    CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      snprintf(err, errlen, "mac_hankel: cuTensorMapEncodeTiled failed");
      return cudaErrorInvalidValue;
    }
  }
  HkParams p{};
  p.x = x;
  p.zero = zero;
  for (int o = 0; o < nys; ++o) p.ys[o] = ys[o];
  p.nys = nys;
  p.Ktot = ktot;
  p.koff = koff;
  p.N = g.N; p.C = g.C; p.H = g.H; p.W = g.W; p.K = g.K; p.P = g.P; p.Q = g.Q;
  p.sh = g.sh; p.sw = g.sw; p.ph = g.ph; p.pw = g.pw;
  p.HW = g.H * g.W;
  p.CHW = g.C * g.H * g.W;
  p.pitch = t.pitch; p.HS = t.HS; p.delta = t.delta;
  p.T = t.T; p.NN = t.NN; p.NB = t.NB; p.Kp = t.Kp; p.Cp = t.Cp; p.nchunks = t.nchunks;
  p.RS = g.R * g.S; p.S = g.S; p.PT = t.PT; p.npairs = t.npairs;
  p.wrows = t.wrows; p.wslots = t.wslots; p.fslots = t.fslots; p.resident = t.resident;
  p.wslot_bytes = t.wslot_bytes; p.fblk_bytes = t.fblk_bytes;
  // instruction descriptor: D = f32, A/B = bf16 (1) or tf32 (2), both K-major, N>>3 @17, M>>4 @24
  const uint32_t ab = tf32 ? 2u : 1u;
  p.idesc = (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(t.NN >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
  p.tmem_cols = t.tmem_cols;
  p.nacc = t.nacc;
  p.fpitch.init((uint32_t)t.pitch);
  p.fHS.init((uint32_t)t.HS);
  p.fsh.init((uint32_t)g.sh);
  p.fsw.init((uint32_t)g.sw);
  p.phase = t.phase;
  p.xC = g0.C; p.xH = g0.H; p.xW = g0.W;
  p.pimg_bytes = t.pimg_bytes; p.pimg_max = t.pimg_max; p.psbufs = t.planes;
  p.dbg = env_int("POLYCONV_HK_DEBUG", 0);
  // kHW2: -1 = general loader, 0 = pair-aligned loader with a runtime plane size, > 0 = the
  // plane size in words baked in (immediate channel offsets) for the ResNet / VGG planes
  void (*kern)(const CUtensorMap, const CUtensorMap, const HkParams);
  CUtensorMap tmY = tmU;  // kRowTile: y as [N*K][P][Q] bf16, boxes of Q pixels x 1 row x NN channels
  if (t.rowtile) {
    cuuint64_t dims[3] = {(cuuint64_t)g0.Q, (cuuint64_t)g0.P, (cuuint64_t)g0.N * g0.K};
    cuuint64_t strides[2] = {(cuuint64_t)g0.Q * 2, (cuuint64_t)g0.P * g0.Q * 2};
    cuuint32_t box[3] = {(cuuint32_t)g0.Q, 1, (cuuint32_t)t.NN};
    cuuint32_t estr[3] = {1, 1, 1};
    if (!enc || enc(&tmY, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, ys[0], dims, strides, box, estr,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      snprintf(err, errlen, "mac_hankel: cuTensorMapEncodeTiled (y) failed");
      return cudaErrorInvalidValue;
    }
  }
  p.rt_stage = t.rowtile ? (uint32_t)(t.NN * g0.Q * 2) : 0u;
  const bool scatter = nys > 1 || ktot != g0.K || koff != 0;
  const int hw2 = g.H * g.W / 2;
  if (!t.phase && t.kc == 16) {
    if (!t.aligned) {
      snprintf(err, errlen, "mac_hankel: small-C mode needs pair-aligned planes");
      return cudaErrorInvalidValue;
    }
    kern = mac_hankel_kernel<__nv_bfloat16, false, 0, 16>;
  } else if (t.phase && t.kc == 16 && t.rowtile) {
    if (!io_bf16 || scatter) {
      snprintf(err, errlen, "mac_hankel: row-tile mode needs bf16 output and one output buffer");
      return cudaErrorInvalidValue;
    }
    kern = mac_hankel_kernel<__nv_bfloat16, false, -2, 16, false, true>;
  } else if (t.phase && t.kc < 64) {
    if (!t.aligned) {
      snprintf(err, errlen, "mac_hankel: small-C phase mode needs pair-aligned phase planes");
      return cudaErrorInvalidValue;
    }
    kern = t.kc == 16 ? mac_hankel_kernel<__nv_bfloat16, false, -2, 16> : mac_hankel_kernel<__nv_bfloat16, false, -2, 32>;
  } else if (t.phase) {
    kern = t.aligned ? mac_hankel_kernel<__nv_bfloat16, false, -2> : mac_hankel_kernel<__nv_bfloat16, false, -4>;
  } else if (t.planes) {
    kern = mac_hankel_kernel<__nv_bfloat16, false, kHkPlanes>;
  } else if (!t.aligned) {
    kern = tf32 ? mac_hankel_kernel<float, true, -1>
                : (io_bf16 ? mac_hankel_kernel<__nv_bfloat16, false, -1> : mac_hankel_kernel<float, false, -1>);
  } else if (tf32) {
    kern = mac_hankel_kernel<float, true, 0>;
  } else if (!io_bf16) {
    kern = mac_hankel_kernel<float, false, 0>;
  } else {
    kern = hw2 == 1568 ? mac_hankel_kernel<__nv_bfloat16, false, 1568>
           : hw2 == 392 ? mac_hankel_kernel<__nv_bfloat16, false, 392>
           : hw2 == 98  ? mac_hankel_kernel<__nv_bfloat16, false, 98>
                        : mac_hankel_kernel<__nv_bfloat16, false, 0>;
  }
  if (scatter) {
    // the scatter epilogue: stride-1 plans with 128-byte window rows, the general loader
    if (t.phase || t.kc * (tf32 ? 4 : 2) != 128) {
      snprintf(err, errlen, "mac_hankel: forward_scatter needs a stride-1 plan with 128-byte window rows");
      return cudaErrorNotSupported;
    }
    kern = tf32 ? mac_hankel_kernel<float, true, -1, 32, true>
                : (io_bf16 ? mac_hankel_kernel<__nv_bfloat16, false, -1, 64, true> : mac_hankel_kernel<float, false, -1, 64, true>);
  }
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, t.smem_bytes);
  if (e != cudaSuccess) return e;
  {
    // shared-memory carveout: just what the kernel needs, the rest stays L1 (the window loaders'
    // in-flight loads are tracked in L1: experiment POLYCONV_HK_CARVE=percent)
    const int carve = env_int("POLYCONV_HK_CARVE", -1);
    if (carve >= 0) {
      e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
      if (e != cudaSuccess) return e;
    }
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)t.grid);
  cfg.blockDim = dim3(kHkThreads);
  cfg.dynamicSmemBytes = (size_t)t.smem_bytes;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, kern, tmU, tmY, p);
}

}  // namespace polyconv

// Debug only (not part of include/polyconv.h): the per-CTA trace of the last
// POLYCONV_HK_DEBUG&8 launch (160 x 16 u64, globaltimer ns).
extern "C" int polyconv_dbg_hk_trace(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_hk_trace, sizeof(unsigned long long) * 160 * 16);
}
extern "C" int polyconv_dbg_hk_wtrace(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_hk_wtrace, sizeof(unsigned long long) * 64 * 8);
}
extern "C" int polyconv_dbg_hk_ltrace(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_hk_ltrace, sizeof(unsigned long long) * 64 * 16);
}
