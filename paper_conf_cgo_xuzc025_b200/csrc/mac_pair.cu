// mac_pair.cu — the round-1 BF16 path on CTA pairs (tcgen05 cta_group::2): a pack grid for
// a2 + a3, then a4 coefficient MAC + a5 extraction as its programmatic dependent launch.
// Since round 2 `mac_hankel` is the BF16 default; this kernel is selectable (TC_PAIR) and
// kept as the ablation that packs A through HBM.
//
// The coefficient MAC
//   p_{n,k}[m] = sum_c sum_{i,j} A_{n,c}[m - e(i,j)] * U_{k,c}[e(i,j)]   (P.965, P.1350-1352)
// is, per kernel tap (i,j), a GEMM over channels whose position operand is the
// input polynomial shifted by Wp*i + j coefficients (the doubly blocked Hankel
// structure, P.404-437):
//   D[pos][k] += sum_c A[pos + Wp*i + j][c] * U_tap(i,j)[k][c]
// with pos = the base coefficient m - (L_U - 1) of an output (Eq. 12).
//
// Design:
//  * Pack grid (pair_pack_kernel, several CTAs per SM): the tap-major filter
//    U[R*S][NN][Cp] (a3: the nonzero coefficients of the reversed, gap-padded
//    U_{k,c}(t), Eq. 6, grouped by degree e(i,j)) and bands of rb padded rows of the
//    channel-interleaved input polynomial A[N*L_A][Cp] (a2: coefficient r*Wp + s of
//    A_{n,c}(t) = xpad[n][c][r][s], Eq. 10 + zero padding P.1353-1356, BF16 RNE, reading
//    R11): TMA boxes of x rows, a shared-memory transpose into 128-byte swizzled rows, TMA
//    stores.  It triggers the dependent launch at once; the MAC's producer waits
//    (griddepcontrol.wait) before its first TMA read of A / U.
//  * MAC (CTA pairs): UMMA M = 256 positions (128 per CTA = the TMEM lanes: a window of
//    the interleaved input, K-major, TMA), N = NN output channels (B operand = the filter,
//    each CTA holding NN/2 rows of every (chunk, tap) block -- RESIDENT in shared memory:
//    loaded once, reused by every tile).  One window of 128 + (R-1)*Wp + S-1 positions per
//    channel chunk serves all R*S taps through descriptors shifted by (Wp*i + j) rows
//    (tools/umma_probe.cu).  The leader CTA issues tcgen05.mma.cta_group::2 from a per-tap
//    descriptor table; accumulators (fp32) live in TMEM, double buffered, so the epilogue
//    of tile t overlaps the MMAs of tile t+1.  A CTA tile = tr output rows of one image.
//  * Epilogue (a5, fused): positions are TMEM lanes; the Eq. 12 / reading R4
//    extraction y[n][k][oh][ow] = p[Wp*sh*oh + sw*ow + L_U - 1] is a per-lane
//    predicate; bf16 outputs are staged per channel half in shared memory and
//    TMA-stored as [32 channels][tr*Q pixels] boxes of y viewed as [N*K][P*Q]
//    (direct stores for f32 outputs or K % 32 != 0).
//  * Warp roles: warp 0 = TMA producer, warp 1 = TMEM allocator + MMA issuer
//    (leader CTA), warps 2..9 = epilogue (2 per TMEM lane quadrant, each half
//    of the channels).
//  * Synchronisation is pair-local (mbarriers) plus the programmatic launch
//    dependency: no grid-wide counters or flags (the round-1 one-launch variant with a
//    grid counter and band flags, and its experiment switches, were removed).
#include <cuda.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <algorithm>
#include <type_traits>
#include <new>
#include "common.cuh"
#include "sm100.cuh"

namespace polyconv {

namespace {

using namespace sm100;

constexpr int kPairThreads = 320;  // 10 warps
constexpr int kEpi0 = 2;           // first epilogue warp
constexpr int kMaxBlk = 64;        // filter blocks (channel chunks x taps) resident
constexpr int kTileM = 128;        // positions per CTA per tile (TMEM lanes)

struct PairParams {
  const void* x;
  const void* w;
  void* A;  // interleaved input polynomial [N*L_A][Cp] bf16 (plan workspace)
  void* U;  // tap-major filter [R*S][NN][Cp] bf16 (plan workspace)
  void* y;
  long long L_A, G, NLA;
  int N, C, H, W, K, R, S, sh, sw, ph, pw, Hp, Wp, P, Q, PQ;
  int Cp, NN, kc, row_bytes, nchunks, RS, nblk;
  int box_rows, nbox;
  uint32_t wbytes, wbytes_tx, fbytes;
  int ring, num_tiles, num_pairs;
  int urep;  // filter copies in U; pair p reads copy p % urep (spreads the L2 lines all CTAs read)
  uint32_t idesc;
  int tmem_cols;
  int rb, nb, nunits, spitch;
  FastDiv fLA, fWp, fsh, fsw;
  int dbg;
  // TMA pack path (pack_tma): x band [C rows][ne_box elements] in by TMA, the band's
  // A rows out by TMA stores of 64-channel SW128 boxes (rb*Wp rows; the last band
  // of an image through the second map)
  int pack_tma, ne_box, last_rows;
  uint32_t in_bytes, obox_bytes, obox_bytes2;
  // row-aligned tiles: a CTA tile = tr output rows of one image (tpi tiles per image,
  // ntile CTA tiles in all); epilogue by TMA stores of [32 channels][tr*Q pixels]
  // boxes staged in shared memory (epi_tma) or by direct stores
  int tr, tpi, ntile, epi_tma;
  int u_img0;  // first image the pack writes (0)
  // split: a2 + a3 run in a separate pack kernel (pair_pack_kernel) that this kernel
  // follows as a programmatic dependent launch: no grid counter, no band flags
  int split;
  uint32_t estage_bytes;
  FastDiv ftpi;
};

// per-CTA phase trace (POLYCONV_PAIR_DEBUG & 8), globaltimer ns:
// 0 start, 1 pack done, 2 grid counter passed, 3-6 windows 0-3 landed (leader),
// 7/8 tile 0/1 MMAs issued (leader), 9/11 tile 0/1 accumulator ready (epilogue),
// 10/12 tile 0/1 stores done (epilogue warp 0), 13 end, 14 last filter block landed
// (leader), 15 last window TMA issued (producer)
constexpr int kTr = 16;
__device__ unsigned long long g_pair_trace[160 * kTr];
__device__ unsigned long long g_pair_clk[160 * 2];
__device__ unsigned long long g_pair_pk[160 * 4];
__device__ unsigned long long g_pair_iss[160 * 4];  // issuer, tile 0: chunk c filter ready [2c], MMAs issued [2c+1]  // pack sub-phases: filter done, band staged, band written  // clock64 at tr[0] and tr[13]: SM clock = cycles / ns

// ---- pair-specific PTX ---------------------------------------------------------
__device__ __forceinline__ uint32_t mapa_rank0(uint32_t local) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(r) : "r"(local));
  return r;
}
// TMA into this CTA's shared memory, completion signalled on the LEADER's mbarrier
__device__ __forceinline__ void tma_load_2d_pair(uint32_t dst, const void* tmap, uint32_t mbar_cluster, int c0,
                                                 int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(tmap)), "r"(mbar_cluster), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void umma2_f16(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// arrive on the mbarrier at this offset in both CTAs of the pair when all prior MMAs finish
__device__ __forceinline__ void umma2_commit_both(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"((uint16_t)3)
      : "memory");
}
__device__ __forceinline__ void mbar_arrive_remote(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
// mbarrier wait (CTA-scope acquire: a cluster-scope acquire compiles to an L1
// invalidate per poll); sleep_ns > 0 backs off between polls (long waits)
__device__ __forceinline__ void mbar_wait_cl(uint64_t* bar, uint32_t parity, uint32_t sleep_ns = 0) {
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
    if (sleep_ns) __nanosleep(sleep_ns);
  }
}
__device__ __forceinline__ void tmem_alloc2(uint32_t* slot, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(slot)),
               "r"(ncols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc2(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}

template <typename T>
__device__ __forceinline__ uint16_t to_bf16_bits(T v);
template <>
__device__ __forceinline__ uint16_t to_bf16_bits<float>(float v) {
  return __bfloat16_as_ushort(__float2bfloat16_rn(v));  // reading R11: RNE
}
template <>
__device__ __forceinline__ uint16_t to_bf16_bits<__nv_bfloat16>(__nv_bfloat16 v) {
  return __bfloat16_as_ushort(v);
}

// ---- phase 1: a3 + a2 into the workspace ----------------------------------------
template <typename IoT>
__device__ __forceinline__ void pair_pack(const PairParams& p, uint16_t* stg, bool x_too) {
  const int tid = threadIdx.x;
  const int nth = blockDim.x;
  const bool ptr = (p.dbg & 8) && blockIdx.x < 160 && tid == 0;
  // a3: U[tap][k][c] = w[k][c][tap] (tap = i*S + j; k >= K or c >= C: 0).  One flat
  // pass over U spread over every thread of the grid (consecutive threads write
  // consecutive channels), four loads in flight per thread
  {
    const IoT* w = static_cast<const IoT*>(p.w);
    uint16_t* U = static_cast<uint16_t*>(p.U);
    const int total = p.RS * p.NN * p.Cp;  // one copy; urep copies are written
    const int stride = gridDim.x * nth;
    for (int base = blockIdx.x * nth + tid; base < total; base += 4 * stride) {
      uint16_t v[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int idx = base + u * stride;
        v[u] = 0;
        if (idx < total) {
          const int c = idx % p.Cp, tk = idx / p.Cp;
          const int k = tk % p.NN, tap = tk / p.NN;
          if (k < p.K && c < p.C) v[u] = to_bf16_bits<IoT>(w[((long long)k * p.C + c) * p.RS + tap]);
        }
      }
      for (int rep = 0; rep < p.urep; ++rep) {
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int idx = base + u * stride;
          if (idx < total) U[(long long)rep * total + idx] = v[u];
        }
      }
    }
  }
  if (ptr) g_pair_pk[blockIdx.x * 4] = global_ns();
  if (!x_too) return;
  // a2: bands of rb padded rows of one image: stage the band's input rows of
  // every channel (contiguous in NCHW), then write each position's Cp channel
  // words as 16-byte chunks (coalesced: consecutive threads, consecutive chunks)
  const IoT* x = static_cast<const IoT*>(p.x);
  uint4* A4 = static_cast<uint4*>(p.A);
  const int ncg = p.Cp / 8;
  const int HW = p.H * p.W;
  for (int u = blockIdx.x; u < p.nunits; u += gridDim.x) {
    const int n = u / p.nb, b = u - (u / p.nb) * p.nb;
    const int r0 = b * p.rb, r1 = min(p.Hp, r0 + p.rb);
    const int h0 = min(max(r0 - p.ph, 0), p.H), h1 = min(max(r1 - p.ph, 0), p.H);
    const int ne = (h1 - h0) * p.W;
    int eoff = 0;  // staging column of plane element h0*W
    if (ne > 0) {
      constexpr int VE = 16 / (int)sizeof(IoT);  // elements per 16-byte load
      if (HW % VE == 0) {
        // 16-byte loads over [e_lo, e_hi), the band rounded out to whole vectors
        // (planes start 16-byte aligned); batches of 8 loads in flight per thread
        const int e0 = h0 * p.W, e_lo = e0 & ~(VE - 1), e_hi = (e0 + ne + VE - 1) & ~(VE - 1);
        eoff = e0 - e_lo;
        const int nv = (e_hi - e_lo) / VE;
        const uint4* xs = reinterpret_cast<const uint4*>(x + (long long)n * p.C * HW + e_lo);
        const int hwv = HW / VE;
        const int tot = p.C * nv;
        FastDiv fnv;
        fnv.init((uint32_t)nv);
        for (int base = tid; base < tot; base += 8 * nth) {
          uint4 r[8];
#pragma unroll
          for (int u = 0; u < 8; ++u) {
            const int idx = base + u * nth;
            if (idx < tot) {
              const int c = (int)fnv.div((uint32_t)idx), v = idx - c * nv;
              r[u] = __ldg(xs + (long long)c * hwv + v);
            }
          }
#pragma unroll
          for (int u = 0; u < 8; ++u) {
            const int idx = base + u * nth;
            if (idx < tot) {
              const int c = (int)fnv.div((uint32_t)idx), v = idx - c * nv;
              uint16_t* d = stg + c * p.spitch + v * VE;
              if constexpr (VE == 8) {
                const uint32_t wd[4] = {r[u].x, r[u].y, r[u].z, r[u].w};
#pragma unroll
                for (int t = 0; t < 4; ++t) {
                  d[2 * t] = (uint16_t)(wd[t] & 0xFFFFu);
                  d[2 * t + 1] = (uint16_t)(wd[t] >> 16);
                }
              } else {
                const float f[4] = {__uint_as_float(r[u].x), __uint_as_float(r[u].y), __uint_as_float(r[u].z),
                                    __uint_as_float(r[u].w)};
#pragma unroll
                for (int t = 0; t < 4; ++t) d[t] = to_bf16_bits<float>(f[t]);
              }
            }
          }
        }
      } else {
        const IoT* xs = x + ((long long)n * p.C * p.H + h0) * p.W;
        const int tot = p.C * ne;
        FastDiv fne;
        fne.init((uint32_t)ne);
#pragma unroll 8
        for (int idx = tid; idx < tot; idx += nth) {
          const int c = (int)fne.div((uint32_t)idx), e = idx - c * ne;
          stg[c * p.spitch + e] = to_bf16_bits<IoT>(xs[(long long)c * HW + e]);
        }
      }
    }
    __syncthreads();
    if (ptr) g_pair_pk[blockIdx.x * 4 + 1] = global_ns();
    const int npos = (r1 - r0) * p.Wp;
    uint4* dst = A4 + ((long long)n * p.L_A + (long long)r0 * p.Wp) * ncg;
    for (int idx = tid; idx < npos * ncg; idx += nth) {
      const int pp = idx / ncg, q = idx - (idx / ncg) * ncg;
      const int rr = (int)p.fWp.div((uint32_t)pp);
      const int h = r0 + rr - p.ph, ww = pp - rr * p.Wp - p.pw;
      uint32_t v[4] = {0u, 0u, 0u, 0u};
      if (h >= 0 && h < p.H && ww >= 0 && ww < p.W) {
        const int e = (h - h0) * p.W + ww + eoff;
#pragma unroll
        for (int m = 0; m < 4; ++m) {
          const int c0 = q * 8 + 2 * m;
          const uint32_t lo = c0 < p.C ? stg[c0 * p.spitch + e] : 0u;
          const uint32_t hi = c0 + 1 < p.C ? stg[(c0 + 1) * p.spitch + e] : 0u;
          v[m] = lo | (hi << 16);
        }
      }
      dst[idx] = make_uint4(v[0], v[1], v[2], v[3]);
    }
    __syncthreads();
    if (ptr) g_pair_pk[blockIdx.x * 4 + 2] = global_ns();
  }
}

// a2 by TMA: one 2-D TMA box brings the band's input rows of all C channel planes
// (x viewed as [N*C][H*W]; elements past the plane / planes past N*C are
// zero-filled or ignored), the warps transpose it into the band's rows of the
// interleaved layout (coefficient r*Wp + s of A_{n,c}(t) = xpad[n][c][r][s],
// Eq. 10, zero padding P.1353-1356), 128-byte swizzled per 64 channels, and TMA
// stores write them out.  Consecutive threads take consecutive positions, so the
// staging reads are conflict-free and the swizzled 16-byte writes are too.
__device__ __forceinline__ void tma_store_2d(const void* tmap, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(tmap)),
               "r"(src), "r"(c0), "r"(c1)
               : "memory");
}

// a3 straight into shared memory: CTA `rank` of the pair builds its NN/2 output
// channels of every (channel chunk, tap) block of the tap-major filter -- the
// nonzero coefficients of the reversed, gap-padded U_{k,c}(t) (Eq. 6), block
// (ch, tap) row k = w[k][ch*kc .. ch*kc + kc)[tap] -- in the UMMA K-major layout
// (rows of kc bf16 words, 32/64/128-byte swizzle).  One item = 8 channels of one
// output channel: their R*S taps are contiguous in w (one 16-byte vector per tap
// group when RS == 9 and C % 8 == 0), transposed in registers into one 16-byte
// chunk per tap block.  Nothing goes to global memory.
template <typename IoT>
__device__ __forceinline__ void pack_load(const PairParams& p, const CUtensorMap* tmX, uint8_t* stage,
                                          uint64_t* pbar, int u, int bx) {
  const int n = p.u_img0 + u / p.nb, b = u - (u / p.nb) * p.nb;
  const int r0 = b * p.rb;
  const int h0 = min(max(r0 - p.ph, 0), p.H);
  const uint32_t bytes = 64u * p.ne_box * (uint32_t)sizeof(IoT);
  mbar_arrive_expect_tx(pbar + bx, bytes);
  tma_load_2d(stage + (size_t)bx * bytes, tmX, pbar + bx, (h0 * p.W) & ~(16 / (int)sizeof(IoT) - 1),
              n * p.C + bx * 64);
}

// band units of this CTA: x boxes of 64 channel planes in by TMA (the first unit's
// already issued), each transposed into its 128-byte swizzled box of A rows and
// stored by TMA as soon as it is done, then the band is published.
template <typename IoT>
__device__ __forceinline__ void pair_pack_x_tma(const PairParams& p, uint8_t* stage, uint64_t* pbar,
                                                const CUtensorMap* tmX, const CUtensorMap* tmS,
                                                const CUtensorMap* tmS2, bool first_issued) {
  const int tid = threadIdx.x;
  const int nth = blockDim.x;
  const bool ptr = (p.dbg & 8) && blockIdx.x < 160 && tid == 0;
  const int nbx = p.Cp / 64;
  const uint32_t xbox = 64u * p.ne_box * (uint32_t)sizeof(IoT);
  uint8_t* out = stage + p.in_bytes;
  int it = 0;
  for (int u = blockIdx.x; u < p.nunits; u += gridDim.x, ++it) {
    const int n = p.u_img0 + u / p.nb, b = u - (u / p.nb) * p.nb;
    const int r0 = b * p.rb, r1 = min(p.Hp, r0 + p.rb);
    const int h0 = min(max(r0 - p.ph, 0), p.H), h1 = min(max(r1 - p.ph, 0), p.H);
    const bool any = h1 > h0 && !(p.dbg & 2);
    if (tid == 0 && any && !(it == 0 && first_issued))
      for (int bx = 0; bx < nbx; ++bx) pack_load<IoT>(p, tmX, stage, pbar, u, bx);
    const int npos = (r1 - r0) * p.Wp;
    const uint32_t obox = (r1 - r0 == p.rb) ? p.obox_bytes : p.obox_bytes2;
    const int eoff = (h0 * p.W) & (16 / (int)sizeof(IoT) - 1);  // the box starts at h0*W rounded down
    const CUtensorMap* m = (r1 - r0 == p.rb) ? tmS : tmS2;
    for (int bx = 0; bx < nbx; ++bx) {
      if (any) mbar_wait(pbar + bx, (uint32_t)(it & 1));
      if (ptr && bx == 0) g_pair_pk[blockIdx.x * 4 + 1] = global_ns();
      const IoT* in = reinterpret_cast<const IoT*>(stage + (size_t)bx * xbox);
      uint8_t* dbox = out + (size_t)bx * obox;
      const int cbase = bx * 64;
      // one item = one position's 64 channels = one 128-byte row of the box; consecutive
      // threads take consecutive positions (conflict-free staging reads, swizzled writes)
      for (int pos = tid; pos < npos; pos += nth) {
        const int rr = (int)p.fWp.div((uint32_t)pos);
        const int h = r0 + rr - p.ph, ww = pos - rr * p.Wp - p.pw;
        uint8_t* drow = dbox + (size_t)pos * 128;
        const uint32_t sw = (uint32_t)(pos & 7);
        if (any && h >= 0 && h < p.H && ww >= 0 && ww < p.W) {
          const IoT* src = in + (h - h0) * p.W + ww + eoff;
#pragma unroll
          for (int q8 = 0; q8 < 8; ++q8) {
            const int c0 = cbase + q8 * 8;
            uint32_t v[4];
            if (c0 + 8 <= p.C) {
              uint32_t hv[8];
#pragma unroll
              for (int k = 0; k < 8; ++k) hv[k] = to_bf16_bits<IoT>(src[(q8 * 8 + k) * p.ne_box]);
#pragma unroll
              for (int mm = 0; mm < 4; ++mm) v[mm] = hv[2 * mm] | (hv[2 * mm + 1] << 16);
            } else {
#pragma unroll
              for (int mm = 0; mm < 4; ++mm) {
                const int c = c0 + 2 * mm;
                const uint32_t lo = c < p.C ? (uint32_t)to_bf16_bits<IoT>(src[(q8 * 8 + 2 * mm) * p.ne_box]) : 0u;
                const uint32_t hi =
                    c + 1 < p.C ? (uint32_t)to_bf16_bits<IoT>(src[(q8 * 8 + 2 * mm + 1) * p.ne_box]) : 0u;
                v[mm] = lo | (hi << 16);
              }
            }
            *reinterpret_cast<uint4*>(drow + (((uint32_t)q8 ^ sw) << 4)) = make_uint4(v[0], v[1], v[2], v[3]);
          }
        } else {
#pragma unroll
          for (int q8 = 0; q8 < 8; ++q8)
            *reinterpret_cast<uint4*>(drow + (((uint32_t)q8 ^ sw) << 4)) = make_uint4(0u, 0u, 0u, 0u);
        }
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // staging -> TMA store / next load
      __syncthreads();
      if (tid == 0) {
        if (ptr && bx == nbx - 1) g_pair_pk[blockIdx.x * 4 + 3] = global_ns();
        tma_store_2d(m, smem_u32(dbox), bx * 64, (int)((long long)n * p.L_A + (long long)r0 * p.Wp));
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    }
    if (tid == 0) {
      asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");  // written (before publishing / reuse)
      if (ptr) g_pair_pk[blockIdx.x * 4 + 2] = global_ns();
    }
    __syncthreads();
  }
}

template <typename IoT>
__global__ void __launch_bounds__(256) pair_pack_kernel(const __grid_constant__ CUtensorMap tmX,
                                                        const __grid_constant__ CUtensorMap tmS,
                                                        const __grid_constant__ CUtensorMap tmS2,
                                                        const PairParams p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t* stage = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  __shared__ uint64_t pbar[4];
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) mbar_init(pbar + i, 1);
    fence_barrier_init();
  }
  __syncthreads();
  const bool first = (int)blockIdx.x < p.nunits;
  if (threadIdx.x == 0 && first) {
    const int u = (int)blockIdx.x;
    const int b = u - (u / p.nb) * p.nb;
    const int r0 = b * p.rb, r1 = min(p.Hp, r0 + p.rb);
    const int h0 = min(max(r0 - p.ph, 0), p.H), h1 = min(max(r1 - p.ph, 0), p.H);
    if (h1 > h0) {
      prefetch_tmap(&tmX);
      for (int bx = 0; bx < p.Cp / 64; ++bx) pack_load<IoT>(p, &tmX, stage, pbar, u, bx);
    }
  }
  pair_pack<IoT>(p, nullptr, false);
  pair_pack_x_tma<IoT>(p, stage, pbar, &tmX, &tmS, &tmS2, first);
}

// One channel chunk's MMAs (all taps, all K-steps): the whole warp runs the loop,
// one elected lane issues.  Out of line so that the warm-up issue at launch and
// every later chunk execute the same instructions (after an L2 flush the first
// execution of a code path otherwise waits for instruction fetches from DRAM).
__device__ __noinline__ void issue_chunk(uint32_t d_tmem, uint64_t ad0, uint64_t bd0, const uint32_t* mtab, int RS,
                                         int ksteps, uint32_t idesc, uint32_t acc_first) {
  for (int ti = 0; ti < RS; ++ti) {
    const uint64_t ad = ad0 + mtab[2 * ti], bd = bd0 + mtab[2 * ti + 1];
    const uint32_t acc0 = (acc_first | (uint32_t)ti) != 0 ? 1u : 0u;
    if (elect_one()) {
      umma2_f16(d_tmem, ad, bd, idesc, acc0);
      // K step = 32 bytes = +2 in the start field
      if (ksteps > 1) umma2_f16(d_tmem, ad + 2, bd + 2, idesc, 1u);
      if (ksteps > 2) {
        umma2_f16(d_tmem, ad + 4, bd + 4, idesc, 1u);
        umma2_f16(d_tmem, ad + 6, bd + 6, idesc, 1u);
      }
    }
    __syncwarp();
  }
}

template <typename IoT>
__global__ void __launch_bounds__(kPairThreads, 1)
    mac_pair_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmU,
                    const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmS,
                    const __grid_constant__ CUtensorMap tmS2, const __grid_constant__ CUtensorMap tmY,
                    const PairParams p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  uint8_t* sF = smem;                                        // filter blocks [nblk][NN/2][row]
  uint8_t* sWin = sF + (size_t)p.nblk * p.fbytes;            // window ring [ring][rows][row]
  uint8_t* sEpi = sWin + (size_t)p.ring * p.wbytes;          // epilogue staging [NN][tr*Q] bf16
  uint64_t* bars = reinterpret_cast<uint64_t*>(sEpi + p.estage_bytes);
  uint64_t* ffull = bars;                 // [kMaxBlk] filter block landed (leader: both halves)
  uint64_t* wfull = ffull + kMaxBlk;      // [ring] window landed (leader: both CTAs' windows)
  uint64_t* wempty = wfull + 8;           // [ring] window consumed (both CTAs, MMA commit)
  uint64_t* tfull = wempty + 8;           // [2] accumulator ready (both CTAs, MMA commit)
  uint64_t* tempty = tfull + 2;           // [2] accumulator drained (leader: 16 epilogue warps)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  uint32_t* mtab = tmem_slot + 4;  // [kMaxBlk][2]: per tap, A shift and B offset (16-byte units)
  uint64_t* pbar = reinterpret_cast<uint64_t*>(mtab + 2 * kMaxBlk);  // [6] pack: x boxes [0,4), w slabs [4,6)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const int pair = (int)blockIdx.x >> 1;
  const bool trace = (p.dbg & 8) && blockIdx.x < 160;
  unsigned long long* tr = g_pair_trace + blockIdx.x * kTr;
  if (trace && threadIdx.x == 0) {
    tr[0] = global_ns();
    g_pair_clk[blockIdx.x * 2] = clock64();
  }

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmU);
    for (int b = 0; b < p.nblk; ++b) mbar_init(ffull + b, 1);
    for (int s = 0; s < p.ring; ++s) {
      mbar_init(wfull + s, 1);
      mbar_init(wempty + s, 1);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(tfull + s, 1);
      mbar_init(tempty + s, 2 * 8);
    }
    for (int i = 0; i < 6; ++i) mbar_init(pbar + i, 1);
    fence_barrier_init();
  }
  if (warp == 1) {
    tmem_alloc2(tmem_slot, (uint32_t)p.tmem_cols);
    // descriptor offsets per tap, so that the issue loop is a few uniform adds per
    // tap (divisions in it left the tensor pipe idle)
    for (int ti = lane; ti < p.RS; ti += 32) {
      const int i = ti / p.S, j = ti - (ti / p.S) * p.S;
      mtab[2 * ti] = ((uint32_t)(p.Wp * i + j) * (uint32_t)p.row_bytes) >> 4;
      mtab[2 * ti + 1] = ((uint32_t)ti * p.fbytes) >> 4;
    }
  }
  __syncthreads();  // pbar initialised

  // the staging area is overwritten by TMA (async proxy) next
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (trace && threadIdx.x == 0) tr[1] = global_ns();
  tc_fence_before();
  __syncthreads();
  cluster_sync();  // peer barriers initialised, TMEM allocated in both CTAs
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // --------------------------------------------------------------- TMA producer
    const uint32_t lead_wfull = mapa_rank0(smem_u32(wfull));
    const uint32_t lead_ffull = mapa_rank0(smem_u32(ffull));
    const uint32_t sW0 = smem_u32(sWin), sF0 = smem_u32(sF);
    const int half = p.NN / 2;
    // the pack kernel (the programmatic-launch primary) has written A and U
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("fence.proxy.async.global;" ::: "memory");
    if (trace && lane == 0) tr[2] = global_ns();
    __syncwarp();
    // the first chunk's filter blocks go out before the first window (measured +4%)
    const bool f0_early = pair < p.num_tiles;
    if (f0_early && elect_one()) {
      for (int tap = 0; tap < p.RS; ++tap) {
        if (rank == 0) mbar_arrive_expect_tx(ffull + tap, 2u * p.fbytes);
        tma_load_2d_pair(sF0 + (uint32_t)tap * p.fbytes, &tmU, lead_ffull + 8u * (uint32_t)tap, 0,
                         tap * p.NN + (int)rank * half + (pair % p.urep) * p.RS * p.NN);
      }
    }
    __syncwarp();
    int wi = 0, lt = 0;
    // padded rows one window covers
    const int wrows_img = (p.nbox * p.box_rows + p.Wp - 1) / p.Wp + 1;
    for (int t = pair; t < p.num_tiles; t += p.num_pairs, ++lt) {
      // CTA tile 2t + rank = output rows [blk*tr, blk*tr + tr) of image n; its positions
      // start at coefficient n*L_A + blk*tr*sh*Wp (Eq. 12 base of output (blk*tr, 0))
      const int ct = 2 * t + (int)rank;
      const int tn = (int)p.ftpi.div((uint32_t)ct), tb = ct - tn * p.tpi;
      const int g0 = tn * (int)p.L_A + tb * p.tr * p.sh * p.Wp;
      __syncwarp();
      for (int ci = 0; ci < p.nchunks; ++ci, ++wi) {
        // one fixed (chunk, tap) order everywhere: every output sees the same
        // accumulation order whatever tile or batch it is computed in (reading R12)
        const int ch = ci;
        const int slot = wi % p.ring;
        mbar_wait_cl(wempty + slot, (uint32_t)((wi / p.ring) & 1) ^ 1u);
        if (elect_one()) {
          if (rank == 0) mbar_arrive_expect_tx(wfull + slot, 2u * p.wbytes_tx);
          for (int b = 0; b < p.nbox; ++b)
            tma_load_2d_pair(sW0 + (uint32_t)slot * p.wbytes + (uint32_t)(b * p.box_rows * p.row_bytes), &tmA,
                             lead_wfull + 8u * (uint32_t)slot, ch * p.kc, g0 + b * p.box_rows);
        }
        __syncwarp();
        if (elect_one()) {
          if (lt == 0 && !(f0_early && ci == 0)) {  // this chunk's filter blocks
            for (int tap = 0; tap < p.RS; ++tap) {
              const int blk = ch * p.RS + tap;
              if (rank == 0) mbar_arrive_expect_tx(ffull + blk, 2u * p.fbytes);
              tma_load_2d_pair(sF0 + (uint32_t)blk * p.fbytes, &tmU, lead_ffull + 8u * (uint32_t)blk, ch * p.kc,
                               tap * p.NN + (int)rank * half + (pair % p.urep) * p.RS * p.NN);
            }
          }
        }
        __syncwarp();
      }
    }
    if (trace && lane == 0) tr[15] = global_ns();
  } else if (warp == 1) {
    // ---------------------------------------------------- MMA issuer (leader CTA)
    if (rank == 0) {
      const uint32_t sW0 = smem_u32(sWin), sF0 = smem_u32(sF);
      const int ksteps = p.row_bytes / 32;
      int wi = 0, lt = 0;
      for (int t = pair; t < p.num_tiles; t += p.num_pairs, ++lt) {
        const int a = lt & 1;
        mbar_wait_cl(tempty + a, (uint32_t)((lt >> 1) & 1) ^ 1u);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + (uint32_t)(a * p.NN);
        for (int ci = 0; ci < p.nchunks; ++ci, ++wi) {
          const int ch = ci;  // the producer's order
          const int slot = wi % p.ring;
          mbar_wait_cl(wfull + slot, (uint32_t)((wi / p.ring) & 1));
          tc_fence_after();
          if (trace && lane == 0 && wi < 4) tr[3 + wi] = global_ns();
          if (lt == 0) {  // this chunk's filter blocks (first tile only; then resident)
            for (int tap = 0; tap < p.RS; ++tap) mbar_wait_cl(ffull + ch * p.RS + tap, 0u);
            tc_fence_after();
            if (trace && lane == 0 && ci == p.nchunks - 1) tr[12] = global_ns();
          }
          if (trace && lane == 0 && lt == 0 && ci < 2) g_pair_iss[blockIdx.x * 4 + 2 * ci] = global_ns();
          const uint64_t ad0 = make_sdesc(sW0 + (uint32_t)slot * p.wbytes, (uint32_t)p.row_bytes, 0);
          const uint64_t bd0 = make_sdesc(sF0 + (uint32_t)(ch * p.RS) * p.fbytes, (uint32_t)p.row_bytes, 0);
          issue_chunk(d_tmem, ad0, bd0, mtab, p.RS, ksteps, p.idesc, (uint32_t)ci);
          if (trace && lane == 0 && lt == 0 && ci < 2) g_pair_iss[blockIdx.x * 4 + 2 * ci + 1] = global_ns();
          if (elect_one()) umma2_commit_both(wempty + slot);  // window slot free in both CTAs
          __syncwarp();
        }
        if (elect_one()) umma2_commit_both(tfull + a);  // accumulator ready in both CTAs
        __syncwarp();
        if (trace && lane == 0 && lt < 2) tr[7 + lt] = global_ns();
      }
    }
  } else {
    // --------------------------------------------------------------- epilogue (a5)
    const int e = warp - kEpi0;
    const int q = warp & 3;       // TMEM lane quadrant this warp may access
    const int h = e >> 2;         // channel half
    const int half = p.NN / 2;
    const uint32_t lead_tempty = mapa_rank0(smem_u32(tempty));
    int lt = 0;
    for (int t = pair; t < p.num_tiles; t += p.num_pairs, ++lt) {
      const int a = lt & 1;
      mbar_wait_cl(tfull + a, (uint32_t)((lt >> 1) & 1), 64u);
      tc_fence_after();
      if (trace && threadIdx.x == kEpi0 * 32 && lt < 2) tr[9 + 2 * lt] = global_ns();
      // this lane's position m (tile-relative coefficient) -> output pixel (Eq. 12 with
      // stride, reading R4): row r = m / Wp, column s; valid on the stride lattice
      const int ct = 2 * t + (int)rank;
      const int tn = (int)p.ftpi.div((uint32_t)ct), tb = ct - tn * p.tpi;
      const int m = q * 32 + lane;
      const int r = (int)p.fWp.div((uint32_t)m), sc = m - r * p.Wp;
      const int ohr = (int)p.fsh.div((uint32_t)r), ow = (int)p.fsw.div((uint32_t)sc);
      const bool valid = ct < p.ntile && ohr * p.sh == r && ow * p.sw == sc && ohr < p.tr &&
                         tb * p.tr + ohr < p.P && ow < p.Q;
      const int j = ohr * p.Q + ow;  // pixel within the tile's run [tb*tr*Q, (tb*tr + tr)*Q)
      const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(a * p.NN + h * half);
      uint32_t v[64];
      tmem_ld32(taddr, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
      if (half > 32) tmem_ld32(taddr + 32u, *reinterpret_cast<uint32_t(*)[32]>(&v[32]));
      tmem_ld_wait();
      tc_fence_before();  // every TMEM read of this accumulator done: release it
      __syncwarp();
      if (lane == 0) mbar_arrive_remote(lead_tempty + 8u * (uint32_t)a);
      if (p.epi_tma) {
        // stage this half's channels [64][tr*Q] (bf16), then one thread stores the
        // 32-channel boxes; the staging is free once the previous stores were read
        const int trq = p.tr * p.Q;
        __nv_bfloat16* st = reinterpret_cast<__nv_bfloat16*>(sEpi) + (size_t)h * half * trq;
        const bool issuer = (e & 3) == 0 && lane == 0;
        if (issuer) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        asm volatile("bar.sync %0, 128;" ::"r"(1 + h) : "memory");
        if (valid) {
#pragma unroll
          for (int jj = 0; jj < 64; ++jj)
            if (jj < half) st[jj * trq + j] = __float2bfloat16_rn(__uint_as_float(v[jj]));
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("bar.sync %0, 128;" ::"r"(1 + h) : "memory");
        if (issuer && ct < p.ntile) {
          for (int b = 0; b < half / 32; ++b) {
            const int k0 = h * half + b * 32;
            if (k0 >= p.K) break;
            tma_store_2d(&tmY, smem_u32(st + (size_t)b * 32 * trq), tb * trq, tn * p.K + k0);
          }
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
      } else if (valid) {
        IoT* y = static_cast<IoT*>(p.y);
        const long long base = (long long)tn * p.K * p.PQ + (long long)(tb * p.tr + ohr) * p.Q + ow;
#pragma unroll
        for (int jj = 0; jj < 64; ++jj) {
          const int k = h * half + jj;
          if (jj < half && k < p.K) {
            const float f = __uint_as_float(v[jj]);
            if constexpr (std::is_same<IoT, float>::value) y[base + (long long)k * p.PQ] = f;
            else y[base + (long long)k * p.PQ] = __float2bfloat16_rn(f);
          }
        }
      }
      if (trace && threadIdx.x == kEpi0 * 32 && lt < 1) tr[10 + 2 * lt] = global_ns();
    }
    // the staging must outlive the stores' reads; the writes themselves complete with the grid
    if (p.epi_tma && (e & 3) == 0 && lane == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
  }

  tc_fence_before();
  __syncthreads();
  cluster_sync();  // the peer's MMAs / epilogue are done before TMEM is released
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc2(tmem_base, (uint32_t)p.tmem_cols);
  }
  if (trace && threadIdx.x == 0) {
    tr[13] = global_ns();
    g_pair_clk[blockIdx.x * 2 + 1] = clock64();
  }
}

// ---- host side ------------------------------------------------------------------
typedef CUresult (*EncodeTiledFnPair)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                      const cuuint64_t*, const cuuint32_t*, const cuuint32_t*,
                                      CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                                      CUtensorMapFloatOOBfill);

EncodeTiledFnPair get_encode_pair() {
  static EncodeTiledFnPair fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFnPair>(f);
  }
  return fn;
}

// bf16 2-D view [rows][cols], boxes of box_cols x box_rows, swizzle = row width
bool encode_bf16(CUtensorMap* map, const void* base, uint64_t cols, uint64_t rows, uint32_t box_cols,
                 uint32_t box_rows) {
  EncodeTiledFnPair enc = get_encode_pair();
  if (!enc) return false;
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {cols * 2};
  cuuint32_t box[2] = {box_cols, box_rows};
  cuuint32_t estr[2] = {1, 1};
  const uint32_t rb = box_cols * 2;
  CUtensorMapSwizzle sw = rb == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                          : rb == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                     : CU_TENSOR_MAP_SWIZZLE_32B;
  return enc(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
             CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

inline long long cdivp(long long a, long long b) { return (a + b - 1) / b; }

}  // namespace

PairTiling pair_tiling(const Geom& g, int fmt, bool io_bf16, int num_sms) {
  PairTiling t{};
  t.ok = false;
  if (fmt != FMT_BF16) return t;
  if (g.K > 128) return t;  // one output-channel tile of NN <= 128 (64 per CTA of the pair)
  t.kc = g.C >= 64 ? 64 : (g.C >= 32 ? 32 : 16);
  t.row_bytes = t.kc * 2;
  t.Cp = (int)cdivp(g.C, t.kc) * t.kc;
  t.NN = (int)std::max(64LL, cdivp(g.K, 64) * 64);  // halves of whole 32-column TMEM loads
  t.nchunks = t.Cp / t.kc;
  t.RS = g.R * g.S;
  t.nblk = t.nchunks * t.RS;
  if (t.nblk > kMaxBlk) return t;
  const long long wrows = kTileM + (long long)(g.R - 1) * g.Wp + (g.S - 1);
  if (wrows <= 256) {
    t.box_rows = (int)cdivp(wrows, 8) * 8;
    t.nbox = 1;
  } else {
    t.box_rows = 128;
    t.nbox = (int)cdivp(wrows, 128);
  }
  if (t.nbox > 8) return t;
  t.wbytes = (int)cdivp((long long)t.nbox * t.box_rows * t.row_bytes, 1024) * 1024;
  t.wbytes_tx = t.nbox * t.box_rows * t.row_bytes;
  t.fbytes = t.NN / 2 * t.row_bytes;
  const long long fil = (long long)t.nblk * t.fbytes;
  // row-aligned tiles: tr output rows of one image per CTA tile, every valid output
  // inside the 128 TMEM lanes: (tr-1)*sh*Wp + (Q-1)*sw + 1 <= 128
  if ((long long)(g.Q - 1) * g.sw + 1 > kTileM) return t;
  t.tr = 1;
  while ((long long)t.tr * g.sh * g.Wp + (long long)(g.Q - 1) * g.sw + 1 <= kTileM && t.tr < g.P) ++t.tr;
  t.tpi = (int)cdivp(g.P, t.tr);
  if ((long long)g.N * t.tpi >= (1LL << 30)) return t;
  t.ntile = g.N * t.tpi;
  // epilogue by TMA stores: y viewed as [N*K][P*Q] bf16, boxes of tr*Q pixels x 32 channels
  const long long trq = (long long)t.tr * g.Q;
  t.epi_tma = io_bf16 && g.K % 32 == 0 && (trq * 2) % 16 == 0 && ((long long)g.P * g.Q * 2) % 16 == 0 &&
              trq <= 256 && !getenv("POLYCONV_PAIR_EPI_ST");
  t.estage_bytes = t.epi_tma ? (int)(cdivp((long long)t.NN * trq * 2, 1024) * 1024) : 0;
  const long long budget = 227LL * 1024 - 1024 - 2048;  // alignment slack, barriers + tap table
  const long long left = budget - fil - t.estage_bytes;
  if (left < 2LL * t.wbytes) {
    if (!t.epi_tma) return t;
    t.epi_tma = 0;  // no room to stage the epilogue: direct stores
    t.estage_bytes = 0;
    if (budget - fil < 2LL * t.wbytes) return t;
  }
  t.ring = (int)std::min(4LL, (budget - fil - t.estage_bytes) / t.wbytes);
  t.smem_bytes = (int)(1024 + fil + (long long)t.ring * t.wbytes + t.estage_bytes + 2048);
  t.tmem_cols = 64;
  while (t.tmem_cols < 2 * t.NN) t.tmem_cols *= 2;
  if (t.tmem_cols > 512) return t;
  if ((long long)g.N * g.L_A + 4096 >= (1LL << 31)) return t;  // 32-bit TMA row coordinates / decode
  t.num_tiles = (int)cdivp(t.ntile, 2);
  t.num_pairs = std::min(t.num_tiles, num_sms / 2);
  t.grid = 2 * t.num_pairs;
  // packing bands: about one band per CTA, staged in the (then unused) operand area
  const long long stage_cap = fil + (long long)t.ring * t.wbytes + t.estage_bytes;
  t.nb = std::max(1, t.grid / g.N);
  if (t.nb > g.Hp) t.nb = g.Hp;
  for (;;) {
    t.rb = (int)cdivp(g.Hp, t.nb);
    t.spitch = (t.rb * g.W + 16) | 1;  // + rounding of the band to whole 16-byte vectors; odd
    if ((long long)t.Cp * t.spitch * 2 <= stage_cap || t.rb == 1) break;
    ++t.nb;
  }
  if ((long long)t.Cp * t.spitch * 2 > stage_cap) return t;
  t.nb = (int)cdivp(g.Hp, t.rb);
  t.nunits = g.N * t.nb;
  // TMA pack path: x band by one TMA box, A rows out by TMA stores (64-channel SW128 boxes).
  t.pack_tma = 0;
  t.u_img0 = 0;
  {
    const int eb_in = io_bf16 ? 2 : 4;
    const int ve = 16 / eb_in;
    const int rb_cap = std::min(256 / g.Wp, 256 / g.W);
    const bool tma_ok = t.Cp % 64 == 0 && t.Cp <= 256 && ((long long)g.H * g.W * eb_in) % 16 == 0 &&
                        !getenv("POLYCONV_PAIR_PACK_LD");
    {
      const int img0 = 0;
      const int nimg = g.N;
      int nb2 = std::max(1, nimg > 0 ? t.grid / nimg : 1);
      if (nb2 > g.Hp) nb2 = g.Hp;
      int rb2 = (int)cdivp(g.Hp, nb2);
      if (rb2 > rb_cap) rb2 = rb_cap;
      if (rb2 < 1 || !tma_ok) goto no_tma;
      const int nbb = (int)cdivp(g.Hp, rb2);
      const int last = g.Hp - (nbb - 1) * rb2;
      const int ne_box = (int)cdivp((long long)rb2 * g.W + ve - 1, ve) * ve;  // + the start's rounding
      const long long in_b = cdivp((long long)(t.Cp / 64) * 64 * ne_box * eb_in, 1024) * 1024;
      const long long ob = cdivp((long long)rb2 * g.Wp * 128, 1024) * 1024;
      const long long ob2 = cdivp((long long)last * g.Wp * 128, 1024) * 1024;
      const long long band_b = in_b + (long long)(t.Cp / 64) * std::max(ob, ob2);
      if (ne_box > 256 || band_b > stage_cap) goto no_tma;
      t.pack_tma = 1;
      t.u_img0 = img0;
      t.rb = rb2;
      t.nb = nbb;
      t.nunits = nimg * nbb;
      t.last_rows = last;
      t.ne_box = ne_box;
      t.in_bytes = (int)in_b;
      t.obox_bytes = (int)ob;
      t.obox_bytes2 = (int)ob2;
    }
  no_tma:;
  }
  // split: the packing runs as its own grid (pair_pack_kernel, several CTAs per SM,
  // small bands), the pair kernel follows it as a programmatic dependent launch.  This is
  // the only mode: the one-launch variant met on a grid counter and per-band flags, which
  // needed the whole grid co-resident and broke on CUDA-graph replay (the counters only
  // grew while the targets were baked into the captured launch); split measured 2% slower.
  t.split = 0;
  if (t.pack_tma) {
    const int eb_in = io_bf16 ? 2 : 4;
    const int ve = 16 / eb_in;
    const int rb_cap = std::min(256 / g.Wp, 256 / g.W);
    int nb2 = std::max(1, (4 * num_sms) / g.N);
    if (nb2 > g.Hp) nb2 = g.Hp;
    int rb2 = std::max(1, std::min((int)cdivp(g.Hp, nb2), rb_cap));
    const int nbb = (int)cdivp(g.Hp, rb2);
    const int last = g.Hp - (nbb - 1) * rb2;
    const int ne_box = (int)cdivp((long long)rb2 * g.W + ve - 1, ve) * ve;
    const long long in_b = cdivp((long long)(t.Cp / 64) * 64 * ne_box * eb_in, 1024) * 1024;
    const long long ob = cdivp((long long)rb2 * g.Wp * 128, 1024) * 1024;
    const long long ob2 = cdivp((long long)last * g.Wp * 128, 1024) * 1024;
    const long long band_b = in_b + (long long)(t.Cp / 64) * std::max(ob, ob2);
    if (ne_box <= 256 && band_b + 1024 <= 100 * 1024 && (long long)g.N * nbb < (1LL << 30)) {
      t.split = 1;
      t.u_img0 = 0;
      t.rb = rb2;
      t.nb = nbb;
      t.nunits = g.N * nbb;
      t.last_rows = last;
      t.ne_box = ne_box;
      t.in_bytes = (int)in_b;
      t.obox_bytes = (int)ob;
      t.obox_bytes2 = (int)ob2;
      t.pack_smem = (int)(band_b + 1024);
      t.pack_grid = std::max(t.nunits, num_sms);
    }
  }
  t.ok = t.split != 0;  // no split packing grid for this shape: not supported (no grid barrier)
  return t;
}

namespace {
// Everything a launch needs, built once per (x, w, y, workspace) pointer set: the host path
// of a repeated forward is two cudaLaunchKernelEx calls (tensor-map encoding and the
// cluster-occupancy check cost microseconds that an idle stream would wait for).
struct PairLaunchState {
  const void *x = nullptr, *w = nullptr, *y = nullptr, *A = nullptr, *U = nullptr;
  bool io_bf16 = false, valid = false;
  CUtensorMap tmA, tmU, tmX, tmS, tmS2, tmY;
  PairParams p;
};

cudaError_t prepare_mac_pair(PairLaunchState& S, const Geom& g, const PairTiling& t, const void* x, const void* w,
                             bool io_bf16, void* A, void* U, void* y, char* err, size_t errlen) {
  S.valid = false;
  CUtensorMap& tmA = S.tmA;
  CUtensorMap& tmU = S.tmU;
  if (!encode_bf16(&tmA, A, (uint64_t)t.Cp, (uint64_t)g.N * g.L_A, (uint32_t)t.kc, (uint32_t)t.box_rows) ||
      !encode_bf16(&tmU, U, (uint64_t)t.Cp, (uint64_t)g.urep * t.RS * t.NN, (uint32_t)t.kc, (uint32_t)(t.NN / 2))) {
    snprintf(err, errlen, "mac_pair: cuTensorMapEncodeTiled failed");
    return cudaErrorInvalidValue;
  }
  CUtensorMap& tmX = S.tmX;
  CUtensorMap& tmS = S.tmS;
  CUtensorMap& tmS2 = S.tmS2;
  memset(&tmX, 0, sizeof(tmX));
  memset(&tmS, 0, sizeof(tmS));
  memset(&tmS2, 0, sizeof(tmS2));
  if (t.pack_tma) {
    EncodeTiledFnPair enc = get_encode_pair();
    const int eb_in = io_bf16 ? 2 : 4;
    cuuint64_t dims[2] = {(cuuint64_t)g.H * g.W, (cuuint64_t)g.N * g.C};
    cuuint64_t strides[1] = {(cuuint64_t)g.H * g.W * eb_in};
    cuuint32_t box[2] = {(cuuint32_t)t.ne_box, 64};
    cuuint32_t estr[2] = {1, 1};
    bool ok = enc && enc(&tmX, io_bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2,
                         const_cast<void*>(x), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
    ok = ok && encode_bf16(&tmS, A, (uint64_t)t.Cp, (uint64_t)g.N * g.L_A, 64, (uint32_t)(t.rb * g.Wp)) &&
         encode_bf16(&tmS2, A, (uint64_t)t.Cp, (uint64_t)g.N * g.L_A, 64, (uint32_t)(t.last_rows * g.Wp));
    if (!ok) {
      snprintf(err, errlen, "mac_pair: cuTensorMapEncodeTiled (pack) failed");
      return cudaErrorInvalidValue;
    }
  }
  CUtensorMap& tmY = S.tmY;
  memset(&tmY, 0, sizeof(tmY));
  if (t.epi_tma) {
    EncodeTiledFnPair enc = get_encode_pair();
    cuuint64_t dims[2] = {(cuuint64_t)g.P * g.Q, (cuuint64_t)g.N * g.K};
    cuuint64_t strides[1] = {(cuuint64_t)g.P * g.Q * 2};
    cuuint32_t box[2] = {(cuuint32_t)(t.tr * g.Q), 32};
    cuuint32_t estr[2] = {1, 1};
    if (!enc || enc(&tmY, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, y, dims, strides, box, estr,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      snprintf(err, errlen, "mac_pair: cuTensorMapEncodeTiled (output) failed");
      return cudaErrorInvalidValue;
    }
  }
  PairParams& p = S.p;
  p = PairParams{};
  p.x = x; p.w = w; p.A = A; p.U = U; p.y = y;
  p.tr = t.tr; p.tpi = t.tpi; p.ntile = t.ntile; p.epi_tma = t.epi_tma;
  p.u_img0 = t.u_img0;
  p.split = t.split;
  p.estage_bytes = (uint32_t)t.estage_bytes;
  p.ftpi.init((uint32_t)t.tpi);
  p.pack_tma = t.pack_tma; p.ne_box = t.ne_box; p.last_rows = t.last_rows;
  p.in_bytes = (uint32_t)t.in_bytes; p.obox_bytes = (uint32_t)t.obox_bytes; p.obox_bytes2 = (uint32_t)t.obox_bytes2;
  p.L_A = g.L_A;
  p.G = (long long)(g.N - 1) * g.L_A + g.M_ext;
  p.NLA = (long long)g.N * g.L_A;
  p.N = g.N; p.C = g.C; p.H = g.H; p.W = g.W; p.K = g.K; p.R = g.R; p.S = g.S;
  p.sh = g.sh; p.sw = g.sw; p.ph = g.ph; p.pw = g.pw; p.Hp = g.Hp; p.Wp = g.Wp; p.P = g.P; p.Q = g.Q;
  p.PQ = g.P * g.Q;
  p.Cp = t.Cp; p.NN = t.NN; p.kc = t.kc; p.row_bytes = t.row_bytes; p.nchunks = t.nchunks; p.RS = t.RS;
  p.nblk = t.nblk; p.box_rows = t.box_rows; p.nbox = t.nbox;
  p.wbytes = (uint32_t)t.wbytes; p.wbytes_tx = (uint32_t)t.wbytes_tx; p.fbytes = (uint32_t)t.fbytes;
  p.ring = t.ring; p.num_tiles = t.num_tiles; p.num_pairs = t.num_pairs;
  p.urep = g.urep;
  // instruction descriptor: D=f32 @4, A/B = bf16 @7/@10, both K-major, N>>3 @17, M>>4 @24 (M = 256)
  p.idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(t.NN >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
  p.tmem_cols = t.tmem_cols;
  p.rb = t.rb; p.nb = t.nb; p.nunits = t.nunits; p.spitch = t.spitch;
  p.fLA.init((uint32_t)g.L_A);
  p.fWp.init((uint32_t)g.Wp);
  p.fsh.init((uint32_t)g.sh);
  p.fsw.init((uint32_t)g.sw);
  auto kern = io_bf16 ? mac_pair_kernel<__nv_bfloat16> : mac_pair_kernel<float>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, t.smem_bytes);
  if (e != cudaSuccess) return e;
  if (t.split) {
    auto pk = io_bf16 ? pair_pack_kernel<__nv_bfloat16> : pair_pack_kernel<float>;
    e = cudaFuncSetAttribute(pk, cudaFuncAttributeMaxDynamicSharedMemorySize, t.pack_smem);
    if (e != cudaSuccess) return e;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)t.grid);
  cfg.blockDim = dim3(kPairThreads);
  cfg.dynamicSmemBytes = (size_t)t.smem_bytes;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  // the grid counter needs every CTA co-resident
  int max_clusters = 0;
  if (cudaOccupancyMaxActiveClusters(&max_clusters, kern, &cfg) == cudaSuccess && max_clusters > 0 &&
      max_clusters < t.num_pairs) {
    snprintf(err, errlen, "mac_pair: only %d co-resident clusters for %d pairs", max_clusters, t.num_pairs);
    return cudaErrorInvalidConfiguration;
  }
  cudaGetLastError();
  S.x = x; S.w = w; S.y = y; S.A = A; S.U = U; S.io_bf16 = io_bf16;
  S.valid = true;
  return cudaSuccess;
}
}  // namespace

void* pair_state_new() { return new (std::nothrow) PairLaunchState(); }
void pair_state_free(void* s) { delete static_cast<PairLaunchState*>(s); }

cudaError_t launch_mac_pair(const Geom& g, const PairTiling& t, const void* x, const void* w, bool io_bf16,
                            void* A, void* U, void* y, cudaStream_t st, char* err, size_t errlen, void* state) {
  if (!t.ok) {
    snprintf(err, errlen, "mac_pair: shape not supported");
    return cudaErrorInvalidValue;
  }
  PairLaunchState local;
  PairLaunchState& S = state ? *static_cast<PairLaunchState*>(state) : local;
  if (!S.valid || S.x != x || S.w != w || S.y != y || S.A != A || S.U != U ||
      S.io_bf16 != io_bf16) {
    cudaError_t e = prepare_mac_pair(S, g, t, x, w, io_bf16, A, U, y, err, errlen);
    if (e != cudaSuccess) return e;
  }
  const char* dbg = getenv("POLYCONV_PAIR_DEBUG");
  S.p.dbg = dbg ? atoi(dbg) : 0;
  if (t.split) {
    auto pk = io_bf16 ? pair_pack_kernel<__nv_bfloat16> : pair_pack_kernel<float>;
    cudaLaunchConfig_t pc = {};
    pc.gridDim = dim3((unsigned)t.pack_grid);
    pc.blockDim = dim3(256);
    pc.dynamicSmemBytes = (size_t)t.pack_smem;
    pc.stream = st;
    cudaError_t e = cudaLaunchKernelEx(&pc, pk, S.tmX, S.tmS, S.tmS2, S.p);
    if (e != cudaSuccess) return e;
  }
  auto kern = io_bf16 ? mac_pair_kernel<__nv_bfloat16> : mac_pair_kernel<float>;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)t.grid);
  cfg.blockDim = dim3(kPairThreads);
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
  cfg.numAttrs = t.split ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, S.tmA, S.tmU, S.tmX, S.tmS, S.tmS2, S.tmY, S.p);
}

}  // namespace polyconv

// Debug only (not part of include/polyconv.h): the per-CTA phase trace of the
// last POLYCONV_PAIR_DEBUG&8 launch (160 x 16 u64).
extern "C" int polyconv_dbg_pair_iss(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_pair_iss, sizeof(unsigned long long) * 160 * 4);
}
extern "C" int polyconv_dbg_pair_pk(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_pair_pk, sizeof(unsigned long long) * 160 * 4);
}
extern "C" int polyconv_dbg_pair_clk(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_pair_clk, sizeof(unsigned long long) * 160 * 2);
}
extern "C" int polyconv_dbg_pair_trace(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_pair_trace, sizeof(unsigned long long) * 160 * polyconv::kTr);
}
