// mac_pair.cu — the BF16 hot path in ONE launch on CTA pairs (tcgen05
// cta_group::2): a2 + a3 packing, a4 coefficient MAC, a5 extraction.
//
// The coefficient MAC
//   p_{n,k}[m] = sum_c sum_{i,j} A_{n,c}[m - e(i,j)] * U_{k,c}[e(i,j)]   (P.965, P.1350-1352)
// is, per kernel tap (i,j), a GEMM over channels whose position operand is the
// input polynomial shifted by Wp*i + j coefficients (the doubly blocked Hankel
// structure, P.404-437):
//   D[pos][k] += sum_c A[pos + Wp*i + j][c] * U_tap(i,j)[k][c]
// with pos = the base coefficient m - (L_U - 1) of an output (Eq. 12).
//
// Design (DESIGN.md §4 "mac_pair"):
//  * Phase 1 (every CTA, all warps): pack a slice of the filter into the
//    tap-major layout U[R*S][NN][Cp] (a3: the nonzero coefficients of the
//    reversed, gap-padded U_{k,c}(t), Eq. 6, grouped by degree e(i,j)) and a
//    band of images rows into the channel-interleaved input polynomial
//    A[N*L_A][Cp] (a2: coefficient r*Wp + s of A_{n,c}(t) = xpad[n][c][r][s],
//    Eq. 10 + zero padding P.1353-1356), converted to BF16 (RNE, reading R11).
//    The packed copies are written to the plan workspace (they stay in L2);
//    the CTAs then meet on a grid counter (all CTAs are co-resident: one per
//    SM, grid <= the co-resident cluster count).
//  * Phase 2 (CTA pairs): UMMA M = 256 positions (128 per CTA: A operand =
//    a window of the interleaved input, K-major, loaded by TMA), N = NN output
//    channels (B operand = the filter, each CTA holding NN/2 rows of every
//    (tap, channel chunk) block -- RESIDENT in shared memory for the whole
//    kernel: loaded once, reused by every tile).  One window of
//    128 + (R-1)*Wp + S-1 positions per channel chunk serves all R*S taps: each
//    tap's MMA reads it through a descriptor whose start is shifted by
//    (Wp*i + j) rows (tools/umma_probe.cu).  The leader CTA issues
//    tcgen05.mma.cta_group::2; accumulators (fp32) live in TMEM, double
//    buffered, so the epilogue of tile t overlaps the MMAs of tile t+1.
//  * Epilogue (a5, fused): positions are TMEM lanes, so every warp-wide store
//    of one output channel writes 32 consecutive output pixels (Eq. 12 /
//    reading R4 extraction: y[n][k][oh][ow] = p[Wp*sh*oh + sw*ow + L_U - 1];
//    positions off the lattice are junk and dropped).
//  * Warp roles: warp 0 = TMA producer, warp 1 = TMEM allocator + MMA issuer
//    (leader CTA), warps 2..9 = epilogue (2 per TMEM lane quadrant, each half
//    of the channels).  All ten warps pack in phase 1.
#include <cuda.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <algorithm>
#include <type_traits>
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
  unsigned long long* fcount;
  unsigned long long ftarget;
  long long L_A, G, NLA;
  int N, C, H, W, K, R, S, sh, sw, ph, pw, Hp, Wp, P, Q, PQ;
  int Cp, NN, kc, row_bytes, nchunks, RS, nblk;
  int box_rows, nbox;
  uint32_t wbytes, wbytes_tx, fbytes;
  int ring, num_tiles, num_pairs;
  uint32_t idesc;
  int tmem_cols;
  int rb, nb, nunits, spitch;
  FastDiv fLA, fWp, fsh, fsw;
  int dbg;
};

// per-CTA phase trace (POLYCONV_PAIR_DEBUG & 8), globaltimer ns:
// 0 start, 1 pack done, 2 grid counter passed, 3-6 windows 0-3 landed (leader),
// 7/8 tile 0/1 MMAs issued (leader), 9/11 tile 0/1 accumulator ready (epilogue),
// 10/12 tile 0/1 stores done (epilogue warp 0), 13 end, 14 last filter block landed
// (leader), 15 last window TMA issued (producer)
constexpr int kTr = 16;
__device__ unsigned long long g_pair_trace[160 * kTr];
__device__ unsigned long long g_pair_clk[160 * 2];  // clock64 at tr[0] and tr[13]: SM clock = cycles / ns

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
  uint32_t spins = 0;
  uint64_t t0 = 0;
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
    if ((++spins & 0xFFFu) == 0 || sleep_ns) {
      const uint64_t t = global_ns();
      if (t0 == 0) t0 = t;
      else if (t - t0 > 500000000ull) __trap();
    }
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
__device__ __forceinline__ void pair_pack(const PairParams& p, uint16_t* stg) {
  const int tid = threadIdx.x;
  const int nth = blockDim.x;
  // a3: U[tap][k][c] = w[k][c][tap] (tap = i*S + j; k >= K or c >= C: 0)
  {
    const IoT* w = static_cast<const IoT*>(p.w);
    uint16_t* U = static_cast<uint16_t*>(p.U);
    const int nkc = p.NN * p.Cp;
    for (int idx = blockIdx.x * nth + tid; idx < nkc; idx += gridDim.x * nth) {
      const int k = idx / p.Cp, c = idx - (idx / p.Cp) * p.Cp;
      const bool ok = k < p.K && c < p.C;
      const IoT* src = w + ((long long)k * p.C + c) * p.RS;
      for (int t = 0; t < p.RS; ++t)
        U[((long long)t * p.NN + k) * p.Cp + c] = ok ? to_bf16_bits<IoT>(src[t]) : (uint16_t)0;
    }
  }
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
  }
}

template <typename IoT>
__global__ void __launch_bounds__(kPairThreads, 1)
    mac_pair_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmU,
                    const PairParams p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  uint8_t* sF = smem;                                        // filter blocks [nblk][NN/2][row]
  uint8_t* sWin = sF + (size_t)p.nblk * p.fbytes;            // window ring [ring][rows][row]
  uint64_t* bars = reinterpret_cast<uint64_t*>(sWin + (size_t)p.ring * p.wbytes);
  uint64_t* ffull = bars;                 // [kMaxBlk] filter block landed (leader: both halves)
  uint64_t* wfull = ffull + kMaxBlk;      // [ring] window landed (leader: both CTAs' windows)
  uint64_t* wempty = wfull + 8;           // [ring] window consumed (both CTAs, MMA commit)
  uint64_t* tfull = wempty + 8;           // [2] accumulator ready (both CTAs, MMA commit)
  uint64_t* tempty = tfull + 2;           // [2] accumulator drained (leader: 16 epilogue warps)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  uint32_t* mtab = tmem_slot + 4;  // [kMaxBlk][2]: per rotated tap, A shift and B offset (16-byte units)

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
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc2(tmem_slot, (uint32_t)p.tmem_cols);

  // phase 1: packing (all warps); the window ring and filter area are the staging buffer
  if (!(p.dbg & 2)) pair_pack<IoT>(p, reinterpret_cast<uint16_t*>(sF));  // dbg&2: skip (timing only)
  // the staging area is overwritten by TMA (async proxy) next
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(p.fcount, 1ull);
  }
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
    if ((p.dbg & 1) && elect_one()) {  // timing experiment: filter loads before the pack is done (stale U)
      for (int ch = 0; ch < p.nchunks; ++ch)
        for (int tap = 0; tap < p.RS; ++tap) {
          const int blk = ch * p.RS + tap;
          if (rank == 0) mbar_arrive_expect_tx(ffull + blk, 2u * p.fbytes);
          tma_load_2d_pair(sF0 + (uint32_t)blk * p.fbytes, &tmU, lead_ffull + 8u * (uint32_t)blk, ch * p.kc,
                           tap * p.NN + (int)rank * half);
        }
    }
    __syncwarp();
    if (lane == 0) {
      unsigned long long v;
      uint64_t t0 = 0;
      for (;;) {
        asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p.fcount) : "memory");
        if (v >= p.ftarget) break;
        const uint64_t t = global_ns();
        if (t0 == 0) t0 = t;
        else if (t - t0 > 500000000ull) __trap();
      }
      asm volatile("fence.proxy.async.global;" ::: "memory");  // generic writes -> TMA reads
      if (trace) tr[2] = global_ns();
    }
    __syncwarp();
    int wi = 0, lt = 0;
    for (int t = pair; t < p.num_tiles; t += p.num_pairs, ++lt) {
      const int g0 = t * (2 * kTileM) + (int)rank * kTileM;
      for (int ci = 0; ci < p.nchunks; ++ci, ++wi) {
        // every pair walks the (chunk, tap) blocks in its own rotated order, so
        // that the 148 CTAs do not all stream the same filter lines at once
        const int ch = (ci + pair) % p.nchunks;
        const int slot = wi % p.ring;
        mbar_wait_cl(wempty + slot, (uint32_t)((wi / p.ring) & 1) ^ 1u, (p.dbg & 16) ? 500u : 0u);
        if (elect_one()) {
          if (rank == 0) mbar_arrive_expect_tx(wfull + slot, 2u * p.wbytes_tx);
          for (int b = 0; b < p.nbox; ++b)
            tma_load_2d_pair(sW0 + (uint32_t)slot * p.wbytes + (uint32_t)(b * p.box_rows * p.row_bytes), &tmA,
                             lead_wfull + 8u * (uint32_t)slot, ch * p.kc, g0 + b * p.box_rows);
          if (lt == 0 && !(p.dbg & 1)) {  // the filter blocks of this chunk: loaded once, resident
            for (int ti = 0; ti < p.RS; ++ti) {
              const int tap = (ti + pair) % p.RS;
              const int blk = ch * p.RS + tap;
              if (rank == 0) mbar_arrive_expect_tx(ffull + blk, 2u * p.fbytes);
              tma_load_2d_pair(sF0 + (uint32_t)blk * p.fbytes, &tmU, lead_ffull + 8u * (uint32_t)blk, ch * p.kc,
                               tap * p.NN + (int)rank * half);
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
      // descriptor offsets of the pair's rotated tap order, so that the issue loop
      // is a few uniform adds per tap (divisions in it left the tensor pipe idle)
      for (int ti = lane; ti < p.RS; ti += 32) {
        const int tap = (ti + pair) % p.RS;
        const int i = tap / p.S, j = tap - (tap / p.S) * p.S;
        mtab[2 * ti] = ((uint32_t)(p.Wp * i + j) * (uint32_t)p.row_bytes) >> 4;
        mtab[2 * ti + 1] = ((uint32_t)tap * p.fbytes) >> 4;
      }
      __syncwarp();
      int wi = 0, lt = 0;
      for (int t = pair; t < p.num_tiles; t += p.num_pairs, ++lt) {
        const int a = lt & 1;
        if (!(p.dbg & 4)) mbar_wait_cl(tempty + a, (uint32_t)((lt >> 1) & 1) ^ 1u);  // dbg&4: no waits (timing)
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + (uint32_t)(a * p.NN);
        for (int ci = 0; ci < p.nchunks; ++ci, ++wi) {
          const int ch = (ci + pair) % p.nchunks;  // the producer's rotated order
          const int slot = wi % p.ring;
          if (!(p.dbg & 4)) mbar_wait_cl(wfull + slot, (uint32_t)((wi / p.ring) & 1));
          tc_fence_after();
          if (trace && lane == 0 && wi < 4) tr[3 + wi] = global_ns();
          if (lt == 0 && !(p.dbg & 4)) {  // this chunk's filter blocks (first tile only; then resident)
            for (int tap = 0; tap < p.RS; ++tap) mbar_wait_cl(ffull + ch * p.RS + tap, 0u);
            tc_fence_after();
            if (trace && lane == 0 && ci == p.nchunks - 1) tr[14] = global_ns();
          }
          const uint64_t ad0 = make_sdesc(sW0 + (uint32_t)slot * p.wbytes, (uint32_t)p.row_bytes, 0);
          const uint64_t bd0 = make_sdesc(sF0 + (uint32_t)(ch * p.RS) * p.fbytes, (uint32_t)p.row_bytes, 0);
          for (int ti = 0; ti < p.RS; ++ti) {
            const uint64_t ad = ad0 + mtab[2 * ti], bd = bd0 + mtab[2 * ti + 1];
            const uint32_t acc0 = (ci | ti) != 0 ? 1u : 0u;
            if (elect_one()) {
              umma2_f16(d_tmem, ad, bd, p.idesc, acc0);
              // K step = 32 bytes = +2 in the start field
              if (ksteps > 1) umma2_f16(d_tmem, ad + 2, bd + 2, p.idesc, 1u);
              if (ksteps > 2) {
                umma2_f16(d_tmem, ad + 4, bd + 4, p.idesc, 1u);
                umma2_f16(d_tmem, ad + 6, bd + 6, p.idesc, 1u);
              }
            }
            __syncwarp();
          }
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
    IoT* y = static_cast<IoT*>(p.y);
    int lt = 0;
    for (int t = pair; t < p.num_tiles; t += p.num_pairs, ++lt) {
      const int a = lt & 1;
      mbar_wait_cl(tfull + a, (uint32_t)((lt >> 1) & 1), (p.dbg & 16) ? 1000u : 64u);
      tc_fence_after();
      if (trace && threadIdx.x == kEpi0 * 32 && lt < 2) tr[9 + 2 * lt] = global_ns();
      // this lane's position -> output pixel (Eq. 12 with stride, reading R4)
      const long long gpos = (long long)t * (2 * kTileM) + rank * kTileM + q * 32 + lane;
      long long base = -1;
      if (gpos < p.G) {
        const int n = (int)p.fLA.div((uint32_t)gpos);
        const int rem = (int)(gpos - (long long)n * p.L_A);
        const int r = (int)p.fWp.div((uint32_t)rem), s = rem - r * p.Wp;
        const int oh = (int)p.fsh.div((uint32_t)r), ow = (int)p.fsw.div((uint32_t)s);
        if (oh * p.sh == r && ow * p.sw == s && oh < p.P && ow < p.Q)
          base = (long long)n * p.K * p.PQ + (long long)oh * p.Q + ow;
      }
      const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(a * p.NN + h * half);
      for (int cc = 0; cc < half; cc += 32) {
        uint32_t v[32];
        tmem_ld32(taddr + (uint32_t)cc, v);
        tmem_ld_wait();
        if (cc + 32 >= half) {  // every TMEM read of this accumulator done: release it
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive_remote(lead_tempty + 8u * (uint32_t)a);
        }
        const int k0 = h * half + cc;
        if (base >= 0) {
#pragma unroll
          for (int jj = 0; jj < 32; ++jj) {
            const int k = k0 + jj;
            if (k < p.K) {
              const float f = __uint_as_float(v[jj]);
              if constexpr (std::is_same<IoT, float>::value) y[base + (long long)k * p.PQ] = f;
              else y[base + (long long)k * p.PQ] = __float2bfloat16_rn(f);
            }
          }
        }
      }
      if (trace && threadIdx.x == kEpi0 * 32 && lt < 2) tr[10 + 2 * lt] = global_ns();
    }
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

PairTiling pair_tiling(const Geom& g, int fmt, int num_sms) {
  PairTiling t{};
  t.ok = false;
  if (fmt != FMT_BF16) return t;
  if (g.K > 256) return t;
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
  const long long budget = 227LL * 1024 - 1024 - 2048;  // alignment slack, barriers + tap table
  const long long left = budget - fil;
  if (left < 2LL * t.wbytes) return t;
  t.ring = (int)std::min(4LL, left / t.wbytes);
  t.smem_bytes = (int)(1024 + fil + (long long)t.ring * t.wbytes + 2048);
  t.tmem_cols = 64;
  while (t.tmem_cols < 2 * t.NN) t.tmem_cols *= 2;
  if (t.tmem_cols > 512) return t;
  const long long G = (long long)(g.N - 1) * g.L_A + g.M_ext;
  if ((long long)g.N * g.L_A + 4096 >= (1LL << 31)) return t;  // 32-bit TMA row coordinates / decode
  t.num_tiles = (int)cdivp(G, 2 * kTileM);
  t.num_pairs = std::min(t.num_tiles, num_sms / 2);
  t.grid = 2 * t.num_pairs;
  // packing bands: about one band per CTA, staged in the (then unused) operand area
  const long long stage_cap = fil + (long long)t.ring * t.wbytes;
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
  t.ok = true;
  return t;
}

cudaError_t launch_mac_pair(const Geom& g, const PairTiling& t, const void* x, const void* w, bool io_bf16,
                            void* A, void* U, void* y, unsigned long long* fcount, unsigned long long ftarget,
                            cudaStream_t st, char* err, size_t errlen) {
  if (!t.ok) {
    snprintf(err, errlen, "mac_pair: shape not supported");
    return cudaErrorInvalidValue;
  }
  CUtensorMap tmA, tmU;
  if (!encode_bf16(&tmA, A, (uint64_t)t.Cp, (uint64_t)g.N * g.L_A, (uint32_t)t.kc, (uint32_t)t.box_rows) ||
      !encode_bf16(&tmU, U, (uint64_t)t.Cp, (uint64_t)t.RS * t.NN, (uint32_t)t.kc, (uint32_t)(t.NN / 2))) {
    snprintf(err, errlen, "mac_pair: cuTensorMapEncodeTiled failed");
    return cudaErrorInvalidValue;
  }
  PairParams p{};
  p.x = x; p.w = w; p.A = A; p.U = U; p.y = y;
  p.fcount = fcount; p.ftarget = ftarget;
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
  // instruction descriptor: D=f32 @4, A/B = bf16 @7/@10, both K-major, N>>3 @17, M>>4 @24 (M = 256)
  p.idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(t.NN >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
  p.tmem_cols = t.tmem_cols;
  p.rb = t.rb; p.nb = t.nb; p.nunits = t.nunits; p.spitch = t.spitch;
  p.fLA.init((uint32_t)g.L_A);
  p.fWp.init((uint32_t)g.Wp);
  p.fsh.init((uint32_t)g.sh);
  p.fsw.init((uint32_t)g.sw);
  const char* dbg = getenv("POLYCONV_PAIR_DEBUG");
  p.dbg = dbg ? atoi(dbg) : 0;
  auto kern = io_bf16 ? mac_pair_kernel<__nv_bfloat16> : mac_pair_kernel<float>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, t.smem_bytes);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)t.grid);
  cfg.blockDim = dim3(kPairThreads);
  cfg.dynamicSmemBytes = (size_t)t.smem_bytes;
  cfg.stream = st;
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
  return cudaLaunchKernelEx(&cfg, kern, tmA, tmU, p);
}

}  // namespace polyconv

// Debug only (not part of include/polyconv.h): the per-CTA phase trace of the
// last POLYCONV_PAIR_DEBUG&8 launch (160 x 16 u64).
extern "C" int polyconv_dbg_pair_clk(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_pair_clk, sizeof(unsigned long long) * 160 * 2);
}
extern "C" int polyconv_dbg_pair_trace(unsigned long long* host) {
  return (int)cudaMemcpyFromSymbol(host, polyconv::g_pair_trace, sizeof(unsigned long long) * 160 * polyconv::kTr);
}
