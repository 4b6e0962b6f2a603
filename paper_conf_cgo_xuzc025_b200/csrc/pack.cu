// pack.cu — a2/a3: build the paper's polynomials from x and w.
//
//  A_{n,c}(t): coefficient r*Wp + s = xpad[n][c][r][s]       (Eq. 10, P.941-950;
//              zero padding P.1353-1356, Fig. 1; Iw := Wp, reading R2)
//  U_{k,c}(t): coefficient e(i,j) = Wp*(R-1-i) + (S-1-j) = w[k][c][i][j]
//              (Eq. 6 P.768-771, reversed + gap-padded kernel P.1365-1382;
//               Eq. 11 corrected, reading R1)
// Conversion to the math mode's operand format happens here (reading R11):
// fp32 stays fp32, TF32 = cvt.rna, BF16 = RNE.  All kernels are pure copies
// with index math (HBM-bound); the outputs are bit-exact by construction.
#include <cuda.h>
#include <algorithm>
#include <cstdlib>
#include "common.cuh"
#include "sm100.cuh"

namespace polyconv {

namespace {

constexpr int kThreads = 256;

inline unsigned grid_for(long long total, int per_block) {
  long long b = (total + per_block - 1) / per_block;
  if (b > (1LL << 20)) b = 1LL << 20;  // grid-stride beyond this
  return (unsigned)(b < 1 ? 1 : b);
}

// ---- planar input [N][C][L_A] ---------------------------------------------
// Grid over (plane n*C+c, padded row r): one block row writes the Wp
// coefficients r*Wp .. r*Wp+Wp-1 of A_{n,c}(t); 32-bit index math (the plan
// guarantees every tensor indexes below 2^31).
template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_input_planar_kernel(Geom g, const InT* __restrict__ x,
                                                                     typename Word<F>::T* __restrict__ dst) {
  const int rows = g.N * g.C * g.Hp;  // (plane, padded row) pairs
  const int per = kThreads / g.Wp;  // rows per block (0: rows wider than the block)
  if (per >= 1) {
    // several rows per block: thread -> (row, s)
    const int sub = threadIdx.x / g.Wp, s = threadIdx.x - sub * g.Wp;
    if (sub >= per) return;
    for (int rr = blockIdx.x * per + sub; rr < rows; rr += gridDim.x * per) {
      const int nc = rr / g.Hp, r = rr - nc * g.Hp;
      const int h = r - g.ph, w = s - g.pw;
      float v = 0.f;
      if (h >= 0 && h < g.H && w >= 0 && w < g.W) v = load_io(x, ((long long)nc * g.H + h) * g.W + w);
      dst[(long long)nc * g.L_A + (long long)r * g.Wp + s] = Word<F>::enc(v);
    }
  } else {
    // wide rows: a block per row
    for (int rr = blockIdx.x; rr < rows; rr += gridDim.x) {
      const int nc = rr / g.Hp, r = rr - nc * g.Hp;
      const int h = r - g.ph;
      for (int s = threadIdx.x; s < g.Wp; s += kThreads) {
        const int w = s - g.pw;
        float v = 0.f;
        if (h >= 0 && h < g.H && w >= 0 && w < g.W) v = load_io(x, ((long long)nc * g.H + h) * g.W + w);
        dst[(long long)nc * g.L_A + (long long)r * g.Wp + s] = Word<F>::enc(v);
      }
    }
  }
}

// ---- interleaved input [N*L_A][Cp] ------------------------------------------
// One block per (image n, chunk of kRowCh channels, band of `rb` padded rows):
// the block stages the band's input rows -- a contiguous run of rb*W elements
// per channel plane -- in shared memory (coalesced, sequential reads), then
// writes the band's rb*Wp output coefficients, each as 16-byte chunks of
// consecutive channels.  Padding rows/columns (Eq. 10 + reading R3) and
// channels C..Cp-1 are written as zeros.  32-bit index math (the plan
// guarantees every count < 2^31).
constexpr int kRowCh = 64;
constexpr int kBandBytes = 32 * 1024;  // staged bytes per block: kRowCh planes x rb rows

__device__ __forceinline__ float to_f32(float v) { return v; }
__device__ __forceinline__ uint32_t word_bits(float w) { return __float_as_uint(w); }
__device__ __forceinline__ uint32_t word_bits(uint32_t w) { return w; }
__device__ __forceinline__ uint32_t word_bits(__nv_bfloat16 w) { return (uint32_t)__bfloat16_as_ushort(w); }
__device__ __forceinline__ float to_f32(__nv_bfloat16 v) { return __bfloat162float(v); }

struct BandGeom {
  int rb;     // padded rows per band
  int nband;  // bands per image
  int nch;    // channel chunks
  int tw;     // staged elements per channel (rb*W rounded to an odd number of words)
};

inline BandGeom band_geom(const Geom& g, int elem_bytes) {
  BandGeom b;
  const int elems = kBandBytes / (kRowCh * elem_bytes);  // staged elements per channel
  b.rb = g.W >= elems ? 1 : elems / g.W;
  if (b.rb > g.Hp) b.rb = g.Hp;
  b.nband = (g.Hp + b.rb - 1) / b.rb;
  b.nch = (g.Cp + kRowCh - 1) / kRowCh;
  int tw = (b.rb * g.W + 1) & ~1;
  if (((tw / 2) & 1) == 0) tw += 2;
  b.tw = tw;
  return b;
}

template <typename InT, int F>
__device__ __forceinline__ void pack_band(const Geom& g, const BandGeom& bg, const InT* __restrict__ x,
                                          typename Word<F>::T* __restrict__ dst, int blk, InT* tile) {
  using WT = typename Word<F>::T;
  constexpr int EPC = 16 / (int)sizeof(WT);  // channels per 16-byte chunk
  const int band = blk % bg.nband;
  const int rest = blk / bg.nband;
  const int chunk = rest % bg.nch, n = rest / bg.nch;
  const int pr0 = band * bg.rb, pr1 = min(g.Hp, pr0 + bg.rb);  // padded rows of this band
  const int h0 = max(0, pr0 - g.ph), h1 = min(g.H, pr1 - g.ph);  // input rows they contain
  const int c0 = chunk * kRowCh;
  const int cw = min(kRowCh, g.Cp - c0);         // channels of this chunk in the output
  const int cv = max(0, min(kRowCh, g.C - c0));  // of which real
  const int nel = h1 > h0 ? (h1 - h0) * g.W : 0;  // contiguous elements per channel plane
  {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const InT* src = x + ((size_t)(n * g.C + c0) * g.H + h0) * g.W;
    const int cs = g.H * g.W;
    for (int c = warp; c < cv; c += kThreads / 32) {
      const InT* sc = src + (size_t)c * cs;
      InT* tc = tile + c * bg.tw;
      for (int e0 = 0; e0 < nel; e0 += 4 * 32) {  // four independent loads in flight per lane
        InT v[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int e = e0 + k * 32 + lane;
          if (e < nel) v[k] = sc[e];
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int e = e0 + k * 32 + lane;
          if (e < nel) tc[e] = v[k];
        }
      }
    }
  }
  __syncthreads();
  WT* out = dst + ((size_t)n * (size_t)g.L_A + (size_t)(pr0 * g.Wp)) * g.Cp + c0;
  const int npos = (pr1 - pr0) * g.Wp;
  if (g.Cp % EPC == 0) {
    // 16-byte chunks of EPC consecutive channels (Cp is a multiple of EPC)
    const int cpp = cw / EPC;
    const bool pow2 = (cpp & (cpp - 1)) == 0;
    const int sh = __ffs(cpp) - 1;
    const int total = npos * cpp;
    for (int u = threadIdx.x; u < total; u += kThreads) {
      const int pos = pow2 ? (u >> sh) : u / cpp, cg = u - pos * cpp;
      const int r = pos / g.Wp, ps = pos - r * g.Wp;
      const int h = pr0 + r - g.ph, w = ps - g.pw;
      const bool in = h >= h0 && h < h1 && w >= 0 && w < g.W;
      const int e = (h - h0) * g.W + w;
      uint32_t word[EPC];
#pragma unroll
      for (int t = 0; t < EPC; ++t) {
        const int c = cg * EPC + t;
        const float v = (in && c < cv) ? to_f32(tile[c * bg.tw + e]) : 0.f;
        word[t] = word_bits(Word<F>::enc(v));
      }
      uint4 q;
      if constexpr (sizeof(WT) == 2)
        q = make_uint4(word[0] | (word[1] << 16), word[2] | (word[3] << 16), word[4] | (word[5] << 16),
                       word[6] | (word[7] << 16));
      else
        q = make_uint4(word[0], word[1], word[2], word[3]);
      *reinterpret_cast<uint4*>(out + pos * g.Cp + cg * EPC) = q;
    }
  } else {
    // unaligned channel count (thin plans): one word per thread
    const int total = npos * cw;
    for (int u = threadIdx.x; u < total; u += kThreads) {
      const int pos = u / cw, c = u - pos * cw;
      const int r = pos / g.Wp, ps = pos - r * g.Wp;
      const int h = pr0 + r - g.ph, w = ps - g.pw;
      const bool in = h >= h0 && h < h1 && w >= 0 && w < g.W && c < cv;
      out[pos * g.Cp + c] = Word<F>::enc(in ? to_f32(tile[c * bg.tw + (h - h0) * g.W + w]) : 0.f);
    }
  }
  __syncthreads();
}

template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_input_interleaved_kernel(Geom g, BandGeom bg,
                                                                          const InT* __restrict__ x,
                                                                          typename Word<F>::T* __restrict__ dst) {
  extern __shared__ __align__(16) unsigned char pk_smem[];
  InT* tile = reinterpret_cast<InT*>(pk_smem);
  const int nblk = g.N * bg.nch * bg.nband;
  for (int b = blockIdx.x; b < nblk; b += gridDim.x) pack_band<InT, F>(g, bg, x, dst, b, tile);
}

// ---- planar filter [K][C][L_U] ----------------------------------------------
template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_filter_planar_kernel(Geom g, const InT* __restrict__ w,
                                                                      typename Word<F>::T* __restrict__ dst) {
  const long long total = (long long)g.K * g.C * g.L_U;
  for (long long idx = blockIdx.x * (long long)kThreads + threadIdx.x; idx < total;
       idx += (long long)gridDim.x * kThreads) {
    long long kc = idx / g.L_U;
    int e = (int)(idx - kc * g.L_U);
    int ib = e / g.Wp, jb = e - ib * g.Wp;  // e = Wp*(R-1-i) + (S-1-j)
    float v = 0.f;
    if (jb < g.S) {
      int i = g.R - 1 - ib, j = g.S - 1 - jb;
      v = load_io(w, (kc * g.R + i) * g.S + j);
    }
    dst[idx] = Word<F>::enc(v);
  }
}

// ---- tap-major filter [R*S][Kp][Cp] -------------------------------------------
// The nonzero coefficients of U_{k,c}(t) grouped by degree e(i,j) (tap), k, c.
// One thread per (k, c) of [Kp][Cp]: reads the R*S contiguous taps w[k][c][*]
// and writes coefficient e(i,j) of U_{k,c} into row (tap, k) -- consecutive
// threads write consecutive channels.  32-bit index math (plan guarantees < 2^31).
template <typename InT, int F>
__device__ __forceinline__ void pack_tapmajor_kc(const Geom& g, const InT* __restrict__ w,
                                                 typename Word<F>::T* __restrict__ dst, int Kp, int Cp, int idx) {
  const int k = idx / Cp, c = idx - k * Cp;
  const int RS = g.R * g.S;
  const bool in = k < g.K && c < g.C;
  const InT* src = w + ((long long)k * g.C + c) * RS;
  const long long rep_stride = (long long)RS * Kp * Cp;
  // eight taps' loads in flight before their stores (one dependent load per tap took ~4 us
  // for the conv3_x filter, all of it latency)
  for (int t0 = 0; t0 < RS; t0 += 8) {
    float v[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) v[j] = (in && t0 + j < RS) ? load_io(src, t0 + j) : 0.f;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      if (t0 + j >= RS) break;
      const auto e = Word<F>::enc(v[j]);
      for (int r = 0; r < g.urep; ++r) dst[r * rep_stride + ((long long)(t0 + j) * Kp + k) * Cp + c] = e;
    }
  }
}

template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_filter_tapmajor_kernel(Geom g, const InT* __restrict__ w,
                                                                        typename Word<F>::T* __restrict__ dst,
                                                                        int Kp, int Cp) {
  // let a programmatic dependent (the tensor-core MAC) start its prologue now;
  // it waits (griddepcontrol.wait) for this grid's completion before reading dst
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int total = Kp * Cp;
  for (int idx = blockIdx.x * kThreads + threadIdx.x; idx < total; idx += gridDim.x * kThreads)
    pack_tapmajor_kc<InT, F>(g, w, dst, Kp, Cp, idx);
}

// ---- interleaved input, TMA band path (the hot-path pack) -------------------
// One block per (image n, band of rb padded rows, chunk of kc2 channels).
//  1. One TMA 2-D load brings the band's input rows of kc2 channel planes
//     (x viewed as [N*C][H*W]: plane elements [e_lo, e_lo+seg) of planes
//     n*C + c0 ..) into S1 = [kc2][seg]; elements past H*W / planes past N*C
//     are zero-filled by the TMA unit.
//  2. Transpose S1 -> S2 = [rb*Wp positions][kc2 words]: thread (position p,
//     16-byte chunk j) reads the chunk's channels at p's input element (zero in
//     the padding, Eq. 10 + reading R3, and for channels >= C), converts them to
//     the operand format (reading R11) and stores one 16-byte chunk, XOR-swizzled
//     by p so that neither the S1 reads nor the S2 writes conflict in banks.
//  3. Coalesced copy-out: each position's kc2 words are one contiguous run of
//     the interleaved layout [N*L_A][Cp].
struct TBand {
  int rb;     // padded rows per block
  int nband;  // bands per image
  int kc2;    // channels per block
  int nch;    // Cp / kc2
  int seg;    // staged plane elements per channel (TMA box dim 0)
  int ealign; // 16 / sizeof(input element)
};

template <typename InT, int F>
__device__ __forceinline__ void pack_tband(const Geom& g, const TBand& b, const CUtensorMap* tmX,
                                           typename Word<F>::T* __restrict__ dst, int blk, unsigned char* smem) {
  using WT = typename Word<F>::T;
  constexpr int EPC = 16 / (int)sizeof(WT);  // channels per 16-byte chunk
  const int band = blk % b.nband;
  const int rest = blk / b.nband;
  const int ch = rest % b.nch, n = rest / b.nch;
  const int pr0 = band * b.rb, pr1 = min(g.Hp, pr0 + b.rb);
  const int h0 = max(0, pr0 - g.ph), h1 = min(g.H, pr1 - g.ph);
  const int e_lo = (h0 * g.W) & ~(b.ealign - 1);
  const int c0 = ch * b.kc2;
  const InT* S1 = reinterpret_cast<const InT*>(smem);
  const size_t s1_bytes = ((size_t)b.kc2 * b.seg * sizeof(InT) + 127) & ~(size_t)127;
  unsigned char* S2 = smem + s1_bytes;
  uint64_t* bar = reinterpret_cast<uint64_t*>(S2 + (size_t)b.rb * g.Wp * b.kc2 * sizeof(WT));
  const bool has = h1 > h0;
  if (threadIdx.x == 0 && has) {
    sm100::mbar_init(bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    sm100::mbar_arrive_expect_tx(bar, (uint32_t)(b.kc2 * b.seg * sizeof(InT)));
    sm100::tma_load_2d(smem, tmX, bar, e_lo, n * g.C + c0);
  }
  __syncthreads();
  if (has) sm100::mbar_wait(bar, 0);
  const int npos = (pr1 - pr0) * g.Wp;
  const int ncg = b.kc2 / EPC;              // 16-byte chunks per position
  const int rowb = b.kc2 * (int)sizeof(WT);  // bytes per position in S2
  const int cv = min(b.kc2, g.C - c0);       // real channels of this chunk
  for (int i = threadIdx.x; i < npos * ncg; i += kThreads) {
    const int j = i / npos, p = i - j * npos;  // consecutive threads: consecutive positions
    const int r = p / g.Wp, ps = p - r * g.Wp;
    const int h = pr0 + r - g.ph, w = ps - g.pw;
    const bool in = h >= 0 && h < g.H && w >= 0 && w < g.W;
    const int e = h * g.W + w - e_lo;
    uint32_t word[EPC];
#pragma unroll
    for (int t = 0; t < EPC; ++t) {
      const int c = j * EPC + t;
      const float v = (in && c < cv) ? to_f32(S1[c * b.seg + e]) : 0.f;
      word[t] = word_bits(Word<F>::enc(v));
    }
    uint4 q;
    if constexpr (sizeof(WT) == 2)
      q = make_uint4(word[0] | (word[1] << 16), word[2] | (word[3] << 16), word[4] | (word[5] << 16),
                     word[6] | (word[7] << 16));
    else
      q = make_uint4(word[0], word[1], word[2], word[3]);
    *reinterpret_cast<uint4*>(S2 + p * rowb + 16 * (j ^ (p & (ncg - 1)))) = q;
  }
  __syncthreads();
  WT* out = dst + ((size_t)n * (size_t)g.L_A + (size_t)pr0 * g.Wp) * g.Cp + c0;
  for (int i = threadIdx.x; i < npos * ncg; i += kThreads) {
    const int p = i / ncg, j = i - p * ncg;  // consecutive threads: the chunks of one position
    const uint4 q = *reinterpret_cast<const uint4*>(S2 + p * rowb + 16 * (j ^ (p & (ncg - 1))));
    *reinterpret_cast<uint4*>(out + (size_t)p * g.Cp + j * EPC) = q;
  }
  __syncthreads();  // S1/S2/bar reused by the block's next band
  if (threadIdx.x == 0 && has) asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(sm100::smem_u32(bar)) : "memory");
  __syncthreads();
}

inline size_t tband_smem(const Geom& g, const TBand& b, int in_bytes, int word_bytes) {
  return (((size_t)b.kc2 * b.seg * in_bytes + 127) & ~(size_t)127) + (size_t)b.rb * g.Wp * b.kc2 * word_bytes + 16;
}

// Band geometry of the TMA path; rb = 0 when the shape has no TMA view of x
// (H*W*elem not a multiple of 16 bytes) or a band does not fit one box.
inline TBand tband_geom(const Geom& g, int in_bytes, int word_bytes, int num_sms) {
  TBand b{};
  b.ealign = 16 / in_bytes;
  if (((long long)g.H * g.W * in_bytes) % 16 != 0) return b;
  b.kc2 = std::min(g.Cp, 128 / word_bytes);
  if (g.Cp % b.kc2 != 0 || (b.kc2 * word_bytes) % 16 != 0) return b;
  b.nch = g.Cp / b.kc2;
  auto seg_of = [&](int rb) { return (rb * g.W + b.ealign - 1 + b.ealign - 1) / b.ealign * b.ealign; };
  int rb = std::min(g.Hp, 256 / g.Wp);
  while (rb > 1 && (seg_of(rb) > 256 || tband_smem(g, TBand{rb, 0, b.kc2, 0, seg_of(rb), b.ealign}, in_bytes,
                                                   word_bytes) > 64 * 1024))
    --rb;
  // at least ~2 blocks per SM when the problem allows it
  while (rb > 1 && (long long)g.N * b.nch * ((g.Hp + rb - 1) / rb) < 2LL * num_sms) --rb;
  if (rb < 1 || seg_of(rb) > 256 || g.Wp > 256) return TBand{};
  b.rb = rb;
  b.seg = seg_of(rb);
  b.nband = (g.Hp + rb - 1) / rb;
  return b;
}

// ---- fused launch: tap-major filter, then interleaved input bands ------------
template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_both_tma_kernel(const __grid_constant__ CUtensorMap tmX, Geom g,
                                                                 TBand b, const InT* __restrict__ w,
                                                                 typename Word<F>::T* __restrict__ xdst,
                                                                 typename Word<F>::T* __restrict__ wdst,
                                                                 unsigned w_blocks) {
  // let a programmatic dependent (the tensor-core MAC) start its prologue now;
  // it waits (griddepcontrol.wait) for this grid's completion before reading
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  extern __shared__ __align__(128) unsigned char pk_smem[];
  if (blockIdx.x < w_blocks) {
    const int total = g.Kp * g.Cp;
    for (int idx = (int)blockIdx.x * kThreads + threadIdx.x; idx < total; idx += (int)w_blocks * kThreads)
      pack_tapmajor_kc<InT, F>(g, w, wdst, g.Kp, g.Cp, idx);
  } else {
    const int nblk = g.N * b.nch * b.nband;
    const int xb = (int)(gridDim.x - w_blocks);
    for (int blk = (int)(blockIdx.x - w_blocks); blk < nblk; blk += xb)
      pack_tband<InT, F>(g, b, &tmX, xdst, blk, pk_smem);
  }
}

template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_both_kernel(Geom g, BandGeom bg, const InT* __restrict__ x,
                                                             const InT* __restrict__ w,
                                                             typename Word<F>::T* __restrict__ xdst,
                                                             typename Word<F>::T* __restrict__ wdst,
                                                             unsigned w_blocks) {
  // let a programmatic dependent (the tensor-core MAC) start its prologue now;
  // it waits (griddepcontrol.wait) for this grid's completion before reading
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  extern __shared__ __align__(16) unsigned char pk_smem[];
  if (blockIdx.x < w_blocks) {
    const int total = g.Kp * g.Cp;
    for (int idx = (int)blockIdx.x * kThreads + threadIdx.x; idx < total; idx += (int)w_blocks * kThreads)
      pack_tapmajor_kc<InT, F>(g, w, wdst, g.Kp, g.Cp, idx);
  } else {
    InT* tile = reinterpret_cast<InT*>(pk_smem);
    const int nblk = g.N * bg.nch * bg.nband;
    const int xb = (int)(gridDim.x - w_blocks);
    for (int b = (int)(blockIdx.x - w_blocks); b < nblk; b += xb) pack_band<InT, F>(g, bg, x, xdst, b, tile);
  }
}

template <template <typename, int> class Launch, typename... Args>
cudaError_t dispatch(bool in_bf16, int fmt, Args&&... args) {
  if (in_bf16) {
    switch (fmt) {
      case FMT_F32: return Launch<__nv_bfloat16, FMT_F32>::run(args...);
      case FMT_TF32: return Launch<__nv_bfloat16, FMT_TF32>::run(args...);
      default: return Launch<__nv_bfloat16, FMT_BF16>::run(args...);
    }
  }
  switch (fmt) {
    case FMT_F32: return Launch<float, FMT_F32>::run(args...);
    case FMT_TF32: return Launch<float, FMT_TF32>::run(args...);
    default: return Launch<float, FMT_BF16>::run(args...);
  }
}

template <typename InT, int F> struct LInPlanar {
  static cudaError_t run(const Geom& g, const void* x, void* dst, cudaStream_t st) {
    const long long rows = (long long)g.N * g.C * g.Hp;
    const int per = kThreads / g.Wp;
    const long long blocks = per >= 1 ? (rows + per - 1) / per : rows;
    pack_input_planar_kernel<InT, F><<<grid_for(blocks, 1), kThreads, 0, st>>>(
        g, (const InT*)x, (typename Word<F>::T*)dst);
    return cudaGetLastError();
  }
};
template <typename InT>
size_t band_bytes(const BandGeom& bg) { return (size_t)kRowCh * bg.tw * sizeof(InT); }

typedef CUresult (*EncodeTiledFnP)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// TMA view of x as [N*C][H*W] with boxes of b.seg elements x b.kc2 planes.
template <typename InT>
bool encode_x_bands(CUtensorMap* m, const Geom& g, const TBand& b, const void* x) {
  static EncodeTiledFnP fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return false;
    fn = reinterpret_cast<EncodeTiledFnP>(f);
  }
  if ((reinterpret_cast<uintptr_t>(x) & 15) != 0) return false;
  cuuint64_t dims[2] = {(cuuint64_t)g.H * g.W, (cuuint64_t)g.N * g.C};
  cuuint64_t strides[1] = {(cuuint64_t)g.H * g.W * sizeof(InT)};
  cuuint32_t box[2] = {(cuuint32_t)b.seg, (cuuint32_t)b.kc2};
  cuuint32_t estr[2] = {1, 1};
  const CUtensorMapDataType dt =
      sizeof(InT) == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32;
  return fn(m, dt, 2, const_cast<void*>(x), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Interleaved pack (+ tap-major filter pack when w != nullptr) by the TMA band
// kernel; returns cudaErrorNotSupported when the shape has no TMA view.
template <typename InT, int F>
cudaError_t launch_tband(const Geom& g, const void* x, const void* w, void* xd, void* wd, cudaStream_t st) {
  int nsm = 148;
  int dev;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const TBand b = tband_geom(g, (int)sizeof(InT), (int)sizeof(typename Word<F>::T), nsm);
  if (b.rb == 0) return cudaErrorNotSupported;
  CUtensorMap tm;
  if (!encode_x_bands<InT>(&tm, g, b, x)) return cudaErrorNotSupported;
  const size_t smem = tband_smem(g, b, (int)sizeof(InT), (int)sizeof(typename Word<F>::T));
  const long long nblk = (long long)g.N * b.nch * b.nband;
  unsigned xb = grid_for(nblk, 1);
  const unsigned wb = w ? grid_for((long long)g.Kp * g.Cp, kThreads) : 0u;
  cudaError_t e = cudaFuncSetAttribute(pack_both_tma_kernel<InT, F>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  pack_both_tma_kernel<InT, F><<<wb + xb, kThreads, smem, st>>>(tm, g, b, (const InT*)w, (typename Word<F>::T*)xd,
                                                                (typename Word<F>::T*)wd, wb);
  return cudaGetLastError();
}

template <typename InT, int F> struct LInInter {
  static cudaError_t run(const Geom& g, const void* x, void* dst, cudaStream_t st) {
    if (!getenv("POLYCONV_PACK_LEGACY")) {
      const cudaError_t e = launch_tband<InT, F>(g, x, nullptr, dst, nullptr, st);
      if (e != cudaErrorNotSupported) return e;
    }
    const BandGeom bg = band_geom(g, (int)sizeof(InT));
    const long long nblk = (long long)g.N * bg.nch * bg.nband;
    const size_t smem = band_bytes<InT>(bg);
    cudaError_t e = cudaFuncSetAttribute(pack_input_interleaved_kernel<InT, F>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    pack_input_interleaved_kernel<InT, F><<<grid_for(nblk, 1), kThreads, smem, st>>>(
        g, bg, (const InT*)x, (typename Word<F>::T*)dst);
    return cudaGetLastError();
  }
};
template <typename InT, int F> struct LFPlanar {
  static cudaError_t run(const Geom& g, const void* w, void* dst, cudaStream_t st) {
    long long total = (long long)g.K * g.C * g.L_U;
    pack_filter_planar_kernel<InT, F><<<grid_for(total, kThreads), kThreads, 0, st>>>(
        g, (const InT*)w, (typename Word<F>::T*)dst);
    return cudaGetLastError();
  }
};
// bf16 tap-major filter, one thread per (k, 8 consecutive channels): the 8*RS contiguous
// elements w[k][c0..c0+7][*] as RS 16-byte loads, transposed in registers by byte permutes into
// RS 16-byte rows U[tap][k][c0..c0+7].  A few hundred threads instead of one per (k, c): the
// pack occupies a handful of SMs, so the MAC that follows it by programmatic dependent launch
// starts on the others at once (conv3_x: 2048 threads in 16 blocks).  C % 8 == 0.
template <int RS>
__global__ void __launch_bounds__(128) pack_filter_tapmajor_oct_kernel(Geom g, const uint4* __restrict__ w,
                                                                       uint4* __restrict__ dst, int Kp, int Cp) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int noct = Cp >> 3;
  const int idx = blockIdx.x * 128 + threadIdx.x;
  if (idx >= Kp * noct) return;
  const int k = idx / noct, oct = idx - k * noct;
  const bool ok = k < g.K && oct * 8 < g.C;
  uint4 v[RS];
#pragma unroll
  for (int i = 0; i < RS; ++i)
    v[i] = ok ? __ldg(w + ((long long)k * (g.C >> 3) + oct) * RS + i) : make_uint4(0, 0, 0, 0);
  const uint32_t* e = reinterpret_cast<const uint32_t*>(v);  // element j in word j/2, half j%2
#pragma unroll
  for (int t = 0; t < RS; ++t) {
    uint32_t o[4];
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      const int a = (2 * m) * RS + t, b = (2 * m + 1) * RS + t;  // channels 2m, 2m+1 at tap t
      const uint32_t sel = ((b & 1) ? 0x7600u : 0x5400u) | ((a & 1) ? 0x32u : 0x10u);
      o[m] = __byte_perm(e[a >> 1], e[b >> 1], sel);
    }
    dst[((long long)t * Kp + k) * noct + oct] = make_uint4(o[0], o[1], o[2], o[3]);
  }
}

template <typename InT, int F> struct LFTap {
  static cudaError_t run(const Geom& g, const void* w, void* dst, int Kp, int Cp, cudaStream_t st) {
    if constexpr (sizeof(InT) == 2 && F == FMT_BF16) {
      const int RS = g.R * g.S;
      if (g.urep == 1 && g.C % 8 == 0 && Cp % 8 == 0 && (RS == 9 || RS == 25 || RS == 1) &&
          ((uintptr_t)w & 15) == 0 && !getenv("POLYCONV_PACK_LEGACY")) {
        const int n = Kp * (Cp / 8), blocks = (n + 127) / 128;
        const uint4* wv = static_cast<const uint4*>(w);
        uint4* dv = static_cast<uint4*>(dst);
        if (RS == 9) pack_filter_tapmajor_oct_kernel<9><<<blocks, 128, 0, st>>>(g, wv, dv, Kp, Cp);
        else if (RS == 25) pack_filter_tapmajor_oct_kernel<25><<<blocks, 128, 0, st>>>(g, wv, dv, Kp, Cp);
        else pack_filter_tapmajor_oct_kernel<1><<<blocks, 128, 0, st>>>(g, wv, dv, Kp, Cp);
        return cudaGetLastError();
      }
    }
    long long total = (long long)Kp * Cp;
    pack_filter_tapmajor_kernel<InT, F><<<grid_for(total, kThreads), kThreads, 0, st>>>(
        g, (const InT*)w, (typename Word<F>::T*)dst, Kp, Cp);
    return cudaGetLastError();
  }
};
template <typename InT, int F> struct LBoth {
  static cudaError_t run(const Geom& g, const void* x, const void* w, void* xd, void* wd,
                         cudaStream_t st) {
    if (!getenv("POLYCONV_PACK_LEGACY")) {
      const cudaError_t e = launch_tband<InT, F>(g, x, w, xd, wd, st);
      if (e != cudaErrorNotSupported) return e;
    }
    const BandGeom bg = band_geom(g, (int)sizeof(InT));
    const long long nblk = (long long)g.N * bg.nch * bg.nband;
    unsigned xb = grid_for(nblk, 1);
    if (xb > 148 * 8) xb = 148 * 8;
    const unsigned wb = grid_for((long long)g.Kp * g.Cp, kThreads);  // one (k, c) filter row per thread
    const size_t smem = band_bytes<InT>(bg);
    cudaError_t e = cudaFuncSetAttribute(pack_both_kernel<InT, F>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)smem);
    if (e != cudaSuccess) return e;
    pack_both_kernel<InT, F><<<wb + xb, kThreads, smem, st>>>(g, bg, (const InT*)x, (const InT*)w,
                                                              (typename Word<F>::T*)xd,
                                                              (typename Word<F>::T*)wd, wb);
    return cudaGetLastError();
  }
};

}  // namespace

cudaError_t launch_pack_input_planar(const Geom& g, const void* x, bool x_bf16, void* dst, int fmt,
                                     cudaStream_t st) {
  return dispatch<LInPlanar>(x_bf16, fmt, g, x, dst, st);
}
cudaError_t launch_pack_input_interleaved(const Geom& g, const void* x, bool x_bf16, void* dst,
                                          int fmt, cudaStream_t st) {
  return dispatch<LInInter>(x_bf16, fmt, g, x, dst, st);
}
cudaError_t launch_pack_filter_planar(const Geom& g, const void* w, bool w_bf16, void* dst, int fmt,
                                      cudaStream_t st) {
  return dispatch<LFPlanar>(w_bf16, fmt, g, w, dst, st);
}
cudaError_t launch_pack_filter_tapmajor(const Geom& g, const void* w, bool w_bf16, void* dst,
                                        int fmt, int Kp, int Cp, cudaStream_t st) {
  return dispatch<LFTap>(w_bf16, fmt, g, w, dst, Kp, Cp, st);
}
// ---- phase-split filter for the stride-2 pair kernel (reading R19) ----------------------
// U'[t' = i'*S' + j'][k][(a*C + c)*2 + b] = w[k][c][i][j] with i = 2(i' - ph') + a + ph,
// j = 2(j' - pw') + b + pw when inside the kernel, else 0: the taps of the stride-1
// convolution over the phase planes X_{a,c,b}[u][v] = x[c][2u + a][2v + b].  One thread per
// output element (consecutive threads: consecutive virtual channels); bf16 in, bf16 words.
__global__ void __launch_bounds__(kThreads) pack_filter_phase_kernel(Geom g, const __nv_bfloat16* __restrict__ w,
                                                                     __nv_bfloat16* __restrict__ dst, int Rp, int Sp,
                                                                     int php, int pwp, int Kp, int Cp) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const long long total = (long long)Rp * Sp * Kp * Cp;
  for (long long idx = blockIdx.x * (long long)kThreads + threadIdx.x; idx < total;
       idx += (long long)gridDim.x * kThreads) {
    const int vc = (int)(idx % Cp);
    const long long tk = idx / Cp;
    const int k = (int)(tk % Kp), t = (int)(tk / Kp);
    const int ip = t / Sp, jp = t - ip * Sp;
    const int a = vc / (2 * g.C), rem = vc - a * 2 * g.C, c = rem >> 1, b = rem & 1;
    const int i = 2 * (ip - php) + a + g.ph, j = 2 * (jp - pwp) + b + g.pw;
    float v = 0.f;
    if (a < 2 && k < g.K && i >= 0 && i < g.R && j >= 0 && j < g.S)
      v = __bfloat162float(w[(((long long)k * g.C + c) * g.R + i) * g.S + j]);
    dst[idx] = __float2bfloat16_rn(v);
  }
}

cudaError_t launch_pack_filter_phase(const Geom& g, const void* w, void* dst, int Rp, int Sp, int php, int pwp,
                                     int Kp, int Cp, cudaStream_t st) {
  const long long total = (long long)Rp * Sp * Kp * Cp;
  const int grid = (int)std::min<long long>((total + kThreads - 1) / kThreads, 148LL * 8);
  pack_filter_phase_kernel<<<grid, kThreads, 0, st>>>(g, static_cast<const __nv_bfloat16*>(w),
                                                      static_cast<__nv_bfloat16*>(dst), Rp, Sp, php, pwp, Kp, Cp);
  return cudaGetLastError();
}

cudaError_t launch_pack_both_interleaved(const Geom& g, const void* x, const void* w, bool io_bf16,
                                         void* xdst, void* wdst, int fmt, cudaStream_t st) {
  return dispatch<LBoth>(io_bf16, fmt, g, x, w, xdst, wdst, st);
}

}  // namespace polyconv
