// mac_1x1.cu — 1x1 unpadded layers (BF16): a4 + a5 with the input polynomials
// read straight from NCHW x (stride 1, planes of a multiple of 8 pixels), or from a
// gathered copy of the output-lattice pixels (stride > 1, or other plane sizes).
//
// For R = S = 1 the kernel polynomial U_{k,c}(t) is the constant w[k][c] (Eq. 6
// with L_U = 1), the input polynomial A_{n,c}(t) is the plane x[n][c] itself
// (Eq. 10 with no padding: Wp = W), and the product coefficients are
//   p_{n,k}[m] = sum_c A_{n,c}[m] * w[k][c]          (P.965, P.1350-1352)
// with every coefficient an output pixel (Eq. 12: L_U - 1 = 0, m = oh*W + ow).
// That is one GEMM per image, D[k][m] = sum_c W[k][c] * X_n[c][m], whose position
// operand is already laid out by NCHW: x viewed as [N*C][H*W] has positions
// contiguous, i.e. the MN-major B operand of tcgen05.mma (tools/mn_probe.cu:
// SW128, LBO = the next 64-position box, SBO = the next 8 channels).  No packed
// copy of x is made.  The A operand is the tap-major packed filter [1][Kp][Cp]
// (a3, channels past C zero, so the rows a box reads past an image's last channel
// contribute nothing).
//
// Tiles: (image, block of NT positions, 128 output channels); K-chunks of 64
// channels through a ring of stages (TMA); fp32 accumulators in TMEM, double
// buffered; the epilogue holds one output channel per TMEM lane, so each thread
// stores runs of consecutive pixels of its channel as 16-byte vectors.
// Warps: 0 TMA producer, 1 TMEM allocator + MMA issuer, 2..5 epilogue.
#include <cuda.h>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <algorithm>
#include "common.cuh"
#include "sm100.cuh"

namespace polyconv {

namespace {

using namespace sm100;

constexpr int k1Threads = 192;
constexpr int k1MaxStages = 8;

struct P1x1 {
  void* y;
  int N, C, K, HW;   // HW: the operand's plane pitch (positions per [n][c] row of x or of the gathered copy)
  int HWo;           // output pixels per plane (P*Q) <= HW
  int NT, nbox, kchunks, num_pb, num_kt, num_tiles;
  int stages;
  uint32_t a_bytes, b_bytes;  // per stage
  uint32_t idesc;
  int tmem_cols;
  int epi_tma;  // 1: stage each warp's 32 channels x NT pixels (SW128) and TMA-store them;
                // 2: whole planes (one position block): stage the warp's 32 channel planes densely
                //    (a contiguous run of y) and write them with one bulk copy
  int resA;     // 1: each CTA keeps one 128-channel filter block resident (loaded once) and walks
                //    its images / position blocks, so only the x planes stream through the ring
  int groups;   // resA: CTAs per filter block (gridDim.x = groups * num_kt)
  int dbg;      // POLYCONV_1X1_DEBUG ablations (timing probes only): 1 no stores, 2 no MMA, 4 no x loads
  int gimg, NG; // images per tile (planes of <= 64 pixels: one 64-position box each) and image groups
};

// The CTA's i-th tile: (filter block kt, position block pb, image n).  resA: a CTA's tiles
// share kt = blockIdx.x % num_kt; else tiles t = blockIdx.x + i * gridDim.x, kt fastest.
__device__ __forceinline__ bool tile_of(const P1x1& p, int i, int& kt, int& pb, int& n) {
  int rest;
  if (p.resA) {
    kt = blockIdx.x % p.num_kt;
    rest = blockIdx.x / p.num_kt + i * p.groups;
    if (rest >= p.NG * p.num_pb) return false;
  } else {
    const long long t = blockIdx.x + (long long)i * gridDim.x;
    if (t >= p.num_tiles) return false;
    kt = (int)(t % p.num_kt);
    rest = (int)(t / p.num_kt);
  }
  pb = rest % p.num_pb;
  n = rest / p.num_pb;
  return true;
}

__device__ __forceinline__ uint64_t desc_mn(uint32_t saddr) {
  // MN-major, 128-byte swizzle: LBO = 8192 (next 64-position box), SBO = 1024 (next 8 k-rows)
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);
  d |= (uint64_t)(8192u >> 4) << 16;
  d |= (uint64_t)(1024u >> 4) << 32;
  d |= (uint64_t)1u << 46;
  d |= (uint64_t)2u << 61;
  return d;
}

__device__ __forceinline__ void tma_store_2d(const void* tmap, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(tmap)),
               "r"(src), "r"(c0), "r"(c1)
               : "memory");
}

__global__ void __launch_bounds__(k1Threads, 1)
    mac_1x1_kernel(const __grid_constant__ CUtensorMap tmU, const __grid_constant__ CUtensorMap tmX,
                   const __grid_constant__ CUtensorMap tmY, const P1x1 p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  uint8_t* sA = smem;  // [stages][128 rows][128 B], resA: [kchunks][128 rows][128 B] resident
  uint8_t* sB = sA + (p.resA ? (size_t)p.kchunks * p.a_bytes : (size_t)p.stages * p.a_bytes);  // [stages][nbox][64 ch][128 B]
  uint8_t* sE = sB + (size_t)p.stages * p.b_bytes;          // epi_tma: [4 warps][nbox][32 ch][128 B]
  uint64_t* full = reinterpret_cast<uint64_t*>(sE + (p.epi_tma ? (size_t)p.nbox * 16384 : 0));
  uint64_t* empty = full + k1MaxStages;
  uint64_t* tfull = empty + k1MaxStages;
  uint64_t* tempty = tfull + 2;
  uint64_t* afull = tempty + 2;  // resA: the resident filter block landed
  uint32_t* tslot = reinterpret_cast<uint32_t*>(afull + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    prefetch_tmap(&tmU);
    prefetch_tmap(&tmX);
    if (p.epi_tma == 1) prefetch_tmap(&tmY);
    for (int s = 0; s < p.stages; ++s) {
      mbar_init(full + s, 1);
      mbar_init(empty + s, 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(tfull + a, 1);
      mbar_init(tempty + a, 4);
    }
    mbar_init(afull, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc(tslot, (uint32_t)p.tmem_cols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;
  // the packed filter comes from the preceding pack launch (programmatic dependent launch)
  asm volatile("griddepcontrol.wait;" ::: "memory");

  if (warp == 0) {
    int st = 0;
    uint32_t ph = 0;
    int kt, pb, n;
    if (p.resA && tile_of(p, 0, kt, pb, n) && elect_one()) {
      mbar_arrive_expect_tx(afull, (uint32_t)p.kchunks * p.a_bytes);
      for (int kc = 0; kc < p.kchunks; ++kc)
        tma_load_2d(sA + (size_t)kc * p.a_bytes, &tmU, afull, kc * 64, kt * 128);
    }
    __syncwarp();
    for (int i = 0; tile_of(p, i, kt, pb, n); ++i) {
      for (int kc = 0; kc < p.kchunks; ++kc) {
        mbar_wait(empty + st, ph ^ 1u);
        if (elect_one()) {
          mbar_arrive_expect_tx(full + st, (p.resA ? 0u : p.a_bytes) + ((p.dbg & 4) ? 0u : (uint32_t)p.nbox * 8192u));
          if (!p.resA) tma_load_2d(sA + (size_t)st * p.a_bytes, &tmU, full + st, kc * 64, kt * 128);
          if (!(p.dbg & 4))
          for (int b = 0; b < p.nbox; ++b)
            tma_load_2d(sB + (size_t)st * p.b_bytes + (size_t)b * 8192, &tmX, full + st,
                        p.gimg > 1 ? 0 : pb * p.NT + b * 64,
                        (p.gimg > 1 ? (n * p.gimg + b) * p.C : n * p.C) + kc * 64);  // past N: zero fill
        }
        __syncwarp();
        if (++st == p.stages) { st = 0; ph ^= 1u; }
      }
    }
  } else if (warp == 1) {
    int st = 0, lt = 0;
    uint32_t ph = 0;
    int kt, pb, n;
    if (p.resA && tile_of(p, 0, kt, pb, n)) {
      mbar_wait(afull, 0);
      tc_fence_after();
    }
    for (; tile_of(p, lt, kt, pb, n); ++lt) {
      const int a = lt & 1;
      mbar_wait(tempty + a, (uint32_t)((lt >> 1) & 1) ^ 1u);
      tc_fence_after();
      const uint32_t d = tmem + (uint32_t)(a * p.NT);
      for (int kc = 0; kc < p.kchunks; ++kc) {
        mbar_wait(full + st, ph);
        tc_fence_after();
        const uint64_t ad = make_sdesc(smem_u32(sA + (size_t)(p.resA ? kc : st) * p.a_bytes), 128, 0);
        const uint64_t bd = desc_mn(smem_u32(sB + (size_t)st * p.b_bytes));
        if (elect_one()) {
#pragma unroll
          for (int ks = 0; ks < 4; ++ks)  // K step: +32 B (K-major A), +2048 B (MN-major B)
            if (!(p.dbg & 2)) umma<false>(d, ad + 2 * ks, bd + 128 * ks, p.idesc, (kc | ks) != 0 ? 1u : 0u);
          umma_commit(empty + st);
        }
        __syncwarp();
        if (++st == p.stages) { st = 0; ph ^= 1u; }
      }
      if (elect_one()) umma_commit(tfull + a);
      __syncwarp();
    }
  } else {
    // epilogue: lane = output channel (quadrant warp % 4), 32 positions per TMEM load
    const int q = warp & 3;
    __nv_bfloat16* y = static_cast<__nv_bfloat16*>(p.y);
    int lt = 0, kt, pb, n;
    for (; tile_of(p, lt, kt, pb, n); ++lt) {
      const int a = lt & 1;
      mbar_wait_sleep(tfull + a, (uint32_t)((lt >> 1) & 1), 64);
      tc_fence_after();
      const int k = kt * 128 + q * 32 + lane;
      __nv_bfloat16* yrow = y + ((long long)n * p.K + k) * p.HWo + (long long)pb * p.NT;
      const int nvalid = min(p.NT, p.HWo - pb * p.NT);
      const bool vec = (p.HWo & 7) == 0;  // 16-byte aligned 8-pixel groups
      // epi_tma (K % 32 == 0): the warp's 32 channels are all valid or all past K
      const bool wvalid = kt * 128 + q * 32 < p.K && !(p.dbg & 1);
      uint8_t* stg = sE + (size_t)q * p.nbox * 4096;
      if (p.epi_tma) {
        if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // staging free
        __syncwarp();
      }
      for (int c = 0; c < p.NT; c += 32) {
        uint32_t v[32];
        tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(a * p.NT + c), v);
        tmem_ld_wait();
        if (p.epi_tma == 2) {
          // plane `lane` of the warp's dense [32][HWo] run; positions past HWo are not stored
          // gimg > 1: box c/64 is image n*gimg + c/64, staged as its own dense run
          const int cb = p.gimg > 1 ? (c & 63) : c;
          if (wvalid) {
            uint8_t* row = stg + (size_t)(p.gimg > 1 ? (c >> 6) * 4096 : 0) + (size_t)lane * p.HWo * 2;
            if ((p.HWo & 1) == 0) {
#pragma unroll
              for (int j = 0; j < 32; j += 2)
                if (cb + j < p.HWo) {
                  const __nv_bfloat162 h2 = __floats2bfloat162_rn(__uint_as_float(v[j]), __uint_as_float(v[j + 1]));
                  *reinterpret_cast<__nv_bfloat162*>(row + (cb + j) * 2) = h2;
                }
            } else {
#pragma unroll
              for (int j = 0; j < 32; ++j)
                if (cb + j < p.HWo)
                  *reinterpret_cast<__nv_bfloat16*>(row + (cb + j) * 2) = __float2bfloat16_rn(__uint_as_float(v[j]));
            }
          }
          if (c + 32 >= p.NT) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            if (lane == 0 && wvalid) {
              const uint32_t bytes = 64u * (uint32_t)p.HWo;  // 32 planes x HWo x 2 B, a multiple of 16
              for (int b = 0; b < p.gimg; ++b) {
                const int ni = n * p.gimg + b;
                if (ni >= p.N) break;
                __nv_bfloat16* dst = y + ((long long)ni * p.K + kt * 128 + q * 32) * p.HWo;
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst),
                             "r"(smem_u32(stg + (size_t)b * 4096)), "r"(bytes)
                             : "memory");
              }
              asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
          }
        } else if (p.epi_tma) {
          // row `lane` of box c/64 (SW128: 16-byte chunk j at j ^ (lane & 7)); conflict-free
          if (wvalid && c < nvalid) {
            uint8_t* row = stg + (size_t)(c >> 6) * 4096 + lane * 128;
#pragma unroll
            for (int g8 = 0; g8 < 4; ++g8) {
              uint32_t w4[4];
#pragma unroll
              for (int m = 0; m < 4; ++m) {
                const __nv_bfloat162 h2 = __floats2bfloat162_rn(__uint_as_float(v[g8 * 8 + 2 * m]),
                                                                __uint_as_float(v[g8 * 8 + 2 * m + 1]));
                w4[m] = *reinterpret_cast<const uint32_t*>(&h2);
              }
              const int j = (((c & 63) >> 3) + g8) ^ (lane & 7);
              *reinterpret_cast<uint4*>(row + j * 16) = make_uint4(w4[0], w4[1], w4[2], w4[3]);
            }
          }
          if ((c & 63) == 32 || c + 32 >= p.NT) {  // a 64-pixel box is complete
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            const int b = c >> 6;
            if (lane == 0 && wvalid && b * 64 < nvalid) {
              tma_store_2d(&tmY, smem_u32(stg + (size_t)b * 4096), pb * p.NT + b * 64, n * p.K + kt * 128 + q * 32);
              asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
          }
        } else if (p.dbg & 1) {
        } else if (k < p.K && c < nvalid && (p.HWo & 3) != 0) {
#pragma unroll
          for (int j = 0; j < 32; ++j)
            if (c + j < nvalid) yrow[c + j] = __float2bfloat16_rn(__uint_as_float(v[j]));
        } else if (k < p.K && c < nvalid && !vec) {
          // HWo a multiple of 4: 8-byte groups of 4 pixels
#pragma unroll
          for (int g4 = 0; g4 < 8; ++g4) {
            if (c + g4 * 4 < nvalid) {
              const __nv_bfloat162 h0 = __floats2bfloat162_rn(__uint_as_float(v[g4 * 4]), __uint_as_float(v[g4 * 4 + 1]));
              const __nv_bfloat162 h1 =
                  __floats2bfloat162_rn(__uint_as_float(v[g4 * 4 + 2]), __uint_as_float(v[g4 * 4 + 3]));
              *reinterpret_cast<uint2*>(yrow + c + g4 * 4) =
                  make_uint2(*reinterpret_cast<const uint32_t*>(&h0), *reinterpret_cast<const uint32_t*>(&h1));
            }
          }
        } else if (k < p.K && c < nvalid) {
#pragma unroll
          for (int g8 = 0; g8 < 4; ++g8) {
            if (c + g8 * 8 < nvalid) {  // HWo is a multiple of 8: whole 8-pixel groups
              uint32_t w4[4];
#pragma unroll
              for (int m = 0; m < 4; ++m) {
                const __nv_bfloat162 h2 = __floats2bfloat162_rn(__uint_as_float(v[g8 * 8 + 2 * m]),
                                                                __uint_as_float(v[g8 * 8 + 2 * m + 1]));
                w4[m] = *reinterpret_cast<const uint32_t*>(&h2);
              }
              *reinterpret_cast<uint4*>(yrow + c + g8 * 8) = make_uint4(w4[0], w4[1], w4[2], w4[3]);
            }
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(tempty + a);
    }
    if (p.epi_tma && lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, (uint32_t)p.tmem_cols);
  }
}

// The position operand when the planes cannot be read in place (stride > 1, or a plane
// size that is not a multiple of 8 pixels, i.e. no 16-byte TMA row pitch): the output
// lattice pixels of every plane, xq[n*C + c][m] = x[n][c][oh*sh][ow*sw] for m = oh*Q + ow
// < P*Q, zero up to the pitch (Eq. 12 with R = S = 1: the coefficients that become outputs).
__global__ void __launch_bounds__(256) gather1x1_kernel(const __nv_bfloat16* __restrict__ x,
                                                        uint4* __restrict__ xq, long long rows, int H, int W,
                                                        int Q, int PQ, int pitch, int sh, int sw) {
  // one thread per 16-byte vector (8 lattice pixels) of a gathered row r = n*C + c: its 8
  // element loads are independent and in flight together, the (oh, ow) walk is incremental
  // (two divisions per vector), and the row is written with one 16-byte store (measured with
  // one warp per row, 2 pixels per lane and a division per pixel: 2-2.7 TB/s of HBM traffic)
  const int vpr = pitch >> 3;
  const long long nvec = rows * vpr;
  const uint16_t* xs = reinterpret_cast<const uint16_t*>(x);
  // stride 1: the plane is one contiguous run, copied with 8-byte loads when its element
  // offsets are multiples of 4 (ResNet-50 14x14: 18.4 -> 9 us for 25.7 MB)
  const bool contig = sh == 1 && sw == 1 && Q == W && (PQ & 3) == 0;
  // stride 1, any plane size: the 8 elements of a vector are consecutive in x (offset e, any
  // alignment) -- two aligned 16-byte loads and a funnel shift (adjacent lanes' loads overlap
  // in L1; x is read from HBM once)
  const bool funnel = sh == 1 && sw == 1 && Q == W && (PQ & 3) != 0;
  const long long xtotal = rows * H * W;
  for (long long v = (long long)blockIdx.x * 256 + threadIdx.x; v < nvec; v += (long long)gridDim.x * 256) {
    const long long r = v / vpr;
    const int m0 = (int)(v - r * vpr) * 8;
    if (funnel) {
      uint32_t o4[4] = {0u, 0u, 0u, 0u};
      if (m0 < PQ) {
        const long long e = r * PQ + m0, a = e & ~7LL;
        const int sft = (int)(e - a);
        const uint4* x4 = reinterpret_cast<const uint4*>(xs);
        auto vec = [&](long long a8) {  // x[a8 .. a8 + 8), nothing read past the tensor
          if (a8 + 8 <= xtotal) return __ldg(x4 + (a8 >> 3));
          uint32_t t[4] = {0u, 0u, 0u, 0u};
          for (int j = 0; j < 8 && a8 + j < xtotal; ++j) t[j >> 1] |= (uint32_t)xs[a8 + j] << (16 * (j & 1));
          return make_uint4(t[0], t[1], t[2], t[3]);
        };
        const uint4 lo = vec(a);
        const uint4 hi = vec(a + 8);
        const uint32_t w[8] = {lo.x, lo.y, lo.z, lo.w, hi.x, hi.y, hi.z, hi.w};
        const int hw = sft >> 1;
        uint32_t o[5];
#pragma unroll
        for (int i = 0; i < 5; ++i)
          o[i] = hw == 0 ? w[i] : hw == 1 ? w[i + 1] : hw == 2 ? w[i + 2] : w[i + 3 < 8 ? i + 3 : 7];
#pragma unroll
        for (int i = 0; i < 4; ++i) o4[i] = (sft & 1) ? __funnelshift_r(o[i], o[i + 1], 16) : o[i];
        if (m0 + 8 > PQ) {  // the plane's last vector: zeros past PQ
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            if (m0 + 2 * i >= PQ) o4[i] = 0u;
            else if (m0 + 2 * i + 1 >= PQ) o4[i] &= 0xFFFFu;
          }
        }
      }
      xq[v] = make_uint4(o4[0], o4[1], o4[2], o4[3]);
      continue;
    }
    const uint16_t* src = xs + r * H * W;
    if (contig && m0 + 8 <= PQ) {
      const uint2* s2 = reinterpret_cast<const uint2*>(src + m0);
      const uint2 a = __ldg(s2), b = __ldg(s2 + 1);
      xq[v] = make_uint4(a.x, a.y, b.x, b.y);
      continue;
    }
    if (contig) {  // the plane's last partial vector: 4-element groups, zeros past PQ
      const uint2* s2 = reinterpret_cast<const uint2*>(src + m0);
      const uint2 a = m0 < PQ ? __ldg(s2) : make_uint2(0u, 0u);
      const uint2 b = m0 + 4 < PQ ? __ldg(s2 + 1) : make_uint2(0u, 0u);
      xq[v] = make_uint4(a.x, a.y, b.x, b.y);
      continue;
    }
    int oh = m0 / Q, ow = m0 - oh * Q;
    uint32_t e[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      e[k] = (m0 + k < PQ) ? (uint32_t)__ldg(src + (oh * sh) * W + ow * sw) : 0u;
      if (++ow == Q) { ow = 0; ++oh; }
    }
    xq[v] = make_uint4(e[0] | (e[1] << 16), e[2] | (e[3] << 16), e[4] | (e[5] << 16), e[6] | (e[7] << 16));
  }
}

typedef CUresult (*EncFn1)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                           const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                           CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncFn1 get_enc1() {
  static EncFn1 fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncFn1>(f);
  }
  return fn;
}

bool enc2(CUtensorMap* m, const void* base, uint64_t cols, uint64_t rows, uint32_t bc, uint32_t br) {
  EncFn1 enc = get_enc1();
  if (!enc) return false;
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {cols * 2};
  cuuint32_t box[2] = {bc, br};
  cuuint32_t es[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace

bool mac1x1_supported(const Geom& g, int fmt, bool io_bf16) {
  return fmt == FMT_BF16 && io_bf16 && g.R == 1 && g.S == 1 && g.ph == 0 && g.pw == 0 &&
         (long long)g.N * g.C < (1LL << 31) && (long long)g.P * g.Q >= 16;
}

int mac1x1_pitch(const Geom& g) {
  const bool direct = g.sh == 1 && g.sw == 1 && ((long long)g.H * g.W) % 8 == 0;
  return direct ? 0 : (g.P * g.Q + 7) / 8 * 8;
}

cudaError_t launch_gather1x1(const Geom& g, const void* x, void* xq, cudaStream_t st) {
  const int pitch = mac1x1_pitch(g);
  const long long rows = (long long)g.N * g.C;
  long long blocks = (rows * (pitch / 8) + 255) / 256;
  if (blocks > 148LL * 64) blocks = 148LL * 64;
  gather1x1_kernel<<<(unsigned)blocks, 256, 0, st>>>(static_cast<const __nv_bfloat16*>(x), static_cast<uint4*>(xq),
                                                     rows, g.H, g.W, g.Q, g.P * g.Q, pitch, g.sh, g.sw);
  return cudaGetLastError();
}

cudaError_t launch_mac_1x1(const Geom& g, const void* x, const void* U, int Kp, int Cp, void* y, int num_sms,
                           cudaStream_t st, char* err, size_t errlen) {
  P1x1 p{};
  p.y = y;
  const int pitch = mac1x1_pitch(g);
  p.N = g.N; p.C = g.C; p.K = g.K;
  p.HW = pitch ? pitch : g.H * g.W;  // x (direct) or the gathered copy
  p.HWo = g.P * g.Q;
  p.NT = p.HWo >= 256 ? 256 : (p.HWo + 63) / 64 * 64;
  // planes of <= 64 pixels: four images per tile (one 64-position box each), so a streamed
  // filter block serves four images and the MMAs run at N = 256 (POLYCONV_1X1_GIMG=0: one image)
  const char* eg = getenv("POLYCONV_1X1_GIMG");
  const bool gep = g.K % 32 == 0 && (reinterpret_cast<uintptr_t>(y) & 15) == 0 &&
                   (getenv("POLYCONV_1X1_EPI_TMA") == nullptr || getenv("POLYCONV_1X1_EPI_TMA")[0] != '0');
  p.gimg = (p.HWo <= 64 && g.N > 1 && gep && (eg == nullptr || eg[0] != '0')) ? 4 : 1;
  if (p.gimg > 1) p.NT = 256;
  p.NG = (g.N + p.gimg - 1) / p.gimg;
  p.nbox = p.NT / 64;
  p.kchunks = Cp / 64;
  p.num_pb = p.gimg > 1 ? 1 : (p.HWo + p.NT - 1) / p.NT;
  p.num_kt = Kp / 128;
  const long long tiles = (long long)p.NG * p.num_pb * p.num_kt;
  if (tiles >= (1LL << 31) || p.kchunks < 1) {
    snprintf(err, errlen, "mac_1x1: unsupported shape");
    return cudaErrorInvalidValue;
  }
  p.num_tiles = (int)tiles;
  p.a_bytes = 128 * 128;
  p.b_bytes = (uint32_t)p.nbox * 8192;
  const int per = (int)(p.a_bytes + p.b_bytes);
  // TMA-stored epilogue: whole 32-channel row blocks, 16-byte output row pitch and base
  const char* ev = getenv("POLYCONV_1X1_EPI_TMA");
  const bool ep_ok = g.K % 32 == 0 && (reinterpret_cast<uintptr_t>(y) & 15) == 0 && (ev == nullptr || ev[0] != '0');
  p.epi_tma = !ep_ok ? 0 : (p.num_pb == 1 && g.K % 8 == 0) ? 2 : (p.HWo % 8 == 0 ? 1 : 0);
  if (p.gimg > 1 && p.epi_tma != 2) {
    snprintf(err, errlen, "mac_1x1: multi-image tiles need the staged epilogue");
    return cudaErrorInvalidValue;
  }
  const int estage = p.epi_tma ? p.nbox * 16384 : 0;
  // resident filter block: every CTA's tiles share one 128-channel block, which is loaded
  // once, so only x streams (C <= 384: at most 96 KB; POLYCONV_1X1_RESA=0 turns it off)
  const char* er = getenv("POLYCONV_1X1_RESA");
  const int resA_bytes = p.kchunks * (int)p.a_bytes;
  p.resA = (er == nullptr || er[0] != '0') && resA_bytes <= 96 * 1024 && p.num_kt <= num_sms &&
           (long long)p.NG * p.num_pb >= num_sms / p.num_kt;
  p.groups = p.resA ? num_sms / p.num_kt : 0;
  {
    const char* ed = getenv("POLYCONV_1X1_DEBUG");
    p.dbg = ed ? atoi(ed) : 0;
  }
  p.stages = p.resA ? std::min(k1MaxStages, (227 * 1024 - 2048 - estage - resA_bytes) / (int)p.b_bytes)
                    : std::min(k1MaxStages, (227 * 1024 - 2048 - estage) / per);
  if (p.stages < 2) {
    snprintf(err, errlen, "mac_1x1: shared memory");
    return cudaErrorInvalidValue;
  }
  // D f32 @4, A/B bf16 @7/@10, B MN-major (bit 16), N >> 3 @17, M = 128 >> 4 @24
  p.idesc = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(p.NT >> 3) << 17) | ((128u >> 4) << 24);
  p.tmem_cols = 2 * p.NT <= 32 ? 32 : (2 * p.NT <= 64 ? 64 : (2 * p.NT <= 128 ? 128 : (2 * p.NT <= 256 ? 256 : 512)));
  CUtensorMap tmU, tmX, tmY;
  memset(&tmY, 0, sizeof(tmY));
  if (!enc2(&tmU, U, (uint64_t)Cp, (uint64_t)Kp, 64, 128) ||
      !enc2(&tmX, x, (uint64_t)p.HW, (uint64_t)g.N * g.C, 64, 64) ||
      (p.epi_tma == 1 && !enc2(&tmY, y, (uint64_t)p.HWo, (uint64_t)g.N * g.K, 64, 32))) {
    snprintf(err, errlen, "mac_1x1: cuTensorMapEncodeTiled failed");
    return cudaErrorInvalidValue;
  }
  const int smem = p.resA ? 1024 + resA_bytes + p.stages * (int)p.b_bytes + estage + 1024
                         : 1024 + p.stages * per + estage + 1024;
  cudaError_t e = cudaFuncSetAttribute(mac_1x1_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(p.resA ? p.groups * p.num_kt : std::min(p.num_tiles, num_sms)));
  cfg.blockDim = dim3(k1Threads);
  cfg.dynamicSmemBytes = (size_t)smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, mac_1x1_kernel, tmU, tmX, tmY, p);
}

}  // namespace polyconv
