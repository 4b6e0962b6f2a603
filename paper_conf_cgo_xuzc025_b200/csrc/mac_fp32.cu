// mac_fp32.cu — a4+a5 on the FP32 SIMT pipe (math FP32_FMA, the 1e-5 path).
//
// Computes, for one image n, the product coefficients of
//   p_{n,k}(t) = sum_c A_{n,c}(t) U_{k,c}(t)        (P.965, P.1350-1352)
// at the degrees m = base + L_U - 1, base in [0, M_ext), as R*S shifted
// dot products over the planar packed polynomial (the Hankel structure):
//   p[base + L_U - 1] = sum_c sum_{i,j} A_{n,c}[base + Wp*i + j] * U_{k,c}[e(i,j)]
// and stores the ones on the extraction lattice (Eq. 12 + R4) into NCHW y.
//
// CTA tile: 64 output channels x 256 consecutive degrees (two CTAs per SM: one
// stages while the other computes); 8 warps, warp w owns
// 8 channels, lane l owns 8 consecutive degrees (64 fp32 accumulators/thread).
// Per channel chunk (8 channels) the CTA stages R windows of A (one per kernel
// row i, starting at degree m0 + Wp*i) and the 8 x R*S x 64 filter
// coefficients in shared memory.  For each kernel row a thread loads its 8+S-1
// window values once into registers and reuses them for all S taps of the row
// (the shifts j = 0..S-1 slide along the same registers).  Weight loads are
// warp-uniform (smem broadcast).  Windows are padded 4 words per 32 so the
// 128-bit window loads are bank-conflict free.
#include "common.cuh"

namespace polyconv {

namespace {

constexpr int BK = 64, BP = 256, CC = 8, NT = 256;

__host__ __device__ constexpr int nv_for(int smax) { return (8 + smax - 1 + 3) / 4 * 4; }
__host__ __device__ constexpr int winp_for(int smax) { return 8 * 31 + nv_for(smax); }
__host__ __device__ constexpr int phys(int q) { return q + (q >> 5) * 4; }  // bank-conflict pad
__host__ __device__ constexpr int winp_phys(int smax) { return phys(winp_for(smax) - 1) + 1; }

template <int SMAX>
__global__ void __launch_bounds__(NT, 2) mac_fp32_kernel(Geom g, const float* __restrict__ A,
                                                         const float* __restrict__ U, int Kp, int Cp,
                                                         float* __restrict__ y) {
  constexpr int NV = nv_for(SMAX);
  constexpr int WINP = winp_for(SMAX);
  constexpr int WROW = (winp_phys(SMAX) + 3) / 4 * 4;  // floats per staged window row
  extern __shared__ float4 smem4[];
  float* s_in = reinterpret_cast<float*>(smem4);       // [CC][R][WROW]
  float* s_w = s_in + CC * g.R * WROW;                  // [CC][RS][BK]

  const int n = blockIdx.z;
  const int k0 = blockIdx.y * BK;
  const long long m0 = (long long)blockIdx.x * BP;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int RS = g.R * g.S;
  const float* An = A + (long long)n * g.C * g.L_A;

  float acc[8][8];
#pragma unroll
  for (int a = 0; a < 8; ++a)
#pragma unroll
    for (int b = 0; b < 8; ++b) acc[a][b] = 0.f;

  for (int c0 = 0; c0 < g.C; c0 += CC) {
    // stage windows: s_in[cc][i][phys(q)] = A_{n,c0+cc}[m0 + Wp*i + q]
    const int nwin = CC * g.R * WINP;
    for (int e = threadIdx.x; e < nwin; e += NT) {
      int q = e % WINP;
      int ci = e / WINP;
      int cc = ci / g.R, i = ci - cc * g.R;
      long long m = m0 + (long long)g.Wp * i + q;
      float v = 0.f;
      if (c0 + cc < g.C && m < g.L_A) v = __ldg(An + (long long)(c0 + cc) * g.L_A + m);
      s_in[ci * WROW + phys(q)] = v;
    }
    // stage filter coefficients: s_w[cc][tap][kk] = U_tap[k0+kk][c0+cc]
    const int nw = CC * RS * BK;
    for (int e = threadIdx.x; e < nw; e += NT) {
      int cc = e % CC;
      int tk = e / CC;
      int kk = tk % BK, tap = tk / BK;
      s_w[(cc * RS + tap) * BK + kk] = __ldg(U + ((long long)tap * Kp + k0 + kk) * Cp + c0 + cc);
    }
    __syncthreads();
    const int ccn = min(CC, g.C - c0);
    for (int cc = 0; cc < ccn; ++cc) {
      for (int i = 0; i < g.R; ++i) {
        const float* win = s_in + (cc * g.R + i) * WROW;
        float pv[NV];
#pragma unroll
        for (int v = 0; v < NV / 4; ++v) {
          float4 t4 = *reinterpret_cast<const float4*>(win + phys(8 * lane + 4 * v));
          pv[4 * v] = t4.x; pv[4 * v + 1] = t4.y; pv[4 * v + 2] = t4.z; pv[4 * v + 3] = t4.w;
        }
        const float* wrow = s_w + (cc * RS + i * g.S) * BK + warp * 8;
#pragma unroll
        for (int j = 0; j < SMAX; ++j) {
          if (j < g.S) {
            float4 w0 = *reinterpret_cast<const float4*>(wrow + j * BK);
            float4 w1 = *reinterpret_cast<const float4*>(wrow + j * BK + 4);
            float wv[8] = {w0.x, w0.y, w0.z, w0.w, w1.x, w1.y, w1.z, w1.w};
#pragma unroll
            for (int a = 0; a < 8; ++a)
#pragma unroll
              for (int b = 0; b < 8; ++b) acc[a][b] = fmaf(wv[a], pv[b + j], acc[a][b]);
          }
        }
      }
    }
    __syncthreads();
  }

  // fused extraction (Eq. 12 + R4): degree base -> (r, s) of the padded plane
#pragma unroll
  for (int b = 0; b < 8; ++b) {
    long long base = m0 + 8 * lane + b;
    if (base >= g.M_ext) continue;
    int r = (int)(base / g.Wp), s = (int)(base - (long long)r * g.Wp);
    if (r % g.sh || s % g.sw) continue;
    int oh = r / g.sh, ow = s / g.sw;
    if (oh >= g.P || ow >= g.Q) continue;
#pragma unroll
    for (int a = 0; a < 8; ++a) {
      int k = k0 + warp * 8 + a;
      if (k < g.K) y[(((long long)n * g.K + k) * g.P + oh) * g.Q + ow] = acc[a][b];
    }
  }
}

template <int SMAX>
int smem_for(const Geom& g) {
  constexpr int WROW = (winp_phys(SMAX) + 3) / 4 * 4;
  return (CC * g.R * WROW + CC * g.R * g.S * BK) * 4;
}

}  // namespace

Fp32Tiling fp32_tiling(const Geom& g) {
  Fp32Tiling t{CC, 0, 0};
  if (g.S <= 1) { t.smax = 1; t.smem_bytes = smem_for<1>(g); }
  else if (g.S <= 3) { t.smax = 3; t.smem_bytes = smem_for<3>(g); }
  else if (g.S <= 5) { t.smax = 5; t.smem_bytes = smem_for<5>(g); }
  else if (g.S <= 7) { t.smax = 7; t.smem_bytes = smem_for<7>(g); }
  else { t.smax = 0; }
  if (t.smem_bytes > 200 * 1024) t.smax = 0;  // caller falls back to the thin kernel
  return t;
}

cudaError_t launch_mac_fp32(const Geom& g, const Fp32Tiling& t, const float* A, const float* U,
                            int Kp, int Cp, float* y, cudaStream_t st) {
  dim3 grid((unsigned)((g.M_ext + BP - 1) / BP), (unsigned)(Kp / BK), (unsigned)g.N);
  cudaError_t e = cudaSuccess;
#define PC_FP32(SM)                                                                             \
  case SM:                                                                                      \
    e = cudaFuncSetAttribute(mac_fp32_kernel<SM>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                             t.smem_bytes);                                                     \
    if (e != cudaSuccess) return e;                                                             \
    mac_fp32_kernel<SM><<<grid, NT, t.smem_bytes, st>>>(g, A, U, Kp, Cp, y);                    \
    break;
  switch (t.smax) {
    PC_FP32(1) PC_FP32(3) PC_FP32(5) PC_FP32(7)
    default: return cudaErrorInvalidValue;
  }
#undef PC_FP32
  return cudaGetLastError();
}

}  // namespace polyconv
