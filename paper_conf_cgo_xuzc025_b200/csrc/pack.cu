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
#include "common.cuh"

namespace polyconv {

namespace {

constexpr int kThreads = 256;

inline unsigned grid_for(long long total, int per_block) {
  long long b = (total + per_block - 1) / per_block;
  if (b > (1LL << 20)) b = 1LL << 20;  // grid-stride beyond this
  return (unsigned)(b < 1 ? 1 : b);
}

// ---- planar input [N][C][L_A] ---------------------------------------------
template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_input_planar_kernel(Geom g, const InT* __restrict__ x,
                                                                     typename Word<F>::T* __restrict__ dst) {
  const long long total = (long long)g.N * g.C * g.L_A;
  for (long long idx = blockIdx.x * (long long)kThreads + threadIdx.x; idx < total;
       idx += (long long)gridDim.x * kThreads) {
    long long nc = idx / g.L_A;
    int m = (int)(idx - nc * g.L_A);
    int r = m / g.Wp, s = m - r * g.Wp;
    int h = r - g.ph, w = s - g.pw;
    float v = 0.f;
    if (h >= 0 && h < g.H && w >= 0 && w < g.W) v = load_io(x, (nc * g.H + h) * g.W + w);
    dst[idx] = Word<F>::enc(v);
  }
}

// ---- interleaved input [N*L_A][Cp] ------------------------------------------
// Tiled transpose: a block moves 64 coefficients x 32 channels.  Reads walk the
// coefficient axis (consecutive s -> consecutive w in x), writes walk channels.
constexpr int TM = 64, TCH = 32;

template <typename InT, int F>
__device__ __forceinline__ void pack_interleaved_tile(const Geom& g, const InT* __restrict__ x,
                                                      typename Word<F>::T* __restrict__ dst,
                                                      long long tile, float (*sm)[TM + 1]) {
  const int ctiles = (g.Cp + TCH - 1) / TCH;
  const long long mtiles = (g.L_A + TM - 1) / TM;
  const long long per_img = mtiles * ctiles;
  const int n = (int)(tile / per_img);
  long long rem = tile - (long long)n * per_img;
  const long long m0 = (rem / ctiles) * TM;
  const int c0 = (int)(rem % ctiles) * TCH;
  const int t = threadIdx.x;
  // load: thread -> (c = t/64 + 4*it, m = t%64)
  {
    const int mm = t % TM;
    const long long m = m0 + mm;
    int r = (int)(m / g.Wp), s = (int)(m - (long long)r * g.Wp);
    int h = r - g.ph, w = s - g.pw;
    bool inb = m < g.L_A && h >= 0 && h < g.H && w >= 0 && w < g.W;
#pragma unroll
    for (int it = 0; it < TCH / (kThreads / TM); ++it) {
      int cc = t / TM + it * (kThreads / TM);
      int c = c0 + cc;
      float v = 0.f;
      if (inb && c < g.C) v = load_io(x, (((long long)n * g.C + c) * g.H + h) * g.W + w);
      sm[cc][mm] = v;
    }
  }
  __syncthreads();
  {
    const int cc = t % TCH;
#pragma unroll
    for (int it = 0; it < TM / (kThreads / TCH); ++it) {
      int mm = t / TCH + it * (kThreads / TCH);
      long long m = m0 + mm;
      if (m < g.L_A && c0 + cc < g.Cp)
        dst[((long long)n * g.L_A + m) * g.Cp + c0 + cc] = Word<F>::enc(sm[cc][mm]);
    }
  }
  __syncthreads();
}

template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_input_interleaved_kernel(Geom g, const InT* __restrict__ x,
                                                                          typename Word<F>::T* __restrict__ dst) {
  __shared__ float sm[TCH][TM + 1];
  const long long ntiles = (long long)g.N * ((g.L_A + TM - 1) / TM) * ((g.Cp + TCH - 1) / TCH);
  for (long long tile = blockIdx.x; tile < ntiles; tile += gridDim.x)
    pack_interleaved_tile<InT, F>(g, x, dst, tile, sm);
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
template <typename InT, int F>
__device__ __forceinline__ void pack_tapmajor_elem(const Geom& g, const InT* __restrict__ w,
                                                   typename Word<F>::T* __restrict__ dst, int Kp,
                                                   int Cp, long long idx) {
  long long tk = idx / Cp;
  int c = (int)(idx - tk * Cp);
  int tap = (int)(tk / Kp);
  int k = (int)(tk - (long long)tap * Kp);
  float v = 0.f;
  if (k < g.K && c < g.C) v = load_io(w, ((long long)k * g.C + c) * g.R * g.S + tap);
  dst[idx] = Word<F>::enc(v);
}

template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_filter_tapmajor_kernel(Geom g, const InT* __restrict__ w,
                                                                        typename Word<F>::T* __restrict__ dst,
                                                                        int Kp, int Cp) {
  // let a programmatic dependent (the tensor-core MAC) start its prologue now;
  // it waits (griddepcontrol.wait) for this grid's completion before reading dst
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const long long total = (long long)g.R * g.S * Kp * Cp;
  for (long long idx = blockIdx.x * (long long)kThreads + threadIdx.x; idx < total;
       idx += (long long)gridDim.x * kThreads)
    pack_tapmajor_elem<InT, F>(g, w, dst, Kp, Cp, idx);
}

// ---- fused launch: interleaved input tiles, then tap-major filter ------------
template <typename InT, int F>
__global__ void __launch_bounds__(kThreads) pack_both_kernel(Geom g, const InT* __restrict__ x,
                                                             const InT* __restrict__ w,
                                                             typename Word<F>::T* __restrict__ xdst,
                                                             typename Word<F>::T* __restrict__ wdst,
                                                             unsigned x_blocks) {
  __shared__ float sm[TCH][TM + 1];
  if (blockIdx.x < x_blocks) {
    const long long ntiles = (long long)g.N * ((g.L_A + TM - 1) / TM) * ((g.Cp + TCH - 1) / TCH);
    for (long long tile = blockIdx.x; tile < ntiles; tile += x_blocks)
      pack_interleaved_tile<InT, F>(g, x, xdst, tile, sm);
  } else {
    const unsigned wb = gridDim.x - x_blocks;
    const long long total = (long long)g.R * g.S * g.Kp * g.Cp;
    for (long long idx = (blockIdx.x - x_blocks) * (long long)kThreads + threadIdx.x; idx < total;
         idx += (long long)wb * kThreads)
      pack_tapmajor_elem<InT, F>(g, w, wdst, g.Kp, g.Cp, idx);
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
    long long total = (long long)g.N * g.C * g.L_A;
    pack_input_planar_kernel<InT, F><<<grid_for(total, kThreads), kThreads, 0, st>>>(
        g, (const InT*)x, (typename Word<F>::T*)dst);
    return cudaGetLastError();
  }
};
template <typename InT, int F> struct LInInter {
  static cudaError_t run(const Geom& g, const void* x, void* dst, cudaStream_t st) {
    long long nt = (long long)g.N * ((g.L_A + TM - 1) / TM) * ((g.Cp + TCH - 1) / TCH);
    pack_input_interleaved_kernel<InT, F><<<grid_for(nt, 1), kThreads, 0, st>>>(
        g, (const InT*)x, (typename Word<F>::T*)dst);
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
template <typename InT, int F> struct LFTap {
  static cudaError_t run(const Geom& g, const void* w, void* dst, int Kp, int Cp, cudaStream_t st) {
    long long total = (long long)g.R * g.S * Kp * Cp;
    pack_filter_tapmajor_kernel<InT, F><<<grid_for(total, kThreads), kThreads, 0, st>>>(
        g, (const InT*)w, (typename Word<F>::T*)dst, Kp, Cp);
    return cudaGetLastError();
  }
};
template <typename InT, int F> struct LBoth {
  static cudaError_t run(const Geom& g, const void* x, const void* w, void* xd, void* wd,
                         cudaStream_t st) {
    long long nt = (long long)g.N * ((g.L_A + TM - 1) / TM) * ((g.Cp + TCH - 1) / TCH);
    long long wt = (long long)g.R * g.S * g.Kp * g.Cp;
    unsigned xb = grid_for(nt, 1);
    if (xb > 148 * 8) xb = 148 * 8;
    unsigned wb = grid_for(wt, kThreads);
    if (wb > 148) wb = 148;
    pack_both_kernel<InT, F><<<xb + wb, kThreads, 0, st>>>(g, (const InT*)x, (const InT*)w,
                                                           (typename Word<F>::T*)xd,
                                                           (typename Word<F>::T*)wd, xb);
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
cudaError_t launch_pack_both_interleaved(const Geom& g, const void* x, const void* w, bool io_bf16,
                                         void* xdst, void* wdst, int fmt, cudaStream_t st) {
  return dispatch<LBoth>(io_bf16, fmt, g, x, w, xdst, wdst, st);
}

}  // namespace polyconv
