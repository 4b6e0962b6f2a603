// fft.cu — the paper's own solver: the polynomial products by FFT,
//   R = IFFT(FFT(P) . FFT(Q))                       (Eq. 15, P.1050-1058)
// with P = A_{n,c}(t) (Eq. 10) and Q = U_{k,c}(t) (Eq. 11, reading R1), both zero-padded to
// L >= L_A + L_U - 1 (Eq. 14, P.1036-1049), L a power of two (P.1385-1388, reading Z9); one
// FFT per input channel and the channel sum taken in the frequency domain (P.1336-1352,
// P.1390-1393), then the Eq. 12 coefficients extracted (P.1396-1403).
//
//   fft_rows_fwd   RB input polynomials A_{n,c} per CTA in shared memory (bit-reversed
//                  placement), radix-2 DIT FFT, bins 0..L/2 (real input: the rest is the
//                  conjugate mirror) written as X^[f][n][c]
//   fft_filter_eval  U^[f][k][c] by direct evaluation at the roots of unity (R*S nonzero
//                  coefficients per U_{k,c}; cheaper than an FFT of the mostly-zero vector)
//   fft_contract   per frequency a complex GEMM over channels: Y^[f][n][k] = sum_c X^ U^
//                  (fp32 FFMA, register-blocked tiles; the contraction the paper does as
//                  element-wise products summed over channels)
//   fft_rows_inv   RB (n, k) rows per CTA: full spectrum from the half spectrum, inverse FFT,
//                  y[n][k][oh][ow] = Re(p[m(oh,ow)]) / L at the Eq. 12 degrees
// fp32 complex arithmetic throughout (math mode FP32_FMA); twiddles from double-precision
// sincospi, computed once per plan.  RB polynomials per CTA in shared memory (RB*L <= 16384):
// limited to L <= 8192; larger planes take the direct paths.
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <cstdint>
#include <algorithm>
#include "common.cuh"

namespace polyconv {

namespace {

constexpr int kFftThreads = 256;

__device__ __forceinline__ float2 cmul(float2 a, float2 b) {
  return make_float2(fmaf(a.x, b.x, -a.y * b.y), fmaf(a.x, b.y, a.y * b.x));
}

// Shared-memory slot of element i of a row: one float2 of padding per 32 (bit-reversed
// placement would otherwise put 32 consecutive threads on one bank).
__device__ __forceinline__ int pidx(int i) { return i + (i >> 5); }
__host__ __device__ inline int padded_len(int L) { return L + (L >> 5); }

// In-place iterative radix-2 DIT over nrows rows a[r*L .. r*L + L) (input in bit-reversed
// order), twiddles tw[m] = exp(-2 pi i m / L) for m < L/2 in shared memory; one barrier per
// stage for all rows.
__device__ void fft_smem(float2* a, const float2* tw, int L, int logL, int nrows) {
  const int hb = L >> 1;
  for (int s = 1; s <= logL; ++s) {
    const int half = 1 << (s - 1);
    const int tshift = logL - s;  // twiddle index = j * (L >> s)
    for (int e = threadIdx.x; e < nrows * hb; e += blockDim.x) {
      const int r = e >> (logL - 1), b = e & (hb - 1);
      const int j = b & (half - 1);
      const int e0 = ((b >> (s - 1)) << s) + j;
      float2* ar = a + r * padded_len(L);
      const int i0 = pidx(e0), i1 = pidx(e0 + half);
      const float2 w = tw[j << tshift];
      const float2 u = ar[i0];
      const float2 v = cmul(ar[i1], w);
      ar[i0] = make_float2(u.x + v.x, u.y + v.y);
      ar[i1] = make_float2(u.x - v.x, u.y - v.y);
    }
    __syncthreads();
  }
}

struct FftParams {
  const void* x;
  const void* w;
  float2* X;    // [F][N][C]
  float2* U;    // [F][K][C]
  float2* Y;    // [F][N][K]
  const float2* tw;
  void* y;
  int N, C, H, W, K, R, S, sh, sw, ph, pw, P, Q, Wp;
  long long L_A, L_U;
  int L, logL, F, RB;
  int io_bf16;
};

__device__ __forceinline__ float ld_io(const void* p, long long i, int bf16) {
  return bf16 ? __bfloat162float(static_cast<const __nv_bfloat16*>(p)[i]) : static_cast<const float*>(p)[i];
}

__global__ void fft_twiddles_kernel(float2* tw, int L) {
  for (int m = blockIdx.x * blockDim.x + threadIdx.x; m < L / 2; m += gridDim.x * blockDim.x) {
    double s, c;
    sincospi(-2.0 * (double)m / (double)L, &s, &c);
    tw[m] = make_float2((float)c, (float)s);
  }
}

// Input polynomials: RB rows A_{n,c} of consecutive channels per CTA (spectra written as RB-long
// contiguous runs per bin).
__global__ void __launch_bounds__(kFftThreads) fft_rows_fwd_kernel(const FftParams p) {
  extern __shared__ float2 fsm[];
  float2* tw = fsm;
  float2* a0 = fsm + p.L / 2;
  const int Lp = padded_len(p.L);
  for (int m = threadIdx.x; m < p.L / 2; m += blockDim.x) tw[m] = p.tw[m];
  const int cb = (p.C + p.RB - 1) / p.RB;
  const int n = blockIdx.x / cb, c0 = (blockIdx.x - n * cb) * p.RB;
  const int nr = min(p.RB, p.C - c0);
  const int shift = 32 - p.logL;
  for (int e = threadIdx.x; e < nr * p.L; e += blockDim.x) {
    const int r = e >> p.logL, t = e & (p.L - 1);
    // coefficient t of A_{n,c}: xpad[n][c][t / Wp][t % Wp] (Eq. 10 with Iw := Wp, reading R2)
    float v = 0.f;
    if (t < p.L_A) {
      const int rr = t / p.Wp, s = t - (t / p.Wp) * p.Wp;
      const int h = rr - p.ph, w = s - p.pw;
      if (h >= 0 && h < p.H && w >= 0 && w < p.W)
        v = ld_io(p.x, (((long long)n * p.C + c0 + r) * p.H + h) * p.W + w, p.io_bf16);
    }
    a0[r * Lp + pidx(__brev((unsigned)t) >> shift)] = make_float2(v, 0.f);
  }
  __syncthreads();
  fft_smem(a0, tw, p.L, p.logL, nr);
  for (int e = threadIdx.x; e < p.F * nr; e += blockDim.x) {
    const int f = e / nr, r = e - (e / nr) * nr;
    p.X[((long long)f * p.N + n) * p.C + c0 + r] = a0[r * Lp + pidx(f)];
  }
}

// Filter polynomials: U_{k,c}(t) has only R*S nonzero coefficients, so its spectrum is evaluated
// directly at the roots of unity ("evaluate ... over the complex roots of unity", P.1028-1030):
// U^[f] = sum_{i,j} w[k][c][i][j] exp(-2 pi i f e(i,j) / L).  One thread per (k, c) walks the
// bins of a CTA's f-range (consecutive threads = consecutive channels: coalesced stores), with
// the R*S weights and their twiddle indices (f * e(i,j) mod L, advanced by e(i,j)) in registers.
constexpr int kMaxEvalTaps = 49;
template <int TAPS>
__global__ void __launch_bounds__(kFftThreads) fft_filter_eval_kernel(const FftParams p, int fper) {
  extern __shared__ float2 fsm[];
  float2* tw = fsm;
  for (int m = threadIdx.x; m < p.L / 2; m += blockDim.x) tw[m] = p.tw[m];
  __syncthreads();
  const int RS = p.R * p.S;
  const long long kc = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (kc >= (long long)p.K * p.C) return;
  const int f0 = blockIdx.y * fper, f1 = min(p.F, f0 + fper);
  float wv[TAPS];
  int deg[TAPS], m[TAPS];
  const int mask = p.L - 1;
#pragma unroll
  for (int t = 0; t < TAPS; ++t) {
    if (t < RS) {
      const int i = t / p.S, j = t - (t / p.S) * p.S;
      wv[t] = ld_io(p.w, kc * RS + t, p.io_bf16);
      deg[t] = p.Wp * (p.R - 1 - i) + (p.S - 1 - j);  // e(i,j), Eq. 11 (reading R1)
      m[t] = (int)(((long long)f0 * deg[t]) & mask);
    }
  }
  for (int f = f0; f < f1; ++f) {
    float2 acc = make_float2(0.f, 0.f);
#pragma unroll
    for (int t = 0; t < TAPS; ++t) {
      if (t < RS) {
        const int mm = m[t];
        const float2 z = mm < (p.L >> 1) ? tw[mm] : make_float2(-tw[mm - (p.L >> 1)].x, -tw[mm - (p.L >> 1)].y);
        acc.x = fmaf(wv[t], z.x, acc.x);
        acc.y = fmaf(wv[t], z.y, acc.y);
        m[t] = (mm + deg[t]) & mask;
      }
    }
    p.U[(long long)f * p.K * p.C + kc] = acc;  // [F][K][C]
  }
}

// Y^[f][n][k] = sum_c X^[f][n][c] U^[f][k][c]: CTA tile 32 n x 64 k of one frequency, 256
// threads with 2 x 4 outputs each, channels staged 16 at a time.
constexpr int kTN = 32, kTK = 64, kTC = 16;
__global__ void __launch_bounds__(256) fft_contract_kernel(const FftParams p) {
  __shared__ float2 Xs[kTC][kTN + 1];
  __shared__ float2 Us[kTC][kTK + 1];
  const int f = blockIdx.z;
  const int n0 = blockIdx.y * kTN, k0 = blockIdx.x * kTK;
  const int tid = threadIdx.x, ty = tid >> 4, tx = tid & 15;
  float2 acc[2][4];
#pragma unroll
  for (int i = 0; i < 2; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = make_float2(0.f, 0.f);
  const float2* Xf = p.X + (long long)f * p.N * p.C;
  const float2* Uf = p.U + (long long)f * p.K * p.C;
  for (int c0 = 0; c0 < p.C; c0 += kTC) {
    for (int e = tid; e < kTN * kTC; e += 256) {
      const int n = e / kTC, cc = e - (e / kTC) * kTC;
      Xs[cc][n] = (n0 + n < p.N && c0 + cc < p.C) ? Xf[(long long)(n0 + n) * p.C + c0 + cc] : make_float2(0.f, 0.f);
    }
    for (int e = tid; e < kTK * kTC; e += 256) {
      const int k = e / kTC, cc = e - (e / kTC) * kTC;
      Us[cc][k] = (k0 + k < p.K && c0 + cc < p.C) ? Uf[(long long)(k0 + k) * p.C + c0 + cc] : make_float2(0.f, 0.f);
    }
    __syncthreads();
#pragma unroll
    for (int cc = 0; cc < kTC; ++cc) {
      float2 xv[2], uv[4];
#pragma unroll
      for (int i = 0; i < 2; ++i) xv[i] = Xs[cc][ty * 2 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) uv[j] = Us[cc][tx + 16 * j];
#pragma unroll
      for (int i = 0; i < 2; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          acc[i][j].x = fmaf(xv[i].x, uv[j].x, fmaf(-xv[i].y, uv[j].y, acc[i][j].x));
          acc[i][j].y = fmaf(xv[i].x, uv[j].y, fmaf(xv[i].y, uv[j].x, acc[i][j].y));
        }
    }
    __syncthreads();
  }
  float2* Yf = p.Y + (long long)f * p.N * p.K;
#pragma unroll
  for (int i = 0; i < 2; ++i) {
    const int n = n0 + ty * 2 + i;
    if (n >= p.N) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int k = k0 + tx + 16 * j;
      if (k < p.K) Yf[(long long)n * p.K + k] = acc[i][j];
    }
  }
}

// RB consecutive output channels of one image per CTA: spectrum bins 0..L/2 of each row from
// Y^[f][n][k] (RB contiguous values per f), the conjugate mirror for L/2+1..L-1, inverse FFT
// as conj(FFT(conj(.))), then the Eq. 12 extraction (stride: reading R4).
__global__ void __launch_bounds__(kFftThreads) fft_rows_inv_kernel(const FftParams p) {
  extern __shared__ float2 fsm[];
  float2* tw = fsm;
  float2* a0 = fsm + p.L / 2;
  for (int m = threadIdx.x; m < p.L / 2; m += blockDim.x) tw[m] = p.tw[m];
  const int kb = (p.K + p.RB - 1) / p.RB;
  const int n = blockIdx.x / kb, k0 = (blockIdx.x - n * kb) * p.RB;
  const int nr = min(p.RB, p.K - k0);
  const int shift = 32 - p.logL;
  // load: conj of the spectrum, bit-reversed placement (the inverse runs as a forward FFT)
  for (int e = threadIdx.x; e < p.F * nr; e += blockDim.x) {
    const int f = e / nr, r = e - (e / nr) * nr;
    const float2 v = p.Y[((long long)f * p.N + n) * p.K + k0 + r];
    float2* a = a0 + (size_t)r * padded_len(p.L);
    a[pidx(__brev((unsigned)f) >> shift)] = make_float2(v.x, -v.y);
    if (f > 0 && f < p.L / 2) a[pidx(__brev((unsigned)(p.L - f)) >> shift)] = make_float2(v.x, v.y);  // conj(conj(Y_f))
  }
  __syncthreads();
  fft_smem(a0, tw, p.L, p.logL, nr);
  const float inv = 1.f / (float)p.L;
  const long long PQ = (long long)p.P * p.Q;
  for (int e = threadIdx.x; e < nr * PQ; e += blockDim.x) {
    const int r = (int)(e / PQ);
    const int o = (int)(e - (long long)r * PQ);
    const int oh = o / p.Q, ow = o - (o / p.Q) * p.Q;
    const long long m = (long long)p.Wp * p.sh * oh + (long long)p.sw * ow + p.L_U - 1;  // Eq. 12 + R4
    const float v = a0[(size_t)r * padded_len(p.L) + pidx((int)m)].x * inv;  // Re(conj(z)) = Re(z)
    const long long yi = ((long long)n * p.K + k0 + r) * PQ + o;
    if (p.io_bf16) static_cast<__nv_bfloat16*>(p.y)[yi] = __float2bfloat16_rn(v);
    else static_cast<float*>(p.y)[yi] = v;
  }
}

}  // namespace

FftTiling fft_tiling(const Geom& g) {
  FftTiling t{};
  t.ok = false;
  const long long need = g.L_A + g.L_U - 1;  // Eq. 14: both vectors padded to M + N - 1
  int L = 1, logL = 0;
  while (L < need) { L <<= 1; ++logL; }
  if (L > 8192 || L < 2 || g.R * g.S > kMaxEvalTaps) return t;
  t.L = L;
  t.logL = logL;
  t.F = L / 2 + 1;
  t.RB = (int)std::max(1, std::min(8, 16384 / L));  // rows per CTA: RB * L * 8 bytes <= 128 KB
  t.x_bytes = (size_t)t.F * g.N * g.C * sizeof(float2);
  t.u_bytes = (size_t)t.F * g.K * g.C * sizeof(float2);
  t.y_bytes = (size_t)t.F * g.N * g.K * sizeof(float2);
  t.tw_bytes = (size_t)(L / 2) * sizeof(float2);
  if ((long long)g.N * g.C > (1LL << 31) - 1 || (long long)g.K * g.C > (1LL << 31) - 1 ||
      (long long)g.N * ((g.K + t.RB - 1) / t.RB) > (1LL << 31) - 1)
    return t;
  t.ok = true;
  return t;
}

cudaError_t launch_fft_twiddles(const FftTiling& t, void* tw, cudaStream_t st) {
  fft_twiddles_kernel<<<(t.L / 2 + 255) / 256, 256, 0, st>>>(static_cast<float2*>(tw), t.L);
  return cudaGetLastError();
}

cudaError_t launch_fft_conv(const Geom& g, const FftTiling& t, const void* x, const void* w, bool io_bf16, void* ws,
                            const void* tw, void* y, cudaStream_t st) {
  FftParams p{};
  p.x = x; p.w = w; p.y = y;
  char* b = static_cast<char*>(ws);
  p.X = reinterpret_cast<float2*>(b);
  p.U = reinterpret_cast<float2*>(b + t.x_bytes);
  p.Y = reinterpret_cast<float2*>(b + t.x_bytes + t.u_bytes);
  p.tw = static_cast<const float2*>(tw);
  p.N = g.N; p.C = g.C; p.H = g.H; p.W = g.W; p.K = g.K; p.R = g.R; p.S = g.S;
  p.sh = g.sh; p.sw = g.sw; p.ph = g.ph; p.pw = g.pw; p.P = g.P; p.Q = g.Q; p.Wp = g.Wp;
  p.L_A = g.L_A; p.L_U = g.L_U;
  p.L = t.L; p.logL = t.logL; p.F = t.F; p.RB = t.RB;
  p.io_bf16 = io_bf16 ? 1 : 0;
  const size_t fwd_smem = (size_t)t.RB * padded_len(t.L) * sizeof(float2) + t.tw_bytes;
  const size_t inv_smem = fwd_smem;
  cudaError_t e = cudaFuncSetAttribute(fft_rows_fwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fwd_smem);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(fft_rows_inv_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)inv_smem);
  if (e != cudaSuccess) return e;
  const unsigned cb = (unsigned)((g.C + t.RB - 1) / t.RB);
  fft_rows_fwd_kernel<<<(unsigned)g.N * cb, kFftThreads, fwd_smem, st>>>(p);
  const int RS = g.R * g.S;
  auto fev = RS <= 1 ? fft_filter_eval_kernel<1> : RS <= 9 ? fft_filter_eval_kernel<9>
             : RS <= 25 ? fft_filter_eval_kernel<25> : fft_filter_eval_kernel<kMaxEvalTaps>;
  e = cudaFuncSetAttribute(fev, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)t.tw_bytes);
  if (e != cudaSuccess) return e;
  // (k, c) threads x f-ranges: at least ~4 CTAs per SM
  const unsigned kcb = (unsigned)(((long long)g.K * g.C + kFftThreads - 1) / kFftThreads);
  const int fsplit = (int)std::max<long long>(1, std::min<long long>(t.F, (600 + kcb - 1) / kcb));
  const int fper = (t.F + fsplit - 1) / fsplit;
  fev<<<dim3(kcb, (unsigned)((t.F + fper - 1) / fper)), kFftThreads, t.tw_bytes, st>>>(p, fper);
  dim3 cg((unsigned)((g.K + kTK - 1) / kTK), (unsigned)((g.N + kTN - 1) / kTN), (unsigned)t.F);
  fft_contract_kernel<<<cg, 256, 0, st>>>(p);
  const unsigned inv_blocks = (unsigned)(g.N * ((g.K + t.RB - 1) / t.RB));
  fft_rows_inv_kernel<<<inv_blocks, kFftThreads, inv_smem, st>>>(p);
  return cudaGetLastError();
}

}  // namespace polyconv
