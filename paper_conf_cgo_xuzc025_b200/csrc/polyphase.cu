// polyphase.cu — stride-s convolution as a stride-1 one (reading R4b).
//
// The paper has no stride; reading R4 extracts the stride lattice from the
// stride-1 product coefficients, which computes s^2 times the needed outputs.
// With the phases of the zero-padded input split into channels,
//   xq[n][(a*s + b)*C + c][u][v] = xpad[n][c][u*s + a][v*s + b]
//   wq[k][(a*s + b)*C + c][i][j] = w[k][c][i*s + a][j*s + b]   (0 past R, S)
// the stride-s output is the stride-1, unpadded convolution of xq with wq:
//   y[n][k][oh][ow] = sum_{c,i,j} xpad[c][oh*s + i][ow*s + j] w[k][c][i][j]
//                   = sum_{a,b,c,i',j'} xq[(a,b,c)][oh + i'][ow + j'] wq[k][(a,b,c)][i'][j']
// (i = i'*s + a, j = j'*s + b), so the polynomial method of the inner plan runs
// on s^2*C channels of ceil(R/s) x ceil(S/s) kernels and computes only the
// lattice.  xq is cropped to exactly P + Rq - 1 rows and Q + Sq - 1 columns.
// Both transforms are copies (HBM-bound): x one block per output plane (warps over rows,
// lanes along the contiguous output dimension), w one thread per output element.
#include <algorithm>
#include "common.cuh"

namespace polyconv {

namespace {

template <typename T>
__global__ void __launch_bounds__(256) s2d_kernel(const T* __restrict__ x, T* __restrict__ xq, int N, int C, int H,
                                                  int W, int s, int ph, int pw, int Hq, int Wq) {
  // one block per output plane (n, (a, b), c), decoded once; warps over its rows u, lanes
  // along v (contiguous writes; reads strided by s, the other phases hit the same sectors)
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int planes = N * s * s * C;
  for (int pl = blockIdx.x; pl < planes; pl += gridDim.x) {
    const int n = pl / (s * s * C), cq = pl - n * (s * s * C);
    const int ab = cq / C, c = cq - ab * C;
    const int a = ab / s, b = ab - a * s;
    const T* xp = x + ((long long)n * C + c) * H * W;
    T* dp = xq + (long long)pl * Hq * Wq;
    for (int u = warp; u < Hq; u += 8) {
      const int h = u * s + a - ph;
      const bool hin = h >= 0 && h < H;
      const T* src = xp + (long long)(hin ? h : 0) * W;
      T* dst = dp + (long long)u * Wq;
      for (int v = lane; v < Wq; v += 32) {
        const int w = v * s + b - pw;
        dst[v] = (hin && w >= 0 && w < W) ? src[w] : T(0.f);
      }
    }
  }
}

template <typename T>
__global__ void __launch_bounds__(256) wphase_kernel(const T* __restrict__ w, T* __restrict__ wq, int K, int C, int R,
                                                     int S, int s, int Rq, int Sq) {
  const long long total = (long long)K * s * s * C * Rq * Sq;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < total;
       idx += (long long)gridDim.x * blockDim.x) {
    const int jq = (int)(idx % Sq);
    long long r = idx / Sq;
    const int iq = (int)(r % Rq);
    r /= Rq;
    const int cq = (int)(r % ((long long)s * s * C));
    const int k = (int)(r / ((long long)s * s * C));
    const int ab = cq / C, c = cq - ab * C;
    const int a = ab / s, b = ab - a * s;
    const int i = iq * s + a, j = jq * s + b;
    T val = T(0.f);
    if (i < R && j < S) val = w[(((long long)k * C + c) * R + i) * S + j];
    wq[idx] = val;
  }
}

inline unsigned blocks_for(long long n) {
  long long b = (n + 255) / 256;
  return (unsigned)(b < 148LL * 16 ? (b < 1 ? 1 : b) : 148LL * 16);
}

}  // namespace

cudaError_t launch_polyphase(const Geom& g, int Hq, int Wq, int Rq, int Sq, const void* x, const void* w, void* xq,
                             void* wq, bool io_bf16, cudaStream_t st) {
  const int s = g.sh;
  const long long nw = (long long)g.K * s * s * g.C * Rq * Sq;
  const long long planes = (long long)g.N * s * s * g.C;  // < 2^31: the plan's element limits
  const unsigned xblocks = (unsigned)std::min<long long>(std::max<long long>(planes, 1), 148LL * 16);
  if (io_bf16) {
    s2d_kernel<__nv_bfloat16><<<xblocks, 256, 0, st>>>(static_cast<const __nv_bfloat16*>(x),
                                                               static_cast<__nv_bfloat16*>(xq), g.N, g.C, g.H, g.W,
                                                               s, g.ph, g.pw, Hq, Wq);
    wphase_kernel<__nv_bfloat16><<<blocks_for(nw), 256, 0, st>>>(static_cast<const __nv_bfloat16*>(w),
                                                                  static_cast<__nv_bfloat16*>(wq), g.K, g.C, g.R,
                                                                  g.S, s, Rq, Sq);
  } else {
    s2d_kernel<float><<<xblocks, 256, 0, st>>>(static_cast<const float*>(x), static_cast<float*>(xq), g.N,
                                                       g.C, g.H, g.W, s, g.ph, g.pw, Hq, Wq);
    wphase_kernel<float><<<blocks_for(nw), 256, 0, st>>>(static_cast<const float*>(w), static_cast<float*>(wq),
                                                          g.K, g.C, g.R, g.S, s, Rq, Sq);
  }
  return cudaGetLastError();
}

}  // namespace polyconv
