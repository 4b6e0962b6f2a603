// extract.cu — a5 standalone: pick the product coefficients at the Eq. 12
// degrees and store them as NCHW output (P.966-972; selection pattern
// P.1396-1403: skip the first L_U-1 = (Kh-1)*Iw+Kw-1, take Ow, skip Kw-1, ...).
//   y[n][k][oh][ow] = coeffs[n][k][Wp*sh*oh + sw*ow + L_U - 1]   (stride: R4)
// One thread per output element; consecutive threads -> consecutive ow, so
// the stores are coalesced and the loads are unit-stride within a row.
#include "common.cuh"

namespace polyconv {

namespace {
template <typename OutT>
__global__ void __launch_bounds__(256) extract_kernel(Geom g, const float* __restrict__ coeffs,
                                                      OutT* __restrict__ y) {
  const long long Lp = g.L_A + g.L_U - 1;
  const long long total = (long long)g.N * g.K * g.P * g.Q;
  for (long long idx = blockIdx.x * 256LL + threadIdx.x; idx < total; idx += (long long)gridDim.x * 256) {
    long long nk = idx / ((long long)g.P * g.Q);
    int pq = (int)(idx - nk * g.P * g.Q);
    int oh = pq / g.Q, ow = pq - oh * g.Q;
    long long m = (long long)g.Wp * g.sh * oh + (long long)g.sw * ow + g.L_U - 1;
    store_out(y, idx, __ldg(coeffs + nk * Lp + m));
  }
}
}  // namespace

cudaError_t launch_extract(const Geom& g, const float* coeffs, void* y, bool y_bf16,
                           cudaStream_t st) {
  long long total = (long long)g.N * g.K * g.P * g.Q;
  long long b = (total + 255) / 256;
  unsigned grid = (unsigned)(b > (1 << 20) ? (1 << 20) : (b < 1 ? 1 : b));
  if (y_bf16)
    extract_kernel<__nv_bfloat16><<<grid, 256, 0, st>>>(g, coeffs, (__nv_bfloat16*)y);
  else
    extract_kernel<float><<<grid, 256, 0, st>>>(g, coeffs, (float*)y);
  return cudaGetLastError();
}

}  // namespace polyconv
