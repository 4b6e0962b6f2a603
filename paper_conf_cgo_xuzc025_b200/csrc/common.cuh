// common.cuh — device helpers: operand-format conversion (reading R11) and
// packed-word decoding.  Product code only.
#pragma once
#include <cstdint>
#include <cuda_bf16.h>
#include "internal.h"

namespace polyconv {

// Division by a runtime-invariant divisor d >= 1 through a multiply-high
// (round-up reciprocal; exact for 0 <= n < 2^31).  Set up on the host.
struct FastDiv {
  uint32_t d, mul, shr;
  __host__ __device__ void init(uint32_t div) {
    d = div;
    if (div <= 1) { mul = 0; shr = 0; return; }
    uint32_t l = 0;
    while ((1ull << l) < div) ++l;  // ceil(log2(div))
    const uint32_t p = 31 + l;
    mul = (uint32_t)(((1ull << p) + div - 1) / div);
    shr = p - 32;
  }
  __device__ __forceinline__ uint32_t div(uint32_t n) const { return d == 1 ? n : (__umulhi(n, mul) >> shr); }
};

__device__ __forceinline__ float load_io(const float* p, long long i) { return __ldg(p + i); }
__device__ __forceinline__ float load_io(const __nv_bfloat16* p, long long i) {
  return __bfloat162float(p[i]);
}

// fp32 -> tf32 word, round to nearest, ties away (cvt.rna.tf32.f32).
__device__ __forceinline__ uint32_t to_tf32_rna(float v) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(v));
  return r;
}

// Storage word of value v in format F.
template <int F> struct Word;
template <> struct Word<FMT_F32> {
  using T = float;
  __device__ __forceinline__ static float enc(float v) { return v; }
  __device__ __forceinline__ static float dec(float w) { return w; }
};
template <> struct Word<FMT_TF32> {
  using T = uint32_t;
  __device__ __forceinline__ static uint32_t enc(float v) { return to_tf32_rna(v); }
  __device__ __forceinline__ static float dec(uint32_t w) { return __uint_as_float(w); }
};
template <> struct Word<FMT_BF16> {
  using T = __nv_bfloat16;
  __device__ __forceinline__ static __nv_bfloat16 enc(float v) { return __float2bfloat16_rn(v); }
  __device__ __forceinline__ static float dec(__nv_bfloat16 w) { return __bfloat162float(w); }
};

__device__ __forceinline__ void store_out(float* y, long long i, float v) { y[i] = v; }
__device__ __forceinline__ void store_out(__nv_bfloat16* y, long long i, float v) {
  y[i] = __float2bfloat16_rn(v);
}

}  // namespace polyconv
