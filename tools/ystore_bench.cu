// ystore_bench.cu — design probe (not product code): how fast can one CTA per
// SM (140 CTAs, 8 warps each) write a conv3_x-sized output (6.4 MB bf16) from
// registers/shared memory, by store width: 4-byte lanes (128 B per warp
// instruction), 16-byte lanes (512 B), and 1-D bulk copies shared -> global.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ystore_bench tools/ystore_bench.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include <algorithm>
#include "../paper_conf_cgo_xuzc025_b200/csrc/sm100.cuh"

using namespace polyconv::sm100;

constexpr int NCTA = 140, PER = 49152;  // bytes per CTA (128 channels x 192 outputs x 2 B)

__global__ void st_kernel(char* y, int variant, unsigned long long* tout) {
  extern __shared__ __align__(128) uint8_t sm[];
  for (int i = threadIdx.x; i < PER / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = i;
  __syncthreads();
  unsigned long long t0 = global_ns();
  char* dst = y + (size_t)blockIdx.x * PER;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (variant == 0) {  // 4 B per lane; each warp instruction one 128 B run; 16 in flight per warp
    for (int base = warp * 128 * 16; base < PER; base += 8 * 128 * 16) {
      uint32_t v[16];
#pragma unroll
      for (int i = 0; i < 16; ++i) v[i] = reinterpret_cast<uint32_t*>(sm)[(base + i * 128) / 4 + lane];
#pragma unroll
      for (int i = 0; i < 16; ++i)
        if (base + i * 128 < PER) *reinterpret_cast<uint32_t*>(dst + base + i * 128 + 4 * lane) = v[i];
    }
  } else if (variant == 1) {  // 16 B per lane; 512 B per warp instruction
    for (int base = warp * 512 * 4; base < PER; base += 8 * 512 * 4) {
      uint4 v[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) v[i] = reinterpret_cast<uint4*>(sm)[(base + i * 512) / 16 + lane];
#pragma unroll
      for (int i = 0; i < 4; ++i)
        if (base + i * 512 < PER) *reinterpret_cast<uint4*>(dst + base + i * 512 + 16 * lane) = v[i];
    }
  } else if (variant == 2) {  // 4 B per lane, but each lane writes a DIFFERENT channel plane (stride 1568 B)
    for (int i = warp; i < PER / 128; i += 8) {
      const uint32_t v = reinterpret_cast<uint32_t*>(sm)[i * 32 + lane];
      *reinterpret_cast<uint32_t*>(dst + (size_t)lane * 1568 % PER + (i * 4) % 1568) = v;
    }
  } else if (variant >= 4) {
    // the conv3_x epilogue partition: CTA t owns positions [208t, 208t+208) of the
    // concatenated padded planes (Wp = 30, L_A = 900); per pass of 64 positions,
    // warp w stores channels w, w+8, ..: lane l -> positions 2l, 2l+1 (one bf16x2
    // word when both are outputs); variant 5: each lane stores 8 outputs (16 B)
    // of one channel when they are contiguous and 16 B aligned
    uint16_t* yy = reinterpret_cast<uint16_t*>(y);
    for (int c0 = 0; c0 < 208; c0 += 64) {
      const int cc = c0 + 2 * lane;
      int o[2];
      for (int q = 0; q < 2; ++q) {
        o[q] = -1;
        const int gp = blockIdx.x * 208 + cc + q;
        if (cc + q < min(208, c0 + 64)) {
          const int n = gp / 900, m = gp % 900, r = m / 30, s = m % 30;
          if (r < 28 && s < 28) o[q] = n * 128 * 784 + r * 28 + s;
        }
      }
      const uint32_t v = reinterpret_cast<uint32_t*>(sm)[lane];
      if (o[0] >= 0 || o[1] >= 0) {
#pragma unroll 16
        for (int i = 0; i < 16; ++i) {
          const int k = warp + 8 * i;
          if (o[0] >= 0 && o[1] == o[0] + 1 && (o[0] & 1) == 0)
            *reinterpret_cast<uint32_t*>(yy + (size_t)k * 784 + o[0]) = v;
          else {
            if (o[0] >= 0) yy[(size_t)k * 784 + o[0]] = (uint16_t)v;
            if (o[1] >= 0) yy[(size_t)k * 784 + o[1]] = (uint16_t)(v >> 16);
          }
        }
      }
    }
  } else {  // 1-D bulk copies of 4 KB shared -> global
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (tid < PER / 4096) {
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + tid * 4096),
                   "r"(smem_u32(sm + tid * 4096)), "r"(4096)
                   : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
  }
  __syncthreads();
  if (tid == 0) { tout[2 * blockIdx.x] = t0; tout[2 * blockIdx.x + 1] = global_ns(); }
}

__global__ void flush_kernel(float* a, size_t n, float* sink) {
  float s = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) a[i] = 0.f;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    s += a[(i * 7919) % n];
  if (s == 12345.f) *sink = s;
}
__global__ void read_kernel(const float* a, size_t n, float* sink) {
  float s = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) s += a[i];
  if (s == 12345.f) *sink = s;
}

int main() {
  char* y;
  cudaMalloc(&y, (size_t)32 * 128 * 784 * 2 + NCTA * PER);
  float *fl, *ev, *sink;
  size_t fn = (size_t)64 << 20;
  cudaMalloc(&fl, fn * 4);
  cudaMalloc(&ev, fn * 4);
  cudaMalloc(&sink, 4);
  unsigned long long* tout;
  cudaMalloc(&tout, 2 * 160 * 8);
  cudaFuncSetAttribute(st_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, PER);
  const char* names[] = {"STG.32 coalesced (128 B/instr)", "STG.128 coalesced (512 B/instr)",
                         "STG.32 scattered over planes", "bulk 4 KB shared->global", "conv3_x epilogue pattern"};
  for (int v = 0; v < 5; ++v) {
    std::vector<double> meds;
    for (int rep = 0; rep < 8; ++rep) {
      flush_kernel<<<1184, 256>>>(fl, fn, sink);
      read_kernel<<<1184, 256>>>(ev, fn, sink);
      st_kernel<<<NCTA, 256, PER>>>(y, v, tout);
      cudaDeviceSynchronize();
      std::vector<unsigned long long> h(2 * NCTA);
      cudaMemcpy(h.data(), tout, 2 * NCTA * 8, cudaMemcpyDeviceToHost);
      std::vector<double> d;
      for (int b = 0; b < NCTA; ++b) d.push_back((h[2 * b + 1] - h[2 * b]) / 1e3);
      std::sort(d.begin(), d.end());
      if (rep >= 2) meds.push_back(d[NCTA / 2]);
    }
    std::sort(meds.begin(), meds.end());
    printf("%-34s per-CTA store phase: med %.2f us  (%.1f B/clk/SM at 1.9 GHz)\n", names[v], meds[meds.size() / 2],
           PER / (meds[meds.size() / 2] * 1e3 * 1.9));
  }
  return 0;
}
