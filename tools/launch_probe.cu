// Probe: event-timed cost of launching an (almost) empty kernel right after an L2 flush, by
// shared-memory footprint and cluster shape.  Explains the fixed per-forward overhead.
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/launch_probe tools/launch_probe.cu
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>
__global__ void flushk(float4* p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    p[i] = make_float4(0, 0, 0, 0);
}
__global__ void readk(const float4* p, size_t n, float* out) {
  float s = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    s += p[i].x;
  if (s == 12345.f) *out = s;
}
__global__ void emptyk(int* o) {
  extern __shared__ int sm[];
  if (threadIdx.x == 0 && o) sm[0] = 1;
}
__global__ void tinyk(int* o) {  // PDL primary
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (o && threadIdx.x == 0) o[blockIdx.x] = 1;
}
int main() {
  size_t n = (256ull << 20) / 16;
  float4 *buf, *buf2; float* out; int* o;
  cudaMalloc(&buf, n * 16); cudaMalloc(&buf2, n * 16); cudaMalloc(&out, 4); cudaMalloc(&o, 4096);
  cudaStream_t st; cudaStreamCreate(&st);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int smems[] = {0, 48 * 1024, 100 * 1024, 232448 - 2048};
  cudaFuncSetAttribute(emptyk, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448);
  for (int flushmode = 0; flushmode < 3; ++flushmode)
  for (int pdl = 0; pdl < 2; ++pdl)
  for (int cl = 1; cl <= 2; ++cl)
    for (int si = 0; si < 4; ++si) {
      std::vector<float> ts;
      for (int it = 0; it < 25; ++it) {
        if (flushmode >= 1) flushk<<<148 * 4, 512, 0, st>>>(buf, n);
        if (flushmode == 2) readk<<<148 * 4, 512, 0, st>>>(buf2, n, out);
        cudaEventRecord(e0, st);
        if (pdl) tinyk<<<16, 256, 0, st>>>(o);
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(148); cfg.blockDim = dim3(896); cfg.dynamicSmemBytes = smems[si]; cfg.stream = st;
        cudaLaunchAttribute at[2]; int na = 0;
        at[na].id = cudaLaunchAttributeClusterDimension; at[na].val.clusterDim.x = cl; at[na].val.clusterDim.y = 1; at[na].val.clusterDim.z = 1; ++na;
        if (pdl) { at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization; at[na].val.programmaticStreamSerializationAllowed = 1; ++na; }
        cfg.attrs = at; cfg.numAttrs = na;
        cudaError_t e = cudaLaunchKernelEx(&cfg, emptyk, (int*)nullptr);
        if (e != cudaSuccess) { printf("launch err %s\n", cudaGetErrorString(e)); return 1; }
        cudaEventRecord(e1, st);
        cudaStreamSynchronize(st);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (it >= 5) ts.push_back(ms * 1000);
      }
      std::sort(ts.begin(), ts.end());
      printf("flush=%d pdl_tiny=%d cluster=%d smem=%6d  median %.2f us  min %.2f\n", flushmode, pdl, cl, smems[si], ts[ts.size() / 2], ts[0]);
    }
  return 0;
}
