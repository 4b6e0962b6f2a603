// Probe: event-timed floor of (a) back-to-back events, (b) one empty kernel launched directly,
// (c) the same kernel replayed from a CUDA graph, (d) a PDL pair (tiny primary + cluster-2
// 227 KB dependent) directly and from a graph; after an L2 flush each time.
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o tools/graph_probe tools/graph_probe.cu
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>
__global__ void flushk(float4* p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    p[i] = make_float4(0, 0, 0, 0);
}
__global__ void emptyk(int* o) {
  extern __shared__ int sm[];
  if (threadIdx.x == 0 && o) sm[0] = 1;
}
__global__ void tinyk(int* o) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (o && threadIdx.x == 0) o[blockIdx.x] = 1;
}
static cudaStream_t st;
static void launch_pair(bool pdl) {
  tinyk<<<16, 256, 0, st>>>(nullptr);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(148); cfg.blockDim = dim3(896); cfg.dynamicSmemBytes = 230400; cfg.stream = st;
  cudaLaunchAttribute at[2]; int na = 0;
  at[na].id = cudaLaunchAttributeClusterDimension; at[na].val.clusterDim.x = 2; at[na].val.clusterDim.y = 1; at[na].val.clusterDim.z = 1; ++na;
  if (pdl) { at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization; at[na].val.programmaticStreamSerializationAllowed = 1; ++na; }
  cfg.attrs = at; cfg.numAttrs = na;
  cudaLaunchKernelEx(&cfg, emptyk, (int*)nullptr);
}
int main() {
  size_t n = (256ull << 20) / 16;
  float4* buf; cudaMalloc(&buf, n * 16);
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaFuncSetAttribute(emptyk, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448);
  cudaGraph_t g1, g2, g3; cudaGraphExec_t x1, x2, x3;
  cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
  emptyk<<<148, 896, 0, st>>>(nullptr);
  cudaStreamEndCapture(st, &g1); cudaGraphInstantiate(&x1, g1, 0);
  cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
  launch_pair(true);
  cudaStreamEndCapture(st, &g2); cudaGraphInstantiate(&x2, g2, 0);
  cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
  launch_pair(false);
  cudaStreamEndCapture(st, &g3); cudaGraphInstantiate(&x3, g3, 0);
  const char* names[] = {"events only", "empty direct", "empty graph", "pair+pdl direct", "pair+pdl graph",
                         "pair direct", "pair graph"};
  for (int mode = 0; mode < 7; ++mode) {
    std::vector<float> ts;
    for (int it = 0; it < 40; ++it) {
      flushk<<<148 * 4, 512, 0, st>>>(buf, n);
      cudaEventRecord(e0, st);
      if (mode == 1) emptyk<<<148, 896, 0, st>>>(nullptr);
      if (mode == 2) cudaGraphLaunch(x1, st);
      if (mode == 3) launch_pair(true);
      if (mode == 4) cudaGraphLaunch(x2, st);
      if (mode == 5) launch_pair(false);
      if (mode == 6) cudaGraphLaunch(x3, st);
      cudaEventRecord(e1, st);
      cudaStreamSynchronize(st);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      if (it >= 5) ts.push_back(ms * 1000);
    }
    std::sort(ts.begin(), ts.end());
    printf("%-18s median %.2f us  min %.2f  max %.2f\n", names[mode], ts[ts.size() / 2], ts[0], ts.back());
  }
  // same without syncing between steps (host runs ahead, as in bench.py)
  for (int mode = 0; mode < 7; ++mode) {
    const int K = 40;
    std::vector<cudaEvent_t> a(K), b(K);
    for (int i = 0; i < K; ++i) { cudaEventCreate(&a[i]); cudaEventCreate(&b[i]); }
    for (int it = 0; it < K; ++it) {
      flushk<<<148 * 4, 512, 0, st>>>(buf, n);
      cudaEventRecord(a[it], st);
      if (mode == 1) emptyk<<<148, 896, 0, st>>>(nullptr);
      if (mode == 2) cudaGraphLaunch(x1, st);
      if (mode == 3) launch_pair(true);
      if (mode == 4) cudaGraphLaunch(x2, st);
      if (mode == 5) launch_pair(false);
      if (mode == 6) cudaGraphLaunch(x3, st);
      cudaEventRecord(b[it], st);
    }
    cudaStreamSynchronize(st);
    std::vector<float> ts;
    for (int it = 5; it < K; ++it) { float ms; cudaEventElapsedTime(&ms, a[it], b[it]); ts.push_back(ms * 1000); }
    std::sort(ts.begin(), ts.end());
    printf("async %-12s median %.2f us  min %.2f  max %.2f\n", names[mode], ts[ts.size() / 2], ts[0], ts.back());
  }
  return 0;
}
