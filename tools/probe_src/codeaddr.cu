#include <cstdio>
#include <cstdint>
__device__ __noinline__ int anchor(int x) { return x * 3 + 1; }
__global__ void k(int mode, unsigned long long* out) {
  void* fp = (void*)&anchor;
  void* kp = (void*)&k;
  out[0] = (unsigned long long)fp;
  out[1] = (unsigned long long)kp;
  if (mode == 1) {
    unsigned v;
    asm volatile("ld.global.u32 %0, [%1];" : "=r"(v) : "l"(kp));
    out[2] = v;
  }
  if (mode == 2) {
    asm volatile("prefetch.global.L2 [%0];" :: "l"(kp));
    out[2] = 7;
  }
  unsigned g;
  asm volatile("{\n\t.reg .pred p;\n\tisspacep.global p, %1;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(g) : "l"(kp));
  out[3] = g;
}
int main() {
  unsigned long long* d; cudaMalloc(&d, 64);
  for (int mode : {0, 2, 1}) {
    cudaMemset(d, 0, 64);
    k<<<1, 1>>>(mode, d);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[4] = {0};
    cudaMemcpy(h, d, 32, cudaMemcpyDeviceToHost);
    printf("mode %d err=%s anchor=%llx kernel=%llx val=%llx isglobal=%llu\n", mode, cudaGetErrorString(e), h[0], h[1], h[2], h[3]);
    if (e != cudaSuccess) break;
  }
  return 0;
}
