// xload_bench.cu — design probe (not product code): how fast can one CTA per SM
// pull the conv3_x input (bf16 x[32][128][28][28], 6.4 MB, cold L2) into shared
// memory, by access pattern.  Each CTA streams a list of TMA boxes (or 1-D bulk
// copies) through a ring of slots; a consumer warp releases each slot as soon
// as it lands.  Prints the event time of the launch and per-CTA finish spread.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/xload_bench tools/xload_bench.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include "../paper_conf_cgo_xuzc025_b200/csrc/sm100.cuh"

using namespace polyconv::sm100;

constexpr int N = 32, C = 128, H = 28, W = 28, HW = H * W, Wp = 30, Hp = 30, LA = Hp * Wp;
constexpr int NT = 208, BROWS = 272;

struct Item { int a, b; };  // TMA: (dim0 coord, dim1 coord); bulk: (byte offset, bytes)

__global__ void ring_load(const __grid_constant__ CUtensorMap tm, const char* xbase, const Item* items,
                          const int* start, int ring, int slot_bytes, int box_bytes, int bulk,
                          unsigned long long* tout) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = raw + (((smem_u32(raw) + 1023) & ~1023u) - smem_u32(raw));
  __shared__ uint64_t full[32], empty[32];
  const int warp = threadIdx.x >> 5;
  const int i0 = start[blockIdx.x], i1 = start[blockIdx.x + 1];
  if (threadIdx.x == 0) {
    for (int s = 0; s < ring; ++s) { mbar_init(full + s, 1); mbar_init(empty + s, 1); }
    fence_barrier_init();
  }
  __syncthreads();
  unsigned long long t0 = global_ns();
  if (warp == 0) {
    for (int i = i0; i < i1; ++i) {
      const int k = i - i0, s = k % ring;
      mbar_wait(empty + s, ((k / ring) & 1) ^ 1);
      if (elect_one()) {
        const Item it = items[i];
        if (bulk) {
          mbar_arrive_expect_tx(full + s, it.b);
          asm volatile(
              "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                  smem_u32(sm + (size_t)s * slot_bytes)),
              "l"(xbase + it.a), "r"(it.b), "r"(smem_u32(full + s))
              : "memory");
        } else {
          mbar_arrive_expect_tx(full + s, box_bytes);
          tma_load_2d(sm + (size_t)s * slot_bytes, &tm, full + s, it.a, it.b);
        }
      }
      __syncwarp();
    }
  } else if (warp == 1) {
    for (int i = i0; i < i1; ++i) {
      const int k = i - i0, s = k % ring;
      mbar_wait(full + s, (k / ring) & 1);
      __syncwarp();
      if ((threadIdx.x & 31) == 0) mbar_arrive(empty + s);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) { tout[2 * blockIdx.x] = t0; tout[2 * blockIdx.x + 1] = global_ns(); }
}

__global__ void flush_kernel(float* a, size_t n, float* sink) {
  float s = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    a[i] = 0.f;
  }
  __syncthreads();
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    s += a[(i * 7919) % n];
  if (s == 12345.f) *sink = s;
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  const int nsm = 140;
  size_t xbytes = (size_t)N * C * HW * 2;
  char* x;
  cudaMalloc(&x, xbytes);
  cudaMemset(x, 1, xbytes);
  float* fl;
  size_t fn = (size_t)128 << 20;  // 512 MB of floats
  cudaMalloc(&fl, fn * 4);
  float* sink;
  cudaMalloc(&sink, 4);
  EncFn enc;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  unsigned long long* tout;
  cudaMalloc(&tout, 2 * 160 * 8);
  Item* ditems;
  cudaMalloc(&ditems, 1 << 22);
  int* dstart;
  cudaMalloc(&dstart, 4 * 200);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaFuncSetAttribute(ring_load, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);

  // window element ranges of tile b, channel chunk ch: elements [e_lo, e_hi) of image n (up to 2 images)
  auto windows = [&](int b, std::vector<std::pair<int, std::pair<int, int>>>& segs) {
    segs.clear();
    long long wrow = (long long)b * NT;
    for (int n = 0; n < N; ++n) {
      long long base = (long long)n * LA - wrow;
      if (base >= BROWS || base + LA <= 0) continue;
      int pr_lo = base >= 0 ? 0 : (int)((-base) / Wp);
      int pr_hi = std::min(Hp - 1, (int)((BROWS - 1 - base) / Wp));
      int h_lo = std::max(0, pr_lo - 1), h_hi = std::min(H - 1, pr_hi - 1);
      if (h_lo > h_hi) continue;
      segs.push_back({n, {(h_lo * W) & ~7, (h_hi + 1) * W}});
    }
  };
  struct Var { const char* name; int box_e, box_c, swz, bulk, ring; };
  const bool noflush = getenv("NOFLUSH") != nullptr;  // x L2-warm
  printf("L2 %s between reps\n", noflush ? "NOT flushed" : "flushed");
  std::vector<Var> vars = {{"box 232el x 64ch noswz ring2 (mac_pair)", 232, 64, 0, 0, 2},
                           {"box 256el x 64ch noswz ring2 line-aligned", 256, 64, 0, 0, 2},
                           {"mx: box 64el x 64ch sw128 ring6", 64, 64, 1, 0, 6},
                           {"mx: box 64el x 64ch sw128 ring12", 64, 64, 1, 0, 12},
                           {"box 256el x 32ch noswz ring8", 256, 32, 0, 0, 8},
                           {"box 256el x 16ch noswz ring12", 256, 16, 0, 0, 12},
                           {"bulk per-plane segment ring16", 0, 0, 0, 1, 16},
                           {"bulk contiguous 8KB ring12", 0, 0, 0, 2, 12}};
  for (const Var& v : vars) {
    std::vector<Item> items;
    std::vector<int> start(1, 0);
    for (int b = 0; b < nsm; ++b) {
      std::vector<std::pair<int, std::pair<int, int>>> segs;
      windows(b, segs);
      if (v.bulk == 2) {
        size_t per = (xbytes + nsm - 1) / nsm;
        per = (per + 15) & ~(size_t)15;
        for (size_t o = b * per; o < std::min(xbytes, (b + 1) * per); o += 8192)
          items.push_back({(int)o, (int)std::min((size_t)8192, std::min(xbytes, (b + 1) * per) - o)});
      } else {
        for (int ch = 0; ch < 2; ++ch)
          for (auto& s : segs) {
            int n = s.first, elo = s.second.first, ehi = s.second.second;
            if (v.bulk == 1) {
              for (int c = 0; c < 64; ++c) {
                int bytes = ((ehi - elo) * 2 + 15) & ~15;
                size_t off = ((size_t)(n * C + ch * 64 + c) * HW + elo) * 2;
                if (off + bytes > xbytes) bytes = (int)(xbytes - off);
                items.push_back({(int)off, bytes});
              }
            } else {
              for (int cc = 0; cc < 64; cc += v.box_c)
                for (int e = (v.box_e == 256 && v.box_c == 64) ? (elo & ~63) : elo; e < ehi; e += v.box_e)
                  items.push_back({e, n * C + ch * 64 + cc});
            }
          }
      }
      start.push_back((int)items.size());
    }
    cudaMemcpy(ditems, items.data(), items.size() * sizeof(Item), cudaMemcpyHostToDevice);
    cudaMemcpy(dstart, start.data(), start.size() * 4, cudaMemcpyHostToDevice);
    CUtensorMap tm{};
    int box_bytes = 0, slot = 8192;
    if (!v.bulk) {
      cuuint64_t dims[2] = {(cuuint64_t)HW, (cuuint64_t)N * C};
      cuuint64_t str[1] = {(cuuint64_t)HW * 2};
      cuuint32_t box[2] = {(cuuint32_t)v.box_e, (cuuint32_t)v.box_c};
      cuuint32_t es[2] = {1, 1};
      CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, x, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                       v.swz ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                       CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) { printf("encode failed %d\n", r); continue; }
      box_bytes = v.box_e * v.box_c * 2;
      slot = (box_bytes + 1023) & ~1023;
    }
    std::vector<float> ts;
    double spread = 0, medend = 0;
    for (int rep = 0; rep < 12; ++rep) {
      if (!noflush) flush_kernel<<<1184, 256>>>(fl, fn, sink);
      cudaEventRecord(e0);
      ring_load<<<nsm, 64, v.ring * slot + 2048>>>(tm, x, ditems, dstart, v.ring, slot, box_bytes, v.bulk ? 1 : 0,
                                                   tout);
      cudaEventRecord(e1);
      cudaError_t err = cudaDeviceSynchronize();
      if (err != cudaSuccess) { printf("%s: %s\n", v.name, cudaGetErrorString(err)); return 1; }
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (rep >= 2) ts.push_back(ms * 1000);
      std::vector<unsigned long long> h(2 * nsm);
      cudaMemcpy(h.data(), tout, 2 * nsm * 8, cudaMemcpyDeviceToHost);
      unsigned long long t0 = ~0ull;
      std::vector<double> ends;
      for (int b = 0; b < nsm; ++b) t0 = std::min(t0, h[2 * b]);
      for (int b = 0; b < nsm; ++b) ends.push_back((h[2 * b + 1] - t0) / 1e3);
      std::sort(ends.begin(), ends.end());
      spread = ends.back();
      medend = ends[nsm / 2];
    }
    std::sort(ts.begin(), ts.end());
    printf("%-36s items/CTA %4d  event med %6.2f us min %6.2f | CTA end med %5.2f max %5.2f us\n", v.name,
           (int)(items.size() / nsm), ts[ts.size() / 2], ts[0], medend, spread);
  }
  return 0;
}
