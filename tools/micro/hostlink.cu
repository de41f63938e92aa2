// Host-link microbenchmark for the extract miss path (a7 misses, PAPER.md L79:
// Extract is "dominated by loading features ... due to the limited PCIe
// bandwidth").  Measures on one B200, over a pinned host region of G GB:
//   1. DMA H2D (copy engine), one 1 GiB copy and 4 MB chunks;
//   2. zero-copy row gathers by a kernel (n random rows of 512 B / 1 KB,
//      density of PA at alpha=0.22) in three orders: random, binned by 2 MB
//      page, fully sorted by address;
//   3. a host-thread row gather (memcpy of the same rows into a pinned
//      staging buffer) with T threads -- the CPU side of a gather+DMA path;
//   4. zero-copy gather and a DMA running concurrently (does the link add up?).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o hostlink hostlink.cu -lpthread -lcuda
// Run:   ./hostlink [GB=32] [mode: 0 cudaHostAlloc | 1 aligned_alloc+cudaHostRegister |
//                             2 cuMemCreate(HOST_NUMA) mapped for the GPU and the CPU]
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <thread>
#include <vector>

#define CK(x)                                                               \
  do {                                                                      \
    cudaError_t e = (x);                                                    \
    if (e != cudaSuccess) {                                                 \
      printf("%s: %s\n", #x, cudaGetErrorString(e));                        \
      exit(1);                                                              \
    }                                                                       \
  } while (0)

// 8 independent 16-byte loads per thread, rows spread over the block (as k_gather)
__global__ void __launch_bounds__(256) gather(const float4* __restrict__ src, const unsigned* __restrict__ rows,
                                              int n, int vpr, float4* __restrict__ out) {
  const long long total = (long long)n * vpr;
  const long long stride = (long long)gridDim.x * blockDim.x * 8;
  for (long long base = ((long long)blockIdx.x * blockDim.x) * 8 + threadIdx.x; base < total; base += stride) {
    float4 x[8];
    long long dst[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const long long v = base + (long long)q * blockDim.x;
      if (v < total) {
        const long long r = v / vpr, c = v - r * vpr;
        x[q] = __ldg(src + (size_t)rows[r] * vpr + c);
        dst[q] = v;
      }
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const long long v = base + (long long)q * blockDim.x;
      if (v < total) __stcs(out + dst[q], x[q]);
    }
  }
}

static double now() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main(int argc, char** argv) {
  const size_t G = (size_t)(argc > 1 ? atoll(argv[1]) : 32) << 30;
  const int mode = argc > 2 ? atoi(argv[2]) : 0;
  const bool reg = mode == 1;
  char* h = nullptr;
  double t0 = now();
  size_t gran = 0;
  if (mode == 2) {  // VMM host allocation: the GPU maps it with the allocation granularity
    CK(cudaFree(0));
    CUmemAllocationProp prop = {};
    prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop.location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA;
    prop.location.id = 0;
    if (cuMemGetAllocationGranularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS) {
      printf("granularity query failed\n");
      return 1;
    }
    size_t mgran = 0;
    cuMemGetAllocationGranularity(&mgran, &prop, CU_MEM_ALLOC_GRANULARITY_MINIMUM);
    printf("vmm host granularity recommended %zu minimum %zu\n", gran, mgran);
    CUdeviceptr va;
    CUmemGenericAllocationHandle hd;
    CUresult r;
    if ((r = cuMemAddressReserve(&va, G, gran, 0, 0)) != CUDA_SUCCESS ||
        (r = cuMemCreate(&hd, G, &prop, 0)) != CUDA_SUCCESS || (r = cuMemMap(va, G, 0, hd, 0)) != CUDA_SUCCESS) {
      printf("vmm alloc failed: %d\n", (int)r);
      return 1;
    }
    CUmemAccessDesc acc[2] = {};
    acc[0].location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    acc[0].location.id = 0;
    acc[0].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    acc[1].location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA;
    acc[1].location.id = 0;
    acc[1].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    if ((r = cuMemSetAccess(va, G, acc, 2)) != CUDA_SUCCESS) {
      printf("cuMemSetAccess failed: %d\n", (int)r);
      return 1;
    }
    h = (char*)va;
  } else if (reg) {
    h = (char*)aligned_alloc(1 << 21, G);
  } else {
    CK(cudaHostAlloc((void**)&h, G, cudaHostAllocMapped | cudaHostAllocPortable));
  }
  {  // first touch in parallel
    const int T = std::max(1u, std::thread::hardware_concurrency());
    std::vector<std::thread> th;
    for (int t = 0; t < T; ++t)
      th.emplace_back([=] {
        const size_t a = G / T * t, b = t == T - 1 ? G : G / T * (t + 1);
        for (size_t i = a; i < b; i += 4096) memset(h + i, (int)(i >> 12) & 0x7f, std::min<size_t>(4096, b - i));
      });
    for (auto& x : th) x.join();
  }
  if (reg) CK(cudaHostRegister(h, G, cudaHostRegisterMapped | cudaHostRegisterPortable));
  printf("host region %zu GB (%s) ready in %.1f s; host threads %u\n", G >> 30,
         mode == 2 ? "cuMemCreate HOST_NUMA" : reg ? "aligned_alloc + cudaHostRegister" : "cudaHostAlloc",
         now() - t0, std::thread::hardware_concurrency());
  char* hd = h;
  if (mode != 2) CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
  float* d = nullptr;
  CK(cudaMalloc(&d, 1ull << 30));
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float ms;
  cudaStream_t s1, s2;
  cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);

  // ---- 1. DMA
  CK(cudaMemcpy(d, h, 1 << 30, cudaMemcpyHostToDevice));
  double best = 0;
  for (int it = 0; it < 3; ++it) {
    cudaEventRecord(a);
    cudaMemcpy(d, h + ((size_t)it << 30), 1 << 30, cudaMemcpyHostToDevice);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    best = std::max(best, (1 << 30) / ms / 1e6);
  }
  printf("dma_h2d_1GiB %.1f GB/s\n", best);
  best = 0;
  for (int it = 0; it < 3; ++it) {
    cudaEventRecord(a, s1);
    for (int c = 0; c < 256; ++c)
      cudaMemcpyAsync((char*)d + ((size_t)c << 22), h + ((size_t)c << 22) + ((size_t)it << 30), 1 << 22,
                      cudaMemcpyHostToDevice, s1);
    cudaEventRecord(b, s1);
    cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    best = std::max(best, (1 << 30) / ms / 1e6);
  }
  printf("dma_h2d_4MB_chunks %.1f GB/s\n", best);

  // ---- 2. zero-copy gathers
  const int n = 442000;  // PA alpha=0.22 misses per batch
  unsigned* drows;
  CK(cudaMalloc(&drows, n * 4ull));
  float4* out;
  CK(cudaMalloc(&out, (size_t)n * 1024));
  std::mt19937_64 rng(7);
  for (int rowb : {512, 1024}) {
    const size_t nrows = G / rowb;
    std::vector<unsigned> r(n);
    for (int i = 0; i < n; ++i) r[i] = (unsigned)(rng() % nrows);
    const int vpr = rowb / 16;
    for (int order = 0; order < 3; ++order) {
      std::vector<unsigned> o = r;
      const char* name = "random";
      if (order == 1) {
        const int sh = 21 - __builtin_ctz(rowb);
        std::stable_sort(o.begin(), o.end(), [&](unsigned x, unsigned y) { return (x >> sh) < (y >> sh); });
        name = "bin2MB";
      } else if (order == 2) {
        std::sort(o.begin(), o.end());
        name = "sorted";
      }
      CK(cudaMemcpy(drows, o.data(), n * 4ull, cudaMemcpyHostToDevice));
      for (int blocks : {296, 592, 1184}) {
        gather<<<blocks, 256>>>((const float4*)hd, drows, n, vpr, out);
        best = 0;
        for (int it = 0; it < 3; ++it) {
          cudaEventRecord(a);
          gather<<<blocks, 256>>>((const float4*)hd, drows, n, vpr, out);
          cudaEventRecord(b);
          cudaEventSynchronize(b);
          cudaEventElapsedTime(&ms, a, b);
          best = std::max(best, (double)n * rowb / ms / 1e6);
        }
        printf("zerocopy rows=%d order=%s blocks=%d %.1f GB/s\n", rowb, name, blocks, best);
      }
    }
    // ---- 3. host-thread gather into pinned staging
    char* stage;
    CK(cudaMallocHost((void**)&stage, (size_t)n * rowb));
    for (int T : {1, 4, 8, 16, 32}) {
      if (T > (int)std::thread::hardware_concurrency() * 2 || getenv("SKIP_CPU")) break;
      for (int order = 0; order < 3; order += 2) {
        std::vector<unsigned> o = r;
        if (order == 2) std::sort(o.begin(), o.end());
        double tb = 1e9;
        for (int it = 0; it < 3; ++it) {
          const double t1 = now();
          std::vector<std::thread> th;
          for (int t = 0; t < T; ++t)
            th.emplace_back([&, t] {
              const int lo = (int)((long long)n * t / T), hi = (int)((long long)n * (t + 1) / T);
              for (int i = lo; i < hi; ++i) memcpy(stage + (size_t)i * rowb, h + (size_t)o[i] * rowb, rowb);
            });
          for (auto& x : th) x.join();
          tb = std::min(tb, now() - t1);
        }
        printf("cpu_gather rows=%d order=%s threads=%d %.1f GB/s\n", rowb, order ? "sorted" : "random", T,
               (double)n * rowb / tb / 1e9);
      }
    }
    // ---- 4. concurrent: zero-copy gather (sorted) + DMA of the staging buffer
    {
      std::vector<unsigned> o = r;
      std::sort(o.begin(), o.end());
      CK(cudaMemcpy(drows, o.data(), n * 4ull, cudaMemcpyHostToDevice));
      const size_t dbytes = (size_t)n * rowb;
      cudaEvent_t c0, c1;
      cudaEventCreate(&c0);
      cudaEventCreate(&c1);
      CK(cudaDeviceSynchronize());
      cudaEventRecord(a, s1);
      cudaStreamWaitEvent(s2, a, 0);
      gather<<<592, 256, 0, s1>>>((const float4*)hd, drows, n, vpr, out);
      cudaMemcpyAsync(d, stage, std::min(dbytes, (size_t)1 << 30), cudaMemcpyHostToDevice, s2);
      cudaEventRecord(c0, s1);
      cudaEventRecord(c1, s2);
      cudaEventSynchronize(c0);
      cudaEventSynchronize(c1);
      float m0, m1;
      cudaEventElapsedTime(&m0, a, c0);
      cudaEventElapsedTime(&m1, a, c1);
      const double tot = (double)dbytes + std::min(dbytes, (size_t)1 << 30);
      printf("concurrent rows=%d zerocopy %.3f ms + dma %.3f ms: aggregate %.1f GB/s\n", rowb, m0, m1,
             tot / std::max(m0, m1) / 1e6);
    }
    cudaFreeHost(stage);
  }
  return 0;
}
