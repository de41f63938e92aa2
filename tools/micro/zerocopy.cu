// Host-link microbenchmark (B200 over PCIe): DMA H2D bandwidth and zero-copy
// kernel reads of pinned host memory -- sequential, and random rows of 512 B /
// 1 KB over a small (64 MB) and a large (32 GB) region.  Sets the host-link
// roofline of the extract miss path.
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include <vector>
#include <algorithm>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)
__global__ void rows_read(const float4* __restrict__ src, const unsigned* __restrict__ rows, int n,
                          int vpr, float4* __restrict__ out) {
  // one warp per row group, lanes over 16-byte vectors
  const int lane = threadIdx.x & 31;
  const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, nw = (gridDim.x * blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (int r = w; r < n; r += nw) {
    const float4* p = src + (size_t)rows[r] * vpr;
    for (int c = lane; c < vpr; c += 32) { float4 x = p[c]; acc.x += x.x; acc.y += x.y; acc.z += x.z; acc.w += x.w; }
  }
  if (acc.x == 12345.f) out[0] = acc;
}
int main(int argc, char** argv) {
  const size_t big = (argc > 1 ? atoll(argv[1]) : 32) << 30;
  float* h; CK(cudaHostAlloc(&h, big, cudaHostAllocMapped | cudaHostAllocPortable));
  for (size_t i = 0; i < big / 4; i += 1024) h[i] = 1.f;
  float* d; CK(cudaMalloc(&d, 1 << 30));
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float ms;
  cudaMemcpy(d, h, 1 << 30, cudaMemcpyHostToDevice);
  cudaEventRecord(a); cudaMemcpy(d, h, 1 << 30, cudaMemcpyHostToDevice); cudaEventRecord(b); cudaEventSynchronize(b);
  cudaEventElapsedTime(&ms, a, b); printf("DMA H2D 1 GiB: %.1f GB/s\n", (1 << 30) / ms / 1e6);
  float4* hd; CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
  float4* o; cudaMalloc(&o, 64);
  for (int rowb : {512, 1024}) {
    const int vpr = rowb / 16;
    for (size_t region : {(size_t)64 << 20, big}) {
      const int n = 400000;
      std::vector<unsigned> r(n);
      const size_t nrows = region / rowb;
      srand(7);
      for (int i = 0; i < n; ++i) r[i] = (unsigned)(((size_t)rand() * 65536 + rand()) % nrows);
      unsigned* dr; cudaMalloc(&dr, n * 4);
      if (getenv("SORTED")) std::sort(r.begin(), r.end());
      cudaMemcpy(dr, r.data(), n * 4, cudaMemcpyHostToDevice);
      for (int blocks : {148, 592, 1184}) {
        rows_read<<<blocks, 256>>>(hd, dr, n, vpr, o);
        cudaEventRecord(a); rows_read<<<blocks, 256>>>(hd, dr, n, vpr, o); cudaEventRecord(b); cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("zero-copy random %4d B rows over %6zu MB, %4d blocks: %.1f GB/s (%.1f M rows/s)\n", rowb, region >> 20, blocks,
               (double)n * rowb / ms / 1e6, n / ms / 1e3);
      }
      // sequential rows
      for (int i = 0; i < n; ++i) r[i] = i;
      cudaMemcpy(dr, r.data(), n * 4, cudaMemcpyHostToDevice);
      cudaEventRecord(a); rows_read<<<592, 256>>>(hd, dr, n, vpr, o); cudaEventRecord(b); cudaEventSynchronize(b);
      cudaEventElapsedTime(&ms, a, b);
      printf("zero-copy sequential %4d B rows: %.1f GB/s\n", rowb, (double)n * rowb / ms / 1e6);
      cudaFree(dr);
    }
  }
  return 0;
}
