// Microbenchmark: dependent global-load latency (pointer chase) and kernel
// launch gap on this B200.  nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cstdio>
#include <cuda_runtime.h>
#include <vector>
__global__ void chase(const unsigned* __restrict__ p, int steps, unsigned* out, long long* cyc) {
  unsigned x = 0;
  long long t0 = clock64();
  for (int i = 0; i < steps; ++i) x = p[x];
  long long t1 = clock64();
  out[0] = x;
  cyc[0] = t1 - t0;
}
__global__ void empty() {}
int main() {
  for (size_t n : {1u << 12, 1u << 20, 1u << 24, 1u << 28}) {  // 16 KB .. 1 GB
    std::vector<unsigned> h(n);
    unsigned stride = 4099;  // odd stride in words, visits all entries (n power of 2)
    for (size_t i = 0; i < n; ++i) h[i] = (unsigned)((i + stride * 8) % n);
    unsigned *d, *o; long long* c;
    cudaMalloc(&d, n * 4); cudaMalloc(&o, 4); cudaMalloc(&c, 8);
    cudaMemcpy(d, h.data(), n * 4, cudaMemcpyHostToDevice);
    chase<<<1, 1>>>(d, 1000, o, c);
    chase<<<1, 1>>>(d, 20000, o, c);
    long long cy; cudaMemcpy(&cy, c, 8, cudaMemcpyDeviceToHost);
    printf("footprint %8zu KB: %.1f cycles/load\n", n * 4 / 1024, cy / 20000.0);
    cudaFree(d); cudaFree(o); cudaFree(c);
  }
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int w = 0; w < 3; ++w) empty<<<148, 256>>>();
  cudaEventRecord(a);
  for (int i = 0; i < 1000; ++i) empty<<<148, 256>>>();
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  printf("empty kernel back-to-back: %.2f us/launch\n", ms);
  return 0;
}
