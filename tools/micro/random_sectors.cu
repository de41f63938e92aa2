// Microbenchmark: random-access throughput of B200 HBM (what bounds the sampling
// kernels: every pick touches one random 32-byte sector of the CSR, the relabel table
// and the CSR offsets).  Random 4-byte loads (one sector each) and random 16-byte loads
// over footprints from L2-resident to 8 GB, with U independent loads in flight per
// thread; and random 64-bit atomicMin (RED) over a 40 MB table.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o random_sectors random_sectors.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long mix(unsigned long long x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull;
  return x ^ (x >> 33);
}

template <int U, typename T>
__global__ void rnd_load(const T* __restrict__ a, unsigned long long n, int iters, T* out) {
  const unsigned long long tid = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x;
  T acc{};
  for (int it = 0; it < iters; ++it) {
    T x[U];
#pragma unroll
    for (int u = 0; u < U; ++u) x[u] = __ldcg(a + mix(tid * 1315423911ull + it * 977ull + u) % n);
#pragma unroll
    for (int u = 0; u < U; ++u) acc = acc + x[u];
  }
  if (acc == (T)123456789) out[0] = acc;
}

__global__ void rnd_red(unsigned long long* a, unsigned long long n, int iters) {
  const unsigned long long tid = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x;
  for (int it = 0; it < iters; ++it) {
    const unsigned long long i = mix(tid * 7919ull + it) % n;
    atomicMin(a + 2 * i, tid);
  }
}

int main() {
  const int grid = 148 * 8, block = 256, iters = 16;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  unsigned* buf;
  const size_t maxb = 8ull << 30;
  cudaMalloc(&buf, maxb);
  cudaMemset(buf, 1, maxb);
  unsigned* out;
  cudaMalloc(&out, 64);
  for (size_t fp : {32ull << 20, 256ull << 20, 1ull << 30, 8ull << 30}) {
    float ms;
#define RUN(U)                                                                          \
  {                                                                                     \
    rnd_load<U, unsigned><<<grid, block>>>(buf, fp / 4, iters, out);                    \
    cudaEventRecord(e0);                                                                \
    rnd_load<U, unsigned><<<grid, block>>>(buf, fp / 4, iters, out);                    \
    cudaEventRecord(e1);                                                                \
    cudaEventSynchronize(e1);                                                           \
    cudaEventElapsedTime(&ms, e0, e1);                                                  \
    const double acc = (double)grid * block * iters * U;                                \
    printf("footprint %5zu MB  u32 random loads U=%d: %7.2f G accesses/s = %7.1f GB/s of 32B sectors\n", \
           fp >> 20, U, acc / ms / 1e6, acc * 32 / ms / 1e6);                           \
  }
    RUN(1) RUN(4) RUN(8)
  }
  // random 64-bit atomicMin over a 40 MB table of 16-byte entries (the relabel table)
  {
    const unsigned long long n = (40ull << 20) / 16;
    float ms;
    rnd_red<<<grid, block>>>((unsigned long long*)buf, n, iters);
    cudaEventRecord(e0);
    rnd_red<<<grid, block>>>((unsigned long long*)buf, n, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("RED.MIN.64 random over 40 MB: %.2f G atomics/s\n", (double)grid * block * iters / ms / 1e6);
  }
  return 0;
}
