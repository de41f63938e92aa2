// Host-link split microbenchmark (extract misses): can a zero-copy gather of
// random 512-byte rows confined to the LOWER half of a 57 GB pinned matrix (so its 2 MB
// address translations stay cached) and a sequential zero-copy read of a separate pinned
// staging buffer (the host-gathered upper half) share the PCIe link at full rate?
//   A: random rows from the lower half (sorted), n_a rows
//   B: sequential read of an n_b-row staging buffer (written by the CPU long before, or
//      just before each repetition: "fresh")
// Each alone and both on two streams; a new random row set per repetition (same regions).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o split split.cu -lpthread
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <thread>
#include <vector>

#define CK(x)                                                  \
  do {                                                         \
    cudaError_t e = (x);                                       \
    if (e != cudaSuccess) {                                    \
      printf("%s: %s\n", #x, cudaGetErrorString(e));           \
      exit(1);                                                 \
    }                                                          \
  } while (0)

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

__global__ void __launch_bounds__(256) seqread(const float4* __restrict__ src, long long nvec, float4* __restrict__ out) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v0 = (long long)blockIdx.x * blockDim.x + threadIdx.x; v0 < nvec; v0 += stride * 4) {
    float4 x[4];
#pragma unroll
    for (int q = 0; q < 4; ++q)
      if (v0 + q * stride < nvec) x[q] = __ldcs(src + v0 + q * stride);
#pragma unroll
    for (int q = 0; q < 4; ++q)
      if (v0 + q * stride < nvec) __stcs(out + v0 + q * stride, x[q]);
  }
}

int main(int argc, char** argv) {
  const size_t G = (size_t)(argc > 1 ? atoll(argv[1]) : 57) << 30;
  const int rowb = 512, vpr = rowb / 16;
  const size_t nrows = G / rowb;
  char* h = (char*)aligned_alloc(1 << 21, G);
  {
    const int T = std::max(1u, std::thread::hardware_concurrency());
    std::vector<std::thread> th;
    for (int t = 0; t < T; ++t)
      th.emplace_back([=] {
        const size_t a = G / T * t, b = t == T - 1 ? G : G / T * (t + 1);
        for (size_t i = a; i < b; i += 4096) memset(h + i, 1, std::min<size_t>(4096, b - i));
      });
    for (auto& x : th) x.join();
  }
  CK(cudaHostRegister(h, G, cudaHostRegisterMapped | cudaHostRegisterPortable));
  char* hd;
  CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
  for (double fb : {0.25, 0.5}) {
    const int n = 442000, nb = (int)(n * fb), na = n - nb;
    char* stage;
    CK(cudaHostAlloc((void**)&stage, (size_t)nb * rowb, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(stage, 2, (size_t)nb * rowb);
    char* sd;
    CK(cudaHostGetDevicePointer((void**)&sd, stage, 0));
    unsigned* drows;
    CK(cudaMalloc(&drows, n * 4ull));
    float4 *oa, *ob;
    CK(cudaMalloc(&oa, (size_t)n * rowb));
    CK(cudaMalloc(&ob, (size_t)n * rowb));
    cudaStream_t s1, s2;
    cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaEvent_t e0, ea, eb;
    cudaEventCreate(&e0);
    cudaEventCreate(&ea);
    cudaEventCreate(&eb);
    std::mt19937_64 rng(11);
    const size_t lower = (size_t)(nrows * (1.0 - fb));  // A draws from rows [0, lower)
    for (int mode = 0; mode < 4; ++mode) {  // 0 A alone, 1 B alone, 2 both, 3 both + fresh B
      double best = 1e9, ta = 0, tb = 0;
      for (int rep = 0; rep < 6; ++rep) {
        std::vector<unsigned> r(na);
        for (int i = 0; i < na; ++i) r[i] = (unsigned)(rng() % lower);
        std::sort(r.begin(), r.end());
        CK(cudaMemcpy(drows, r.data(), na * 4ull, cudaMemcpyHostToDevice));
        if (mode == 3) memset(stage, rep, (size_t)nb * rowb);
        CK(cudaDeviceSynchronize());
        cudaEventRecord(e0, s1);
        cudaStreamWaitEvent(s2, e0, 0);
        if (mode != 1) gather<<<148, 256, 0, s1>>>((const float4*)hd, drows, na, vpr, oa);
        if (mode != 0) seqread<<<148, 256, 0, s2>>>((const float4*)sd, (long long)nb * vpr, ob);
        cudaEventRecord(ea, s1);
        cudaEventRecord(eb, s2);
        CK(cudaDeviceSynchronize());
        float ma, mb;
        cudaEventElapsedTime(&ma, e0, ea);
        cudaEventElapsedTime(&mb, e0, eb);
        const double t = std::max(mode == 1 ? 0.f : ma, mode == 0 ? 0.f : mb);
        if (rep >= 2 && t < best) { best = t; ta = ma; tb = mb; }
      }
      const double bytes = (mode == 0 ? (double)na : mode == 1 ? (double)nb : (double)n) * rowb;
      printf("fb=%.2f mode=%s: %.3f ms (A %.3f, B %.3f) -> %.1f GB/s\n", fb,
             mode == 0 ? "A_lower_random" : mode == 1 ? "B_staged_seq" : mode == 2 ? "both" : "both_freshB",
             best, ta, tb, bytes / best / 1e6);
    }
    cudaFreeHost(stage);
    cudaFree(drows);
    cudaFree(oa);
    cudaFree(ob);
  }
  return 0;
}
