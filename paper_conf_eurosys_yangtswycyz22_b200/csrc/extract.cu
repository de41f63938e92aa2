// extract.cu -- a4 (mark) for arbitrary id lists and a7 (extract) for sm_100a.
//
// Paper: "the Trainer will simultaneously extract their features from host
// memory and the feature cache in GPU memory" (§5.2); Extract
// time is "mainly dominated by loading features ... from host memory ... due
// to the limited PCIe bandwidth" (L79 §2).
//
// One persistent launch serves both halves: blocks [0, H) gather cache hits
// from HBM, blocks [H, grid) gather misses straight from the mapped pinned
// host matrix (zero copy over PCIe), so the HBM gather never waits behind
// PCIe latency and no CPU thread touches feature bytes.  Rows move as 16-byte
// vectors (LDG.128/STG.128), each row handled by a group of lanes, four rows
// in flight per group.
#include <cuda_runtime.h>

#include "glb_internal.cuh"

namespace glb {

namespace {

constexpr unsigned kFull = 0xFFFFFFFFu;

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__global__ void __launch_bounds__(kThreads)
    k_mark(const uint32_t* __restrict__ vertices, uint64_t n, uint64_t V,
           const int32_t* __restrict__ slot, DevState* st, uint32_t* __restrict__ hit_dst,
           uint32_t* __restrict__ hit_src, uint32_t* __restrict__ miss_dst,
           uint32_t* __restrict__ miss_src) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i0 = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u); i0 < n; i0 += stride) {
    const uint64_t i = i0 + (threadIdx.x & 31);
    const bool act = i < n;
    uint32_t u = 0;
    int32_t s = -1;
    if (act) {
      u = vertices[i];
      if (u >= V) {
        atomicOr(&st->err, kErrRange);
        u = 0;
      }
      s = __ldg(slot + u);
    }
    const bool hit = act && s >= 0, miss = act && s < 0;
    const uint32_t mh = __ballot_sync(kFull, hit), mm = __ballot_sync(kFull, miss);
    const int lane = threadIdx.x & 31;
    uint32_t bh = 0, bm = 0;
    if (lane == 0) {
      if (mh) bh = atomicAdd(&st->nhit, (uint32_t)__popc(mh));
      if (mm) bm = atomicAdd(&st->nmiss, (uint32_t)__popc(mm));
    }
    bh = __shfl_sync(kFull, bh, 0);
    bm = __shfl_sync(kFull, bm, 0);
    if (hit) {
      const uint32_t r = bh + __popc(mh & lanemask_lt());
      hit_dst[r] = (uint32_t)i;
      hit_src[r] = (uint32_t)s;
    }
    if (miss) {
      const uint32_t r = bm + __popc(mm & lanemask_lt());
      miss_dst[r] = (uint32_t)i;
      miss_src[r] = u;
    }
  }
}

// Gather rows src[src_idx[r]] -> out[dst_idx ? dst_idx[r] : r] for both lists.
// LPR lanes per row; VEC: 16-byte vectors (row bytes % 16 == 0).
template <int LPR, bool VEC>
__global__ void __launch_bounds__(kThreads)
    k_gather(float* __restrict__ out, const float* __restrict__ src_hit,
             const float* __restrict__ src_miss, const uint32_t* __restrict__ hit_dst,
             const uint32_t* __restrict__ hit_src, const uint32_t* __restrict__ miss_dst,
             const uint32_t* __restrict__ miss_src, const uint32_t* __restrict__ dev_counts,
             uint64_t nh_host, uint64_t nm_host, uint32_t D, unsigned long long* xcount) {
  const uint64_t nh = dev_counts ? dev_counts[0] : nh_host;
  const uint64_t nm = dev_counts ? dev_counts[1] : nm_host;
  const uint32_t G = gridDim.x;
  uint32_t miss_blocks = 0;
  if (nm) miss_blocks = nh ? max(1u, G / 4) : G;
  const bool is_miss = blockIdx.x >= G - miss_blocks;
  const uint32_t rb = is_miss ? blockIdx.x - (G - miss_blocks) : blockIdx.x;
  const uint32_t nrb = is_miss ? miss_blocks : G - miss_blocks;
  const uint64_t n = is_miss ? nm : nh;
  const uint32_t* dlist = is_miss ? miss_dst : hit_dst;
  const uint32_t* slist = is_miss ? miss_src : hit_src;
  const float* src = is_miss ? src_miss : src_hit;
  if (xcount && blockIdx.x == 0 && threadIdx.x == 0) {
    xcount[0] = nh;
    xcount[1] = nm;
  }
  if (n == 0) return;
  const uint32_t li = threadIdx.x % LPR;
  const uint64_t grp = ((uint64_t)rb * blockDim.x + threadIdx.x) / LPR;
  const uint64_t ngrp = (uint64_t)nrb * blockDim.x / LPR;
  constexpr int U = 4;
  if (VEC) {
    const uint32_t vpr = D / 4;
    const float4* s4 = reinterpret_cast<const float4*>(src);
    float4* o4 = reinterpret_cast<float4*>(out);
    for (uint64_t r0 = grp; r0 < n; r0 += U * ngrp) {
      uint64_t so[U], dof[U];
      bool ok[U];
#pragma unroll
      for (int q = 0; q < U; ++q) {
        const uint64_t r = r0 + q * ngrp;
        ok[q] = r < n;
        so[q] = ok[q] ? (uint64_t)__ldg(slist + r) * vpr : 0;
        dof[q] = ok[q] ? (uint64_t)(dlist ? __ldg(dlist + r) : r) * vpr : 0;
      }
      for (uint32_t c = li; c < vpr; c += LPR) {
        float4 x[U];
#pragma unroll
        for (int q = 0; q < U; ++q)
          if (ok[q]) x[q] = __ldg(s4 + so[q] + c);
#pragma unroll
        for (int q = 0; q < U; ++q)
          if (ok[q]) o4[dof[q] + c] = x[q];
      }
    }
  } else {
    for (uint64_t r0 = grp; r0 < n; r0 += U * ngrp) {
      uint64_t so[U], dof[U];
      bool ok[U];
#pragma unroll
      for (int q = 0; q < U; ++q) {
        const uint64_t r = r0 + q * ngrp;
        ok[q] = r < n;
        so[q] = ok[q] ? (uint64_t)__ldg(slist + r) * D : 0;
        dof[q] = ok[q] ? (uint64_t)(dlist ? __ldg(dlist + r) : r) * D : 0;
      }
      for (uint32_t c = li; c < D; c += LPR) {
        float x[U];
#pragma unroll
        for (int q = 0; q < U; ++q)
          if (ok[q]) x[q] = __ldg(src + so[q] + c);
#pragma unroll
        for (int q = 0; q < U; ++q)
          if (ok[q]) out[dof[q] + c] = x[q];
      }
    }
  }
}

}  // namespace

cudaError_t launch_mark(glb_ctx* c, const uint32_t* vertices, uint64_t n) {
  int grid = (int)((n + kThreads - 1) / kThreads);
  if (grid < 1) grid = 1;
  if (grid > c->num_sms * 8) grid = c->num_sms * 8;
  k_mark<<<grid, kThreads, 0, c->stream>>>(vertices, n, c->V, c->slot, c->st_x, c->xb.hit_dst,
                                           c->xb.hit_src, c->xb.miss_dst, c->xb.miss_src);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_gather(glb_ctx* c, float* out, const float* src_hit, const float* src_miss,
                          const uint32_t* hit_dst, const uint32_t* hit_src,
                          const uint32_t* miss_dst, const uint32_t* miss_src,
                          const uint32_t* dev_counts, uint64_t nhit_host, uint64_t nmiss_host) {
  const uint32_t D = c->D;
  const bool vec = (D % 4) == 0;
  const uint32_t units = vec ? D / 4 : D;  // per-row work units
  const int grid = c->num_sms * 8;
#define GLB_GATHER_ARGS                                                                   \
  out, src_hit, src_miss, hit_dst, hit_src, miss_dst, miss_src, dev_counts, nhit_host, \
      nmiss_host, D, c->xcount
  if (vec) {
    if (units <= 8) k_gather<8, true><<<grid, kThreads, 0, c->stream>>>(GLB_GATHER_ARGS);
    else if (units <= 16) k_gather<16, true><<<grid, kThreads, 0, c->stream>>>(GLB_GATHER_ARGS);
    else k_gather<32, true><<<grid, kThreads, 0, c->stream>>>(GLB_GATHER_ARGS);
  } else {
    if (units <= 8) k_gather<8, false><<<grid, kThreads, 0, c->stream>>>(GLB_GATHER_ARGS);
    else if (units <= 16) k_gather<16, false><<<grid, kThreads, 0, c->stream>>>(GLB_GATHER_ARGS);
    else k_gather<32, false><<<grid, kThreads, 0, c->stream>>>(GLB_GATHER_ARGS);
  }
#undef GLB_GATHER_ARGS
  count_launch(c);
  return cudaGetLastError();
}

}  // namespace glb
