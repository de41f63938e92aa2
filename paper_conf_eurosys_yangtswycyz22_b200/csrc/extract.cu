// extract.cu -- a4 (mark) for arbitrary id lists and a7 (extract) for sm_100a.
//
// Paper: "the Trainer will simultaneously extract their features from host
// memory and the feature cache in GPU memory" (§5.2); Extract
// time is "mainly dominated by loading features ... from host memory ... due
// to the limited PCIe bandwidth" (L79 §2).
//
// One persistent launch serves both halves: chunks of cache hits (HBM) are handed
// out by one device counter and chunks of misses, read straight from mapped pinned
// host memory (zero copy over PCIe), by a second.  Which blocks take which: by
// default every block drains the hits and then takes misses; with a miss-block cap
// (one block per SM when host threads assist or on the pipelined extract stream)
// only the first blocks take misses, and on the extract stream they start on them
// ("misses first": the host link is the critical path) while the rest of the grid
// gathers the hits.  Misses arrive ordered by host address (launch_sort_misses),
// from the cold store when there is one (rank-ordered copy of the non-cached rows);
// a share of them can be gathered by host threads instead (hostgather.cu).
//
// A block copies a chunk of R rows per iteration: the chunk's (dst, src)
// work-list entries are staged in shared memory (double-buffered, the next
// chunk's entries are loaded while this chunk's rows are in flight), then the
// R*U 16-byte vectors (U = vectors per row) are spread over all 256 threads,
// 8 independent LDG.128 per thread issued before any store (MLP ~128 B per
// thread), stores streamed (st.global.cs).
#include <cuda_runtime.h>

#include "glb_internal.cuh"

namespace glb {

namespace {

constexpr unsigned kFull = 0xFFFFFFFFu;
#ifndef GLB_GATHER_VEC  // 16-byte vectors in flight per thread (A/B builds: -DGLB_GATHER_VEC=4)
#define GLB_GATHER_VEC 8
#endif
constexpr int kVecPerThread = GLB_GATHER_VEC;
constexpr int kChunkUnits = kThreads * kVecPerThread;  // vectors per chunk

struct ShardTab {
  const void* base[kMaxShards];
  uint32_t W, rank;
};

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__global__ void __launch_bounds__(kThreads)
    k_mark(const uint32_t* __restrict__ vertices, uint64_t n, const uint32_t* n_dev, uint64_t V,
           const int32_t* __restrict__ slot, DevState* st, uint2* __restrict__ hit_list,
           uint2* __restrict__ miss_list, int32_t* __restrict__ lidslot) {
  if (n_dev) n = *n_dev;  // count produced on the device (e.g. a received sample's n_L)
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
    if (lidslot && act) lidslot[i] = s;
    if (hit) hit_list[bh + __popc(mh & lanemask_lt())] = make_uint2((uint32_t)i, (uint32_t)s);
    if (miss) miss_list[bm + __popc(mm & lanemask_lt())] = make_uint2((uint32_t)i, u);
  }
}

// Feature-row loads.  GLB_GATHER_LD 0: __ldg; 1: ld.global.cs (evict-first in L1/L2);
// 2: ld.global.nc.L1::no_allocate with an L2 evict_first policy -- the gather streams
// hundreds of MB through L2 per batch, and evict-first keeps the next batch's relabel
// table / CSR offsets resident.
#ifndef GLB_GATHER_LD
#define GLB_GATHER_LD 0
#endif
__device__ __forceinline__ uint64_t l2_evict_first_policy() {
  uint64_t pol = 0;
#if GLB_GATHER_LD == 2
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
#endif
  return pol;
}
template <typename T>
__device__ __forceinline__ T ld_row(const T* p, uint64_t pol);
template <>
__device__ __forceinline__ float4 ld_row<float4>(const float4* p, uint64_t pol) {
#if GLB_GATHER_LD == 2
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
  return v;
#elif GLB_GATHER_LD == 3  // explicit 64-byte L2 prefetch size (A/B: DRAM over-fetch per row)
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
#elif GLB_GATHER_LD == 4  // 256-byte L2 prefetch size
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
#elif GLB_GATHER_LD == 1
  return __ldcs(p);
#else
  return __ldg(p);
#endif
}
template <>
__device__ __forceinline__ float ld_row<float>(const float* p, uint64_t pol) {
#if GLB_GATHER_LD == 2
  float v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;"
               : "=f"(v) : "l"(p), "l"(pol));
  return v;
#elif GLB_GATHER_LD == 3
  float v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
#elif GLB_GATHER_LD == 4
  float v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::256B.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
#elif GLB_GATHER_LD == 1
  return __ldcs(p);
#else
  return __ldg(p);
#endif
}
template <typename T>
__device__ __forceinline__ void st_row(T* p, T v) { __stcs(p, v); }

// T = float4 (row bytes % 16 == 0) or float.  U = T-units per row.
// Work: hit chunks first (HBM, fast), then miss chunks (host, PCIe); chunks are
// handed out by two device counters, so every block works on hits while there
// are any and then every block keeps PCIe requests in flight.
//
// SHARD (NEXT-3, peer-sharded cache): a hit's slot is a global cache rank i, owned
// by shard i % W at row i / W; tab.base[w] is shard w's rows (this GPU's own HBM or
// a peer's, mapped over NVLink).  The owner is resolved once per entry when the
// entry is staged, so the per-vector loop only indexes the shard table.
#ifndef GLB_GATHER_MINB  // min resident gather blocks per SM (register cap; A/B builds)
#define GLB_GATHER_MINB 4
#endif
template <typename T, bool SHARD>
__global__ void __launch_bounds__(kThreads, GLB_GATHER_MINB)
    k_gather(T* __restrict__ out, const T* __restrict__ src_hit, const T* __restrict__ src_miss,
             const uint2* __restrict__ hit_list, const uint2* __restrict__ miss_list,
             const uint32_t* __restrict__ fill_src, const uint32_t* __restrict__ dev_counts,
             uint64_t nh_host, uint64_t nm_host, uint32_t U, uint32_t R, uint32_t Sh, uint32_t So,
             int st_wb, int misses_only, unsigned long long* xcount, unsigned int* work,
             ShardTab tab, const int32_t* __restrict__ lidslot, const uint32_t* __restrict__ nl_dev) {
  // U: T-units per row moved; Sh: row stride of src_hit (the HBM cache may pad its rows);
  // So: row stride of out; host rows (src_miss) are dense (stride U)
  // lidslot (GLB_GATHER_LIDORDER): the hit phase walks lids 0..n_L-1 in order (nl_dev = n_L)
  // and takes the cached ones (lidslot[lid] >= 0) instead of the hit list, so a chunk writes
  // consecutive output rows: row boundaries that share a 32-byte sector are written by the
  // same block at nearly the same time
  pdl_enter();
  // staged work entry: source row address and destination element offset, resolved once
  // per row so the per-vector loop is one LDS.128 + two adds
  struct __align__(16) RowEnt {
    const T* src;
    unsigned long long dst;
  };
  __shared__ RowEnt ent[2][kThreads];
  __shared__ unsigned int s_next;
  uint32_t npeer = 0;
  const uint64_t nh_all = dev_counts ? dev_counts[0] : nh_host;
  const uint64_t nm_all = dev_counts ? dev_counts[1] : nm_host;
  if (xcount && blockIdx.x == 0 && threadIdx.x == 0) {
    xcount[0] = nh_all;
    xcount[1] = nm_all;
  }
  const uint64_t nm = (misses_only & 2) ? 0 : nm_all;
  // skip bit 0: hits gathered by k_gather_bulk instead; bit 1: misses gathered by it;
  // bits 8..: how many blocks take host-miss chunks (0 = all; GLB_MISS_BLOCKS) -- fewer
  // requests in flight over the link touch fewer host pages at a time
  const uint64_t nh = (misses_only & 1) ? 0 : (lidslot ? (uint64_t)*nl_dev : nh_all);
  const uint32_t miss_blocks = (uint32_t)misses_only >> 8;
  const uint32_t t = threadIdx.x;
  const uint64_t nch = (nh + R - 1) / R, ncm = (nm + R - 1) / R;  // hit / miss chunks
  const float inv_u = 1.0f / (float)U;
  const uint64_t pol = l2_evict_first_policy();
  // chunk id g: g < nch -> hit chunk g; else miss chunk g - nch
  // bit 2 (misses first): the miss-taking blocks start on the host misses -- the critical
  // path of a host-bound extract -- and only then help with the hits, which the other
  // blocks gather meanwhile
  const bool misses_first = (misses_only & 4) && miss_blocks;
  auto claim = [&]() -> uint64_t {
    if (t == 0) {
      unsigned int g;
      if (misses_first && blockIdx.x < miss_blocks) {
        const unsigned int m = atomicAdd(&work[1], 1u);
        if (m < ncm) {
          g = (unsigned int)nch + m;
        } else {
          const unsigned int h = atomicAdd(&work[0], 1u);
          g = h < nch ? h : (unsigned int)(nch + ncm);
        }
      } else {
        g = atomicAdd(&work[0], 1u);
        if (g >= nch)  // only the first miss_blocks blocks take host chunks (0 = all)
          g = (miss_blocks && blockIdx.x >= miss_blocks) ? (unsigned int)(nch + ncm)
                                                         : (unsigned int)nch + atomicAdd(&work[1], 1u);
      }
      s_next = g;
    }
    __syncthreads();
    const uint64_t g = s_next;
    __syncthreads();
    return g;
  };
  // raw work-list entry of this thread in chunk g (kept in 2 registers while the current
  // chunk's rows are in flight) ...
  auto load_ent = [&](uint64_t g) -> uint2 {
    if (g >= nch + ncm || t >= R) return make_uint2(0u, 0u);
    const bool miss = g >= nch;
    const uint64_t r = (miss ? g - nch : g) * R + t;
    if (r >= (miss ? nm : nh)) return make_uint2(0u, 0u);
    if (!miss && lidslot) {  // lid order: a miss lid is a hole in this chunk
      const int32_t sl = __ldg(lidslot + r);
      return make_uint2((uint32_t)r, sl >= 0 ? (uint32_t)sl : kEmpty);
    }
    if (!miss) return __ldg(hit_list + r);
    return fill_src ? make_uint2((uint32_t)r, __ldg(fill_src + r)) : __ldg(miss_list + r);
  };
  // ... and resolved to (source row address, destination offset) when staged
  auto stage = [&](uint64_t g, uint2 h) -> RowEnt {
    RowEnt re;
    if (g >= nch) {
      re.src = src_miss + (uint64_t)h.y * U;
    } else if (h.y == kEmpty) {  // lid order: not cached (the miss phase gathers it)
      re.src = nullptr;
    } else if (SHARD) {
      const uint32_t w = h.y % tab.W;
      re.src = (const T*)tab.base[w] + (uint64_t)(h.y / tab.W) * Sh;
      npeer += (w != tab.rank) && (g * R + t < nh);
    } else {
      re.src = src_hit + (uint64_t)h.y * Sh;
    }
    re.dst = (unsigned long long)h.x * So;
    return re;
  };
  uint64_t g = claim();
  uint2 e = load_ent(g);
  int buf = 0;
  while (g < nch + ncm) {
    if (t < R) ent[buf][t] = stage(g, e);
    const uint64_t gn = claim();  // (its barrier also publishes ent[buf])
    e = load_ent(gn);             // prefetch the next chunk's entries
    const bool miss = g >= nch;
    const uint64_t c = miss ? g - nch : g;
    const uint64_t rows = min((uint64_t)R, (miss ? nm : nh) - c * R);
    const uint32_t total = (uint32_t)rows * U;
    for (uint32_t base = 0; base < total; base += kChunkUnits) {
      T x[kVecPerThread];
      unsigned long long dst[kVecPerThread];
      uint32_t live = 0;  // vectors of this thread that move a row (holes: lid order)
#pragma unroll
      for (int q = 0; q < kVecPerThread; ++q) {
        const uint32_t v = base + q * kThreads + t;
        if (v < total) {
          uint32_t row = (uint32_t)(((float)v + 0.5f) * inv_u);  // exact for v < 2^20
          const uint32_t col = v - row * U;
          const RowEnt en = ent[buf][row];
          if (en.src) {
            x[q] = ld_row(en.src + col, pol);
            dst[q] = en.dst + col;
            live |= 1u << q;
          }
        }
      }
#pragma unroll
      for (int q = 0; q < kVecPerThread; ++q) {
        if (live >> q & 1u) {
          if (st_wb) out[dst[q]] = x[q];
          else st_row(out + dst[q], x[q]);
        }
      }
    }
    buf ^= 1;
    g = gn;
  }
  if (SHARD) {  // rows this launch read from other GPUs' shards
    const uint32_t wsum = __reduce_add_sync(kFull, npeer);
    if ((t & 31) == 0 && wsum && xcount) atomicAdd(&xcount[2], (unsigned long long)wsum);
  }
  // the last block out re-arms the counters for the next launch on this stream
  if (t == 0) {
    __threadfence();
    if (atomicAdd(&work[2], 1u) == gridDim.x - 1) {
      work[0] = 0u;
      work[1] = 0u;
      work[2] = 0u;
    }
  }
}

// Warp-independent variant (GLB_GATHER_WARP=1): no block barrier anywhere.  Warp gw of
// NW takes chunks gw, gw + NW, ... of Rw rows (hit chunks first, then miss chunks, so all
// warps drain the HBM hits before the host misses); lane i < Rw loads and resolves the
// entry of row i of the chunk (prefetched one chunk ahead), and every 16-byte vector
// fetches its row's (source, destination) from the owning lane with two 64-bit shuffles.
// A block barrier per chunk makes every warp of the block wait for the slowest one -- on
// the PCIe path the slowest of 256 zero-copy rows carries the address-translation tail.
template <typename T, bool SHARD>
__global__ void __launch_bounds__(kThreads)
    k_gather_w(T* __restrict__ out, const T* __restrict__ src_hit, const T* __restrict__ src_miss,
               const uint2* __restrict__ hit_list, const uint2* __restrict__ miss_list,
               const uint32_t* __restrict__ fill_src, const uint32_t* __restrict__ dev_counts,
               uint64_t nh_host, uint64_t nm_host, uint32_t U, uint32_t Rw, uint32_t Sh,
               uint32_t So, int st_wb, int skip, unsigned long long* xcount, ShardTab tab) {
  pdl_enter();
  const uint64_t nh_all = dev_counts ? dev_counts[0] : nh_host;
  const uint64_t nm_all = dev_counts ? dev_counts[1] : nm_host;
  if (xcount && blockIdx.x == 0 && threadIdx.x == 0) {
    xcount[0] = nh_all;
    xcount[1] = nm_all;
  }
  const uint64_t nm = (skip & 2) ? 0 : nm_all;
  const uint64_t nh = (skip & 1) ? 0 : nh_all;
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t NW = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  const uint64_t nch = (nh + Rw - 1) / Rw, ncm = (nm + Rw - 1) / Rw, nc = nch + ncm;
  const float inv_u = 1.0f / (float)U;
  const uint64_t pol = l2_evict_first_policy();
  uint32_t npeer = 0;
  // this lane's work-list entry of chunk g (raw), and its resolved (source, destination)
  auto load_ent = [&](uint64_t g) -> uint2 {
    if (g >= nc || lane >= Rw) return make_uint2(0u, 0u);
    const bool miss = g >= nch;
    const uint64_t r = (miss ? g - nch : g) * Rw + lane;
    if (r >= (miss ? nm : nh)) return make_uint2(0u, 0u);
    if (!miss) return __ldg(hit_list + r);
    return fill_src ? make_uint2((uint32_t)r, __ldg(fill_src + r)) : __ldg(miss_list + r);
  };
  uint64_t g = gw;
  uint2 e = load_ent(g);
  while (g < nc) {
    const bool miss = g >= nch;
    const uint64_t c = miss ? g - nch : g;
    const uint32_t rows = (uint32_t)min((uint64_t)Rw, (miss ? nm : nh) - c * Rw);
    unsigned long long srcp = 0, dsto = (unsigned long long)e.x * So;
    if (miss) {
      srcp = (unsigned long long)(src_miss + (uint64_t)e.y * U);
    } else if (SHARD) {
      const uint32_t w = e.y % tab.W;
      srcp = (unsigned long long)((const T*)tab.base[w] + (uint64_t)(e.y / tab.W) * Sh);
      npeer += (w != tab.rank) && lane < rows;
    } else {
      srcp = (unsigned long long)(src_hit + (uint64_t)e.y * Sh);
    }
    const uint64_t gn = g + NW;
    e = load_ent(gn);  // next chunk's entry, in flight with this chunk's rows
    const uint32_t total = rows * U;
    for (uint32_t base = 0; base < total; base += 32 * kVecPerThread) {
      T x[kVecPerThread];
      unsigned long long dst[kVecPerThread];
#pragma unroll
      for (int q = 0; q < kVecPerThread; ++q) {
        const uint32_t v = base + q * 32 + lane;
        const uint32_t row = (uint32_t)(((float)v + 0.5f) * inv_u);  // exact for v < 2^20
        const unsigned long long s = __shfl_sync(kFull, srcp, row & 31);
        const unsigned long long d = __shfl_sync(kFull, dsto, row & 31);
        if (v < total) {
          const uint32_t col = v - row * U;
          x[q] = ld_row((const T*)s + col, pol);
          dst[q] = d + col;
        }
      }
#pragma unroll
      for (int q = 0; q < kVecPerThread; ++q) {
        const uint32_t v = base + q * 32 + lane;
        if (v < total) {
          if (st_wb) out[dst[q]] = x[q];
          else st_row(out + dst[q], x[q]);
        }
      }
    }
    g = gn;
  }
  if (SHARD) {
    const uint32_t wsum = __reduce_add_sync(kFull, npeer);
    if (lane == 0 && wsum && xcount) atomicAdd(&xcount[2], (unsigned long long)wsum);
  }
}

// ---- host-miss ordering: a one-pass counting sort of the miss list by the 2 MB
// host page its source row lives in, so consecutive zero-copy reads share GPU
// address translations (measured: random 512 B rows over 64 GB 35 -> 47 GB/s).
// cold_row (nullable): the cold store's row of each vertex (rank-ordered host copy of the
// non-cached rows, glb_set_cold_store) -- the misses are translated while they are ordered
__device__ __forceinline__ uint32_t host_row(uint32_t gid, const uint32_t* cold_row) {
  return cold_row ? __ldg(cold_row + gid) : gid;
}

__global__ void k_miss_hist(const uint2* __restrict__ miss, const uint32_t* __restrict__ nmiss,
                            uint32_t page_shift, unsigned int* __restrict__ bins,
                            const uint32_t* __restrict__ cold_row) {
  const uint32_t n = *nmiss;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    atomicAdd(&bins[host_row(miss[i].y, cold_row) >> page_shift], 1u);
}

__global__ void __launch_bounds__(1024) k_miss_scan(unsigned int* bins, uint32_t nb) {
  __shared__ unsigned int warp_tot[32];
  __shared__ unsigned int carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (uint32_t b0 = 0; b0 < nb; b0 += 1024) {
    const uint32_t i = b0 + threadIdx.x;
    const unsigned int x = i < nb ? bins[i] : 0u;
    unsigned int inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned int y = __shfl_up_sync(kFull, inc, o);
      if (lane >= o) inc += y;
    }
    if (lane == 31) warp_tot[w] = inc;
    __syncthreads();
    if (w == 0) {
      unsigned int t = warp_tot[lane], ti = t;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned int y = __shfl_up_sync(kFull, ti, o);
        if (lane >= o) ti += y;
      }
      warp_tot[lane] = ti - t;
    }
    __syncthreads();
    if (i < nb) bins[i] = carry + warp_tot[w] + inc - x;
    __syncthreads();
    if (threadIdx.x == 1023) carry += warp_tot[31] + inc;
    __syncthreads();
  }
}

__global__ void k_miss_scatter(const uint2* __restrict__ miss, const uint32_t* __restrict__ nmiss,
                               uint32_t page_shift, unsigned int* __restrict__ offs,
                               uint2* __restrict__ sorted, const uint32_t* __restrict__ cold_row) {
  const uint32_t n = *nmiss;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    uint2 m = miss[i];
    m.y = host_row(m.y, cold_row);
    sorted[atomicAdd(&offs[m.y >> page_shift], 1u)] = m;
  }
}

// ---- a7 hits through the TMA bulk-copy engine (cp.async.bulk, no tensor map):
// k_gather moves every 16-byte vector through registers, so it needs many resident
// threads (and registers) per SM -- exactly what the latency-bound sampler of the next
// batch, running concurrently at pipeline depth 2, needs too.  Here each lane of a
// one- or two-warp block owns a ring of P row slots in shared memory and streams its
// rows through it: bulk load global -> smem (completion on a per-slot mbarrier with the
// row's byte count), then bulk store smem -> out (bulk_group).  The copy engine keeps
// 32*NW*(P-1) rows in flight per SM with a handful of registers; the SM's warps stay
// free for the sampler.  Rows are 16-byte multiples (D % 4 == 0), all addresses
// 16-byte aligned.  Lane gl takes hit rows gl, gl + NL, ... (static; rows are uniform).
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(bar), "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_load(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
      ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
__device__ __forceinline__ void bulk_store(void* dst, uint32_t src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
               ::"l"(dst), "r"(src), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}

template <bool SHARD>
__global__ void __launch_bounds__(64)
    k_gather_bulk(uint8_t* __restrict__ out, const uint8_t* __restrict__ src_hit,
                  const uint2* __restrict__ hit_list, const uint32_t* __restrict__ dev_counts,
                  uint64_t nh_host, uint32_t row_bytes, uint64_t src_stride, uint32_t P,
                  unsigned long long* xcount, ShardTab tab, int which) {
  // which 0: hit list (dst row, cache slot) from the HBM cache; 1: miss list (dst row, gid)
  // from the mapped host matrix (src_hit = its device alias, dense rows)
  extern __shared__ __align__(128) uint8_t smem[];
  pdl_enter();
  const uint32_t lanes = blockDim.x;  // lanes of this block
  const uint32_t lane = threadIdx.x;
  // layout: [P][lanes] mbarriers (8 B), [P][lanes] destination rows (4 B), then the
  // [P][lanes] row slots (128-byte aligned)
  const uint32_t bar0 = smem_u32(smem);
  uint32_t* dstrow = reinterpret_cast<uint32_t*>(smem + (uint64_t)P * lanes * 8);
  const uint32_t slot0 = smem_u32(smem + (((uint64_t)P * lanes * 12 + 127) & ~127ull));
  auto bar = [&](uint32_t s) { return bar0 + (s * lanes + lane) * 8u; };
  auto slot = [&](uint32_t s) { return slot0 + (s * lanes + lane) * row_bytes; };
  for (uint32_t s = 0; s < P; ++s) mbar_init(bar(s), 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  // the bulk-copy instructions take uniform operands: the compiler issues every lane's copy
  // from one thread in turn, so another lane's barrier must be initialised first
  __syncthreads();
  const uint64_t nh = dev_counts ? dev_counts[which] : nh_host;
  if (xcount && blockIdx.x == 0 && lane == 0 && dev_counts) {
    xcount[0] = dev_counts[0];
    xcount[1] = dev_counts[1];
  }
  const uint64_t NL = (uint64_t)gridDim.x * lanes;
  const uint64_t gl = (uint64_t)blockIdx.x * lanes + lane;
  const uint64_t nk = gl < nh ? (nh - gl + NL - 1) / NL : 0;  // rows of this lane
  uint32_t npeer = 0;
  auto src_of = [&](uint2 h) -> const uint8_t* {
    if (SHARD) {
      const uint32_t w = h.y % tab.W;
      npeer += w != tab.rank;
      return (const uint8_t*)tab.base[w] + (uint64_t)(h.y / tab.W) * src_stride;
    }
    return src_hit + (uint64_t)h.y * src_stride;
  };
  auto issue = [&](uint64_t k) {  // load row k of this lane into slot k % P
    const uint2 h = __ldg(hit_list + gl + k * NL);
    const uint32_t s = (uint32_t)(k % P);
    dstrow[s * lanes + lane] = h.x;
    mbar_expect_tx(bar(s), row_bytes);
    bulk_load(slot(s), src_of(h), row_bytes, bar(s));
  };
  const uint64_t pro = nk < P ? nk : P;
#pragma unroll 1
  for (uint64_t k = 0; k < pro; ++k) issue(k);
#pragma unroll 1
  for (uint64_t k = 0; k < nk; ++k) {
    const uint32_t s = (uint32_t)(k % P);
    mbar_wait(bar(s), (uint32_t)((k / P) & 1));
    bulk_store(out + (uint64_t)dstrow[s * lanes + lane] * row_bytes, slot(s), row_bytes);
    // refill the slot of the previous row (P >= 2) once its store has read it; the store
    // just issued may stay in flight
    if (k >= 1 && k - 1 + P < nk) {
      asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      issue(k - 1 + P);
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");  // stores complete before exit
  if (SHARD) {
    const uint32_t wsum = __reduce_add_sync(kFull, npeer);
    if ((lane & 31) == 0 && wsum && xcount) atomicAdd(&xcount[2], (unsigned long long)wsum);
  }
}

}  // namespace

cudaError_t launch_sort_misses(glb_ctx* c, const uint2* miss, const uint32_t* nmiss_dev,
                               uint2* sorted) {
  // bins of 2^miss_bin_log2 bytes of the host matrix (rounded down to a power-of-2 row count);
  // with a cold store the entries' host rows are cold-store rows, ordered the same way
  const uint64_t row_bytes = 4ull * c->D;
  uint32_t shift = 0;
  const uint32_t lg = c->miss_bin_log2 ? c->miss_bin_log2 : 21;  // the cold store needs the pass
  while ((row_bytes << (shift + 1)) <= (1ull << lg)) ++shift;
  const uint32_t nb = (uint32_t)((c->V >> shift) + 1);
  if (nb > c->miss_bins_cap) return cudaErrorInvalidValue;
  cudaError_t e = cudaMemsetAsync(c->miss_bins, 0, sizeof(unsigned int) * nb, c->stream);
  if (e != cudaSuccess) return e;
  const int grid = c->num_sms * 4;
  k_miss_hist<<<grid, kThreads, 0, c->stream>>>(miss, nmiss_dev, shift, c->miss_bins, c->cold_row);
  count_launch(c);
  unsigned int* offs = c->miss_bins;
  if (nb <= 8192) {  // a few coarse bins: one block scans them in place
    k_miss_scan<<<1, 1024, 0, c->stream>>>(c->miss_bins, nb);
    count_launch(c);
  } else {  // many fine bins: the three-phase device scan
    offs = c->miss_bins + c->miss_bins_cap;
    e = scan_exclusive_u32(c, c->miss_bins, nb, offs, offs + c->miss_bins_cap);
    if (e != cudaSuccess) return e;
  }
  k_miss_scatter<<<grid, kThreads, 0, c->stream>>>(miss, nmiss_dev, shift, offs, sorted, c->cold_row);
  count_launch(c);
  return cudaGetLastError();
}

uint32_t miss_bins_needed(const glb_ctx* c, uint64_t V, uint32_t D, uint32_t* scan_sums) {
  const uint64_t row_bytes = 4ull * D;
  uint32_t shift = 0;
  while ((row_bytes << (shift + 1)) <= (1ull << c->miss_bin_log2)) ++shift;
  const uint32_t nb = (uint32_t)((V >> shift) + 1);
  *scan_sums = (uint32_t)((nb + kThreads * 16 - 1) / (kThreads * 16)) + 1;
  return nb;
}

cudaError_t launch_mark(glb_ctx* c, const uint32_t* vertices, uint64_t n) {
  return launch_mark_to(c, vertices, n, nullptr, c->st_x, c->xb.hit_list, c->xb.miss_list, nullptr);
}

cudaError_t launch_mark_to(glb_ctx* c, const uint32_t* vertices, uint64_t n, const uint32_t* n_dev,
                           DevState* st, uint2* hit_list, uint2* miss_list, int32_t* lidslot) {
  int grid = (int)((n + kThreads - 1) / kThreads);
  if (grid < 1) grid = 1;
  if (grid > c->num_sms * 8) grid = c->num_sms * 8;
  k_mark<<<grid, kThreads, 0, c->stream>>>(vertices, n, n_dev, c->V, c->slot, st, hit_list,
                                           miss_list, lidslot);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_gather(glb_ctx* c, float* out, const float* src_hit, const float* src_miss,
                          const uint2* hit_list, const uint2* miss_list, const uint32_t* fill_src,
                          const uint32_t* dev_counts, uint64_t nhit_host, uint64_t nmiss_host,
                          const int32_t* lidslot, const uint32_t* nl_dev) {
  const uint32_t D = c->D;
  const bool vec = (D % 4) == 0;
  const uint32_t U = vec ? D / 4 : D;
  uint32_t R = kChunkUnits / U;
  if (R > (uint32_t)kThreads) R = kThreads;
  if (R < 1) R = 1;
  const int grid = c->num_sms * (c->stream == c->xstream ? c->gather_bps_pipe : c->gather_bps);
  // row strides in T units: the HBM cache's rows may be padded (glb_ctx::cache_stride)
  const uint32_t cs = c->cache_stride ? c->cache_stride : D;
  const uint32_t Sh = vec ? cs / 4 : cs;
  const uint32_t So = out == c->cache ? Sh : U;
  const int wb = c->gather_st_wb;
  int mo = 0;
  // hits through the bulk-copy engine (sample / generic extracts, rows of 16-byte vectors)
  if (c->gather_bulk && vec && hit_list && !fill_src && out != c->cache) {
    const uint32_t lanes = 64, row_bytes = 4 * D;
    uint32_t P = (uint32_t)((uint64_t)c->gather_bulk_smem / ((uint64_t)lanes * row_bytes));
    if (P > 16) P = 16;
    if (P >= 2) {
      const size_t smem = (((size_t)P * lanes * 12 + 127) & ~(size_t)127) + (size_t)P * lanes * row_bytes;
      const bool shard = c->shard_world > 1 && src_hit == c->cache;
      ShardTab tab = {};
      tab.W = c->shard_world;
      tab.rank = c->shard_rank;
      for (uint32_t w = 0; w < c->shard_world; ++w) tab.base[w] = c->shard_base[w];
      cudaError_t e;
      if (shard && (e = cudaMemsetAsync(c->xcount + 2, 0, sizeof(unsigned long long), c->stream)) != cudaSuccess)
        return e;
      auto kern = shard ? k_gather_bulk<true> : k_gather_bulk<false>;
      if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) != cudaSuccess)
        return e;
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(c->num_sms);
      cfg.blockDim = dim3(lanes);
      cfg.dynamicSmemBytes = smem;
      cfg.stream = c->stream;
      cudaLaunchAttribute attr[1];
      attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      attr[0].val.programmaticStreamSerializationAllowed = 1;
      cfg.attrs = attr;
      cfg.numAttrs = 1;
      const uint64_t stride = 4ull * (c->cache_stride ? c->cache_stride : D);
      e = cudaLaunchKernelEx(&cfg, kern, (uint8_t*)out, (const uint8_t*)src_hit, hit_list,
                             dev_counts, (uint64_t)nhit_host, row_bytes, stride, P, c->xcount, tab, 0);
      count_launch(c);
      if (e != cudaSuccess) return e;
      if (c->C >= c->V) return cudaSuccess;  // every vertex cached: no misses to gather
      mo = 1;  // the misses follow on the LSU path (host memory over PCIe)
    }
  }
  // misses through the bulk-copy engine (GLB_MISS_BULK=1): one cp.async.bulk per host row
  if (c->miss_bulk && vec && hit_list && miss_list && !fill_src && out != c->cache &&
      dev_counts && c->C < c->V) {
    const uint32_t lanes = 32, row_bytes = 4 * D;
    uint32_t P = (uint32_t)((uint64_t)c->gather_bulk_smem / ((uint64_t)lanes * row_bytes));
    if (P > 16) P = 16;
    if (P >= 2) {
      const size_t smem = (((size_t)P * lanes * 12 + 127) & ~(size_t)127) + (size_t)P * lanes * row_bytes;
      cudaError_t e;
      if ((e = cudaFuncSetAttribute(k_gather_bulk<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) != cudaSuccess)
        return e;
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(c->num_sms);
      cfg.blockDim = dim3(lanes);
      cfg.dynamicSmemBytes = smem;
      cfg.stream = c->stream;
      cudaLaunchAttribute attr[1];
      attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      attr[0].val.programmaticStreamSerializationAllowed = 1;
      cfg.attrs = attr;
      cfg.numAttrs = 1;
      ShardTab tab0 = {};
      e = cudaLaunchKernelEx(&cfg, k_gather_bulk<false>, (uint8_t*)out, (const uint8_t*)src_miss,
                             miss_list, dev_counts, (uint64_t)0, row_bytes, (uint64_t)row_bytes, P,
                             c->xcount, tab0, 1);
      count_launch(c);
      if (e != cudaSuccess) return e;
      if (mo) return cudaSuccess;  // hits were bulk-gathered too
      mo = 2;                      // the LSU gather does the hits only
    }
  }
  // blocks that take host-miss chunks: GLB_MISS_BLOCKS, else one per SM while the host
  // takes a share of the misses (measured on PA: fewer zero-copy rows in flight touch
  // fewer host pages at once -- 5.20-5.23 vs 5.35 ms per step; profiles/r02_missblocks.txt)
  // On the extract stream (pipeline depth 2) a sample's host misses are the critical path:
  // one block per SM takes them, and those blocks start on them (misses first) while the
  // other half of the grid gathers the HBM hits -- measured on PA / UK / TW at the paper's
  // R%: 5.08-5.14 vs 5.29-5.39, 6.07-6.15 vs 6.36, 7.80 vs 8.18-8.54 ms per step
  // (profiles/r02_missesfirst_ab.txt).  GLB_MISS_BLOCKS / GLB_MISSES_FIRST override.
  const bool pipe_misses = c->stream == c->xstream && miss_list && c->C < c->V;
  const uint32_t mb = c->miss_blocks ? c->miss_blocks
                      : ((c->hg_inflight || pipe_misses) ? (uint32_t)c->num_sms : 0u);
  const bool first = c->misses_first >= 0 ? c->misses_first != 0 : pipe_misses;
  const int mfirst = (mb && first) ? 4 : 0;
  // chunk counters of the launching stream (this ctx's gathers are serial on it; each
  // launch leaves them zeroed for the next)
  unsigned int* work = c->stream == c->xstream ? c->work + 4 : c->work;
  // sharded only for sample/extract gathers that read the cache (not the cache fill)
  const bool shard = c->shard_world > 1 && src_hit == c->cache && hit_list;
  ShardTab tab = {};
  tab.W = c->shard_world;
  tab.rank = c->shard_rank;
  for (uint32_t w = 0; w < c->shard_world; ++w) tab.base[w] = c->shard_base[w];
  cudaError_t e;
  if (shard && !mo && (e = cudaMemsetAsync(c->xcount + 2, 0, sizeof(unsigned long long), c->stream)) != cudaSuccess)
    return e;
  if (c->gather_warp) {  // warp-independent gather (no block barriers; hit list order)
    uint32_t Rw = (uint32_t)(32 * kVecPerThread) / U;
    Rw = Rw < 1 ? 1 : Rw > 32 ? 32 : Rw;
    const int gridw = c->num_sms * (c->stream == c->xstream ? c->gather_bps_pipe : c->gather_bps);
    if (vec && shard)
      e = launch_pdl(k_gather_w<float4, true>, gridw, kThreads, c->stream, (float4*)out,
                     (const float4*)src_hit, (const float4*)src_miss, hit_list, miss_list, fill_src,
                     dev_counts, nhit_host, nmiss_host, U, Rw, Sh, So, wb, mo, c->xcount, tab);
    else if (vec)
      e = launch_pdl(k_gather_w<float4, false>, gridw, kThreads, c->stream, (float4*)out,
                     (const float4*)src_hit, (const float4*)src_miss, hit_list, miss_list, fill_src,
                     dev_counts, nhit_host, nmiss_host, U, Rw, Sh, So, wb, mo, c->xcount, tab);
    else if (shard)
      e = launch_pdl(k_gather_w<float, true>, gridw, kThreads, c->stream, out, src_hit, src_miss,
                     hit_list, miss_list, fill_src, dev_counts, nhit_host, nmiss_host, U, Rw, Sh,
                     So, wb, mo, c->xcount, tab);
    else
      e = launch_pdl(k_gather_w<float, false>, gridw, kThreads, c->stream, out, src_hit, src_miss,
                     hit_list, miss_list, fill_src, dev_counts, nhit_host, nmiss_host, U, Rw, Sh,
                     So, wb, mo, c->xcount, tab);
    count_launch(c);
    return e;
  }
  if (vec && shard)
    e = launch_pdl(k_gather<float4, true>, grid, kThreads, c->stream, (float4*)out,
                   (const float4*)src_hit, (const float4*)src_miss, hit_list, miss_list, fill_src,
                   dev_counts, nhit_host, nmiss_host, U, R, Sh, So, wb, mo | mfirst | (int)(mb << 8), c->xcount, work, tab, lidslot, nl_dev);
  else if (vec)
    e = launch_pdl(k_gather<float4, false>, grid, kThreads, c->stream, (float4*)out,
                   (const float4*)src_hit, (const float4*)src_miss, hit_list, miss_list, fill_src,
                   dev_counts, nhit_host, nmiss_host, U, R, Sh, So, wb, mo | mfirst | (int)(mb << 8), c->xcount, work, tab, lidslot, nl_dev);
  else if (shard)
    e = launch_pdl(k_gather<float, true>, grid, kThreads, c->stream, out, src_hit, src_miss,
                   hit_list, miss_list, fill_src, dev_counts, nhit_host, nmiss_host, U, R,
                   Sh, So, wb, mo | mfirst | (int)(mb << 8), c->xcount, work, tab, lidslot, nl_dev);
  else
    e = launch_pdl(k_gather<float, false>, grid, kThreads, c->stream, out, src_hit, src_miss,
                   hit_list, miss_list, fill_src, dev_counts, nhit_host, nmiss_host, U, R,
                   Sh, So, wb, mo | mfirst | (int)(mb << 8), c->xcount, work, tab, lidslot, nl_dev);
  count_launch(c);
  return e;
}

}  // namespace glb
