// presc.cu -- a1 (epoch shuffle), a5/a6 (PreSC ranking + cache slots) and the
// hit-rate statistics, for sm_100a.
//
// Paper: "shuffle the training set T at the beginning of each epoch" (PAPER.md
// L305 §6.2); load_cache(hotness_map, alpha) "identifies and loads the
// features of the top-ranked alpha|V| vertices ... It also builds a hash table
// to indicate the location in feature cache" (L301 §6.1); PreSC uses the
// visit counts of K pre-sampling epochs as h_v (L333 §6.3); the Optimal policy
// caches the most visited vertices of the recorded footprints (L148 fn4).
//
// Both orders are strict total orders resolved by a STABLE LSD radix sort
// (8-bit digits): shuffle keys (64-bit Philox draw, ties by index) and
// hotness keys (maxcount - count, ties by gid).  One pass = tile histogram ->
// device-wide exclusive scan (digit-major) -> stable in-tile ranking with
// __match_any_sync and a scatter.
#include <cuda_runtime.h>

#include "glb_internal.cuh"

namespace glb {

namespace {

constexpr unsigned kFull = 0xFFFFFFFFu;
constexpr int kSortItems = 16;
constexpr int kSortTile = kThreads * kSortItems;  // 4096 keys
constexpr int kWarps = kThreads / 32;
constexpr int kScanChunk = kThreads * 16;

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

template <typename K>
__device__ __forceinline__ uint32_t digit_of(K k, int shift) {
  return (uint32_t)(k >> shift) & 0xFFu;
}

// key index handled by (tile, warp, iteration j, lane): warps own contiguous
// 512-key runs, iterations walk them in order -> rank order == index order.
__device__ __forceinline__ uint64_t sort_index(uint64_t tile, int w, int j, int lane) {
  return tile * kSortTile + (uint64_t)w * (kSortTile / kWarps) + (uint64_t)j * 32 + lane;
}

template <typename K>
__global__ void __launch_bounds__(kThreads)
    k_radix_hist(const K* __restrict__ keys, uint64_t n, int shift, uint32_t* __restrict__ hist,
                 uint64_t ntiles) {
  __shared__ uint32_t h[256];
  h[threadIdx.x] = 0;
  __syncthreads();
  const uint64_t tile = blockIdx.x;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
#pragma unroll 4
  for (int j = 0; j < kSortItems; ++j) {
    const uint64_t i = sort_index(tile, w, j, lane);
    if (i < n) atomicAdd(&h[digit_of(keys[i], shift)], 1u);
  }
  __syncthreads();
  hist[(uint64_t)threadIdx.x * ntiles + tile] = h[threadIdx.x];
}

template <typename K>
__global__ void __launch_bounds__(kThreads)
    k_radix_scatter(const K* __restrict__ keys, const uint32_t* __restrict__ vals, uint64_t n,
                    int shift, const uint32_t* __restrict__ offsets, uint64_t ntiles,
                    K* __restrict__ keys_out, uint32_t* __restrict__ vals_out) {
  __shared__ uint32_t wcnt[kWarps][256];
  __shared__ uint32_t goff[256];
  const uint64_t tile = blockIdx.x;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < kWarps * 256; i += kThreads) (&wcnt[0][0])[i] = 0;
  goff[threadIdx.x] = offsets[(uint64_t)threadIdx.x * ntiles + tile];
  __syncthreads();
  K k[kSortItems];
  uint32_t v[kSortItems], r[kSortItems];
#pragma unroll
  for (int j = 0; j < kSortItems; ++j) {
    const uint64_t i = sort_index(tile, w, j, lane);
    const bool ok = i < n;
    k[j] = ok ? keys[i] : (K)0;
    v[j] = ok ? vals[i] : 0u;
    const uint32_t dg = ok ? digit_of(k[j], shift) : 256u + lane;
    const uint32_t peers = __match_any_sync(kFull, dg);
    uint32_t before = 0;
    if (ok) before = wcnt[w][dg];
    r[j] = before + __popc(peers & lanemask_lt());
    __syncwarp();
    if (ok && (peers >> lane) == 1u) wcnt[w][dg] = before + __popc(peers);  // highest peer lane
    __syncwarp();
  }
  __syncthreads();
  {  // exclusive prefix over warps, per digit
    uint32_t run = 0;
    for (int ww = 0; ww < kWarps; ++ww) {
      const uint32_t t = wcnt[ww][threadIdx.x];
      wcnt[ww][threadIdx.x] = run;
      run += t;
    }
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < kSortItems; ++j) {
    const uint64_t i = sort_index(tile, w, j, lane);
    if (i < n) {
      const uint32_t dg = digit_of(k[j], shift);
      const uint64_t pos = (uint64_t)goff[dg] + wcnt[w][dg] + r[j];
      keys_out[pos] = k[j];
      vals_out[pos] = v[j];
    }
  }
}

// ---- device-wide exclusive scan of u32 (3 phases) ----
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t x, uint32_t* total) {
  __shared__ uint32_t s[kWarps];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t inc = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) s[w] = inc;
  __syncthreads();
  if (w == 0) {
    uint32_t t = lane < kWarps ? s[lane] : 0;
    uint32_t ti = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, ti, o);
      if (lane >= o) ti += y;
    }
    if (lane < kWarps) s[lane] = ti - t;
    if (lane == kWarps - 1) *total = ti;
  }
  __syncthreads();
  const uint32_t res = s[w] + inc - x;
  __syncthreads();
  return res;
}

__global__ void __launch_bounds__(kThreads)
    k_scan_reduce(const uint32_t* __restrict__ a, uint64_t n, uint32_t* __restrict__ sums) {
  __shared__ uint32_t red[kWarps];
  const uint64_t b = (uint64_t)blockIdx.x * kScanChunk;
  uint32_t s = 0;
  for (int i = threadIdx.x; i < kScanChunk; i += kThreads)
    if (b + i < n) s += a[b + i];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int w = 0; w < kWarps; ++w) t += red[w];
    sums[blockIdx.x] = t;
  }
}

__global__ void __launch_bounds__(kThreads) k_scan_sums(uint32_t* sums, uint64_t m) {
  __shared__ uint32_t total;
  uint32_t carry = 0;
  for (uint64_t b = 0; b < m; b += kThreads) {
    const uint64_t i = b + threadIdx.x;
    const uint32_t x = i < m ? sums[i] : 0u;
    const uint32_t ex = block_excl_scan(x, &total);
    if (i < m) sums[i] = carry + ex;
    carry += total;
    __syncthreads();
  }
}

__global__ void __launch_bounds__(kThreads)
    k_scan_down(const uint32_t* __restrict__ a, uint64_t n, const uint32_t* __restrict__ sums,
                uint32_t* __restrict__ out) {
  __shared__ uint32_t total;
  const uint64_t b = (uint64_t)blockIdx.x * kScanChunk;
  constexpr int kPer = kScanChunk / kThreads;  // 16 consecutive per thread
  uint32_t x[kPer];
  uint32_t s = 0;
#pragma unroll
  for (int q = 0; q < kPer; ++q) {
    const uint64_t i = b + (uint64_t)threadIdx.x * kPer + q;
    x[q] = i < n ? a[i] : 0u;
    s += x[q];
  }
  uint32_t run = sums[blockIdx.x] + block_excl_scan(s, &total);
#pragma unroll
  for (int q = 0; q < kPer; ++q) {
    const uint64_t i = b + (uint64_t)threadIdx.x * kPer + q;
    if (i < n) out[i] = run;
    run += x[q];
  }
}

__global__ void k_shuffle_keys(uint64_t n, uint64_t seed, uint32_t epoch,
                               unsigned long long* __restrict__ keys, uint32_t* __restrict__ vals) {
  const uint32_t c3 = ctr3(epoch, 0, kDomShuffle);
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    keys[i] = draw64(seed, (uint32_t)i, 0, 0, c3, 0);
    vals[i] = (uint32_t)i;
  }
}

__global__ void k_permute(const uint32_t* __restrict__ table, const uint32_t* __restrict__ idx,
                          uint64_t n, uint32_t* __restrict__ out) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = table[idx[i]];
}

__global__ void k_max_u32(const uint32_t* __restrict__ a, uint64_t n, uint32_t* out) {
  uint32_t m = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    m = max(m, a[i]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(kFull, m, o));
  if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}

__global__ void k_rank_keys(const uint32_t* __restrict__ hot, uint64_t n, uint32_t maxc,
                            uint32_t* __restrict__ keys, uint32_t* __restrict__ vals) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    keys[i] = maxc - hot[i];  // ascending key == descending hotness
    vals[i] = (uint32_t)i;    // ties keep gid order (stable sort)
  }
}

__global__ void k_assign_slots(const uint32_t* __restrict__ order, uint64_t C, int32_t* slot) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < C;
       i += (uint64_t)gridDim.x * blockDim.x)
    slot[order[i]] = (int32_t)i;
}

// NEXT-3: the vertices of shard r of a peer-sharded cache, in local-row order
// (global rank i = j*W + r is local row j of shard r).
__global__ void k_shard_rows(const uint32_t* __restrict__ order, uint32_t W, uint32_t r,
                             uint64_t n, uint32_t* __restrict__ out) {
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n;
       j += (uint64_t)gridDim.x * blockDim.x)
    out[j] = order[j * W + r];
}

__global__ void k_vmap_reset(VEntry* __restrict__ vmap, const int32_t* __restrict__ slot,
                             uint64_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    VEntry e;
    e.gp = ~0ull;
    e.aux = (unsigned long long)(uint32_t)slot[i];
    vmap[i] = e;
  }
}

__global__ void k_policy_hotness(int policy, uint64_t seed, const uint64_t* __restrict__ indptr,
                                 const uint32_t* __restrict__ counts, uint64_t n,
                                 uint32_t* __restrict__ out) {
  const uint32_t c3 = ctr3(0, 0, kDomPolicy);
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n;
       v += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t h;
    if (policy == GLB_POLICY_DEGREE) {
      const uint64_t d = indptr[v + 1] - indptr[v];
      h = d > 0xFFFFFFFFull ? 0xFFFFFFFFu : (uint32_t)d;
    } else if (policy == GLB_POLICY_RANDOM) {
      h = (uint32_t)(draw64(seed, (uint32_t)v, 0, 0, c3, 0) >> 32);
    } else {
      h = counts[v];
    }
    out[v] = h;
  }
}

__global__ void k_topmark(const uint32_t* __restrict__ order, uint64_t C, uint8_t* __restrict__ flag) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < C;
       i += (uint64_t)gridDim.x * blockDim.x)
    flag[order[i]] = 1;
}

// num = sum over T_i and T_j of min(f_i, f_j); den = sum over T_j of f_j
__global__ void k_similarity(const uint32_t* __restrict__ fi, const uint32_t* __restrict__ fj,
                             const uint8_t* __restrict__ ti, const uint8_t* __restrict__ tj,
                             uint64_t n, unsigned long long* out2) {
  unsigned long long num = 0, den = 0;
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n;
       v += (uint64_t)gridDim.x * blockDim.x) {
    if (tj[v]) {
      den += fj[v];
      if (ti[v]) num += min(fi[v], fj[v]);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    num += __shfl_xor_sync(kFull, num, o);
    den += __shfl_xor_sync(kFull, den, o);
  }
  if ((threadIdx.x & 31) == 0) {
    if (num) atomicAdd(out2 + 0, num);
    if (den) atomicAdd(out2 + 1, den);
  }
}

__global__ void k_hit_stats(const uint32_t* __restrict__ acc, const int32_t* __restrict__ slot,
                            uint64_t n, unsigned long long* out3) {
  unsigned long long tot = 0, hit = 0;
  uint32_t mx = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t a = acc[i];
    tot += a;
    if (slot[i] >= 0) hit += a;
    mx = max(mx, a);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    tot += __shfl_xor_sync(kFull, tot, o);
    hit += __shfl_xor_sync(kFull, hit, o);
    mx = max(mx, __shfl_xor_sync(kFull, mx, o));
  }
  if ((threadIdx.x & 31) == 0) {
    if (tot) atomicAdd(out3 + 0, tot);
    if (hit) atomicAdd(out3 + 1, hit);
    if (mx) atomicMax(out3 + 2, (unsigned long long)mx);
  }
}

__global__ void k_value_hist(const uint32_t* __restrict__ a, uint64_t n,
                             unsigned long long* bins, uint32_t nbins) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t x = a[i];
    if (x && x < nbins) atomicAdd(bins + x, 1ull);
  }
}

// ---- inclusive u64 prefix of u32 values (edge weights; 3 phases, any length) ----
__global__ void __launch_bounds__(kThreads)
    k_scan64_reduce(const uint32_t* __restrict__ a, uint64_t n, unsigned long long* __restrict__ sums) {
  __shared__ unsigned long long red[kWarps];
  const uint64_t b = (uint64_t)blockIdx.x * kScanChunk;
  unsigned long long s = 0;
  for (int i = threadIdx.x; i < kScanChunk; i += kThreads)
    if (b + i < n) s += a[b + i];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
    for (int w = 0; w < kWarps; ++w) t += red[w];
    sums[blockIdx.x] = t;
  }
}

__device__ __forceinline__ unsigned long long block_excl_scan64(unsigned long long x,
                                                                unsigned long long* total) {
  __shared__ unsigned long long s[kWarps];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  unsigned long long inc = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long y = __shfl_up_sync(kFull, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) s[w] = inc;
  __syncthreads();
  if (w == 0) {
    unsigned long long t = lane < kWarps ? s[lane] : 0, ti = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(kFull, ti, o);
      if (lane >= o) ti += y;
    }
    if (lane < kWarps) s[lane] = ti - t;
    if (lane == kWarps - 1) *total = ti;
  }
  __syncthreads();
  const unsigned long long res = s[w] + inc - x;
  __syncthreads();
  return res;
}

__global__ void __launch_bounds__(kThreads) k_scan64_sums(unsigned long long* sums, uint64_t m) {
  __shared__ unsigned long long total;
  unsigned long long carry = 0;
  for (uint64_t b = 0; b < m; b += kThreads) {
    const uint64_t i = b + threadIdx.x;
    const unsigned long long x = i < m ? sums[i] : 0ull;
    const unsigned long long ex = block_excl_scan64(x, &total);
    if (i < m) sums[i] = carry + ex;
    carry += total;
    __syncthreads();
  }
}

__global__ void __launch_bounds__(kThreads)
    k_scan64_down(const uint32_t* __restrict__ a, uint64_t n,
                  const unsigned long long* __restrict__ sums, unsigned long long* __restrict__ out) {
  __shared__ unsigned long long total;
  const uint64_t b = (uint64_t)blockIdx.x * kScanChunk;
  constexpr int kPer = kScanChunk / kThreads;
  uint32_t x[kPer];
  unsigned long long s = 0;
#pragma unroll
  for (int q = 0; q < kPer; ++q) {
    const uint64_t i = b + (uint64_t)threadIdx.x * kPer + q;
    x[q] = i < n ? a[i] : 0u;
    s += x[q];
  }
  unsigned long long run = sums[blockIdx.x] + block_excl_scan64(s, &total);
#pragma unroll
  for (int q = 0; q < kPer; ++q) {
    const uint64_t i = b + (uint64_t)threadIdx.x * kPer + q;
    run += x[q];
    if (i < n) out[i] = run;  // inclusive
  }
}

cudaError_t scan_excl_u32(glb_ctx* c, const uint32_t* a, uint64_t n, uint32_t* out,
                          uint32_t* sums) {
  const uint64_t m = (n + kScanChunk - 1) / kScanChunk;
  if (m == 0) return cudaSuccess;
  k_scan_reduce<<<(unsigned)m, kThreads, 0, c->stream>>>(a, n, sums);
  k_scan_sums<<<1, kThreads, 0, c->stream>>>(sums, m);
  k_scan_down<<<(unsigned)m, kThreads, 0, c->stream>>>(a, n, sums, out);
  count_launch(c, 3);
  return cudaGetLastError();
}

cudaError_t ensure_tmp(glb_ctx* c, size_t bytes) {
  if (c->sort_tmp_bytes >= bytes) return cudaSuccess;
  if (c->sort_tmp) cudaFree(c->sort_tmp);
  c->sort_tmp = nullptr;
  c->sort_tmp_bytes = 0;
  cudaError_t e = cudaMalloc(&c->sort_tmp, bytes);
  if (e == cudaSuccess) c->sort_tmp_bytes = bytes;
  return e;
}

template <typename K>
cudaError_t radix_sort_pairs(glb_ctx* c, K* keys, uint32_t* vals, K* keys_alt, uint32_t* vals_alt,
                             uint64_t n, int bits, K** keys_out, uint32_t** vals_out) {
  K* kin = keys;
  K* kout = keys_alt;
  uint32_t* vin = vals;
  uint32_t* vout = vals_alt;
  if (n > 0) {
    const uint64_t ntiles = (n + kSortTile - 1) / kSortTile;
    const uint64_t hn = 256 * ntiles;
    const uint64_t nsums = (hn + kScanChunk - 1) / kScanChunk;
    cudaError_t e = ensure_tmp(c, (2 * hn + nsums + 1) * sizeof(uint32_t));
    if (e != cudaSuccess) return e;
    uint32_t* hist = (uint32_t*)c->sort_tmp;
    uint32_t* offs = hist + hn;
    uint32_t* sums = offs + hn;
    for (int shift = 0; shift < bits; shift += 8) {
      k_radix_hist<K><<<(unsigned)ntiles, kThreads, 0, c->stream>>>(kin, n, shift, hist, ntiles);
      count_launch(c);
      if ((e = scan_excl_u32(c, hist, hn, offs, sums)) != cudaSuccess) return e;
      k_radix_scatter<K><<<(unsigned)ntiles, kThreads, 0, c->stream>>>(kin, vin, n, shift, offs,
                                                                      ntiles, kout, vout);
      count_launch(c);
      if ((e = cudaGetLastError()) != cudaSuccess) return e;
      K* tk = kin; kin = kout; kout = tk;
      uint32_t* tv = vin; vin = vout; vout = tv;
    }
  }
  *keys_out = kin;
  *vals_out = vin;
  return cudaGetLastError();
}

inline int grid_for(glb_ctx* c) { return c->num_sms * 8; }

}  // namespace

cudaError_t scan_exclusive_u32(glb_ctx* c, const uint32_t* a, uint64_t n, uint32_t* out,
                               uint32_t* sums) {
  return scan_excl_u32(c, a, n, out, sums);
}

cudaError_t radix_sort_pairs_u64(glb_ctx* c, unsigned long long* keys, uint32_t* vals,
                                 unsigned long long* keys_alt, uint32_t* vals_alt, uint64_t n,
                                 int bits, unsigned long long** keys_out, uint32_t** vals_out) {
  return radix_sort_pairs<unsigned long long>(c, keys, vals, keys_alt, vals_alt, n, bits,
                                              keys_out, vals_out);
}
cudaError_t radix_sort_pairs_u32(glb_ctx* c, uint32_t* keys, uint32_t* vals, uint32_t* keys_alt,
                                 uint32_t* vals_alt, uint64_t n, int bits, uint32_t** keys_out,
                                 uint32_t** vals_out) {
  return radix_sort_pairs<uint32_t>(c, keys, vals, keys_alt, vals_alt, n, bits, keys_out,
                                    vals_out);
}

cudaError_t scan_inclusive_u64(glb_ctx* c, const uint32_t* a, uint64_t n, unsigned long long* out) {
  const uint64_t m = (n + kScanChunk - 1) / kScanChunk;
  if (m == 0) return cudaSuccess;
  unsigned long long* sums = nullptr;
  cudaError_t e = cudaMalloc(&sums, sizeof(unsigned long long) * m);
  if (e != cudaSuccess) return e;
  k_scan64_reduce<<<(unsigned)m, kThreads, 0, c->stream>>>(a, n, sums);
  k_scan64_sums<<<1, kThreads, 0, c->stream>>>(sums, m);
  k_scan64_down<<<(unsigned)m, kThreads, 0, c->stream>>>(a, n, sums, out);
  count_launch(c, 3);
  e = cudaStreamSynchronize(c->stream);
  cudaFree(sums);
  return e == cudaSuccess ? cudaGetLastError() : e;
}

cudaError_t launch_shuffle_keys(glb_ctx* c, uint32_t epoch, unsigned long long* keys,
                                uint32_t* vals) {
  k_shuffle_keys<<<grid_for(c), kThreads, 0, c->stream>>>(c->n_train, c->seed, epoch, keys, vals);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_permute(glb_ctx* c, const uint32_t* table, const uint32_t* idx, uint64_t n,
                           uint32_t* out) {
  k_permute<<<grid_for(c), kThreads, 0, c->stream>>>(table, idx, n, out);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_max_u32(glb_ctx* c, const uint32_t* a, uint64_t n, uint32_t* out_dev) {
  k_max_u32<<<grid_for(c), kThreads, 0, c->stream>>>(a, n, out_dev);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_rank_keys(glb_ctx* c, const uint32_t* hot, uint32_t maxc, uint32_t* keys,
                             uint32_t* vals) {
  k_rank_keys<<<grid_for(c), kThreads, 0, c->stream>>>(hot, c->V, maxc, keys, vals);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_assign_slots(glb_ctx* c, const uint32_t* order, uint64_t C) {
  if (C == 0) return cudaSuccess;
  k_assign_slots<<<grid_for(c), kThreads, 0, c->stream>>>(order, C, c->slot);
  count_launch(c);
  return cudaGetLastError();
}

__global__ void k_cold_rows(const uint32_t* __restrict__ order, uint64_t C, uint64_t V,
                            uint32_t* __restrict__ cold_row) {
  for (uint64_t i = C + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < V;
       i += (uint64_t)gridDim.x * blockDim.x)
    cold_row[order[i]] = (uint32_t)(i - C);  // rank C + j -> cold-store row j
}

cudaError_t launch_cold_rows(glb_ctx* c, const uint32_t* order, uint64_t C) {
  k_cold_rows<<<c->num_sms * 8, kThreads, 0, c->stream>>>(order, C, c->V, c->cold_row);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_shard_rows(glb_ctx* c, const uint32_t* order, uint32_t W, uint32_t r,
                              uint64_t n, uint32_t* out) {
  if (n == 0) return cudaSuccess;
  k_shard_rows<<<grid_for(c), kThreads, 0, c->stream>>>(order, W, r, n, out);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_vmap_reset(glb_ctx* c) {
  if (!c->vmap) return cudaSuccess;
  k_vmap_reset<<<grid_for(c), kThreads, 0, c->stream>>>(c->vmap, c->slot, c->V);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_policy_hotness(glb_ctx* c, int policy, uint64_t seed, uint32_t* out) {
  k_policy_hotness<<<grid_for(c), kThreads, 0, c->stream>>>(policy, seed, c->indptr, c->counts,
                                                             c->V, out);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_topmark(glb_ctx* c, const uint32_t* order, uint64_t C, uint8_t* flag) {
  if (C == 0) return cudaSuccess;
  k_topmark<<<grid_for(c), kThreads, 0, c->stream>>>(order, C, flag);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_similarity(glb_ctx* c, const uint32_t* fi, const uint32_t* fj,
                              const uint8_t* ti, const uint8_t* tj, unsigned long long* out2) {
  k_similarity<<<grid_for(c), kThreads, 0, c->stream>>>(fi, fj, ti, tj, c->V, out2);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_hit_stats(glb_ctx* c, unsigned long long* out3) {
  k_hit_stats<<<grid_for(c), kThreads, 0, c->stream>>>(c->access, c->slot, c->V, out3);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_value_hist(glb_ctx* c, const uint32_t* a, uint64_t n, unsigned long long* bins,
                              uint32_t nbins) {
  k_value_hist<<<grid_for(c), kThreads, 0, c->stream>>>(a, n, bins, nbins);
  count_launch(c);
  return cudaGetLastError();
}

}  // namespace glb
