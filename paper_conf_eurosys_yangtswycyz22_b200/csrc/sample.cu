// sample.cu -- a2 (k-hop uniform), a2' (random walk), a3 (dedup + relabel into
// blocks) and a4 (mark) for sm_100a.
//
// Paper: k-hop sampling "uniformly selects ... neighbors for each vertex"
// (§2, Fig 7), "a variant of the Fisher-Yates
// algorithm ... GPU-friendly since the workload is more balanced for each
// vertex" (L410 §7.3); samples are "deduplicated and reassigned with
// consecutive IDs (starting from 0)" (L67, L250 §5.2); cached vertices are
// marked during Sample (L252).
//
// Design:
//  * k_khop: k lanes per frontier vertex (floor(32/k) vertices per warp), one
//    lane per slot.  Floyd's draws are independent per slot (counter-based
//    RNG), so every lane computes its t_s at once; the sequential "t already
//    chosen?" test is resolved exactly with __match_any_sync + a short
//    fixed-point over the j-chain (proof in DESIGN.md).
//  * relabel: direct-address table vmap[gid] = (~gen << 32 | first position),
//    one atomicMin per pick (filtered by a plain read), then a single-pass
//    decoupled-look-back scan over the padded (vertex, slot) array assigns new
//    lids in first-occurrence order and writes the block CSR with src lids
//    directly (no separate remap pass).
#include <cuda_runtime.h>

#include "glb_internal.cuh"

#ifdef GLB_TRACE
// debug timeline of the compaction tiles: [hop][tile][event] = %globaltimer (ns)
__device__ unsigned long long g_trace[GLB_MAX_HOPS][4096][8];
extern "C" glb_status glb_trace_dump(void* host, size_t bytes) {
  return cudaMemcpyFromSymbol(host, g_trace, bytes) == cudaSuccess ? GLB_OK : GLB_ECUDA;
}
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));  // ns, comparable across SMs
  return t;
}
// [hop][0] = first block start, [hop][1] = last block end of k_khop (ns)
__device__ unsigned long long g_ktrace[GLB_MAX_HOPS][2];
extern "C" glb_status glb_trace_reset() {
  unsigned long long h[GLB_MAX_HOPS][2];
  for (int i = 0; i < GLB_MAX_HOPS; ++i) { h[i][0] = ~0ull; h[i][1] = 0; }
  static unsigned long long z[GLB_MAX_HOPS][4096][8];
  if (cudaMemcpyToSymbol(g_trace, z, sizeof(z)) != cudaSuccess) return GLB_ECUDA;
  return cudaMemcpyToSymbol(g_ktrace, h, sizeof(h)) == cudaSuccess ? GLB_OK : GLB_ECUDA;
}
extern "C" glb_status glb_ktrace_dump(void* host) {
  return cudaMemcpyFromSymbol(host, g_ktrace, sizeof(g_ktrace)) == cudaSuccess ? GLB_OK : GLB_ECUDA;
}
#define KTRACE_BEGIN(h) do { if (threadIdx.x == 0) atomicMin(&::g_ktrace[h][0], gtime()); } while (0)
#define KTRACE_END(h) do { __syncthreads(); if (threadIdx.x == 0) atomicMax(&::g_ktrace[h][1], gtime()); } while (0)
#define TRACE(h, t, ev) \
  do { if (threadIdx.x == 0 && (t) < 4096) ::g_trace[h][t][ev] = gtime(); } while (0)
#else
#define TRACE(h, t, ev) do {} while (0)
#define KTRACE_BEGIN(h) do {} while (0)
#define KTRACE_END(h) do {} while (0)
#endif

namespace glb {

namespace {

constexpr unsigned kFull = 0xFFFFFFFFu;

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// Random 4-byte reads of the CSR: a non-coherent load that does not allocate in L1 and asks L2
// for a 64-byte fill (the sampler touches one 4-byte word of each sector it pulls in).
// Measured against the plain __ldg (GLB_SAMPLE_LD=0 A/B build, profiles/r02_ldhint_ab.txt):
// PR 206.7 vs 208.0, UK 429.8 vs 432.9, TW 590.3 vs 597.5 us/step at alpha = 1.
#ifndef GLB_SAMPLE_LD
#define GLB_SAMPLE_LD 1
#endif
__device__ __forceinline__ uint32_t ld_csr(const uint32_t* p) {
#if GLB_SAMPLE_LD == 1
  uint32_t v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
#else
  return __ldg(p);
#endif
}

// The (indptr[v], indptr[v+1]) pair of a random frontier vertex.  A plain load of one random
// 8-byte word pulls in a 128-byte line (ncu on PA's last random-walk hop: ~200 DRAM bytes
// per walk step).  GLB_INDPTR_LD=1 (A/B builds) asks for a 64-byte fill like ld_csr: TW
// 578.6 vs 580.2, UK 433.0 vs 433.4, PR 207.2 vs 207.0 us/step, but PA (random walks)
// 595 vs 574 -- slower, so plain loads stay (profiles/r02t_indptr_ld_ab.txt).
#ifndef GLB_INDPTR_LD
#define GLB_INDPTR_LD 0
#endif
__device__ __forceinline__ uint64_t ld_indptr(const uint64_t* p) {
#if GLB_INDPTR_LD == 1
  uint64_t v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::64B.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
#else
  return *p;
#endif
}

// Insert one pick into the relabel table: keep the smallest position of this
// generation.  Values only decrease over time, so a (possibly stale) read that
// is already <= e proves the atomic would be a no-op.
__device__ __forceinline__ unsigned long long vmap_insert(VEntry* vmap, uint32_t u,
                                                          unsigned long long e) {
  const unsigned long long old = __ldcg(&vmap[u].gp);
  if (old > e) atomicMin(&vmap[u].gp, e);  // no return value needed: RED, no round trip
  return old;  // <= e: an earlier position (or a lid) of this generation already held u
}

// The relabel table.  Dense mode: entry index = gid (V entries; aux = cache slot).
// Hash mode (large V): open addressing with linear probing over mask+1 entries
// sized from the batch's unique-vertex bound, so the table stays L2-resident;
// aux = (gen << 32 | gid) -- entries of older generations count as free, so the
// table is never cleared -- and the claimer of an entry copies the vertex's cache
// slot into hslot[index].  Both modes share gp semantics and every later step
// addresses entries by index.
struct Table {
  VEntry* e;
  int32_t* hslot;       // hash mode: cache slot per entry
  const int32_t* slot;  // [V] cache slot map
  uint32_t mask;        // hash mode: capacity - 1
  uint32_t gen;
};

__device__ __forceinline__ uint32_t hash32(uint32_t x) {  // lowbias32 mixer
  x ^= x >> 16;
  x *= 0x7feb352du;
  x ^= x >> 15;
  x *= 0x846ca68bu;
  x ^= x >> 16;
  return x;
}

// Find or claim gid's entry for this generation; kEmpty if the table is full.
__device__ __forceinline__ uint32_t hclaim(const Table& T, uint32_t gid, bool& claimed) {
  const unsigned long long key = ((unsigned long long)T.gen << 32) | gid;
  uint32_t h = hash32(gid) & T.mask;
  claimed = false;
  // bounded probing: a run this long means the table is (nearly) full -> ENOMEM
  const uint32_t max_probe = T.mask < 1023u ? T.mask : 1023u;
  for (uint32_t probe = 0, tries = 0; probe <= max_probe && tries < 4096u; ++tries) {
    unsigned long long* kp = &T.e[h].aux;
    const unsigned long long kg = __ldcg(kp);
    if (kg == key) return h;
    if ((uint32_t)(kg >> 32) != T.gen) {  // free in this generation: try to claim it
      const unsigned long long prev = atomicCAS(kp, kg, key);
      if (prev == kg) {
        claimed = true;
        return h;
      }
      if (prev == key) return h;
      if ((uint32_t)(prev >> 32) != T.gen) continue;  // lost to nothing we know: retry slot
    }
    h = (h + 1) & T.mask;
    ++probe;
  }
  return kEmpty;
}

// Entry index of gid (dense: gid; hash: found / claimed, the claimer records
// the cache slot).  kEmpty (and an error flag) when the hash table is full.
template <bool HASH>
__device__ __forceinline__ uint32_t entry_of(const Table& T, uint32_t gid, DevState* st) {
  if (!HASH) return gid;
  bool claimed;
  const uint32_t h = hclaim(T, gid, claimed);
  if (h == kEmpty) {
    atomicOr(&st->err, kErrCapacity);
    return kEmpty;
  }
  if (claimed) T.hslot[h] = __ldg(T.slot + gid);
  return h;
}

// Encoded pick: the gid, or -- when the sampler already found u relabelled by an
// earlier hop / as a seed (table value (gen, lid) with lid < base) -- lid | kOld,
// so the compaction needs no table access for it.  gids and lids are < 2^31.
constexpr uint32_t kOld = 0x80000000u;
__device__ __forceinline__ uint32_t encode_pick(uint32_t u, unsigned long long old,
                                                unsigned long long e, uint32_t base) {
  if (old <= e && (uint32_t)old < base) return (uint32_t)old | kOld;
  return u;
}

constexpr uint32_t kDefer = 0x80000000u;  // deferred src lid marker (indices < 2^31)

// Resolve deferred src lids of block `hop` (entries = table index | kDefer).
__device__ __forceinline__ void fixup_block(uint32_t nnz, const VEntry* vmap,
                                            uint32_t* __restrict__ bindices) {
  for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += gridDim.x * blockDim.x) {
    const uint32_t x = bindices[e];
    if (x & kDefer) bindices[e] = (uint32_t)__ldcg(&vmap[x & ~kDefer].gp);  // (gen, lid)
  }
}

struct MarkArgs {
  const int32_t* slot;
  int32_t* lidslot;
  uint2* hit_list;   // (lid, slot)
  uint2* miss_list;  // (lid, gid)
  uint32_t* count;   // nullable visit-count target
};

struct StatusArgs {  // look-back status arrays to clear for this batch
  unsigned long long* p[GLB_MAX_HOPS];
  uint32_t n[GLB_MAX_HOPS];
  uint32_t L;
};

// ---------------------------------------------------------------- seeds
template <bool HASH>
__global__ void __launch_bounds__(kThreads)
    k_seed_init(const uint32_t* __restrict__ seeds, uint32_t n0, uint64_t V, DevState* st,
                uint32_t* __restrict__ uniq, Table T, MarkArgs mk, StatusArgs za) {
  pdl_enter();
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    st->n[0] = n0;
    st->base[0] = n0;
  }
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t l = 0; l < za.L; ++l)
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < za.n[l]; i += stride) za.p[l][i] = 0ull;
  const int lane = threadIdx.x & 31;
  // warp-uniform loop bound so that the ballots below see the whole warp
  for (uint32_t i0 = blockIdx.x * blockDim.x + (threadIdx.x & ~31u); i0 < n0; i0 += stride) {
    const uint32_t i = i0 + lane;
    const bool act = i < n0;
    uint32_t u = 0;
    int32_t s = -1;
    if (act) {
      u = seeds[i];
      if (u >= V) {
        atomicOr(&st->err, kErrRange);
        u = 0;  // keep later kernels in bounds; the batch is reported invalid
      }
      uniq[i] = u;
      if (HASH) {
        bool claimed;
        const uint32_t h = hclaim(T, u, claimed);
        if (h == kEmpty) atomicOr(&st->err, kErrCapacity);
        else {
          if (!claimed) atomicOr(&st->err, kErrDupSeed);  // key already inserted this batch
          T.hslot[h] = __ldg(T.slot + u);
          atomicMin(&T.e[h].gp, enc_pos(T.gen, i));  // a seed's position is its lid
        }
      } else {
        atomicMin(&T.e[u].gp, enc_pos(T.gen, i));
      }
      s = __ldg(mk.slot + u);
      mk.lidslot[i] = s;
      if (mk.count) atomicAdd(mk.count + u, 1u);
    }
    const bool hit = act && s >= 0, miss = act && s < 0;
    const uint32_t mh = __ballot_sync(kFull, hit), mm = __ballot_sync(kFull, miss);
    uint32_t bh = 0, bm = 0;
    if (lane == 0) {
      if (mh) bh = atomicAdd(&st->nhit, (uint32_t)__popc(mh));
      if (mm) bm = atomicAdd(&st->nmiss, (uint32_t)__popc(mm));
    }
    bh = __shfl_sync(kFull, bh, 0);
    bm = __shfl_sync(kFull, bm, 0);
    if (hit) mk.hit_list[bh + __popc(mh & lanemask_lt())] = make_uint2(i, (uint32_t)s);
    if (miss) mk.miss_list[bm + __popc(mm & lanemask_lt())] = make_uint2(i, u);
  }
}

// ---------------------------------------------------------------- k-hop (k lanes / vertex)
// Fanout k <= 32: floor(32/k) frontier vertices per warp, lane s of a group
// owns Floyd slot s.
//
// DEDUP (GLB_RELABEL_DEDUP=1, the north star's staged insert at warp scope): picks of the
// same gid within a warp are combined first (__match_any_sync) -- only the lowest lane,
// which holds the smallest flat position, probes / inserts into the relabel table, and
// the value it read is broadcast to its peers, so a hub picked by several frontier
// vertices of one warp costs one table access instead of several.
//
// DEDUP == 2 (GLB_RELABEL_DEDUP=2, the north star's "shared-memory-staged open-addressing
// hash insert"): the whole block's picks of one iteration (8 warps) are first
// inserted into a 512-entry open-addressing table in shared memory keyed by gid, with the
// smallest flat position per gid (smem atomicMin); after a barrier only that pick probes /
// inserts into the global relabel table, and its result is shared through the smem table.
// The loop is block-uniform (same vertex-to-warp mapping as the warp-strided loop).
constexpr uint32_t kStageEntries = 2 * kThreads;  // smem table (load factor <= 1/2)
template <bool HASH, int DEDUP>
__global__ void __launch_bounds__(kThreads)
    k_khop(uint32_t hop, uint32_t k, uint64_t seed, uint32_t epoch, uint32_t batch, Table T,
           const DevState* __restrict__ st, DevState* st_w, const uint64_t* __restrict__ indptr,
           const uint32_t* __restrict__ indices, const uint32_t* __restrict__ uniq,
           uint32_t* __restrict__ picks, uint32_t* __restrict__ pidx, uint32_t* fix_ind) {
  pdl_enter();
  KTRACE_BEGIN(hop);
  if (fix_ind) fixup_block(st->nnz[hop - 1], T.e, fix_ind);  // deferred lids of block hop-1
  const uint32_t gen = T.gen;
  const uint32_t n_l = st->n[hop];
  const uint32_t base = st->base[hop];
  const uint32_t c3 = ctr3(epoch, hop, kDomKhop);
  const int lane = threadIdx.x & 31;
  const uint32_t gpw = 32 / k;                 // groups (vertices) per warp
  const uint32_t gi = (uint32_t)lane / k;      // >= gpw: idle lane
  const uint32_t s = (uint32_t)lane - gi * k;  // slot
  const int gbase = (int)(gi * k);
  const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  __shared__ uint32_t sk[DEDUP == 2 ? kStageEntries : 1];             // gid (kEmpty = free)
  __shared__ uint32_t sp[DEDUP == 2 ? kStageEntries : 1];             // min flat position
  __shared__ unsigned long long so[DEDUP == 2 ? kStageEntries : 1];   // table value read
  __shared__ uint32_t si[DEDUP == 2 ? kStageEntries : 1];             // table index
  if (DEDUP == 2) {
    for (uint32_t i = threadIdx.x; i < kStageEntries; i += blockDim.x) {
      sk[i] = kEmpty;
      sp[i] = kEmpty;
    }
    __syncthreads();
  }
  // block-uniform bound for DEDUP == 2 (barriers inside); warp w of block b starts at the
  // same vertex as in the warp-strided loop
  const uint32_t wib = threadIdx.x >> 5, wpb = blockDim.x >> 5;
  for (uint32_t b0 = blockIdx.x * wpb * gpw; DEDUP == 2 ? b0 < n_l : b0 + wib * gpw < n_l;
       b0 += nwarps * gpw) {
    const uint32_t w0 = b0 + wib * gpw;
    (void)warp_global;
    const uint32_t d = w0 + gi;
    const bool active = gi < gpw && d < n_l;
    uint32_t v = 0, deg = 0;
    uint64_t lo = 0;
    if (active) {
      v = uniq[d];
      lo = ld_indptr(indptr + v);
      deg = (uint32_t)(ld_indptr(indptr + v + 1) - lo);
      if (!HASH && hop == 0 && s == 0 && __ldcg(&T.e[v].gp) != enc_pos(gen, d))
        atomicOr(&st_w->err, kErrDupSeed);
    }
    const bool big = active && deg > k;
    uint32_t t = 0, j = 0;
    if (big) {
      j = deg - k + s;
      t = bounded(draw64(seed, v, s >> 1, batch, c3, s & 1u), j + 1);
    }
    uint32_t sel = kEmpty;
    if (__any_sync(kFull, big)) {
      // D1: an earlier slot of the same vertex drew the same t
      const unsigned long long key =
          big ? (((unsigned long long)gi << 32) | t) : ((1ull << 63) | (unsigned)lane);
      const uint32_t eq = __match_any_sync(kFull, key);
      const bool d1 = (eq & lanemask_lt()) != 0;
      // j-chain: t equals j_{s'} (s' < s), which is taken iff slot s' was displaced
      const bool inr = big && t >= deg - k && t < j;
      const int ref = inr ? gbase + (int)(t - (deg - k)) : lane;
      bool disp = d1;
      for (;;) {
        const bool r = __shfl_sync(kFull, disp, ref);
        const bool nd = d1 || (inr && r);
        const bool done = __ballot_sync(kFull, nd) == __ballot_sync(kFull, disp);
        disp = nd;
        if (done) break;
      }
      if (big) sel = disp ? j : t;
    }
    if (!big && active && s < deg) sel = s;
    uint32_t u = kEmpty, idx = kEmpty;
    if (DEDUP == 2) {
      const uint32_t pos = base + d * k + s;
      uint32_t h = kEmpty;
      if (sel != kEmpty) {  // stage: find / claim the gid's smem entry, keep the min position
        u = ld_csr(indices + lo + sel);
        h = hash32(u) & (kStageEntries - 1);
        for (;;) {
          const uint32_t prev = atomicCAS(&sk[h], kEmpty, u);
          if (prev == kEmpty || prev == u) break;
          h = (h + 1) & (kStageEntries - 1);
        }
        atomicMin(&sp[h], pos);
      }
      __syncthreads();
      if (sel != kEmpty && sp[h] == pos) {  // first occurrence in this block: one table access
        const uint32_t ix = entry_of<HASH>(T, u, st_w);
        si[h] = ix;
        so[h] = ix != kEmpty ? vmap_insert(T.e, ix, enc_pos(gen, pos)) : ~0ull;
      }
      __syncthreads();
      if (sel != kEmpty) {
        idx = si[h];
        const unsigned long long old = so[h];
        u = idx != kEmpty ? encode_pick(u, old, enc_pos(gen, pos), base) : kEmpty;
      }
      __syncthreads();
      if (sel != kEmpty) {  // free the entry for the next iteration
        sk[h] = kEmpty;
        sp[h] = kEmpty;
      }
      __syncthreads();
    } else if (DEDUP == 1) {
      if (sel != kEmpty) u = ld_csr(indices + lo + sel);
      // lanes with the same gid: flat positions grow with the lane, so the lowest lane
      // holds the first occurrence within the warp
      const unsigned long long key =
          sel != kEmpty ? (unsigned long long)u : ((1ull << 63) | (unsigned)lane);
      const uint32_t peers = __match_any_sync(kFull, key);
      const int leader = __ffs(peers) - 1;
      unsigned long long old = ~0ull;
      if (sel != kEmpty && lane == leader) {
        idx = entry_of<HASH>(T, u, st_w);
        if (idx != kEmpty) old = vmap_insert(T.e, idx, enc_pos(gen, base + d * k + s));
      }
      idx = __shfl_sync(kFull, idx, leader);
      old = __shfl_sync(kFull, old, leader);
      if (sel != kEmpty)
        u = idx != kEmpty ? encode_pick(u, old, enc_pos(gen, base + d * k + s), base) : kEmpty;
    } else if (sel != kEmpty) {
      u = ld_csr(indices + lo + sel);
      idx = entry_of<HASH>(T, u, st_w);
      if (idx != kEmpty) {
        const unsigned long long e = enc_pos(gen, base + d * k + s);
        u = encode_pick(u, vmap_insert(T.e, idx, e), e, base);
      } else {
        u = kEmpty;
      }
    }
    if (active) {
      picks[(size_t)d * k + s] = u;
      if (HASH) pidx[(size_t)d * k + s] = idx;
    }
  }
  KTRACE_END(hop);
}

// ---------------------------------------------------------------- weighted k-hop (NEXT-1)
// L81 fn1 / L148 fn5 / L136; reading Q19: slot s of frontier vertex v draws with
// replacement x = floor(r * W / 2^64) over the row's total weight W and picks the
// first position whose inclusive weight prefix exceeds x.  The prefix is global over
// all edges (wprefix, u64), so the row's prefix is wprefix - wprefix[lo - 1].  One
// lane per slot; slots beyond 32 loop.  Binary search over the row.
template <bool HASH>
__global__ void __launch_bounds__(kThreads)
    k_khop_weighted(uint32_t hop, uint32_t k, uint64_t seed, uint32_t epoch, uint32_t batch,
                    Table T, const DevState* __restrict__ st, DevState* st_w,
                    const uint64_t* __restrict__ indptr, const uint32_t* __restrict__ indices,
                    const unsigned long long* __restrict__ wprefix,
                    const uint32_t* __restrict__ uniq, uint32_t* __restrict__ picks,
                    uint32_t* __restrict__ pidx, uint32_t* fix_ind) {
  pdl_enter();
  if (fix_ind) fixup_block(st->nnz[hop - 1], T.e, fix_ind);
  const uint32_t gen = T.gen;
  const uint32_t n_l = st->n[hop];
  const uint32_t base = st->base[hop];
  const uint32_t c3 = ctr3(epoch, hop, kDomWeighted);
  const uint32_t G = k < 32 ? k : 32;         // lanes per vertex
  const int lane = threadIdx.x & 31;
  const uint32_t gpw = 32 / G;
  const uint32_t gi = (uint32_t)lane / G;
  const uint32_t sl = (uint32_t)lane - gi * G;
  const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t w0 = warp_global * gpw; w0 < n_l; w0 += nwarps * gpw) {
    const uint32_t d = w0 + gi;
    if (gi >= gpw || d >= n_l) continue;
    const uint32_t v = uniq[d];
    const uint64_t lo = ld_indptr(indptr + v), hi = ld_indptr(indptr + v + 1);
    const unsigned long long pbase = lo ? wprefix[lo - 1] : 0ull;
    const unsigned long long W = hi > lo ? wprefix[hi - 1] - pbase : 0ull;
    for (uint32_t s = sl; s < k; s += G) {
      uint32_t u = kEmpty, idx = kEmpty;
      if (W) {
        const unsigned long long x =
            __umul64hi(draw64(seed, v, s >> 1, batch, c3, s & 1u), W);  // floor(r*W/2^64)
        const unsigned long long target = pbase + x;
        uint64_t a = lo, b = hi - 1;  // first p in [lo, hi) with wprefix[p] > target
        while (a < b) {
          const uint64_t m = a + ((b - a) >> 1);
          if (__ldg(wprefix + m) > target) b = m;
          else a = m + 1;
        }
        u = ld_csr(indices + a);
        idx = entry_of<HASH>(T, u, st_w);
        if (idx != kEmpty) {
          const unsigned long long e = enc_pos(gen, base + d * k + s);
          u = encode_pick(u, vmap_insert(T.e, idx, e), e, base);
        } else {
          u = kEmpty;
        }
      }
      picks[(size_t)d * k + s] = u;
      if (HASH) pidx[(size_t)d * k + s] = idx;
    }
  }
}

// Fanout > 32: one warp per vertex, Floyd run sequentially by lane 0 in shared memory.
template <bool HASH>
__global__ void __launch_bounds__(kThreads)
    k_khop_wide(uint32_t hop, uint32_t k, uint64_t seed, uint32_t epoch, uint32_t batch,
                Table T, const DevState* __restrict__ st, DevState* st_w,
                const uint64_t* __restrict__ indptr, const uint32_t* __restrict__ indices,
                const uint32_t* __restrict__ uniq, uint32_t* __restrict__ picks,
                uint32_t* __restrict__ pidx, uint32_t* fix_ind) {
  pdl_enter();
  __shared__ uint32_t chosen[kThreads / 32][kMaxFanout];
  if (fix_ind) fixup_block(st->nnz[hop - 1], T.e, fix_ind);
  const uint32_t gen = T.gen;
  const uint32_t n_l = st->n[hop];
  const uint32_t base = st->base[hop];
  const uint32_t c3 = ctr3(epoch, hop, kDomKhop);
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  uint32_t* ch = chosen[wib];
  for (uint32_t d = warp_global; d < n_l; d += nwarps) {
    const uint32_t v = uniq[d];
    const uint64_t lo = ld_indptr(indptr + v);
    const uint32_t deg = (uint32_t)(ld_indptr(indptr + v + 1) - lo);
    if (!HASH && hop == 0 && lane == 0 && __ldcg(&T.e[v].gp) != enc_pos(gen, d))
      atomicOr(&st_w->err, kErrDupSeed);
    if (deg > k) {
      if (lane == 0) {
        for (uint32_t s = 0; s < k; ++s) {
          const uint32_t j = deg - k + s;
          const uint32_t t = bounded(draw64(seed, v, s >> 1, batch, c3, s & 1u), j + 1);
          bool taken = false;
          for (uint32_t q = 0; q < s; ++q) taken |= (ch[q] == t);
          ch[s] = taken ? j : t;
        }
      }
      __syncwarp();
    }
    for (uint32_t s = lane; s < k; s += 32) {
      uint32_t sel = kEmpty;
      if (deg > k) sel = ch[s];
      else if (s < deg) sel = s;
      uint32_t u = sel != kEmpty ? ld_csr(indices + lo + sel) : kEmpty, idx = kEmpty;
      if (u != kEmpty) {
        idx = entry_of<HASH>(T, u, st_w);
        if (idx != kEmpty) {
          const unsigned long long e = enc_pos(gen, base + d * k + s);
          u = encode_pick(u, vmap_insert(T.e, idx, e), e, base);
        } else {
          u = kEmpty;
        }
      }
      picks[(size_t)d * k + s] = u;
      if (HASH) pidx[(size_t)d * k + s] = idx;
    }
    __syncwarp();
  }
}

// ---------------------------------------------------------------- random walk
// PinSAGE (L209, L353): G >= walks lanes per frontier vertex, one walk per lane.
// PinSAGE (L209, L353): G >= walks lanes per frontier vertex, one walk per lane;
// LEN >= walk length (register arrays; 3 for PinSAGE).
#ifndef GLB_RWALK_MINB  // min resident random-walk blocks per SM (register cap; A/B builds)
#define GLB_RWALK_MINB 1
#endif
template <int G, int LEN, bool HASH>
__global__ void __launch_bounds__(kThreads, GLB_RWALK_MINB)
    k_rwalk(uint32_t hop, uint32_t walks, uint32_t len, uint32_t topk, uint64_t seed,
            uint32_t epoch, uint32_t batch, Table T, const DevState* __restrict__ st,
            DevState* st_w, const uint64_t* __restrict__ indptr,
            const uint32_t* __restrict__ indices, const uint32_t* __restrict__ uniq,
            uint32_t* __restrict__ picks, uint32_t* __restrict__ pickw,
            uint32_t* __restrict__ pidx, uint32_t* fix_ind) {
  pdl_enter();
  if (fix_ind) fixup_block(st->nnz[hop - 1], T.e, fix_ind);
  const uint32_t gen = T.gen;
  const uint32_t n_l = st->n[hop];
  const uint32_t base = st->base[hop];
  const uint32_t c3 = ctr3(epoch, hop, kDomRwalk);
  const int lane = threadIdx.x & 31;
  const uint32_t w = lane & (G - 1);
  const int gbase = lane & ~(G - 1);
  constexpr uint32_t kGroupsPerWarp = 32 / G;
  const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t w0 = warp_global * kGroupsPerWarp; w0 < n_l; w0 += nwarps * kGroupsPerWarp) {
    const uint32_t d = w0 + lane / G;
    const bool active = d < n_l;
    uint32_t v = 0;
    uint32_t vis[LEN];
#pragma unroll
    for (int t = 0; t < LEN; ++t) vis[t] = kEmpty;
    if (active) {
      v = uniq[d];
      if (!HASH && hop == 0 && w == 0 && __ldcg(&T.e[v].gp) != enc_pos(gen, d))
        atomicOr(&st_w->err, kErrDupSeed);
      if (w < walks) {
        uint32_t cur = v;
#pragma unroll
        for (int t = 0; t < LEN; ++t) {
          if ((uint32_t)t < len) {
            const uint64_t b = ld_indptr(indptr + cur);
            const uint32_t deg = (uint32_t)(ld_indptr(indptr + cur + 1) - b);
            if (deg == 0) break;
            const uint64_t r = draw64(seed, v, (w << 8) | ((uint32_t)t >> 1), batch, c3, t & 1);
            cur = ld_csr(indices + b + bounded(r, deg));
            if (cur != v) vis[t] = cur;
          }
        }
      }
    }
    // visit counts and first occurrences over the group's walks*len entries
    uint32_t cnt[LEN];
    bool first[LEN];
#pragma unroll
    for (int t = 0; t < LEN; ++t) { cnt[t] = 0; first[t] = true; }
    for (uint32_t src = 0; src < G; ++src) {
#pragma unroll
      for (int tt = 0; tt < LEN; ++tt) {
        const uint32_t x = __shfl_sync(kFull, vis[tt], gbase + src);
#pragma unroll
        for (int t = 0; t < LEN; ++t) {
          if (vis[t] != kEmpty && x == vis[t]) {
            ++cnt[t];
            if (src * LEN + tt < w * LEN + t) first[t] = false;
          }
        }
      }
    }
    // rank of each distinct visited vertex by (count desc, gid asc)
    uint32_t rank[LEN];
    uint32_t ndist = 0;
#pragma unroll
    for (int t = 0; t < LEN; ++t) rank[t] = 0;
    for (uint32_t src = 0; src < G; ++src) {
#pragma unroll
      for (int tt = 0; tt < LEN; ++tt) {
        const uint32_t x = __shfl_sync(kFull, vis[tt], gbase + src);
        const uint32_t xc = __shfl_sync(kFull, cnt[tt], gbase + src);
        const bool xf = __shfl_sync(kFull, first[tt], gbase + src);
        if (x != kEmpty && xf) {
          ++ndist;
#pragma unroll
          for (int t = 0; t < LEN; ++t)
            if (vis[t] != kEmpty && first[t] && (xc > cnt[t] || (xc == cnt[t] && x < vis[t])))
              ++rank[t];
        }
      }
    }
    if (active) {
      for (uint32_t r = w; r < topk; r += G)
        if (r >= ndist) picks[(size_t)d * topk + r] = kEmpty;
#pragma unroll
      for (int t = 0; t < LEN; ++t) {
        if (vis[t] != kEmpty && first[t] && rank[t] < topk) {
          const uint32_t f = d * topk + rank[t];
          const unsigned long long e = enc_pos(gen, base + f);
          const uint32_t idx = entry_of<HASH>(T, vis[t], st_w);
          picks[f] = idx == kEmpty ? kEmpty : encode_pick(vis[t], vmap_insert(T.e, idx, e), e, base);
          if (HASH) pidx[f] = idx;
          pickw[f] = cnt[t];
        }
      }
    }
  }
}

// ---------------------------------------------------------------- compaction scan
// Status word of the decoupled look-back: [flag:2][new:31][valid:31].
// flag 1 = aggregate, 2 = inclusive prefix.
constexpr unsigned long long kFlagAgg = 1ull << 62;
constexpr unsigned long long kFlagInc = 2ull << 62;
constexpr unsigned long long kValMask = (1ull << 62) - 1;
#ifndef GLB_LOOKBACK
#define GLB_LOOKBACK 8
#endif
constexpr int kLookback = GLB_LOOKBACK;  // look-back window = 32 * kLookback tiles

__device__ __forceinline__ unsigned long long pack_status(unsigned long long flag,
                                                          unsigned long long pair) {
  // pair = new << 32 | valid
  return flag | ((pair >> 32) << 31) | (pair & 0x7FFFFFFFull);
}
__device__ __forceinline__ unsigned long long unpack_pair(unsigned long long w) {
  w &= kValMask;
  return ((w >> 31) << 32) | (w & 0x7FFFFFFFull);
}

template <typename T>
__device__ __forceinline__ T warp_incl_scan(T x) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const T y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  return x;
}
__device__ __forceinline__ unsigned long long warp_sum64(unsigned long long x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(kFull, x, o);
  return x;
}

// One tile = kCompactTile consecutive (vertex, slot) positions of hop l; warp
// w owns positions [w*512, w*512+512) of the tile and walks them 32 at a time
// (lane = position), so every load and every compacted store is coalesced.
//  1. valid = pick present; new = this position is the first occurrence
//     (vmap holds the minimum position of this generation).
//  2. warp ballots + block scan + decoupled look-back -> global prefixes:
//     new vertices get lid n_l + new-prefix (first-occurrence order); valid
//     picks get edge slot valid-prefix (block CSR in slot order).
//  3. new vertices: uniq / lidmap / mark lists / visit count.
//  4. every edge's src lid: new -> own; repeat of a vertex first seen at an
//     earlier position p: same tile -> shared memory; relabelled already
//     (vmap holds (gen, lid) with lid < base) -> that lid; earlier tile of
//     this hop -> deferred: the entry holds gid | kDefer and fixup_block (in
//     the next kernel) reads the lid from vmap once every tile has written.
//  vmap doubles as the gid -> lid map: the first-occurrence tile overwrites
//  (gen, position) with (gen, lid); lid <= position, so the table stays
//  monotone (later atomicMins never replace it) and a concurrent reader sees
//  either value, both of which it resolves correctly.

#ifndef GLB_COMPACT_MINB  // min resident compaction blocks per SM (register cap; A/B builds)
#define GLB_COMPACT_MINB 3
#endif
template <bool W, bool HASH>
__global__ void __launch_bounds__(kThreads, GLB_COMPACT_MINB)
    k_compact(uint32_t hop, uint32_t k, Table T, DevState* st,
              const uint32_t* __restrict__ picks, const uint32_t* __restrict__ pickw,
              const uint32_t* __restrict__ pidx,
              uint32_t* __restrict__ uniq, uint32_t* __restrict__ bindptr,
              uint32_t* __restrict__ bindices, uint32_t* __restrict__ bweights,
              unsigned long long* status, MarkArgs mk, uint32_t num_sms) {
  pdl_enter();
  constexpr int NW = kThreads / 32;
  __shared__ uint32_t s_tile;
  __shared__ unsigned long long s_wnv[NW];  // per warp (new << 32 | valid), then exclusive
  __shared__ uint32_t s_whm[NW];            // per warp (hit | miss << 16), then exclusive
  __shared__ unsigned long long s_excl;
  __shared__ uint32_t s_hbase, s_mbase;
  // per position: the cache slot of a new vertex (phase 1 -> 3), then its lid (3 -> 4)
  __shared__ uint32_t s_lid[kCompactTile];
  __shared__ uint32_t s_idx[HASH ? kCompactTile : 1];  // hash mode: table index per position
  const uint32_t gen = T.gen;
  const uint32_t n_l = st->n[hop];
  const uint32_t base = st->base[hop];
  const uint32_t flat = n_l * k;
  const uint32_t items = compact_items(flat, num_sms);  // positions per thread
  const uint32_t tile_n = items * kThreads;
  const uint32_t ntiles = (flat + tile_n - 1) / tile_n;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const uint32_t lt = lanemask_lt();
  if (flat == 0) {
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      st->n[hop + 1] = n_l;
      st->nnz[hop] = 0;
      st->base[hop + 1] = base;
      bindptr[n_l] = 0;
      if (n_l == 0) bindptr[0] = 0;
    }
    return;
  }
  for (;;) {
    if (threadIdx.x == 0) s_tile = atomicAdd(&st->tile_ctr[hop], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    if (tile >= ntiles) break;
    TRACE(hop, tile, 0);
    const uint32_t t0 = tile * tile_n;
    const uint32_t loc0 = wid * items * 32 + lane;  // local position of item 0
    uint32_t u[kCompactItems];
    uint32_t p[kCompactItems];  // first position (this generation) of u[i]
#pragma unroll
    for (int i = 0; i < kCompactItems; ++i) {
      const uint32_t f = t0 + loc0 + i * 32;
      u[i] = ((uint32_t)i < items && f < flat) ? picks[f] : kEmpty;
    }
    uint32_t vmask = 0, nmask = 0, hmask = 0;
#pragma unroll
    for (int i = 0; i < kCompactItems; ++i) {
      p[i] = 0;
      if (u[i] != kEmpty) {
        vmask |= 1u << i;
        if (u[i] & kOld) {
          p[i] = u[i] & ~kOld;  // the sampler resolved it: a lid < base
        } else {
          // dense: one 16-byte load gives (gen, position-or-lid) and the cache slot
          const uint32_t idx = HASH ? pidx[t0 + loc0 + i * 32] : u[i];
          if (HASH) s_idx[loc0 + i * 32] = idx;
          const ulonglong2 ent = __ldcg(reinterpret_cast<const ulonglong2*>(T.e + idx));
          p[i] = (uint32_t)ent.x;
          if (ent.x == enc_pos(gen, base + t0 + loc0 + i * 32)) {
            nmask |= 1u << i;
            const int32_t sl = HASH ? __ldcg(T.hslot + idx) : (int32_t)(uint32_t)ent.y;
            s_lid[loc0 + i * 32] = (uint32_t)sl;
            if (sl >= 0) hmask |= 1u << i;
          }
        }
      }
    }
    TRACE(hop, tile, 1);
    {  // warp totals
      const uint32_t nn = __popc(nmask), nh = __popc(hmask);
      unsigned long long nv = ((unsigned long long)nn << 32) | __popc(vmask);
      uint32_t hm = nh | ((nn - nh) << 16);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        nv += __shfl_xor_sync(kFull, nv, o);
        hm += __shfl_xor_sync(kFull, hm, o);
      }
      if (lane == 0) {
        s_wnv[wid] = nv;
        s_whm[wid] = hm;
      }
    }
    __syncthreads();
    if (wid == 0) {
      const unsigned long long x = lane < NW ? s_wnv[lane] : 0ull;
      const unsigned long long xi = warp_incl_scan(x);
      const uint32_t y = lane < NW ? s_whm[lane] : 0u;
      const uint32_t yi = warp_incl_scan(y);
      if (lane < NW) {
        s_wnv[lane] = xi - x;  // exclusive warp offsets
        s_whm[lane] = yi - y;
      }
      const unsigned long long agg = __shfl_sync(kFull, xi, NW - 1);
      const uint32_t agg_hm = __shfl_sync(kFull, yi, NW - 1);
      if (lane == 0) {  // list space for this tile's marks (independent of the look-back)
        s_hbase = (agg_hm & 0xFFFFu) ? atomicAdd(&st->nhit, agg_hm & 0xFFFFu) : 0u;
        s_mbase = (agg_hm >> 16) ? atomicAdd(&st->nmiss, agg_hm >> 16) : 0u;
      }
      // decoupled look-back
      unsigned long long excl = 0;
      if (tile == 0) {
        if (lane == 0) atomicExch(status + 0, pack_status(kFlagInc, agg));
      } else {
        if (lane == 0) atomicExch(status + tile, pack_status(kFlagAgg, agg));
        // Look-back over a window of 32*kLookback predecessors at once (entry o = q*32 +
        // lane is tile idx - o): all its status words are loaded together and re-polled
        // until published, so an inclusive prefix propagates kLookback*32 tiles per L2
        // round trip instead of 32 (the chain dominated small hops).
        long long idx = (long long)tile - 1;
        for (;;) {
          unsigned long long wv[kLookback];
#pragma unroll
          for (int q = 0; q < kLookback; ++q) {
            const long long jx = idx - (q * 32 + lane);
            wv[q] = jx >= 0 ? (unsigned long long)*((volatile unsigned long long*)(status + jx))
                            : (unsigned long long)kFlagInc;
          }
          for (;;) {
            bool pending = false;
#pragma unroll
            for (int q = 0; q < kLookback; ++q) pending |= (wv[q] >> 62) == 0;
            if (!__any_sync(kFull, pending)) break;
#pragma unroll
            for (int q = 0; q < kLookback; ++q)
              if ((wv[q] >> 62) == 0)
                wv[q] = *((volatile unsigned long long*)(status + idx - (q * 32 + lane)));
          }
          int qmin = -1;
          uint32_t incm = 0;
#pragma unroll
          for (int q = 0; q < kLookback; ++q) {
            const uint32_t b = __ballot_sync(kFull, (wv[q] >> 62) >= 2);
            if (qmin < 0 && b) {
              qmin = q;
              incm = b;
            }
          }
          unsigned long long part = 0;
          if (qmin >= 0) {  // nearest inclusive prefix: entry (qmin, first lane of incm)
            const int lmin = __ffs(incm) - 1;
#pragma unroll
            for (int q = 0; q < kLookback; ++q)
              if (q < qmin || (q == qmin && lane <= lmin)) part += unpack_pair(wv[q]);
            excl += warp_sum64(part);
            break;
          }
#pragma unroll
          for (int q = 0; q < kLookback; ++q) part += unpack_pair(wv[q]);
          excl += warp_sum64(part);
          idx -= 32 * kLookback;
        }
        if (lane == 0) atomicExch(status + tile, pack_status(kFlagInc, excl + agg));
      }
      TRACE(hop, tile, 2);
      if (lane == 0) {
        s_excl = excl;
        if (tile == ntiles - 1) {
          const unsigned long long tot = excl + agg;
          st->n[hop + 1] = n_l + (uint32_t)(tot >> 32);
          st->nnz[hop] = (uint32_t)tot;
          st->base[hop + 1] = base + flat;
          bindptr[n_l] = (uint32_t)tot;
        }
      }
    }
    __syncthreads();
    TRACE(hop, tile, 3);
    const unsigned long long ex = s_excl + s_wnv[wid];
    // 3. new vertices (compacted, coalesced)
    {
      uint32_t rn = (uint32_t)(ex >> 32);
      uint32_t rh = s_hbase + (s_whm[wid] & 0xFFFFu), rm = s_mbase + (s_whm[wid] >> 16);
#pragma unroll
      for (int i = 0; i < kCompactItems; ++i) {
        const bool isn = (nmask >> i) & 1u, ish = (hmask >> i) & 1u;
        const uint32_t nb = __ballot_sync(kFull, isn);
        const uint32_t hb = __ballot_sync(kFull, ish);
        const uint32_t mb = nb & ~hb;
        if (isn) {
          const uint32_t loc = loc0 + i * 32;
          const uint32_t lid = n_l + rn + __popc(nb & lt);
          const int32_t sl = (int32_t)s_lid[loc];
          uniq[lid] = u[i];
          __stcg(&T.e[HASH ? s_idx[loc] : u[i]].gp, enc_pos(gen, lid));  // relabelled: readers get the lid
          mk.lidslot[lid] = sl;
          if (ish) mk.hit_list[rh + __popc(hb & lt)] = make_uint2(lid, (uint32_t)sl);
          else mk.miss_list[rm + __popc(mb & lt)] = make_uint2(lid, u[i]);
          if (mk.count) atomicAdd(mk.count + u[i], 1u);
          s_lid[loc] = lid;
        }
        rn += __popc(nb);
        rh += __popc(hb);
        rm += __popc(mb);
      }
    }
    __syncthreads();
    TRACE(hop, tile, 4);
    // 4. edges (src lids, compacted, coalesced) and block indptr
    {
      uint32_t lid[kCompactItems];
#pragma unroll
      for (int i = 0; i < kCompactItems; ++i) {  // independent loads first
        lid[i] = 0;
        if ((vmask >> i) & 1u) {
          const uint32_t fp = p[i] - base;  // first position as a flat index of this hop
          if ((nmask >> i) & 1u) lid[i] = s_lid[loc0 + i * 32];
          else if (p[i] < base) lid[i] = p[i];                   // relabelled earlier (lid)
          else if (fp >= t0) lid[i] = s_lid[fp - t0];           // earlier in this tile
          else lid[i] = (HASH ? s_idx[loc0 + i * 32] : u[i]) | kDefer;  // earlier tile: fixup
        }
      }
      uint32_t rv = (uint32_t)ex;
#pragma unroll
      for (int i = 0; i < kCompactItems; ++i) {
        const uint32_t f = t0 + loc0 + i * 32;
        const bool isv = (vmask >> i) & 1u;
        const uint32_t vb = __ballot_sync(kFull, isv);
        const uint32_t ev = rv + __popc(vb & lt);
        if ((uint32_t)i < items && f < flat && f % k == 0) bindptr[f / k] = ev;
        if (isv) {
          bindices[ev] = lid[i];
          if (W) bweights[ev] = pickw[f];
        }
        rv += __popc(vb);
      }
    }
    __syncthreads();
    TRACE(hop, tile, 5);
  }
}

__global__ void __launch_bounds__(kThreads)
    k_fixup(uint32_t hop, const DevState* __restrict__ st, const VEntry* vmap,
            uint32_t* __restrict__ bindices) {
  pdl_enter();
  fixup_block(st->nnz[hop], vmap, bindices);
}

__global__ void k_validate(const uint64_t* __restrict__ indptr, const uint32_t* __restrict__ indices,
                           uint64_t V, uint64_t E, DevState* st) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t t0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  bool bad = false;
  for (uint64_t i = t0; i < V; i += stride) bad |= indptr[i + 1] < indptr[i];
  if (t0 == 0) bad |= indptr[0] != 0 || indptr[V] != E;
  for (uint64_t e = t0; e < E; e += stride) bad |= indices[e] >= V;
  if (bad) atomicOr(&st->err, kErrBadGraph);
}

// Hash mode: every entry free (generation 0 is never used) with gp = max.
__global__ void k_table_reset(VEntry* __restrict__ t, uint64_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    t[i].gp = ~0ull;
    t[i].aux = 0ull;
  }
}

// sampler grids: blocks per SM (GLB_SAMPLE_BPS; default 8 = a full SM of 256-thread blocks)
inline int grid_for(glb_ctx* c, int per_sm = 0) {
  return c->num_sms * (per_sm ? per_sm : c->sample_bps);
}

MarkArgs mark_args(glb_ctx* c, int count_mode) {
  MarkArgs m;
  m.slot = c->slot;
  m.lidslot = c->sb.lidslot;
  m.hit_list = c->sb.hit_list;
  m.miss_list = c->sb.miss_list;
  m.count = count_mode == GLB_COUNT_PRESAMPLE ? c->counts
            : count_mode == GLB_COUNT_ACCESS  ? c->access
                                              : nullptr;
  return m;
}

Table table_of(glb_ctx* c) {
  Table T;
  T.e = c->hash_mode ? c->htab : c->vmap;
  T.hslot = c->hslot;
  T.slot = c->slot;
  T.mask = c->hmask;
  T.gen = c->gen;
  return T;
}

}  // namespace

cudaError_t launch_validate_graph(glb_ctx* c) {
  k_validate<<<grid_for(c), kThreads, 0, c->stream>>>(c->indptr, c->indices, c->V, c->E, c->st);
  count_launch(c);
  return cudaGetLastError();
}

cudaError_t launch_seed_init(glb_ctx* c, const uint32_t* seeds, uint32_t n0, int count_mode) {
  int blocks = (int)((n0 + kThreads - 1) / kThreads);
  if (blocks < 1) blocks = 1;
  if (blocks > grid_for(c)) blocks = grid_for(c);
  StatusArgs za = {};
  za.L = c->sb.L;
  for (uint32_t l = 0; l < c->sb.L; ++l) {
    za.p[l] = c->sb.status[l];
    za.n[l] = (uint32_t)c->sb.ntiles[l];
  }
  const Table T = table_of(c);
  const cudaError_t e =
      c->hash_mode
          ? launch_pdl_w(c->pin, k_seed_init<true>, blocks, kThreads, c->stream, seeds, n0, c->V, c->st,
                       c->sb.uniq, T, mark_args(c, count_mode), za)
          : launch_pdl_w(c->pin, k_seed_init<false>, blocks, kThreads, c->stream, seeds, n0, c->V, c->st,
                       c->sb.uniq, T, mark_args(c, count_mode), za);
  count_launch(c);
  return e;
}

cudaError_t launch_khop(glb_ctx* c, uint32_t hop, uint32_t k, uint64_t seed, uint32_t epoch,
                        uint32_t batch) {
  const int grid = grid_for(c);
  const SampleBufs& b = c->sb;
  uint32_t* fix = hop ? b.bindices[hop - 1] : nullptr;
  const DevState* stc = c->st;
  const uint64_t* ip = c->indptr;
  const uint32_t* ix = c->indices;
  const uint32_t* uq = b.uniq;
  const Table T = table_of(c);
  cudaError_t e;
#define GLB_KH_ARGS hop, k, seed, epoch, batch, T, stc, c->st, ip, ix, uq, b.picks, b.pidx, fix
  if (k <= 32 && c->relabel_dedup == 2)
    e = c->hash_mode ? launch_pdl_w(c->pin, k_khop<true, 2>, grid, kThreads, c->stream, GLB_KH_ARGS)
                     : launch_pdl_w(c->pin, k_khop<false, 2>, grid, kThreads, c->stream, GLB_KH_ARGS);
  else if (k <= 32 && c->relabel_dedup == 1)
    e = c->hash_mode ? launch_pdl_w(c->pin, k_khop<true, 1>, grid, kThreads, c->stream, GLB_KH_ARGS)
                     : launch_pdl_w(c->pin, k_khop<false, 1>, grid, kThreads, c->stream, GLB_KH_ARGS);
  else if (k <= 32)
    e = c->hash_mode ? launch_pdl_w(c->pin, k_khop<true, 0>, grid, kThreads, c->stream, GLB_KH_ARGS)
                     : launch_pdl_w(c->pin, k_khop<false, 0>, grid, kThreads, c->stream, GLB_KH_ARGS);
  else
    e = c->hash_mode ? launch_pdl_w(c->pin, k_khop_wide<true>, grid, kThreads, c->stream, GLB_KH_ARGS)
                     : launch_pdl_w(c->pin, k_khop_wide<false>, grid, kThreads, c->stream, GLB_KH_ARGS);
#undef GLB_KH_ARGS
  count_launch(c);
  return e;
}

cudaError_t launch_khop_weighted(glb_ctx* c, uint32_t hop, uint32_t k, uint64_t seed,
                                 uint32_t epoch, uint32_t batch) {
  const int grid = grid_for(c);
  const SampleBufs& b = c->sb;
  uint32_t* fix = hop ? b.bindices[hop - 1] : nullptr;
  const DevState* stc = c->st;
  const uint64_t* ip = c->indptr;
  const uint32_t* ix = c->indices;
  const unsigned long long* wp = c->wprefix;
  const uint32_t* uq = b.uniq;
  const Table T = table_of(c);
  cudaError_t e;
#define GLB_KW_ARGS hop, k, seed, epoch, batch, T, stc, c->st, ip, ix, wp, uq, b.picks, b.pidx, fix
  e = c->hash_mode ? launch_pdl_w(c->pin, k_khop_weighted<true>, grid, kThreads, c->stream, GLB_KW_ARGS)
                   : launch_pdl_w(c->pin, k_khop_weighted<false>, grid, kThreads, c->stream, GLB_KW_ARGS);
#undef GLB_KW_ARGS
  count_launch(c);
  return e;
}

cudaError_t launch_rwalk(glb_ctx* c, uint32_t hop, uint64_t seed, uint32_t epoch, uint32_t batch) {
  const int grid = grid_for(c);
  const SampleBufs& b = c->sb;
#define GLB_RW_ARGS                                                                            \
  hop, c->rw_walks, c->rw_len, c->rw_topk, seed, epoch, batch, T, stc, c->st, ip, ix, uq, b.picks, \
      b.pickw, b.pidx, fix
  uint32_t* fix = hop ? b.bindices[hop - 1] : nullptr;
  const uint32_t w = c->rw_walks;
  const DevState* stc = c->st;
  const uint64_t* ip = c->indptr;
  const uint32_t* ix = c->indices;
  const uint32_t* uq = b.uniq;
  const Table T = table_of(c);
  cudaError_t e;
#define GLB_RW_L(GG, LL)                                                                       \
  (c->hash_mode ? launch_pdl_w(c->pin, k_rwalk<GG, LL, true>, grid, kThreads, c->stream, GLB_RW_ARGS)  \
                : launch_pdl_w(c->pin, k_rwalk<GG, LL, false>, grid, kThreads, c->stream, GLB_RW_ARGS))
#define GLB_RW_G(GG) (c->rw_len <= 3 ? GLB_RW_L(GG, 3) : GLB_RW_L(GG, kMaxWalkLen))
  if (w <= 1) e = GLB_RW_G(1);
  else if (w <= 2) e = GLB_RW_G(2);
  else if (w <= 4) e = GLB_RW_G(4);
  else if (w <= 8) e = GLB_RW_G(8);
  else if (w <= 16) e = GLB_RW_G(16);
  else e = GLB_RW_G(32);
#undef GLB_RW_G
#undef GLB_RW_L
#undef GLB_RW_ARGS
  count_launch(c);
  return e;
}

cudaError_t launch_fixup(glb_ctx* c, uint32_t hop) {
  const DevState* stc = c->st;
  const VEntry* vm = table_of(c).e;
  const cudaError_t e = launch_pdl_w(c->pin, k_fixup, grid_for(c), kThreads, c->stream, hop, stc, vm,
                                   c->sb.bindices[hop]);
  count_launch(c);
  return e;
}

cudaError_t launch_compact(glb_ctx* c, uint32_t hop, uint32_t k, bool weighted, int count_mode) {
  const SampleBufs& b = c->sb;
  const int grid = grid_for(c, GLB_COMPACT_MINB);
  const uint32_t* pk = b.picks;
  const uint32_t* pw = b.pickw;
  const uint32_t* pi = b.pidx;
  const uint32_t nsm = (uint32_t)c->num_sms;
  const Table T = table_of(c);
  const MarkArgs mk = mark_args(c, count_mode);
  cudaError_t e;
#define GLB_CP_ARGS(W)                                                                          \
  hop, k, T, c->st, pk, pw, pi, b.uniq, b.bindptr[hop], b.bindices[hop],                        \
      (W) ? b.bweights[hop] : (uint32_t*)nullptr, b.status[hop], mk, nsm
  if (weighted)
    e = c->hash_mode ? launch_pdl_w(c->pin, k_compact<true, true>, grid, kThreads, c->stream, GLB_CP_ARGS(1))
                     : launch_pdl_w(c->pin, k_compact<true, false>, grid, kThreads, c->stream, GLB_CP_ARGS(1));
  else
    e = c->hash_mode ? launch_pdl_w(c->pin, k_compact<false, true>, grid, kThreads, c->stream, GLB_CP_ARGS(0))
                     : launch_pdl_w(c->pin, k_compact<false, false>, grid, kThreads, c->stream, GLB_CP_ARGS(0));
#undef GLB_CP_ARGS
  count_launch(c);
  return e;
}

cudaError_t launch_table_reset(glb_ctx* c) {
  if (c->hash_mode && c->htab) {
    const uint64_t n = (uint64_t)c->hmask + 1;
    k_table_reset<<<grid_for(c), kThreads, 0, c->stream>>>(c->htab, n);
    count_launch(c);
  }
  return cudaGetLastError();
}

}  // namespace glb
