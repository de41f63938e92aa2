// glb_internal.cuh -- internal declarations of the B200 sample+extract library.
// Not part of the ABI (see include/glb.h).  Shares nothing with oracle/.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "glb.h"

namespace glb {

constexpr uint32_t kEmpty = 0xFFFFFFFFu;
constexpr int kThreads = 256;          // block size of every grid-stride kernel
constexpr int kCompactItems = 16;      // max flat positions per thread in a compaction tile
constexpr int kCompactTile = kThreads * kCompactItems;  // max tile
constexpr int kCompactMinItems = 2;    // tiles shrink to >= 2 per SM for small hops
// positions per thread for a hop of `flat` positions: aim at ~2 tiles per SM
__host__ __device__ inline uint32_t compact_items(uint32_t flat, uint32_t num_sms) {
  const uint32_t per = 2u * num_sms * (uint32_t)kThreads;
  uint32_t it = (flat + per - 1) / per;
  return it < (uint32_t)kCompactMinItems ? (uint32_t)kCompactMinItems
         : it > (uint32_t)kCompactItems ? (uint32_t)kCompactItems : it;
}
constexpr int kMaxFanout = 1024;
constexpr int kMaxShards = 16;  // GLB_MAX_SHARDS: ranks of a peer-sharded cache (NEXT-3)
constexpr int kMaxWalkLen = 8;

// RNG domains (reading Q4): counter word 3 = epoch<<16 | hop<<8 | domain
enum : uint32_t { kDomShuffle = 1, kDomKhop = 2, kDomRwalk = 3, kDomPolicy = 7, kDomWeighted = 8 };

// device error bits (DevState::err)
enum : uint32_t { kErrDupSeed = 1u, kErrRange = 2u, kErrCapacity = 4u, kErrBadGraph = 8u };
// hash-table capacity limit: indices (with the kDefer bit) must stay below 2^31.  The table
// is sized at >= 1.25x the batch's unique-vertex upper bound, so it never fills (no cap
// below the bound: TW's bound is 8.4 M, table 16 M entries = 320 MB)
constexpr uint32_t kMaxHashEntries = 1u << 31;

// Per-batch device state.  Sizes live here so no kernel needs a host sync.
struct DevState {
  uint32_t n[GLB_MAX_HOPS + 1];     // frontier sizes n_0..n_L
  uint32_t nnz[GLB_MAX_HOPS];       // block edge counts
  uint32_t base[GLB_MAX_HOPS + 1];  // first flat position of hop l (relabel order)
  uint32_t tile_ctr[GLB_MAX_HOPS];  // dynamic tile ids of the compaction scans
  uint32_t nhit, nmiss;             // extract work lists (marks)
  uint32_t err;
  uint32_t pad;
};

// Counter-based RNG: Philox4x32-10 (Random123 constants).
__device__ __forceinline__ uint4 philox10(uint4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    if (r) {
      k0 += 0x9E3779B9u;
      k1 += 0xBB67AE85u;
    }
    const uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
    c = make_uint4(hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0);
  }
  return c;
}
__device__ __forceinline__ uint32_t ctr3(uint32_t epoch, uint32_t hop, uint32_t dom) {
  return ((epoch & 0xFFFFu) << 16) | ((hop & 0xFFu) << 8) | (dom & 0xFFu);
}
__device__ __forceinline__ uint64_t draw64(uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2,
                                           uint32_t c3, uint32_t half) {
  const uint4 w = philox10(make_uint4(c0, c1, c2, c3), (uint32_t)seed, (uint32_t)(seed >> 32));
  return half ? (((uint64_t)w.w << 32) | w.z) : (((uint64_t)w.y << 32) | w.x);
}
// floor(r * n / 2^64)
__device__ __forceinline__ uint32_t bounded(uint64_t r, uint32_t n) {
  return (uint32_t)__umul64hi(r, (uint64_t)n);
}

// Relabel table entry: ((0xFFFFFFFF - gen) << 32) | position.  Within one
// generation atomicMin keeps the first position; a newer generation is always
// smaller, so stale entries never need clearing.
__device__ __forceinline__ uint64_t enc_pos(uint32_t gen, uint32_t pos) {
  return ((uint64_t)(0xFFFFFFFFu - gen) << 32) | pos;
}

// Relabel-table entry: gp = ((0xFFFFFFFF - gen) << 32) | first position, then
// | lid once relabelled.  Dense mode (one entry per vertex): aux = the vertex's
// cache slot (-1 = not cached), co-located so one 16-byte load gives both (a4
// mark needs no extra access).  Hash mode: aux = (gen << 32 | gid) key.
struct __align__(16) VEntry {
  unsigned long long gp;
  unsigned long long aux;  // dense: cache slot (low 32 bits); hash: gen << 32 | gid
};

// Optional L2 access-policy window: the relabel table is marked persisting so the
// random CSR / feature traffic between its accesses does not evict it.
struct L2Window {
  void* base = nullptr;
  size_t bytes = 0;
  float hit_ratio = 0.f;
};

struct SampleBufs {
  uint32_t cap_batch = 0;
  uint32_t L = 0;
  uint64_t ub[GLB_MAX_HOPS + 1] = {};
  uint32_t k[GLB_MAX_HOPS] = {};      // slots per frontier vertex (fanout or topk)
  uint32_t* seeds = nullptr;          // u32[cap_batch]
  uint32_t* uniq = nullptr;           // u32[ub[L]]
  int32_t* lidslot = nullptr;         // i32[ub[L]]  (a4 marks)
  uint32_t* picks = nullptr;          // u32[max ub[l]*k[l]]
  uint32_t* pidx = nullptr;           // u32[...] hash mode: table index of each pick
  uint32_t* pickw = nullptr;          // u32[...] random-walk counts
  uint32_t* bindptr[GLB_MAX_HOPS] = {};
  uint32_t* bindices[GLB_MAX_HOPS] = {};
  uint32_t* bweights[GLB_MAX_HOPS] = {};
  unsigned long long* status[GLB_MAX_HOPS] = {};
  uint64_t ntiles[GLB_MAX_HOPS] = {};
  uint2* hit_list = nullptr;          // extract work lists: (dst row, cache slot)
  uint2* miss_list = nullptr;         //                     (dst row, gid)
  uint2* miss_sorted = nullptr;       // miss_list ordered by host page
};

struct ExtractBufs {
  uint64_t cap = 0;
  uint2* hit_list = nullptr;
  uint2* miss_list = nullptr;
  uint2* miss_sorted = nullptr;
};

// a8 factored handoff (handoff.cu).  A trainer owns a ring of receive slots in its HBM;
// each slot holds a pushed sample: [header: DevState + tag | uniq | indptr_l | indices_l |
// weights_l], every array at a 256-byte aligned offset fixed by the trainer's sampler
// capacities (HandoffLayout, shipped to samplers in the trainer's blob).
constexpr int kHandoffMaxSlots = 8;   // GLB_HANDOFF_MAX_SLOTS
constexpr int kHandoffMaxPeers = 16;  // GLB_HANDOFF_MAX_PEERS
struct HandoffLayout {
  uint64_t slot_bytes, off_tag, off_uniq, cap_uniq;
  uint64_t off_indptr[GLB_MAX_HOPS], off_indices[GLB_MAX_HOPS], off_weights[GLB_MAX_HOPS];
  uint64_t cap_indptr[GLB_MAX_HOPS], cap_nnz[GLB_MAX_HOPS];
  uint32_t L, weighted;
};
struct HandoffRecv {  // trainer side
  uint32_t slots = 0;
  HandoffLayout lay = {};
  uint8_t* ring = nullptr;  // device [slots * slot_bytes], IPC-exported
  int32_t* lidslot[kHandoffMaxSlots] = {};  // local per-slot marks (trainer's cache)
  uint2* hit[kHandoffMaxSlots] = {};
  uint2* miss[kHandoffMaxSlots] = {};
  uint2* miss_sorted[kHandoffMaxSlots] = {};
  cudaEvent_t consumed[kHandoffMaxSlots] = {};            // own, interprocess
  cudaEvent_t ready[kHandoffMaxPeers][kHandoffMaxSlots] = {};  // samplers' (opened)
  bool ready_opened[kHandoffMaxPeers] = {};              // opened via IPC (destroy on free)
  int cur = -1;                                          // slot of the current sample
};
struct HandoffSend {  // sampler side, one per attached trainer
  uint32_t slots = 0;
  HandoffLayout lay = {};
  uint8_t* ring = nullptr;  // trainer's ring, mapped (IPC) or borrowed (same process)
  bool ring_ipc = false;
  cudaEvent_t consumed[kHandoffMaxSlots] = {};  // trainer's (opened, or borrowed)
  bool consumed_opened = false;
  cudaEvent_t ready[kHandoffMaxSlots] = {};     // own, interprocess
};

struct HostGather;  // hostgather.cu: host-assisted miss gather (threads, streams, staging)

}  // namespace glb

struct glb_ctx {
  int device = 0;
  cudaStream_t own_stream = nullptr;
  cudaStream_t stream = nullptr;
  int num_sms = 148;
  bool poisoned = false;
  std::string err;
  uint64_t launches = 0;

  // graph (D1, D2)
  uint64_t V = 0, E = 0;
  uint64_t* indptr = nullptr;
  uint32_t* indices = nullptr;
  unsigned long long* wprefix = nullptr;  // [E] inclusive prefix of edge weights (weighted k-hop)
  const void* h_features = nullptr;
  const float* features_mapped = nullptr;  // device alias of the registered host matrix
  bool registered = false;
  uint32_t D = 0;

  // relabel tables (D6): direct-address over gids
  glb::VEntry* vmap = nullptr;  // dense relabel table [V]: (gen, position|lid), cache slot
  glb::VEntry* htab = nullptr;  // hash relabel table [hmask+1]: (gen, position|lid), key
  int32_t* hslot = nullptr;     // [hmask+1] cache slot of each hash entry
  uint32_t hmask = 0;
  bool hash_mode = false;
  int relabel_mode = 0;         // 0 auto, 1 dense, 2 hash (glb_set_relabel_mode)
  int relabel_dedup = 0;        // GLB_RELABEL_DEDUP: 1 warp-level / 2 block smem-staged pre-dedup
                                // of picks before the relabel-table insert (k_khop)
  glb::L2Window pin;            // persisting-L2 window over the relabel table
  int l2_pin = -1;              // -1 auto (small tables only), GLB_L2_PIN=0 off / 1 on
  uint32_t gen = 0;

  // cache (D3, D4, D5)
  int32_t* slot = nullptr;     // i32[V]
  float* cache = nullptr;      // f32[C][cache_stride]
  uint32_t cache_stride = 0;   // floats per cache row: D, or D padded to cache_align bytes
  uint32_t cache_align = 0;    // GLB_CACHE_ALIGN (bytes; 0 = dense rows)
  int gather_st_wb = 0;        // GLB_GATHER_ST=1: write-back stores instead of streaming
  int gather_bulk = 0;         // GLB_GATHER_BULK=1: hits through cp.async.bulk (k_gather_bulk);
                               // measured 2x slower than the LSU gather
  uint32_t gather_bulk_smem = 96 * 1024;  // row-slot bytes per bulk block (GLB_GATHER_BULK_SMEM)
  int miss_bulk = 0;           // GLB_MISS_BULK=1: host misses through cp.async.bulk
  int gather_warp = 0;         // GLB_GATHER_WARP=1: warp-independent gather (k_gather_w)
  uint32_t miss_blocks = 0;    // GLB_MISS_BLOCKS: blocks of k_gather that take host misses (0 all)
  // cold store (glb_set_cold_store): a rank-ordered, pinned host copy of the rows NOT in the
  // HBM cache; misses read it instead of the caller's matrix (fewer host pages per batch)
  int cold_store = 0;             // enabled for the next build_cache
  float* cold_h = nullptr;        // host rows [V - C][D], registered mapped + portable
  const float* cold_d = nullptr;  // device alias
  uint64_t cold_rows = 0;
  size_t cold_bytes = 0;          // registered in 4 GB pieces
  uint32_t* cold_row = nullptr;   // device u32[V]: the cold-store row of a non-cached vertex
  int misses_first = -1;       // miss-taking gather blocks start on the misses: -1 auto (on the
                               // extract stream), GLB_MISSES_FIRST=0/1 forces
  int gather_lidorder = 1;     // sample extracts gather hits in lid order from the marks
                               // (GLB_GATHER_LIDORDER=0: from the hit list; measured 1-2 % slower)
  glb::HostGather* hg = nullptr;  // host-assisted misses (glb_set_host_gather)
  uint32_t hg_permille = 0;       // share of a batch's misses gathered by host threads
  uint32_t hg_threads = 0;
  bool hg_inflight = false;       // the extract being enqueued has a host-assisted part
  uint64_t C = 0;
  // NEXT-3 peer-sharded cache: global rank i < C is owned by shard i % W at row i / W;
  // shard_base[r] = device pointer (valid in this process) of shard r's rows.
  uint32_t shard_rank = 0, shard_world = 1;
  uint64_t C_local = 0;            // rows of this ctx's own shard (== C when W == 1)
  const float* shard_base[glb::kMaxShards] = {};
  void* shard_ipc[glb::kMaxShards] = {};  // opened with cudaIpcOpenMemHandle (closed on rebuild)
  uint32_t shard_attached = 0;     // bitmask of shards with a base pointer
  uint32_t* counts = nullptr;  // u32[V] PreSC hotness
  uint32_t* access = nullptr;  // u32[V] measured accesses
  int count_mode = GLB_COUNT_NONE;

  // sampler config
  bool sampler_set = false;
  int kind = GLB_KHOP_UNIFORM;
  uint32_t L = 0;
  uint32_t fanouts[GLB_MAX_HOPS] = {};
  uint32_t rw_walks = 4, rw_len = 3, rw_topk = 5;
  glb::SampleBufs sb;            // view of the current sample slot (sbs[cur])
  glb::SampleBufs sbs[2];        // double-buffered sample slots (pipeline depth 2)
  glb::ExtractBufs xb;
  int nslots = 1;                // pipeline depth (glb_set_pipeline)
  int cur = 0;                   // slot of the last sample
  cudaStream_t xstream = nullptr;  // extract stream (pipeline depth 2)
  cudaEvent_t ev_sampled[2] = {nullptr, nullptr};
  cudaEvent_t ev_extracted[2] = {nullptr, nullptr};
  int sample_bps = 8;            // sampler kernels' blocks per SM (GLB_SAMPLE_BPS)
  int gather_bps = 4;            // gather blocks per SM
  int gather_bps_pipe = 2;       // ... on the extract stream at pipeline depth 2: leaves SM
                                 // slots to the sampler running concurrently on the main stream
  unsigned int* work = nullptr;  // device [8]: gather chunk counters (main, extract stream)
  unsigned int* miss_bins = nullptr;  // [2*miss_bins_cap + sums] histogram, offsets, scan sums
  uint32_t miss_bins_cap = 0;
  uint32_t miss_bin_log2 = 21;   // host misses ordered by 2^k-byte bins of the matrix
                                 // (GLB_MISS_BIN_LOG2; 0 = unordered)
  int timing = 0;                // record events around every timing-th extract (0: off)
  uint64_t timing_calls = 0;
  std::vector<cudaEvent_t> tev;  // pairs (start, end) of recorded extracts
  size_t tev_used = 0;

  // training set (D9)
  uint32_t* train = nullptr;
  uint32_t* perm = nullptr;       // current epoch permutation (= perm_b[perm_cur])
  // a1 prefetch: the next epoch's permutation is computed on a low-priority side stream
  // while the current epoch's batches run, so no shuffle sits on the step's critical path
  uint32_t* perm_b[2] = {nullptr, nullptr};
  int perm_b_epoch[2] = {-1, -1};
  int perm_cur = 0;
  bool perm_prefetch = true;      // GLB_PERM_PREFETCH=0 disables
  cudaStream_t sstream = nullptr;
  cudaEvent_t ev_perm[2] = {nullptr, nullptr};
  cudaEvent_t ev_mark = nullptr;
  cudaEvent_t ev_xlast = nullptr;  // glb_extract at depth 2: after the extract stream's work
  uint64_t n_train = 0;
  uint32_t batch_size = 0;
  uint64_t seed = 0;
  bool train_set = false;
  int perm_epoch = -1;

  // last sample
  bool have_sample = false;
  uint32_t last_L = 0;
  uint32_t last_k[GLB_MAX_HOPS] = {};
  int last_kind = 0;
  uint32_t last_n0 = 0;

  glb::DevState* st = nullptr;    // device: current sample (sts[cur])
  glb::DevState* sts[2] = {nullptr, nullptr};
  glb::DevState* h_st = nullptr;  // pinned mirror
  glb::DevState* st_x = nullptr;  // device: generic glb_extract (mark lists, errors)
  unsigned long long* scratch = nullptr;  // device [4] u64 reductions
  // shuffle scratch
  unsigned long long* shuf_keys = nullptr;
  uint32_t* shuf_vals = nullptr;
  glb_extract_stats* pending_stats = nullptr;
  unsigned long long* xcount = nullptr;      // device [3] hits/misses/peer hits of the last extract
  unsigned long long* h_xcount = nullptr;    // pinned mirror

  // a8 factored handoff (handoff.cu)
  glb::HandoffRecv* ho_recv = nullptr;
  glb::HandoffSend* ho_send[glb::kHandoffMaxPeers] = {};

  // radix sort scratch
  void* sort_tmp = nullptr;
  size_t sort_tmp_bytes = 0;
};

namespace glb {

// ---- programmatic dependent launch (sm_90+): a kernel of the hot path is
// launched with programmaticStreamSerialization, so it is staged while its
// predecessor drains; every such kernel starts with pdl_enter(): it allows its
// own successor to be staged, then waits for its predecessor's completion and
// memory before touching any data (no RAW/WAR hazard is possible).
__device__ __forceinline__ void pdl_enter() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  asm volatile("griddepcontrol.wait;" ::: "memory");
}

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl_w(const L2Window& w, void (*kern)(KArgs...), unsigned grid,
                                unsigned block, cudaStream_t s, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  int n = 1;
  if (w.bytes) {
    attr[1].id = cudaLaunchAttributeAccessPolicyWindow;
    attr[1].val.accessPolicyWindow.base_ptr = w.base;
    attr[1].val.accessPolicyWindow.num_bytes = w.bytes;
    attr[1].val.accessPolicyWindow.hitRatio = w.hit_ratio;
    attr[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    attr[1].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    n = 2;
  }
  cfg.attrs = attr;
  cfg.numAttrs = n;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), unsigned grid, unsigned block,
                              cudaStream_t s, Args... args) {
  return launch_pdl_w(L2Window(), kern, grid, block, s, args...);
}

// ---- launchers (defined in the .cu files) ----
cudaError_t launch_validate_graph(glb_ctx* c);
cudaError_t launch_seed_init(glb_ctx* c, const uint32_t* seeds, uint32_t n0, int count_mode);
cudaError_t launch_khop(glb_ctx* c, uint32_t hop, uint32_t k, uint64_t seed, uint32_t epoch,
                        uint32_t batch);
cudaError_t launch_rwalk(glb_ctx* c, uint32_t hop, uint64_t seed, uint32_t epoch, uint32_t batch);
cudaError_t launch_compact(glb_ctx* c, uint32_t hop, uint32_t k, bool weighted, int count_mode);
cudaError_t launch_fixup(glb_ctx* c, uint32_t hop);
cudaError_t launch_table_reset(glb_ctx* c);
cudaError_t launch_mark(glb_ctx* c, const uint32_t* vertices, uint64_t n);
// mark into caller-chosen lists; n_dev (nullable) overrides n with a device count; lidslot
// (nullable) receives slot[vertices[i]] per entry
cudaError_t launch_mark_to(glb_ctx* c, const uint32_t* vertices, uint64_t n, const uint32_t* n_dev,
                           DevState* st, uint2* hit_list, uint2* miss_list, int32_t* lidslot);
void handoff_free(glb_ctx* c);  // handoff.cu: drop the a8 ring / peer mappings
// Gather rows: hits src_hit[list.y] -> out[list.x], misses src_miss[list.y] -> out[list.x];
// fill_src (non-null) replaces miss_list with (r, fill_src[r]) (identity destination).
cudaError_t launch_gather(glb_ctx* c, float* out, const float* src_hit, const float* src_miss,
                          const uint2* hit_list, const uint2* miss_list, const uint32_t* fill_src,
                          const uint32_t* dev_counts /* [nhit, nmiss] on device or null */,
                          uint64_t nhit_host, uint64_t nmiss_host,
                          const int32_t* lidslot = nullptr /* hits in lid order (marks) */,
                          const uint32_t* nl_dev = nullptr /* device n_L for lidslot */);
cudaError_t launch_sort_misses(glb_ctx* c, const uint2* miss, const uint32_t* nmiss_dev,
                               uint2* sorted);
// bins of the miss ordering for a V x D matrix; *scan_sums = scratch words of the device scan
uint32_t miss_bins_needed(const glb_ctx* c, uint64_t V, uint32_t D, uint32_t* scan_sums);
cudaError_t scan_exclusive_u32(glb_ctx* c, const uint32_t* a, uint64_t n, uint32_t* out,
                               uint32_t* sums);
cudaError_t scan_inclusive_u64(glb_ctx* c, const uint32_t* a, uint64_t n, unsigned long long* out);
cudaError_t launch_khop_weighted(glb_ctx* c, uint32_t hop, uint32_t k, uint64_t seed,
                                 uint32_t epoch, uint32_t batch);
cudaError_t launch_shuffle_keys(glb_ctx* c, uint32_t epoch, unsigned long long* keys, uint32_t* vals);
cudaError_t radix_sort_pairs_u64(glb_ctx* c, unsigned long long* keys, uint32_t* vals,
                                 unsigned long long* keys_alt, uint32_t* vals_alt, uint64_t n,
                                 int bits, unsigned long long** keys_out, uint32_t** vals_out);
cudaError_t radix_sort_pairs_u32(glb_ctx* c, uint32_t* keys, uint32_t* vals, uint32_t* keys_alt,
                                 uint32_t* vals_alt, uint64_t n, int bits, uint32_t** keys_out,
                                 uint32_t** vals_out);
cudaError_t launch_permute(glb_ctx* c, const uint32_t* table, const uint32_t* idx, uint64_t n,
                           uint32_t* out);
cudaError_t launch_max_u32(glb_ctx* c, const uint32_t* a, uint64_t n, uint32_t* out_dev);
cudaError_t launch_rank_keys(glb_ctx* c, const uint32_t* hot, uint32_t maxc, uint32_t* keys,
                             uint32_t* vals);
cudaError_t launch_assign_slots(glb_ctx* c, const uint32_t* order, uint64_t C);
// out[j] = order[j*W + r] for j < n (the vertices of shard r of a peer-sharded cache)
cudaError_t launch_shard_rows(glb_ctx* c, const uint32_t* order, uint32_t W, uint32_t r,
                              uint64_t n, uint32_t* out);
cudaError_t launch_vmap_reset(glb_ctx* c);   // gp = ~0, slot = c->slot[v]
cudaError_t launch_policy_hotness(glb_ctx* c, int policy, uint64_t seed, uint32_t* out);
cudaError_t launch_topmark(glb_ctx* c, const uint32_t* order, uint64_t C, uint8_t* flag);
cudaError_t launch_similarity(glb_ctx* c, const uint32_t* fi, const uint32_t* fj,
                              const uint8_t* ti, const uint8_t* tj, unsigned long long* out2);
cudaError_t launch_hit_stats(glb_ctx* c, unsigned long long* out3 /* total,hits,max */);
cudaError_t launch_value_hist(glb_ctx* c, const uint32_t* a, uint64_t n, unsigned long long* bins,
                              uint32_t nbins);

// hostgather.cu: a fraction of the misses gathered by host threads into pinned staging,
// read back sequentially by the GPU (glb_set_host_gather)
cudaError_t hg_configure(glb_ctx* c, uint32_t threads);
cudaError_t hg_reserve(glb_ctx* c);  // size the host part's buffers for the sampler config
void hg_free(glb_ctx* c);
bool hg_active(const glb_ctx* c);
cudaError_t hg_enqueue(glb_ctx* c, float* out, const uint2* miss_sorted, uint32_t** dcnt_out);
cudaError_t hg_join(glb_ctx* c);
cudaError_t hg_sync(glb_ctx* c);
// host rows the misses read: the cold store when there is one, else the caller's matrix
inline const void* miss_rows_host(const glb_ctx* c) { return c->cold_h ? (const void*)c->cold_h : c->h_features; }
inline const float* miss_rows_dev(const glb_ctx* c) { return c->cold_d ? c->cold_d : c->features_mapped; }
cudaError_t launch_cold_rows(glb_ctx* c, const uint32_t* order, uint64_t C);  // cold_row map

inline void count_launch(glb_ctx* c, int n = 1) { c->launches += (uint64_t)n; }

}  // namespace glb
