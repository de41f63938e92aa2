// capi.cu -- the extern "C" boundary (include/glb.h): context, buffers, and
// the host-side sequencing of the hot path.  No host sync inside a sampled
// batch: every size a kernel needs lives in DevState on the device.
#include <cuda_runtime.h>

#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstddef>
#include <cstring>
#include <new>
#include <thread>
#include <vector>

#include "glb_internal.cuh"
#include <nvtx3/nvToolsExt.h>

using namespace glb;

namespace {

thread_local std::string g_create_err;

// NVTX range per API call (SURVEY §5 tracing): a profiler (nsys / ncu --nvtx) sees each
// stage's enqueue -- sample, presample, load_cache, extract -- and the kernels it launched.
// Header-only NVTX v3: no cost when no tool is attached.
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

glb_status set_err(glb_ctx* c, glb_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  if (c) c->err = buf;
  else g_create_err = buf;
  return s;
}

glb_status cuda_fail(glb_ctx* c, cudaError_t e, const char* what) {
  if (c) c->poisoned = true;
  return set_err(c, GLB_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define CK(expr)                                          \
  do {                                                    \
    cudaError_t e_ = (expr);                              \
    if (e_ != cudaSuccess) return cuda_fail(c, e_, #expr); \
  } while (0)

#define ENTER(c)                                                            \
  do {                                                                      \
    if (!(c)) return set_err(nullptr, GLB_EINVAL, "null ctx");              \
    if ((c)->poisoned) return set_err(c, GLB_ECUDA, "ctx poisoned: %s", (c)->err.c_str()); \
    cudaError_t e0_ = cudaSetDevice((c)->device);                           \
    if (e0_ != cudaSuccess) return cuda_fail(c, e0_, "cudaSetDevice");     \
  } while (0)

template <typename T>
void dfree(T*& p) {
  if (p) cudaFree((void*)p);
  p = nullptr;
}

template <typename T>
cudaError_t dalloc(T** p, uint64_t count) {
  *p = nullptr;
  return cudaMalloc((void**)p, sizeof(T) * (count ? count : 1));
}

void free_sample_bufs(glb_ctx* c) {
  for (int s = 0; s < 2; ++s) {
    SampleBufs& b = c->sbs[s];
    dfree(b.seeds); dfree(b.uniq); dfree(b.lidslot); dfree(b.picks); dfree(b.pickw);
    dfree(b.pidx);
    for (int l = 0; l < GLB_MAX_HOPS; ++l) {
      dfree(b.bindptr[l]); dfree(b.bindices[l]); dfree(b.bweights[l]); dfree(b.status[l]);
    }
    dfree(b.hit_list); dfree(b.miss_list); dfree(b.miss_sorted);
    b = SampleBufs();
  }
  c->sb = SampleBufs();
  c->sampler_set = false;
  c->have_sample = false;
}

void use_slot(glb_ctx* c, int s) {
  c->cur = s;
  c->sb = c->sbs[s];
  c->st = c->sts[s];
}

cudaError_t sync_all(glb_ctx* c) {
  cudaError_t e = cudaStreamSynchronize(c->stream);
  if (e == cudaSuccess && c->xstream) e = cudaStreamSynchronize(c->xstream);
  if (e == cudaSuccess && c->sstream) e = cudaStreamSynchronize(c->sstream);
  if (e == cudaSuccess) e = hg_sync(c);
  return e;
}

// Drop the peer-shard mapping (IPC-opened peers are closed); the cache becomes local.
void close_shards(glb_ctx* c) {
  for (int r = 0; r < kMaxShards; ++r) {
    if (c->shard_ipc[r]) cudaIpcCloseMemHandle(c->shard_ipc[r]);
    c->shard_ipc[r] = nullptr;
    c->shard_base[r] = nullptr;
  }
  c->shard_rank = 0;
  c->shard_world = 1;
  c->shard_attached = 0;
  c->C_local = 0;
}

// Drop the cold store (host copy + map); callers synchronise first.
void free_cold(glb_ctx* c) {
  if (c->cold_h) {
    constexpr size_t kPiece = 4ull << 30;  // registered in pieces (build_cold_store)
    for (size_t off = 0; off < c->cold_bytes; off += kPiece)
      cudaHostUnregister(reinterpret_cast<uint8_t*>(c->cold_h) + off);
    (void)cudaGetLastError();
    free(c->cold_h);
  }
  c->cold_bytes = 0;
  c->cold_h = nullptr;
  c->cold_d = nullptr;
  c->cold_rows = 0;
  dfree(c->cold_row);
}

void free_graph(glb_ctx* c) {
  close_shards(c);
  free_cold(c);
  dfree(c->indptr); dfree(c->indices); dfree(c->wprefix); dfree(c->vmap); dfree(c->htab);
  c->hslot = nullptr;
  c->hmask = 0;
  c->hash_mode = false;
  if (c->pin.bytes) {  // release this ctx's persisting-L2 set-aside
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, 0);
    cudaCtxResetPersistingL2Cache();
    (void)cudaGetLastError();
  }
  c->pin = L2Window();
  dfree(c->slot); dfree(c->cache); dfree(c->counts); dfree(c->access);
  if (c->registered && c->h_features) cudaHostUnregister((void*)c->h_features);
  c->registered = false;
  c->h_features = nullptr;
  c->features_mapped = nullptr;
  c->V = c->E = 0;
  c->C = 0;
  c->D = 0;
  c->gen = 0;
  c->have_sample = false;
}

bool shards_ready(const glb_ctx* c) {
  return c->shard_world < 2 || c->shard_attached == (uint32_t)((1ull << c->shard_world) - 1);
}

glb_status check_dev_err(glb_ctx* c, DevState* st) {
  uint32_t err = 0;
  CK(cudaMemcpyAsync(&err, &st->err, sizeof(err), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  if (err) {
    CK(cudaMemsetAsync(&st->err, 0, sizeof(uint32_t), c->stream));
    if (err & kErrDupSeed) return set_err(c, GLB_EINVAL, "duplicate seed in batch");
    if (err & kErrRange) return set_err(c, GLB_EINVAL, "vertex id >= V");
    if (err & kErrBadGraph) return set_err(c, GLB_EINVAL, "invalid CSR");
    if (err & kErrCapacity) return set_err(c, GLB_ENOMEM, "relabel hash table full");
    return set_err(c, GLB_EINVAL, "device error 0x%x", err);
  }
  return GLB_OK;
}

// Stats of at most one extract are pending (one pinned mirror): a second extract that
// asks for stats first completes the earlier one.
glb_status flush_pending_stats(glb_ctx* c) {
  if (!c->pending_stats) return GLB_OK;
  CK(sync_all(c));
  c->pending_stats->hits = c->h_xcount[0];
  c->pending_stats->misses = c->h_xcount[1];
  c->pending_stats = nullptr;
  return GLB_OK;
}

// Enqueue one sampled mini-batch (a2/a2' + a3 + a4, and a5 when counting).
glb_status enqueue_sample(glb_ctx* c, const uint32_t* seeds_dev, uint32_t n0, int kind,
                          const uint32_t* k, uint32_t L, uint64_t seed, uint32_t epoch,
                          uint32_t batch) {
  if (epoch > 0xFFFFu) return set_err(c, GLB_ERANGE, "epoch %u >= 2^16", epoch);
  if (n0 > c->sb.cap_batch) return set_err(c, GLB_ENOMEM, "batch %u > max_batch %u", n0, c->sb.cap_batch);
  if (L > c->sb.L) return set_err(c, GLB_ENOMEM, "num_hops %u > configured %u", L, c->sb.L);
  for (uint32_t l = 0; l < L; ++l)
    if (k[l] > c->sb.k[l]) return set_err(c, GLB_ENOMEM, "fanout %u > configured %u at hop %u", k[l], c->sb.k[l], l);
  if (c->gen >= 0xFFFFFFF0u) {  // generation wrap: clear the relabel table once
    CK(launch_vmap_reset(c));
    CK(launch_table_reset(c));
    c->gen = 0;
  }
  c->gen += 1;
  const int slot = c->nslots == 2 ? c->cur ^ 1 : 0;
  // the extract that last read this slot must finish before it is overwritten
  if (c->nslots == 2) CK(cudaStreamWaitEvent(c->stream, c->ev_extracted[slot], 0));
  use_slot(c, slot);
  // sizes and counters restart; the error bits stay (sticky until a call reports them), so
  // an error of any batch of a presample or pipelined run is not lost
  CK(cudaMemsetAsync(c->st, 0, offsetof(DevState, err), c->stream));
  const int mode = c->count_mode;
  CK(launch_seed_init(c, seeds_dev, n0, mode));
  for (uint32_t l = 0; l < L; ++l) {
    if (kind == GLB_KHOP_UNIFORM) CK(launch_khop(c, l, k[l], seed, epoch, batch));
    else if (kind == GLB_KHOP_WEIGHTED) CK(launch_khop_weighted(c, l, k[l], seed, epoch, batch));
    else CK(launch_rwalk(c, l, seed, epoch, batch));
    CK(launch_compact(c, l, k[l], kind == GLB_RANDOM_WALK, mode));
  }
  if (L) CK(launch_fixup(c, L - 1));  // blocks 0..L-2 were fixed inside the next hop's kernel
  c->have_sample = true;
  c->last_L = L;
  c->last_kind = kind;
  c->last_n0 = n0;
  for (uint32_t l = 0; l < L; ++l) c->last_k[l] = k[l];
  return GLB_OK;
}

// Persisting-L2 set-aside + window over the relabel table (skipped if unsupported).
// Auto (GLB_L2_PIN unset): only when the whole table fits in a third of L2 and in the
// persisting set-aside.  Measured at pipeline depth 2 (profiles/r01_ab_experiments.txt):
// PR's 39 MB dense table pinned keeps the sampler's relabel accesses in L2 while the
// previous batch's gather streams ~850 MB through it, 234 -> 206 us/step; tables that
// need most of the set-aside (PR's 80 MB hash table, UK/TW/PA) starve the gather's L2
// share and run 1.3-2.9x slower, so they are never pinned automatically.
void set_l2_window(glb_ctx* c, void* base, size_t bytes) {
  if (c->pin.bytes) {  // drop an earlier set-aside of this ctx
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, 0);
    cudaCtxResetPersistingL2Cache();
    (void)cudaGetLastError();
  }
  c->pin = L2Window();
  if (c->l2_pin == 0 || !base || !bytes) return;
  int max_persist = 0, max_window = 0, l2 = 0;
  cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, c->device);
  cudaDeviceGetAttribute(&max_window, cudaDevAttrMaxAccessPolicyWindowSize, c->device);
  cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, c->device);
  if (max_persist <= 0 || max_window <= 0) return;
  if (c->l2_pin < 0 && (bytes > (size_t)l2 / 3 || bytes > (size_t)max_persist)) return;
  const size_t setaside = bytes < (size_t)max_persist ? bytes : (size_t)max_persist;
  if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, setaside) != cudaSuccess) {
    (void)cudaGetLastError();
    return;
  }
  c->pin.base = base;
  c->pin.bytes = bytes < (size_t)max_window ? bytes : (size_t)max_window;
  const double r = (double)setaside / (double)c->pin.bytes;
  c->pin.hit_ratio = r > 1.0 ? 1.0f : (float)r;
}

// a1: the permutation of `epoch` into dst, on c->stream (Philox keys + stable radix sort;
// reading Q9/§8(c).2).  Uses the shuffle scratch: callers order it after any other user.
cudaError_t compute_perm(glb_ctx* c, uint32_t epoch, uint32_t* dst) {
  const uint64_t n = c->n_train;
  unsigned long long* kout = nullptr;
  uint32_t* vout = nullptr;
  cudaError_t e = launch_shuffle_keys(c, epoch, c->shuf_keys, c->shuf_vals);
  if (e == cudaSuccess)
    e = radix_sort_pairs_u64(c, c->shuf_keys, c->shuf_vals, c->shuf_keys + n, c->shuf_vals + n, n,
                             64, &kout, &vout);
  if (e == cudaSuccess) e = launch_permute(c, c->train, vout, n, dst);
  return e;
}

// Make `epoch`'s permutation current (prefetched, or computed now on the main stream),
// then prefetch epoch + 1 into the other buffer on the side stream.
glb_status ensure_perm(glb_ctx* c, uint32_t epoch) {
  int& cur = c->perm_cur;
  if (c->perm_b_epoch[cur] != (int)epoch) {
    const int o = cur ^ 1;
    if (c->perm_b_epoch[o] == (int)epoch) {  // prefetched: order the main stream after it
      CK(cudaStreamWaitEvent(c->stream, c->ev_perm[o], 0));
    } else {  // compute now, after any side-stream shuffle (shared scratch)
      CK(cudaStreamWaitEvent(c->stream, c->ev_perm[o], 0));
      CK(cudaStreamWaitEvent(c->stream, c->ev_perm[cur], 0));
      CK(compute_perm(c, epoch, c->perm_b[o]));
      c->perm_b_epoch[o] = (int)epoch;
    }
    cur = o;
    c->perm = c->perm_b[cur];
  }
  c->perm_epoch = (int)epoch;
  const int o = cur ^ 1;
  if (c->perm_prefetch && epoch < 0xFFFFu && c->perm_b_epoch[o] != (int)epoch + 1) {
    // buffer o may still be read by batches enqueued on the main stream: wait for them
    CK(cudaEventRecord(c->ev_mark, c->stream));
    CK(cudaStreamWaitEvent(c->sstream, c->ev_mark, 0));
    cudaStream_t main = c->stream;
    c->stream = c->sstream;
    const cudaError_t e = compute_perm(c, epoch + 1, c->perm_b[o]);
    c->stream = main;
    if (e != cudaSuccess) return cuda_fail(c, e, "prefetch shuffle");
    CK(cudaEventRecord(c->ev_perm[o], c->sstream));
    c->perm_b_epoch[o] = (int)epoch + 1;
  }
  return GLB_OK;
}

}  // namespace

extern "C" {

const char* glb_last_error(const glb_ctx* ctx) {
  return ctx ? ctx->err.c_str() : g_create_err.c_str();
}

uint64_t glb_kernel_launches(const glb_ctx* ctx) { return ctx ? ctx->launches : 0; }

glb_status glb_create(int device, glb_ctx** out) {
  if (!out) return set_err(nullptr, GLB_EINVAL, "null out");
  *out = nullptr;
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess || n == 0) return set_err(nullptr, GLB_ECUDA, "no CUDA device: %s", cudaGetErrorString(e));
  if (device < 0 || device >= n) return set_err(nullptr, GLB_EINVAL, "device %d out of range", device);
  glb_ctx* c = new (std::nothrow) glb_ctx();
  if (!c) return set_err(nullptr, GLB_ENOMEM, "host alloc");
  c->device = device;
  int prio_low = 0, prio_high = 0;
  if ((e = cudaSetDevice(device)) != cudaSuccess ||
      (e = cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device)) != cudaSuccess ||
      (e = cudaStreamCreateWithFlags(&c->own_stream, cudaStreamNonBlocking)) != cudaSuccess ||
      (e = cudaDeviceGetStreamPriorityRange(&prio_low, &prio_high)) != cudaSuccess ||
      // the extract stream (pipeline depth 2) yields SMs to the latency-bound sampler
      (e = cudaStreamCreateWithPriority(&c->xstream, cudaStreamNonBlocking,
                                        getenv("GLB_XSTREAM_HIGH") && atoi(getenv("GLB_XSTREAM_HIGH"))
                                            ? prio_high : prio_low)) != cudaSuccess ||
      (e = cudaStreamCreateWithPriority(&c->sstream, cudaStreamNonBlocking, prio_low)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_perm[0], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_perm[1], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_mark, cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_xlast, cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_sampled[0], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_sampled[1], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_extracted[0], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&c->ev_extracted[1], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaMalloc(&c->sts[0], sizeof(DevState))) != cudaSuccess ||
      (e = cudaMalloc(&c->sts[1], sizeof(DevState))) != cudaSuccess ||
      (e = cudaMalloc(&c->st_x, sizeof(DevState))) != cudaSuccess ||
      (e = cudaMalloc(&c->scratch, 4 * sizeof(unsigned long long))) != cudaSuccess ||
      (e = cudaMalloc(&c->xcount, 3 * sizeof(unsigned long long))) != cudaSuccess ||
      (e = cudaMemset(c->xcount, 0, 3 * sizeof(unsigned long long))) != cudaSuccess ||
      (e = cudaMalloc(&c->work, 8 * sizeof(unsigned int))) != cudaSuccess ||
      (e = cudaMemset(c->work, 0, 8 * sizeof(unsigned int))) != cudaSuccess ||
      (e = cudaMallocHost(&c->h_st, sizeof(DevState))) != cudaSuccess ||
      (e = cudaMallocHost(&c->h_xcount, 3 * sizeof(unsigned long long))) != cudaSuccess ||
      (e = cudaMemset(c->sts[0], 0, sizeof(DevState))) != cudaSuccess ||
      (e = cudaMemset(c->sts[1], 0, sizeof(DevState))) != cudaSuccess ||
      (e = cudaMemset(c->st_x, 0, sizeof(DevState))) != cudaSuccess) {
    glb_status s = set_err(nullptr, GLB_ECUDA, "glb_create: %s", cudaGetErrorString(e));
    glb_destroy(c);
    return s;
  }
  c->stream = c->own_stream;
  c->st = c->sts[0];
  if (const char* g = getenv("GLB_GATHER_BPS")) c->gather_bps = atoi(g) > 0 ? atoi(g) : 4;
  c->gather_bps_pipe = getenv("GLB_GATHER_BPS") ? c->gather_bps : 2;
  if (const char* g = getenv("GLB_GATHER_BPS_PIPE")) c->gather_bps_pipe = atoi(g) > 0 ? atoi(g) : 2;
  if (const char* g = getenv("GLB_L2_PIN")) c->l2_pin = atoi(g) != 0 ? 1 : 0;
  if (const char* g = getenv("GLB_SAMPLE_BPS")) c->sample_bps = atoi(g) > 0 ? atoi(g) : 8;
  if (const char* g = getenv("GLB_CACHE_ALIGN")) c->cache_align = (uint32_t)atoi(g);
  if (const char* g = getenv("GLB_GATHER_ST")) c->gather_st_wb = atoi(g) != 0;
  if (const char* g = getenv("GLB_GATHER_BULK")) c->gather_bulk = atoi(g) != 0;
  if (const char* g = getenv("GLB_MISS_BULK")) c->miss_bulk = atoi(g) != 0;
  if (const char* g = getenv("GLB_GATHER_WARP")) c->gather_warp = atoi(g) != 0;
  if (const char* g = getenv("GLB_GATHER_LIDORDER")) c->gather_lidorder = atoi(g) != 0;
  if (const char* g = getenv("GLB_MISSES_FIRST")) c->misses_first = atoi(g) != 0;
  if (const char* g = getenv("GLB_COLD_STORE")) c->cold_store = atoi(g) != 0;
  if (const char* g = getenv("GLB_MISS_BLOCKS")) c->miss_blocks = atoi(g) > 0 ? (uint32_t)atoi(g) : 0u;
  if (const char* g = getenv("GLB_RELABEL_DEDUP")) {  // 1 warp-level, 2 block smem-staged
    const int m = atoi(g);
    c->relabel_dedup = m >= 0 && m <= 2 ? m : 0;
  }
  if (const char* g = getenv("GLB_HOST_GATHER")) {  // permille of the misses, host-gathered
    const int pm = atoi(g);
    const char* t = getenv("GLB_HOST_GATHER_THREADS");
    if (pm > 0 && pm < 1000 &&
        glb_set_host_gather(c, t ? (uint32_t)atoi(t) : 0u, pm / 1000.0) != GLB_OK) {
      glb_status s = set_err(nullptr, GLB_ECUDA, "glb_create: host gather: %s", c->err.c_str());
      glb_destroy(c);
      return s;
    }
  }
  if (const char* g = getenv("GLB_GATHER_BULK_SMEM")) c->gather_bulk_smem = (uint32_t)atoi(g);
  if (const char* g = getenv("GLB_PERM_PREFETCH")) c->perm_prefetch = atoi(g) != 0;
  if (const char* g = getenv("GLB_MISS_BIN_LOG2")) {
    const int k = atoi(g);
    c->miss_bin_log2 = k >= 0 && k <= 40 ? (uint32_t)k : 21u;
  }
  *out = c;
  return GLB_OK;
}

glb_status glb_destroy(glb_ctx* c) {
  if (!c) return GLB_OK;
  cudaSetDevice(c->device);
  if (c->stream) cudaStreamSynchronize(c->stream);
  if (c->xstream) cudaStreamSynchronize(c->xstream);
  if (c->sstream) cudaStreamSynchronize(c->sstream);
  hg_free(c);
  handoff_free(c);
  free_sample_bufs(c);
  free_graph(c);
  dfree(c->xb.hit_list); dfree(c->xb.miss_list); dfree(c->xb.miss_sorted);
  dfree(c->miss_bins);
  dfree(c->train); dfree(c->perm_b[0]); dfree(c->perm_b[1]); dfree(c->shuf_keys); dfree(c->shuf_vals);
  c->perm = nullptr;
  if (c->ev_perm[0]) cudaEventDestroy(c->ev_perm[0]);
  if (c->ev_perm[1]) cudaEventDestroy(c->ev_perm[1]);
  if (c->ev_mark) cudaEventDestroy(c->ev_mark);
  if (c->ev_xlast) cudaEventDestroy(c->ev_xlast);
  if (c->sstream) cudaStreamDestroy(c->sstream);
  dfree(c->sts[0]); dfree(c->sts[1]); dfree(c->st_x); dfree(c->scratch); dfree(c->xcount);
  dfree(c->work);
  for (int i = 0; i < 2; ++i) {
    if (c->ev_sampled[i]) cudaEventDestroy(c->ev_sampled[i]);
    if (c->ev_extracted[i]) cudaEventDestroy(c->ev_extracted[i]);
  }
  for (cudaEvent_t ev : c->tev) cudaEventDestroy(ev);
  if (c->xstream) cudaStreamDestroy(c->xstream);
  if (c->sort_tmp) cudaFree(c->sort_tmp);
  if (c->h_st) cudaFreeHost(c->h_st);
  if (c->h_xcount) cudaFreeHost(c->h_xcount);
  if (c->own_stream) cudaStreamDestroy(c->own_stream);
  delete c;
  return GLB_OK;
}

glb_status glb_set_stream(glb_ctx* c, void* s) {
  ENTER(c);
  c->stream = (cudaStream_t)s;  // NULL = the legacy default stream
  return GLB_OK;
}

glb_status glb_sync(glb_ctx* c) {
  ENTER(c);
  CK(sync_all(c));
  if (c->pending_stats) {
    c->pending_stats->hits = c->h_xcount[0];
    c->pending_stats->misses = c->h_xcount[1];
    c->pending_stats = nullptr;
  }
  glb_status s = check_dev_err(c, c->st_x);
  if (s != GLB_OK) return s;
  s = check_dev_err(c, c->sts[0]);
  return s != GLB_OK ? s : check_dev_err(c, c->sts[1]);
}

glb_status glb_load_graph(glb_ctx* c, uint64_t V, uint64_t E, const uint64_t* indptr,
                          const uint32_t* indices, const void* features, uint32_t D) {
  NvtxRange nvtx_("glb_load_graph");
  ENTER(c);
  if (V == 0 || V >= 0x80000000ull) return set_err(c, GLB_EINVAL, "V=%llu out of range [1, 2^31)", (unsigned long long)V);
  if (!indptr || (E && !indices)) return set_err(c, GLB_EINVAL, "null CSR");
  if (indptr[0] != 0 || indptr[V] != E) return set_err(c, GLB_EINVAL, "indptr[0]!=0 or indptr[V]!=E");
  if (features && D == 0) return set_err(c, GLB_EINVAL, "feat_dim 0");
  CK(sync_all(c));
  free_graph(c);
  free_sample_bufs(c);
  c->V = V;
  c->E = E;
  CK(dalloc(&c->indptr, V + 1));
  CK(dalloc(&c->indices, E));
  CK(dalloc(&c->slot, V));
  CK(dalloc(&c->counts, V));
  CK(dalloc(&c->access, V));
  CK(cudaMemcpy(c->indptr, indptr, sizeof(uint64_t) * (V + 1), cudaMemcpyHostToDevice));
  if (E) CK(cudaMemcpy(c->indices, indices, sizeof(uint32_t) * E, cudaMemcpyHostToDevice));
  CK(cudaMemsetAsync(c->slot, 0xFF, sizeof(int32_t) * V, c->stream));
  CK(cudaMemsetAsync(c->counts, 0, sizeof(uint32_t) * V, c->stream));
  CK(cudaMemsetAsync(c->access, 0, sizeof(uint32_t) * V, c->stream));
  CK(cudaMemsetAsync(c->st, 0, sizeof(DevState), c->stream));
  CK(launch_validate_graph(c));
  glb_status s = check_dev_err(c, c->st);
  if (s != GLB_OK) {
    free_graph(c);
    return s;
  }
  if (features) {
    const size_t bytes = (size_t)V * D * sizeof(float);
    cudaPointerAttributes pa;
    const bool pinned = cudaPointerGetAttributes(&pa, features) == cudaSuccess &&
                        pa.type == cudaMemoryTypeHost;  // e.g. cudaHostAlloc'ed by the caller
    (void)cudaGetLastError();
    cudaError_t e = pinned ? cudaErrorHostMemoryAlreadyRegistered
                           : cudaHostRegister((void*)features, bytes,
                                              cudaHostRegisterMapped | cudaHostRegisterPortable);
    if (e == cudaErrorHostMemoryAlreadyRegistered) {
      (void)cudaGetLastError();
      c->registered = false;
    } else if (e != cudaSuccess) {
      (void)cudaGetLastError();
      free_graph(c);
      return set_err(c, GLB_ENOMEM, "cudaHostRegister(%zu bytes): %s", bytes, cudaGetErrorString(e));
    } else {
      c->registered = true;
    }
    void* dp = nullptr;
    CK(cudaHostGetDevicePointer(&dp, (void*)features, 0));
    c->h_features = features;
    c->features_mapped = (const float*)dp;
    c->D = D;
    uint32_t sums = 0;
    dfree(c->miss_bins);
    c->miss_bins_cap = miss_bins_needed(c, V, D, &sums);
    CK(dalloc(&c->miss_bins, 2ull * c->miss_bins_cap + sums));
  }
  return GLB_OK;
}

glb_status glb_load_edge_weights(glb_ctx* c, const uint32_t* weights) {
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "edge weights before load_graph");
  if (c->E && !weights) return set_err(c, GLB_EINVAL, "null weights");
  CK(sync_all(c));
  dfree(c->wprefix);
  uint32_t* dw = nullptr;
  CK(dalloc(&dw, c->E));
  CK(dalloc(&c->wprefix, c->E));
  if (c->E) CK(cudaMemcpy(dw, weights, sizeof(uint32_t) * c->E, cudaMemcpyHostToDevice));
  cudaError_t e = scan_inclusive_u64(c, dw, c->E, c->wprefix);
  cudaFree(dw);
  if (e != cudaSuccess) return cuda_fail(c, e, "weight prefix scan");
  return GLB_OK;
}

glb_status glb_set_sampler(glb_ctx* c, int kind, const uint32_t* fanouts, uint32_t L,
                           uint32_t walks, uint32_t len, uint32_t topk, uint32_t max_batch) {
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "set_sampler before load_graph");
  if (L > GLB_MAX_HOPS) return set_err(c, GLB_EINVAL, "num_hops %u > %d", L, GLB_MAX_HOPS);
  uint32_t k[GLB_MAX_HOPS] = {};
  if (kind == GLB_KHOP_WEIGHTED && !c->wprefix)
    return set_err(c, GLB_ESTATE, "weighted sampler before glb_load_edge_weights");
  if (kind == GLB_KHOP_UNIFORM || kind == GLB_KHOP_WEIGHTED) {
    if (L && !fanouts) return set_err(c, GLB_EINVAL, "null fanouts");
    for (uint32_t l = 0; l < L; ++l) {
      if (fanouts[l] == 0 || fanouts[l] > (uint32_t)kMaxFanout)
        return set_err(c, GLB_EINVAL, "fanout %u not in [1,%d]", fanouts[l], kMaxFanout);
      k[l] = fanouts[l];
    }
  } else if (kind == GLB_RANDOM_WALK) {
    if (walks == 0 || walks > 32 || len == 0 || len > (uint32_t)kMaxWalkLen || topk == 0 || topk > 32)
      return set_err(c, GLB_EINVAL, "random walk needs walks in [1,32], len in [1,%d], topk in [1,32]", kMaxWalkLen);
    for (uint32_t l = 0; l < L; ++l) k[l] = topk;
  } else {
    return set_err(c, GLB_EINVAL, "unknown sampler kind %d", kind);
  }
  CK(sync_all(c));
  handoff_free(c);  // the ring is sized from the sampler config
  free_sample_bufs(c);
  SampleBufs b;
  b.cap_batch = max_batch;
  b.L = L;
  b.ub[0] = max_batch < c->V ? max_batch : c->V;
  uint64_t pos = b.ub[0], maxflat = 1;
  for (uint32_t l = 0; l < L; ++l) {
    b.k[l] = k[l];
    const uint64_t flat = b.ub[l] * k[l];
    if (flat >= (1ull << 31)) return set_err(c, GLB_ENOMEM, "hop %u capacity %llu >= 2^31", l, (unsigned long long)flat);
    pos += flat;
    maxflat = flat > maxflat ? flat : maxflat;
    const uint64_t nx = b.ub[l] * (1ull + k[l]);
    b.ub[l + 1] = nx < c->V ? nx : c->V;
  }
  if (pos >= 0xFFFFFFFFull) return set_err(c, GLB_ENOMEM, "relabel positions overflow 2^32");
  const uint64_t un = b.ub[L] > max_batch ? b.ub[L] : max_batch;
  // relabel table: dense (one entry per vertex) unless the vertex count dwarfs the
  // batch's unique-vertex bound -- then an L2-sized open-addressing hash table
  uint64_t H = 1024;
  while (H < un + un / 4 && H < kMaxHashEntries) H <<= 1;
  if (c->relabel_mode == 2 && H < un + un / 4)
    return set_err(c, GLB_ENOMEM, "hash relabel table would need > 2^31 entries");
  if (const char* hc = getenv("GLB_HASH_LOG2")) {  // experiment: explicit capacity
    const int lg = atoi(hc);
    if (lg >= 10 && lg <= 30) H = 1ull << lg;
  }
  // auto = dense: measured equal or faster than the hash table on every config
  // (DESIGN.md §7); hash only when the dense table would not fit comfortably.
  size_t free_b = 0, total_b = 0;
  cudaMemGetInfo(&free_b, &total_b);
  const bool hash = c->relabel_mode == 2 ||
                    (c->relabel_mode == 0 && c->V * sizeof(VEntry) > free_b / 4);
  dfree(c->vmap); dfree(c->htab);
  c->hslot = nullptr;
  c->hmask = 0;
  c->hash_mode = hash;
  if (hash) {
    // one allocation: entries then their cache slots, so one L2 window covers both
    CK(dalloc(&c->htab, H + (H * sizeof(int32_t) + sizeof(VEntry) - 1) / sizeof(VEntry)));
    c->hslot = reinterpret_cast<int32_t*>(c->htab + H);
    c->hmask = (uint32_t)(H - 1);
    CK(launch_table_reset(c));
  } else {
    CK(dalloc(&c->vmap, c->V));
    CK(launch_vmap_reset(c));
  }
  set_l2_window(c, hash ? (void*)c->htab : (void*)c->vmap,
                hash ? H * (sizeof(VEntry) + sizeof(int32_t)) : c->V * sizeof(VEntry));
  for (int s = 1; s >= 0; --s) {  // two slots: pipeline depth 2 double-buffers samples
    SampleBufs& bs = c->sbs[s];
    bs = b;
    CK(dalloc(&bs.seeds, max_batch));
    CK(dalloc(&bs.uniq, un));
    CK(dalloc(&bs.lidslot, un));
    CK(dalloc(&bs.picks, maxflat));
    if (hash) CK(dalloc(&bs.pidx, maxflat));
    if (kind == GLB_RANDOM_WALK) CK(dalloc(&bs.pickw, maxflat));
    for (uint32_t l = 0; l < L; ++l) {
      const uint64_t flat = bs.ub[l] * k[l];
      CK(dalloc(&bs.bindptr[l], bs.ub[l] + 1));
      CK(dalloc(&bs.bindices[l], flat));
      if (kind == GLB_RANDOM_WALK) CK(dalloc(&bs.bweights[l], flat));
      const uint64_t min_tile = (uint64_t)kThreads * kCompactMinItems;
      bs.ntiles[l] = (flat + min_tile - 1) / min_tile;
      CK(dalloc(&bs.status[l], bs.ntiles[l]));
    }
    CK(dalloc(&bs.hit_list, un));
    CK(dalloc(&bs.miss_list, un));
    CK(dalloc(&bs.miss_sorted, un));
  }
  use_slot(c, 0);
  c->kind = kind;
  c->L = L;
  for (uint32_t l = 0; l < L; ++l) c->fanouts[l] = k[l];
  c->rw_walks = walks;
  c->rw_len = len;
  c->rw_topk = topk;
  c->sampler_set = true;
  CK(hg_reserve(c));  // host-assisted staging for the new capacity (no-op when off)
  return GLB_OK;
}

glb_status glb_set_train_set(glb_ctx* c, const uint32_t* train, uint64_t n, uint32_t B,
                             uint64_t seed) {
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "set_train_set before load_graph");
  if (B == 0 || (n && !train) || n >= 0xFFFFFFFFull) return set_err(c, GLB_EINVAL, "bad train set");
  {  // T is a set (L305; reading Q6): ids < V, no duplicates
    std::vector<uint64_t> seen((c->V + 63) / 64, 0);
    for (uint64_t i = 0; i < n; ++i) {
      const uint32_t t = train[i];
      if (t >= c->V) return set_err(c, GLB_EINVAL, "train id %u >= V", t);
      if (seen[t >> 6] >> (t & 63) & 1) return set_err(c, GLB_EINVAL, "duplicate train id %u", t);
      seen[t >> 6] |= 1ull << (t & 63);
    }
  }
  CK(sync_all(c));
  dfree(c->train); dfree(c->perm_b[0]); dfree(c->perm_b[1]); dfree(c->shuf_keys); dfree(c->shuf_vals);
  c->perm = nullptr;
  CK(dalloc(&c->train, n));
  CK(dalloc(&c->perm_b[0], n));
  CK(dalloc(&c->perm_b[1], n));
  c->perm_b_epoch[0] = c->perm_b_epoch[1] = -1;
  c->perm_cur = 0;
  c->perm = c->perm_b[0];
  CK(dalloc(&c->shuf_keys, 2 * n));
  CK(dalloc(&c->shuf_vals, 2 * n));
  if (n) CK(cudaMemcpy(c->train, train, sizeof(uint32_t) * n, cudaMemcpyHostToDevice));
  c->n_train = n;
  c->batch_size = B;
  c->seed = seed;
  c->train_set = true;
  c->perm_epoch = -1;
  return GLB_OK;
}

glb_status glb_num_batches(const glb_ctx* c, uint32_t* out) {
  if (!c || !out) return GLB_EINVAL;
  if (!c->train_set) return GLB_ESTATE;
  *out = (uint32_t)((c->n_train + c->batch_size - 1) / c->batch_size);
  return GLB_OK;
}

glb_status glb_shuffle(glb_ctx* c, uint32_t epoch) {
  ENTER(c);
  if (!c->train_set) return set_err(c, GLB_ESTATE, "shuffle before set_train_set");
  if (epoch > 0xFFFFu) return set_err(c, GLB_ERANGE, "epoch %u >= 2^16", epoch);
  return ensure_perm(c, epoch);
}

glb_status glb_get_permutation(glb_ctx* c, uint32_t* host_out) {
  ENTER(c);
  if (c->perm_epoch < 0) return set_err(c, GLB_ESTATE, "no permutation yet");
  CK(cudaMemcpyAsync(host_out, c->perm, sizeof(uint32_t) * c->n_train, cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  return GLB_OK;
}

glb_status glb_sample_result(glb_ctx* c, glb_blocks* out) {
  ENTER(c);
  if (!c->have_sample) return set_err(c, GLB_ESTATE, "no sample");
  CK(cudaMemcpyAsync(c->h_st, c->st, sizeof(DevState), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  const DevState& h = *c->h_st;
  if (h.err) {
    CK(cudaMemsetAsync(&c->st->err, 0, sizeof(uint32_t), c->stream));
    if (h.err & kErrDupSeed) return set_err(c, GLB_EINVAL, "duplicate seed in batch");
    if (h.err & kErrRange) return set_err(c, GLB_EINVAL, "seed id >= V");
    if (h.err & kErrCapacity) return set_err(c, GLB_ENOMEM, "relabel hash table full");
    return set_err(c, GLB_EINVAL, "device error 0x%x", h.err);
  }
  if (!out) return GLB_OK;
  memset(out, 0, sizeof(*out));
  out->num_hops = c->last_L;
  out->num_seeds = h.n[0];
  out->uniq = c->sb.uniq;
  out->cache_slot = c->sb.lidslot;
  for (uint32_t l = 0; l <= c->last_L; ++l) out->sizes[l] = h.n[l];
  for (uint32_t l = 0; l < c->last_L; ++l) {
    out->nnz[l] = h.nnz[l];
    out->indptr[l] = c->sb.bindptr[l];
    out->indices[l] = c->sb.bindices[l];
    out->weights[l] = c->last_kind == GLB_RANDOM_WALK ? c->sb.bweights[l] : nullptr;
  }
  return GLB_OK;
}

glb_status glb_sample(glb_ctx* c, const uint32_t* seeds, uint32_t n0, const uint32_t* fanouts,
                      uint32_t L, uint64_t seed, uint32_t epoch, uint32_t batch, glb_blocks* out) {
  NvtxRange nvtx_("glb_sample");
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "sample before load_graph");
  if (!c->sampler_set) return set_err(c, GLB_ESTATE, "sample before set_sampler");
  if (n0 && !seeds) return set_err(c, GLB_EINVAL, "null seeds");
  const uint32_t* k = c->fanouts;
  if ((c->kind == GLB_KHOP_UNIFORM || c->kind == GLB_KHOP_WEIGHTED) && fanouts) {
    for (uint32_t l = 0; l < L; ++l)
      if (fanouts[l] == 0) return set_err(c, GLB_EINVAL, "fanout 0");
    k = fanouts;
  } else {
    L = c->L;
  }
  if (n0 > c->sb.cap_batch) return set_err(c, GLB_ENOMEM, "batch %u > max_batch %u", n0, c->sb.cap_batch);
  const uint32_t* sd = seeds;
  cudaPointerAttributes at;
  const bool on_dev = n0 && cudaPointerGetAttributes(&at, seeds) == cudaSuccess &&
                      at.type == cudaMemoryTypeDevice;
  (void)cudaGetLastError();
  if (!on_dev) {
    if (n0) CK(cudaMemcpyAsync(c->sb.seeds, seeds, sizeof(uint32_t) * n0, cudaMemcpyHostToDevice, c->stream));
    sd = c->sb.seeds;
  }
  glb_status s = enqueue_sample(c, sd, n0, c->kind, k, L, seed, epoch, batch);
  if (s != GLB_OK) return s;
  return glb_sample_result(c, out);
}

glb_status glb_sample_async(glb_ctx* c, const uint32_t* seeds, uint32_t n0, uint64_t seed,
                            uint32_t epoch, uint32_t batch) {
  NvtxRange nvtx_("glb_sample_async");
  ENTER(c);
  if (!c->V || !c->sampler_set) return set_err(c, GLB_ESTATE, "sample before load_graph/set_sampler");
  if (n0 && !seeds) return set_err(c, GLB_EINVAL, "null seeds");
  if (n0 > c->sb.cap_batch) return set_err(c, GLB_ENOMEM, "batch %u > max_batch %u", n0, c->sb.cap_batch);
  const uint32_t* sd = seeds;
  cudaPointerAttributes at;
  const bool on_dev = n0 && cudaPointerGetAttributes(&at, seeds) == cudaSuccess &&
                      at.type == cudaMemoryTypeDevice;
  (void)cudaGetLastError();
  if (!on_dev) {  // stream-ordered H2D (asynchronous when the host buffer is pinned)
    if (n0) CK(cudaMemcpyAsync(c->sb.seeds, seeds, sizeof(uint32_t) * n0, cudaMemcpyHostToDevice, c->stream));
    sd = c->sb.seeds;
  }
  return enqueue_sample(c, sd, n0, c->kind, c->fanouts, c->L, seed, epoch, batch);
}

glb_status glb_extract_counts_device_ptr(glb_ctx* c, void** out) {
  ENTER(c);
  if (!out) return set_err(c, GLB_EINVAL, "null out");
  *out = c->xcount;
  return GLB_OK;
}

glb_status glb_sample_batch(glb_ctx* c, uint32_t epoch, uint32_t b) {
  NvtxRange nvtx_("glb_sample_batch");
  ENTER(c);
  if (!c->V || !c->sampler_set || !c->train_set) return set_err(c, GLB_ESTATE, "sample_batch needs graph, sampler, train set");
  const uint64_t nb = (c->n_train + c->batch_size - 1) / c->batch_size;
  if (b >= nb) return set_err(c, GLB_EINVAL, "batch %u >= %llu", b, (unsigned long long)nb);
  if (epoch > 0xFFFFu) return set_err(c, GLB_ERANGE, "epoch %u >= 2^16", epoch);
  glb_status s = ensure_perm(c, epoch);
  if (s != GLB_OK) return s;
  const uint64_t lo = (uint64_t)b * c->batch_size;
  const uint64_t hi = lo + c->batch_size < c->n_train ? lo + c->batch_size : c->n_train;
  return enqueue_sample(c, c->perm + lo, (uint32_t)(hi - lo), c->kind, c->fanouts, c->L, c->seed,
                        epoch, b);
}

glb_status glb_set_count_mode(glb_ctx* c, int mode) {
  ENTER(c);
  if (mode < GLB_COUNT_NONE || mode > GLB_COUNT_ACCESS) return set_err(c, GLB_EINVAL, "bad count mode");
  c->count_mode = mode;
  return GLB_OK;
}

glb_status glb_reset_counts(glb_ctx* c, int which) {
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "no graph");
  uint32_t* p = which == GLB_COUNT_PRESAMPLE ? c->counts : which == GLB_COUNT_ACCESS ? c->access : nullptr;
  if (!p) return set_err(c, GLB_EINVAL, "bad count target");
  CK(cudaMemsetAsync(p, 0, sizeof(uint32_t) * c->V, c->stream));
  return GLB_OK;
}

glb_status glb_presample(glb_ctx* c, uint32_t K, uint32_t rank, uint32_t world) {
  NvtxRange nvtx_("glb_presample");
  ENTER(c);
  if (!c->V || !c->sampler_set || !c->train_set) return set_err(c, GLB_ESTATE, "presample needs graph, sampler, train set");
  if (world == 0 || rank >= world) return set_err(c, GLB_EINVAL, "bad rank/world");
  const int saved = c->count_mode;
  c->count_mode = GLB_COUNT_PRESAMPLE;
  const uint32_t nb = (uint32_t)((c->n_train + c->batch_size - 1) / c->batch_size);
  glb_status s = GLB_OK;
  for (uint32_t e = 0; e < K && s == GLB_OK; ++e)
    for (uint32_t b = rank; b < nb && s == GLB_OK; b += world) s = glb_sample_batch(c, e, b);
  c->count_mode = saved;
  if (s != GLB_OK) return s;
  c->have_sample = false;
  s = check_dev_err(c, c->sts[0]);
  return s != GLB_OK ? s : check_dev_err(c, c->sts[1]);
}

glb_status glb_counts_device_ptr(glb_ctx* c, int which, void** out) {
  ENTER(c);
  if (!out) return set_err(c, GLB_EINVAL, "null out");
  *out = which == GLB_COUNT_PRESAMPLE ? (void*)c->counts : which == GLB_COUNT_ACCESS ? (void*)c->access : nullptr;
  return *out ? GLB_OK : set_err(c, GLB_EINVAL, "bad count target");
}

glb_status glb_get_counts(glb_ctx* c, int which, uint32_t* host_out) {
  void* p = nullptr;
  glb_status s = glb_counts_device_ptr(c, which, &p);
  if (s != GLB_OK) return s;
  CK(cudaMemcpyAsync(host_out, p, sizeof(uint32_t) * c->V, cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  return GLB_OK;
}

// Order all vertices by (hotness desc, gid asc) (reading Q10): a stable LSD radix sort
// of maxc - h over gid order.  tmp: device u32[4V]; returns the order (inside tmp).
static glb_status rank_vertices(glb_ctx* c, const uint32_t* hot, uint32_t* tmp, uint32_t** order_out) {
  const uint64_t V = c->V;
  CK(sync_all(c));  // the radix-sort scratch is shared with the side-stream shuffle prefetch
  uint32_t *k0 = tmp, *v0 = tmp + V, *k1 = tmp + 2 * V, *v1 = tmp + 3 * V;
  uint32_t* dmax = (uint32_t*)c->scratch;
  CK(cudaMemsetAsync(dmax, 0, sizeof(uint32_t), c->stream));
  CK(launch_max_u32(c, hot, V, dmax));
  uint32_t maxc = 0;
  CK(cudaMemcpyAsync(&maxc, dmax, sizeof(uint32_t), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  int bits = 0;
  while (bits < 32 && (maxc >> bits)) ++bits;
  CK(launch_rank_keys(c, hot, maxc, k0, v0));
  uint32_t* ko = nullptr;
  CK(radix_sort_pairs_u32(c, k0, v0, k1, v1, V, bits, &ko, order_out));
  return GLB_OK;
}

// Cold store (glb_set_cold_store): the rows of ranks C..V-1 copied, in rank order, into a
// pinned host buffer the misses read instead of the caller's gid-ordered matrix.  A batch's
// misses then fall in the non-cached part only and the warmer (more often missed) rows sit
// together, so the zero-copy reads touch fewer 2 MB host regions (the host link's cost is
// per region).  Bytes are the same rows, so results are unchanged.
// MemAvailable of /proc/meminfo in bytes (0 if unreadable)
static size_t host_mem_available() {
  FILE* f = fopen("/proc/meminfo", "r");
  if (!f) return 0;
  char line[256];
  size_t kb = 0;
  while (fgets(line, sizeof line, f))
    if (sscanf(line, "MemAvailable: %zu kB", &kb) == 1) break;
  fclose(f);
  return kb << 10;
}

static glb_status build_cold_store(glb_ctx* c, const uint32_t* order, uint64_t C) {
  const uint64_t V = c->V, n = V - C;
  const size_t rb = 4ull * c->D;
  std::vector<uint32_t> ord(n);
  CK(cudaMemcpyAsync(ord.data(), order + C, sizeof(uint32_t) * n, cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  const size_t bytes = n * rb;
  // a second host copy of up to most of the matrix: only when the host can hold it with room
  // to spare (an over-committed copy is not a recoverable failure -- the kernel OOM-kills the
  // process while the rows are copied); otherwise the misses read the caller's matrix
  const size_t avail = host_mem_available();
  if (avail && bytes + (16ull << 30) > avail) {
    fprintf(stderr, "glb: cold store of %zu bytes skipped (%zu bytes of host memory available); "
            "misses read the caller's matrix\n", bytes, avail);
    return GLB_OK;
  }
  uint8_t* h = (uint8_t*)aligned_alloc(1 << 21, (bytes + (1 << 21) - 1) & ~(size_t)((1 << 21) - 1));
  if (!h) return set_err(c, GLB_ENOMEM, "cold store: host alloc of %zu bytes", bytes);
  const uint8_t* src = static_cast<const uint8_t*>(c->h_features);
  unsigned T = std::thread::hardware_concurrency();
  T = T ? T : 1;
  std::vector<std::thread> th;
  for (unsigned t = 0; t < T; ++t)
    th.emplace_back([&, t] {
      const uint64_t a = n * t / T, b = n * (t + 1) / T;
      for (uint64_t i = a; i < b; ++i) memcpy(h + i * rb, src + (size_t)ord[i] * rb, rb);
    });
  for (auto& x : th) x.join();
  // register in 4 GB pieces (one huge registration has failed on a VM host that allows the
  // same total in pieces); with unified addressing every piece maps at its host address, so
  // the pieces form one device range.  Any failure: no cold store (misses read the caller's
  // matrix, as without it) -- a cold store is an optimisation, not a requirement.
  constexpr size_t kPiece = 4ull << 30;
  size_t done = 0;
  bool ok = true;
  for (size_t off = 0; off < bytes && ok; off += kPiece) {
    const size_t len = bytes - off < kPiece ? bytes - off : kPiece;
    void* dp = nullptr;
    ok = cudaHostRegister(h + off, len, cudaHostRegisterMapped | cudaHostRegisterPortable) == cudaSuccess;
    if (ok) {
      done = off + len;
      ok = cudaHostGetDevicePointer(&dp, h + off, 0) == cudaSuccess && dp == (void*)(h + off);
    }
  }
  (void)cudaGetLastError();
  if (!ok) {
    for (size_t off = 0; off < done; off += kPiece) cudaHostUnregister(h + off);
    (void)cudaGetLastError();
    free(h);
    fprintf(stderr, "glb: cold store of %zu bytes could not be pinned; misses read the caller's matrix\n", bytes);
    return GLB_OK;
  }
  c->cold_h = (float*)h;
  c->cold_d = (const float*)h;  // unified addressing: the device address is the host address
  c->cold_rows = n;
  c->cold_bytes = bytes;
  CK(dalloc(&c->cold_row, V));
  CK(cudaMemsetAsync(c->cold_row, 0xFF, sizeof(uint32_t) * V, c->stream));
  CK(launch_cold_rows(c, order, C));
  return GLB_OK;
}

// load_cache (L301) for a cache of C global rows split over `world` shards: the
// vertex of global rank i is cached iff i < C, slot[v] = i; shard i % world holds it
// at row i / world (world == 1: the whole cache is local, row = rank).
static glb_status build_cache_impl(glb_ctx* c, uint64_t C, const uint32_t* hotness, uint32_t rank,
                                   uint32_t world) {
  const uint64_t V = c->V;
  const uint32_t* hot = hotness ? hotness : c->counts;
  CK(sync_all(c));  // an in-flight extract may still read the old cache
  close_shards(c);
  uint32_t* tmp = nullptr;
  CK(dalloc(&tmp, 5 * V));
  uint32_t* order = nullptr;
  glb_status s = rank_vertices(c, hot, tmp, &order);
  if (s != GLB_OK) { cudaFree(tmp); return s; }
  CK(cudaMemsetAsync(c->slot, 0xFF, sizeof(int32_t) * V, c->stream));
  CK(launch_assign_slots(c, order, C));
  CK(launch_vmap_reset(c));  // dense mode: copy the slots into the relabel entries
  free_cold(c);
  if (c->cold_store && world == 1 && c->features_mapped && C < V) {
    glb_status cs = build_cold_store(c, order, C);
    if (cs != GLB_OK) { cudaFree(tmp); return cs; }
  }
  dfree(c->cache);
  c->C = C;
  c->shard_rank = rank;
  c->shard_world = world;
  const uint64_t Cl = C > rank ? (C - rank + world - 1) / world : 0;  // rows i = j*world + rank
  c->C_local = Cl;
  if (c->features_mapped && (Cl || world > 1)) {
    // cache rows: D floats, padded to cache_align bytes when rows are 16-byte vectors
    c->cache_stride = c->D;
    if (c->cache_align >= 16 && c->D % 4 == 0) {
      const uint32_t a = c->cache_align / 4;
      c->cache_stride = (c->D + a - 1) / a * a;
    }
    CK(dalloc(&c->cache, Cl * (uint64_t)c->cache_stride));  // >= 1 element: a shard always has a base
    const uint32_t* rows = order;
    if (world > 1) {
      uint32_t* sub = tmp + 4 * V;
      CK(launch_shard_rows(c, order, world, rank, Cl, sub));
      rows = sub;
    }
    // cache rows come over PCIe from the mapped host matrix (zero copy)
    if (Cl)
      CK(launch_gather(c, c->cache, nullptr, c->features_mapped, nullptr, nullptr, rows, nullptr,
                       0, Cl));
  }
  c->shard_base[rank] = c->cache;
  c->shard_attached = 1u << rank;
  CK(cudaStreamSynchronize(c->stream));
  cudaFree(tmp);
  c->have_sample = false;  // marks of an earlier sample refer to the old cache
  return GLB_OK;
}

glb_status glb_build_cache(glb_ctx* c, double alpha, const uint32_t* hotness) {
  NvtxRange nvtx_("glb_build_cache");
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "build_cache before load_graph");
  if (!(alpha >= 0.0 && alpha <= 1.0)) return set_err(c, GLB_EINVAL, "alpha %g not in [0,1]", alpha);
  uint64_t C = (uint64_t)std::floor(alpha * (double)c->V);
  if (C > c->V) C = c->V;
  return build_cache_impl(c, C, hotness, 0, 1);
}

glb_status glb_build_cache_sharded(glb_ctx* c, double alpha, const uint32_t* hotness,
                                   uint32_t rank, uint32_t world) {
  NvtxRange nvtx_("glb_build_cache_sharded");
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "build_cache before load_graph");
  if (!(alpha >= 0.0 && alpha <= 1.0)) return set_err(c, GLB_EINVAL, "alpha %g not in [0,1]", alpha);
  if (world < 1 || world > (uint32_t)kMaxShards || rank >= world)
    return set_err(c, GLB_EINVAL, "shard rank %u / world %u (world <= %d)", rank, world, kMaxShards);
  uint64_t C = (uint64_t)std::floor(alpha * (double)c->V) * world;
  if (C > c->V) C = c->V;
  if (world > 1 && !c->features_mapped)
    return set_err(c, GLB_ESTATE, "a sharded cache needs a graph with features");
  return build_cache_impl(c, C, hotness, rank, world);
}

glb_status glb_cache_device_ptr(glb_ctx* c, void** out, uint64_t* rows) {
  ENTER(c);
  if (!out) return set_err(c, GLB_EINVAL, "null out");
  *out = c->cache;
  if (rows) *rows = c->C_local;
  return GLB_OK;
}

glb_status glb_cache_ipc_handle(glb_ctx* c, void* handle_out) {
  ENTER(c);
  if (!handle_out) return set_err(c, GLB_EINVAL, "null out");
  if (!c->cache) return set_err(c, GLB_ESTATE, "no cache shard (build_cache_sharded first)");
  static_assert(sizeof(cudaIpcMemHandle_t) == GLB_IPC_HANDLE_BYTES, "IPC handle size");
  cudaIpcMemHandle_t h;
  CK(cudaIpcGetMemHandle(&h, c->cache));
  memcpy(handle_out, &h, sizeof(h));
  return GLB_OK;
}

glb_status glb_attach_peer_cache(glb_ctx* c, uint32_t peer, const void* ipc_handle,
                                 const void* dev_ptr) {
  ENTER(c);
  if (c->shard_world < 2) return set_err(c, GLB_ESTATE, "cache is not sharded");
  if (peer >= c->shard_world || peer == c->shard_rank)
    return set_err(c, GLB_EINVAL, "peer %u (rank %u of %u)", peer, c->shard_rank, c->shard_world);
  if (!ipc_handle == !dev_ptr) return set_err(c, GLB_EINVAL, "pass exactly one of ipc_handle, dev_ptr");
  CK(sync_all(c));  // an in-flight extract may read the old mapping
  if (c->shard_ipc[peer]) {
    cudaIpcCloseMemHandle(c->shard_ipc[peer]);
    c->shard_ipc[peer] = nullptr;
  }
  const void* base = dev_ptr;
  if (ipc_handle) {
    cudaIpcMemHandle_t h;
    memcpy(&h, ipc_handle, sizeof(h));
    void* p = nullptr;
    CK(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
    c->shard_ipc[peer] = p;
    base = p;
  } else {
    cudaPointerAttributes a;
    CK(cudaPointerGetAttributes(&a, dev_ptr));
    if (a.type != cudaMemoryTypeDevice) return set_err(c, GLB_EINVAL, "dev_ptr is not device memory");
    if (a.device != c->device) {  // same process, another GPU: NVLink peer access
      int ok = 0;
      CK(cudaDeviceCanAccessPeer(&ok, c->device, a.device));
      if (!ok) return set_err(c, GLB_EINVAL, "device %d cannot access device %d", c->device, a.device);
      cudaError_t e = cudaDeviceEnablePeerAccess(a.device, 0);
      if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
      else if (e != cudaSuccess) return cuda_fail(c, e, "cudaDeviceEnablePeerAccess");
    }
  }
  c->shard_base[peer] = (const float*)base;
  c->shard_attached |= 1u << peer;
  return GLB_OK;
}

glb_status glb_last_extract_counts(glb_ctx* c, uint64_t* out3) {
  ENTER(c);
  if (!out3) return set_err(c, GLB_EINVAL, "null out");
  CK(sync_all(c));
  unsigned long long h[3];
  CK(cudaMemcpy(h, c->xcount, sizeof(h), cudaMemcpyDeviceToHost));
  out3[0] = h[0];
  out3[1] = h[1];
  out3[2] = c->shard_world > 1 ? h[2] : 0;
  return GLB_OK;
}

glb_status glb_policy_hotness(glb_ctx* c, int policy, uint64_t seed, uint32_t* out) {
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "no graph");
  if (!out) return set_err(c, GLB_EINVAL, "null out");
  if (policy < GLB_POLICY_PRESC || policy > GLB_POLICY_RANDOM) return set_err(c, GLB_EINVAL, "bad policy");
  CK(launch_policy_hotness(c, policy, seed, out));
  return GLB_OK;
}

glb_status glb_footprint_similarity(glb_ctx* c, const uint32_t* fi, const uint32_t* fj,
                                    double top_frac, uint64_t* num, uint64_t* den, double* out) {
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "no graph");
  if (!fi || !fj) return set_err(c, GLB_EINVAL, "null counts");
  if (!(top_frac >= 0.0 && top_frac <= 1.0)) return set_err(c, GLB_EINVAL, "top_frac not in [0,1]");
  const uint64_t V = c->V;
  const uint64_t C = (uint64_t)std::floor(top_frac * (double)V);
  uint32_t* tmp = nullptr;
  uint8_t* flags = nullptr;
  CK(dalloc(&tmp, 4 * V));
  CK(dalloc(&flags, 2 * V));
  CK(cudaMemsetAsync(flags, 0, 2 * V, c->stream));
  for (int x = 0; x < 2; ++x) {
    uint32_t* order = nullptr;
    glb_status s = rank_vertices(c, x == 0 ? fi : fj, tmp, &order);
    if (s != GLB_OK) { cudaFree(tmp); cudaFree(flags); return s; }
    CK(launch_topmark(c, order, C, flags + x * V));
  }
  CK(cudaMemsetAsync(c->scratch, 0, 2 * sizeof(unsigned long long), c->stream));
  CK(launch_similarity(c, fi, fj, flags, flags + V, c->scratch));
  unsigned long long h2[2];
  CK(cudaMemcpyAsync(h2, c->scratch, sizeof(h2), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  cudaFree(tmp);
  cudaFree(flags);
  if (num) *num = h2[0];
  if (den) *den = h2[1];
  if (out) *out = h2[1] ? (double)h2[0] / (double)h2[1] : 0.0;
  return GLB_OK;
}

glb_status glb_get_cache_slots(glb_ctx* c, int32_t* host_out) {
  ENTER(c);
  if (!c->V) return set_err(c, GLB_ESTATE, "no graph");
  CK(cudaMemcpyAsync(host_out, c->slot, sizeof(int32_t) * c->V, cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  return GLB_OK;
}

glb_status glb_cache_size(const glb_ctx* c, uint64_t* out) {
  if (!c || !out) return GLB_EINVAL;
  *out = c->C;
  return GLB_OK;
}

glb_status glb_hit_stats_get(glb_ctx* c, glb_hit_stats* out) {
  ENTER(c);
  if (!c->V || !out) return set_err(c, GLB_ESTATE, "no graph");
  unsigned long long h3[3];
  CK(cudaMemsetAsync(c->scratch, 0, 3 * sizeof(unsigned long long), c->stream));
  CK(launch_hit_stats(c, c->scratch));
  CK(cudaMemcpyAsync(h3, c->scratch, sizeof(h3), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  out->total = h3[0];
  out->hits = h3[1];
  out->cache_rows = c->C;
  const uint32_t mx = (uint32_t)h3[2];
  unsigned long long* bins = nullptr;
  CK(dalloc(&bins, (uint64_t)mx + 1));
  CK(cudaMemsetAsync(bins, 0, sizeof(unsigned long long) * ((uint64_t)mx + 1), c->stream));
  CK(launch_value_hist(c, c->access, c->V, bins, mx + 1));
  unsigned long long* hb = new (std::nothrow) unsigned long long[(uint64_t)mx + 1];
  if (!hb) { cudaFree(bins); return set_err(c, GLB_ENOMEM, "host alloc"); }
  CK(cudaMemcpyAsync(hb, bins, sizeof(unsigned long long) * ((uint64_t)mx + 1), cudaMemcpyDeviceToHost, c->stream));
  CK(cudaStreamSynchronize(c->stream));
  cudaFree(bins);
  // Optimal policy: the C largest access counts (L148 fn4)
  uint64_t left = c->C, opt = 0;
  for (uint64_t x = mx; x >= 1 && left; --x) {
    const uint64_t take = hb[x] < left ? hb[x] : left;
    opt += take * x;
    left -= take;
  }
  delete[] hb;
  out->optimal_hits = opt;
  return GLB_OK;
}

glb_status glb_extract(glb_ctx* c, const uint32_t* vertices, uint64_t n, void* out,
                       glb_extract_stats* stats) {
  NvtxRange nvtx_("glb_extract");
  ENTER(c);
  if (!c->V || !c->features_mapped) return set_err(c, GLB_ESTATE, "extract needs a graph with features");
  if (!shards_ready(c)) return set_err(c, GLB_ESTATE, "peer cache shards not all attached");
  if (n && (!vertices || !out)) return set_err(c, GLB_EINVAL, "null pointer");
  if (n >= 0xFFFFFFFFull) return set_err(c, GLB_EINVAL, "n too large");
  if (n > c->xb.cap) {
    CK(cudaStreamSynchronize(c->stream));
    dfree(c->xb.hit_list); dfree(c->xb.miss_list); dfree(c->xb.miss_sorted);
    c->xb.cap = 0;
    CK(dalloc(&c->xb.hit_list, n));
    CK(dalloc(&c->xb.miss_list, n));
    CK(dalloc(&c->xb.miss_sorted, n));
    c->xb.cap = n;
  }
  if (stats) {
    glb_status ps = flush_pending_stats(c);
    if (ps != GLB_OK) return ps;
  }
  if (c->nslots == 2) {  // the extract stream's gathers share the miss-sort scratch and the
    // extract counters with this one: order after them (glb.h, pipeline depth 2)
    CK(cudaEventRecord(c->ev_xlast, c->xstream));
    CK(cudaStreamWaitEvent(c->stream, c->ev_xlast, 0));
  }
  CK(cudaMemsetAsync(&c->st_x->nhit, 0, 2 * sizeof(uint32_t), c->stream));
  if (n) CK(launch_mark(c, vertices, n));
  const uint2* misses = c->xb.miss_list;
  if (n && c->C < c->V && (c->miss_bin_log2 || c->cold_row)) {  // rows may come over PCIe: order them by address
    CK(launch_sort_misses(c, c->xb.miss_list, &c->st_x->nmiss, c->xb.miss_sorted));
    misses = c->xb.miss_sorted;
  }
  CK(launch_gather(c, (float*)out, c->cache, miss_rows_dev(c), c->xb.hit_list, misses,
                   nullptr, &c->st_x->nhit, 0, 0));
  if (stats) {
    CK(cudaMemcpyAsync(c->h_xcount, c->xcount, 3 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, c->stream));
    c->pending_stats = stats;
  }
  return GLB_OK;
}

glb_status glb_extract_sample(glb_ctx* c, void* out, glb_extract_stats* stats) {
  NvtxRange nvtx_("glb_extract_sample");
  ENTER(c);
  if (!c->have_sample) return set_err(c, GLB_ESTATE, "extract_sample without a current sample");
  if (!c->features_mapped) return set_err(c, GLB_ESTATE, "graph loaded without features");
  if (!shards_ready(c)) return set_err(c, GLB_ESTATE, "peer cache shards not all attached");
  if (!out) return set_err(c, GLB_EINVAL, "null out");
  if (stats) {
    glb_status ps = flush_pending_stats(c);
    if (ps != GLB_OK) return ps;
  }
  cudaStream_t main = c->stream;
  const int slot = c->cur;
  if (c->nslots == 2) {  // extract on its own stream, overlapping the next sample;
    // it is ordered after everything enqueued on the main stream so far (the sample it
    // reads and any caller work, e.g. allocating `out`)
    CK(cudaEventRecord(c->ev_sampled[slot], main));
    CK(cudaStreamWaitEvent(c->xstream, c->ev_sampled[slot], 0));
    c->stream = c->xstream;
  }
  cudaEvent_t t0 = nullptr, t1 = nullptr;
  if (c->timing && (c->timing_calls++ % (uint64_t)c->timing) == 0) {
    if (c->tev_used + 2 > c->tev.size()) {
      for (int i = 0; i < 2; ++i) {
        cudaEvent_t ev;
        cudaError_t e = cudaEventCreate(&ev);
        if (e != cudaSuccess) { c->stream = main; return cuda_fail(c, e, "cudaEventCreate"); }
        c->tev.push_back(ev);
      }
    }
    t0 = c->tev[c->tev_used];
    t1 = c->tev[c->tev_used + 1];
    c->tev_used += 2;
    cudaEventRecord(t0, c->stream);
  }
  const uint2* misses = c->sb.miss_list;
  cudaError_t e = cudaSuccess;
  if (c->C < c->V && (c->miss_bin_log2 || c->cold_row)) {  // rows may come over PCIe: order them by address
    e = launch_sort_misses(c, c->sb.miss_list, &c->st->nmiss, c->sb.miss_sorted);
    misses = c->sb.miss_sorted;
  }
  // host-assisted misses: the tail of the ordered list is gathered by host threads
  const bool hg = hg_active(c);
  uint32_t* dcnt = nullptr;
  if (e == cudaSuccess && hg) e = hg_enqueue(c, (float*)out, misses, &dcnt);
  c->hg_inflight = hg && dcnt;
  if (e == cudaSuccess)
    e = launch_gather(c, (float*)out, c->cache, miss_rows_dev(c), c->sb.hit_list, misses,
                      nullptr, dcnt ? dcnt : &c->st->nhit, 0, 0,
                      c->gather_lidorder && !c->gather_warp ? c->sb.lidslot : nullptr,
                      &c->st->n[c->last_L]);
  c->hg_inflight = false;
  if (e == cudaSuccess && hg) e = hg_join(c);
  if (e == cudaSuccess && t1) e = cudaEventRecord(t1, c->stream);
  if (e == cudaSuccess && stats) {
    e = cudaMemcpyAsync(c->h_xcount, c->xcount, 3 * sizeof(unsigned long long),
                        cudaMemcpyDeviceToHost, c->stream);
    c->pending_stats = stats;
  }
  if (e == cudaSuccess && c->nslots == 2) e = cudaEventRecord(c->ev_extracted[slot], c->stream);
  c->stream = main;
  if (e != cudaSuccess) return cuda_fail(c, e, "extract_sample");
  return GLB_OK;
}

glb_status glb_set_relabel_mode(glb_ctx* c, int mode) {
  ENTER(c);
  if (mode < 0 || mode > 2) return set_err(c, GLB_EINVAL, "relabel mode must be 0 (auto), 1 (dense) or 2 (hash)");
  c->relabel_mode = mode;
  return GLB_OK;
}

glb_status glb_relabel_l2_window(const glb_ctx* c, uint64_t* out) {
  if (!c || !out) return GLB_EINVAL;
  *out = c->pin.bytes;
  return GLB_OK;
}

glb_status glb_relabel_mode(const glb_ctx* c, int* out) {
  if (!c || !out) return GLB_EINVAL;
  *out = c->hash_mode ? 2 : 1;
  return GLB_OK;
}

glb_status glb_set_pipeline(glb_ctx* c, int depth) {
  ENTER(c);
  if (depth != 1 && depth != 2) return set_err(c, GLB_EINVAL, "pipeline depth must be 1 or 2");
  CK(sync_all(c));
  c->nslots = depth;
  return GLB_OK;
}

glb_status glb_extract_stream(glb_ctx* c, void** out) {
  ENTER(c);
  if (!out) return set_err(c, GLB_EINVAL, "null out");
  *out = c->nslots == 2 ? (void*)c->xstream : (void*)c->stream;
  return GLB_OK;
}

glb_status glb_set_timing(glb_ctx* c, int enable /* period */) {
  ENTER(c);
  CK(sync_all(c));
  if (enable < 0) return set_err(c, GLB_EINVAL, "timing period < 0");
  c->timing = enable;
  c->timing_calls = 0;
  c->tev_used = 0;
  return GLB_OK;
}

glb_status glb_set_host_gather(glb_ctx* c, uint32_t threads, double fraction) {
  ENTER(c);
  if (!(fraction >= 0.0 && fraction < 1.0)) return set_err(c, GLB_EINVAL, "fraction %g not in [0,1)", fraction);
  if (threads > 256) return set_err(c, GLB_EINVAL, "threads %u > 256", threads);
  CK(sync_all(c));
  const uint32_t pm = (uint32_t)std::lround(fraction * 1000.0);
  if (pm == 0) {
    hg_free(c);
    c->hg_permille = 0;
    c->hg_threads = 0;
    return GLB_OK;
  }
  if (threads == 0) {  // auto: the usable cores minus two (the caller's thread, the driver's)
    const unsigned n = std::thread::hardware_concurrency();
    threads = n > 3 ? n - 2 : 1;
  }
  CK(hg_configure(c, threads - 1));  // the host-function thread itself is the last worker
  c->hg_permille = pm;
  c->hg_threads = threads;
  CK(hg_reserve(c));  // pinned staging now, not in the first extract
  return GLB_OK;
}

glb_status glb_set_cold_store(glb_ctx* c, int enable) {
  ENTER(c);
  c->cold_store = enable != 0;
  if (!c->cold_store) {
    CK(sync_all(c));
    free_cold(c);
  }
  return GLB_OK;
}

glb_status glb_cold_store_rows(const glb_ctx* c, uint64_t* rows) {
  if (!c || !rows) return GLB_EINVAL;
  *rows = c->cold_rows;
  return GLB_OK;
}

glb_status glb_host_gather(const glb_ctx* c, uint32_t* threads, double* fraction) {
  if (!c) return GLB_EINVAL;
  if (threads) *threads = c->hg_threads;
  if (fraction) *fraction = c->hg_permille / 1000.0;
  return GLB_OK;
}

glb_status glb_extract_times(glb_ctx* c, float* out_ms, uint64_t max, uint64_t* n) {
  ENTER(c);
  CK(sync_all(c));
  const uint64_t have = c->tev_used / 2;
  if (n) *n = have;
  for (uint64_t i = 0; i < have && i < max; ++i)
    CK(cudaEventElapsedTime(out_ms + i, c->tev[2 * i], c->tev[2 * i + 1]));
  c->tev_used = 0;
  return GLB_OK;
}

}  // extern "C"
