// hostgather.cu -- a7 misses, host-assisted ("the Trainer will
// simultaneously extract their features from host memory and the feature cache
// in GPU memory"; L79: Extract is bound by "the limited PCIe bandwidth").
//
// Zero-copy reads of 512-byte host rows scattered over a 57 GB matrix are bound by
// per-row address translation on the host link (measured, profiles/r02_hostlink.txt:
// ~41 GB/s at best for random rows over 60 GB, 51 GB/s for 1 KB rows or a 14 GB span,
// 55.6 GB/s for a DMA), not by the link's bandwidth: a second, translation-cheap
// stream over the same link adds up (zero-copy random rows + a contiguous copy:
// 53 GB/s together).  So a fraction f of a batch's (address-ordered) misses -- the
// tail of the ordered list -- is gathered by host threads into a contiguous pinned
// staging buffer, which crosses the link as a DMA (copy engine, one translation per
// page; or, GLB_HOST_GATHER_DMA=0, read sequentially by the scatter kernel itself)
// and is scattered to the output rows, while the extract kernel reads the other
// misses directly.  Every step is enqueued asynchronously: the host part runs in
// stream host functions (cudaLaunchHostFunc: pure memcpy on a thread pool, no CUDA
// calls) ordered between a device->host copy of the part's work list and the copies
// and scatter kernels, on two side streams that the extract stream joins before it
// completes.  The host part's row count is chosen on the host (f x the miss count of
// a recent batch, so every copy has a size known at enqueue time) and clipped on the
// device to the batch's real miss count.  Bytes are moved, never computed: the result
// is identical for every f.
#include <cuda_runtime.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <condition_variable>
#include <cstring>
#include <functional>
#include <mutex>
#include <thread>
#include <vector>

#include "glb_internal.cuh"

namespace glb {

namespace {

constexpr int kMaxChunks = 16;       // host-function / scatter pairs per extract (max)
constexpr uint32_t kTaskRows = 256;  // rows per pool task
constexpr int kSlots = 2;            // sample slots (pipeline depth 2)

// A fixed pool of host threads running a parallel-for; the calling thread helps.
class HostPool {
 public:
  explicit HostPool(int n) {
    for (int i = 0; i < n; ++i) th_.emplace_back([this] { loop(); });
  }
  ~HostPool() {
    {
      std::lock_guard<std::mutex> l(m_);
      stop_ = true;
    }
    cv_.notify_all();
    for (auto& t : th_) t.join();
  }
  int size() const { return (int)th_.size(); }
  void run(uint32_t n, const std::function<void(uint32_t)>& f) {
    std::lock_guard<std::mutex> one(run_m_);  // host functions of two streams: one at a time
    {
      std::lock_guard<std::mutex> l(m_);
      fn_ = &f;
      ntasks_ = n;
      next_.store(0);
      active_ = (int)th_.size();
      ++gen_;
    }
    cv_.notify_all();
    work();
    std::unique_lock<std::mutex> l(m_);
    done_.wait(l, [&] { return active_ == 0; });
    fn_ = nullptr;
  }

 private:
  void work() {
    for (;;) {
      const uint32_t t = next_.fetch_add(1);
      if (t >= ntasks_) break;
      (*fn_)(t);
    }
  }
  void loop() {
    uint64_t seen = 0;
    for (;;) {
      {
        std::unique_lock<std::mutex> l(m_);
        cv_.wait(l, [&] { return stop_ || gen_ != seen; });
        if (stop_) return;
        seen = gen_;
      }
      work();
      {
        std::lock_guard<std::mutex> l(m_);
        if (--active_ == 0) done_.notify_all();
      }
    }
  }
  std::vector<std::thread> th_;
  std::mutex m_, run_m_;
  std::condition_variable cv_, done_;
  const std::function<void(uint32_t)>* fn_ = nullptr;
  uint32_t ntasks_ = 0;
  std::atomic<uint32_t> next_{0};
  int active_ = 0;
  uint64_t gen_ = 0;
  bool stop_ = false;
};

struct HgJob {
  glb_ctx* c;
  int slot, k;
  int nch;          // chunks of this extract's host part
  uint64_t target;  // rows of the host part chosen at enqueue (the device clips to n_cpu)
  std::atomic<int> done{1};  // the host function ran (the ring entry may be reused)
};
constexpr int kJobRing = 64 * kMaxChunks;  // host functions the caller may enqueue ahead

// chunk k of nch of the host part: rows [target*k/nch, target*(k+1)/nch) clipped to n_cpu
inline uint64_t chunk_lo(uint64_t target, int k, int nch) { return target * (uint64_t)k / nch; }

// [0] nh, [1] n_zc (misses the extract kernel reads), [2] n_cpu (host part), [3] nm
__global__ void k_hg_split(const DevState* __restrict__ st, uint32_t target,
                           const uint2* __restrict__ miss_sorted, uint32_t* __restrict__ dcnt,
                           uint2* __restrict__ ent) {
  const uint32_t nm = st->nmiss;
  const uint32_t ncpu = nm < target ? nm : target;
  const uint32_t nzc = nm - ncpu;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    dcnt[0] = st->nhit;
    dcnt[1] = nzc;
    dcnt[2] = ncpu;
    dcnt[3] = nm;
  }
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < ncpu; i += gridDim.x * blockDim.x)
    ent[i] = miss_sorted[nzc + i];  // the host part: the tail of the address-ordered list
}

// rows of chunk k: out[ent[i].x, :] = stage[i, :] (stage: the DMA'd device copy, or the
// pinned buffer itself read sequentially over the link)
template <typename T>
__global__ void __launch_bounds__(kThreads)
    k_hg_scatter(T* __restrict__ out, const T* __restrict__ stage, const uint2* __restrict__ ent,
                 const uint32_t* __restrict__ dcnt, uint64_t lo, uint64_t hi, uint32_t U,
                 uint32_t So) {
  const uint64_t ncpu = dcnt[2];
  if (hi > ncpu) hi = ncpu;
  if (hi <= lo) return;
  const uint64_t total = (hi - lo) * U;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  constexpr int kIn = 4;
  for (uint64_t v0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v0 < total; v0 += stride * kIn) {
    T x[kIn];
    uint64_t d[kIn];
#pragma unroll
    for (int q = 0; q < kIn; ++q) {
      const uint64_t v = v0 + q * stride;
      if (v < total) {
        const uint64_t r = lo + v / U, col = v % U;
        x[q] = __ldcs(stage + r * U + col);
        d[q] = (uint64_t)__ldg(&ent[r].x) * So + col;
      }
    }
#pragma unroll
    for (int q = 0; q < kIn; ++q) {
      const uint64_t v = v0 + q * stride;
      if (v < total) __stcs(out + d[q], x[q]);
    }
  }
}

__global__ void k_hg_fix(const uint32_t* __restrict__ dcnt, unsigned long long* xcount) {
  xcount[1] = dcnt[3];  // the extract kernel counted only its own misses
}

}  // namespace

struct HostGather {
  HostPool* pool = nullptr;
  cudaStream_t cs[2] = {nullptr, nullptr};
  cudaEvent_t ev_split = nullptr, ev_d2h = nullptr, ev_end[2] = {nullptr, nullptr};
  cudaEvent_t ev_chunk[kMaxChunks] = {};  // host function k done (its staged rows are ready)
  bool dma = false;  // staged rows cross the link by DMA (GLB_HOST_GATHER_DMA=1; measured slower)
  int nch = 4;       // chunks per extract (GLB_HOST_GATHER_CHUNKS)
  int sblocks = 0;   // scatter grid (GLB_HOST_GATHER_SCATTER_BLOCKS; 0 = one per SM)
  uint64_t cap = 0;  // rows of the host part per slot
  uint32_t D = 0;
  double nm_est = 0;                 // misses per batch (recent batches)
  uint32_t* dcnt[kSlots] = {};       // device [4]
  uint2* ent_dev[kSlots] = {};       // device [cap]
  uint8_t* dstage[kSlots] = {};      // device [cap][4D] (DMA target)
  uint32_t* cnt[kSlots] = {};        // pinned [4]
  uint2* ent[kSlots] = {};           // pinned [cap]
  uint8_t* stage[kSlots] = {};       // pinned, mapped [cap][4D]
  uint8_t* stage_dev[kSlots] = {};   // device alias of stage
  HgJob job[kJobRing];
  uint64_t njobs = 0;
  // GLB_HG_STATS=1: host-function wall time, printed by hg_free (A/B instrumentation)
  bool stats = false;
  std::atomic<uint64_t> st_ns{0}, st_rows{0}, st_calls{0};
};

namespace {

void hg_free_bufs(HostGather* h) {
  for (int s = 0; s < kSlots; ++s) {
    if (h->dcnt[s]) cudaFree(h->dcnt[s]);
    if (h->ent_dev[s]) cudaFree(h->ent_dev[s]);
    if (h->dstage[s]) cudaFree(h->dstage[s]);
    if (h->cnt[s]) cudaFreeHost(h->cnt[s]);
    if (h->ent[s]) cudaFreeHost(h->ent[s]);
    if (h->stage[s]) cudaFreeHost(h->stage[s]);
    h->dcnt[s] = nullptr;
    h->ent_dev[s] = nullptr;
    h->dstage[s] = nullptr;
    h->cnt[s] = nullptr;
    h->ent[s] = nullptr;
    h->stage[s] = nullptr;
    h->stage_dev[s] = nullptr;
  }
  h->cap = 0;
  h->D = 0;
}

void hg_gather(const HgJob* j);

void CUDART_CB hg_host_fn(void* p) {
  HgJob* j = static_cast<HgJob*>(p);
  HostGather* h = j->c->hg;
  const auto t0 = std::chrono::steady_clock::now();
  hg_gather(j);
  if (h->stats) {
    h->st_ns += (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
                    std::chrono::steady_clock::now() - t0).count();
    h->st_calls += 1;
  }
  j->done.store(1, std::memory_order_release);
}

void hg_gather(const HgJob* j) {
  glb_ctx* c = j->c;
  HostGather* h = c->hg;
  const uint64_t ncpu = h->cnt[j->slot][2];
  const uint64_t lo = chunk_lo(j->target, j->k, j->nch);
  uint64_t hi = chunk_lo(j->target, j->k + 1, j->nch);
  if (hi > ncpu) hi = ncpu;
  if (hi <= lo) return;
  const size_t rb = 4ull * c->D;
  const uint8_t* feats = static_cast<const uint8_t*>(miss_rows_host(c));
  uint8_t* stage = h->stage[j->slot];
  const uint2* ent = h->ent[j->slot];
  const uint32_t ntask = (uint32_t)((hi - lo + kTaskRows - 1) / kTaskRows);
  if (h->stats) h->st_rows += hi - lo;
  std::function<void(uint32_t)> fn = [&](uint32_t t) {
    const uint64_t a = lo + (uint64_t)t * kTaskRows;
    const uint64_t b = a + kTaskRows < hi ? a + kTaskRows : hi;
    constexpr uint64_t kAhead = 8;  // rows prefetched ahead (random rows: no HW prefetch)
    for (uint64_t i = a; i < a + kAhead && i < b; ++i)
      for (size_t o = 0; o < rb; o += 64) __builtin_prefetch(feats + (size_t)ent[i].y * rb + o);
    for (uint64_t i = a; i < b; ++i) {
      if (i + kAhead < b)
        for (size_t o = 0; o < rb; o += 64)
          __builtin_prefetch(feats + (size_t)ent[i + kAhead].y * rb + o);
      memcpy(stage + i * rb, feats + (size_t)ent[i].y * rb, rb);
    }
  };
  h->pool->run(ntask, fn);
}

}  // namespace

void hg_free(glb_ctx* c) {
  HostGather* h = c->hg;
  if (!h) return;
  for (int i = 0; i < 2; ++i)
    if (h->cs[i]) cudaStreamSynchronize(h->cs[i]);
  if (h->stats && h->st_calls)
    fprintf(stderr, "glb host gather: %llu host functions, %.3f ms total, %.1f us mean, "
            "%llu rows, %.2f GB/s while gathering\n",
            (unsigned long long)h->st_calls.load(), h->st_ns.load() / 1e6,
            h->st_ns.load() / 1e3 / h->st_calls.load(), (unsigned long long)h->st_rows.load(),
            h->st_rows.load() * 4.0 * c->D / (h->st_ns.load() ? h->st_ns.load() : 1));
  delete h->pool;
  hg_free_bufs(h);
  for (int i = 0; i < 2; ++i) {
    if (h->cs[i]) cudaStreamDestroy(h->cs[i]);
    if (h->ev_end[i]) cudaEventDestroy(h->ev_end[i]);
  }
  if (h->ev_split) cudaEventDestroy(h->ev_split);
  if (h->ev_d2h) cudaEventDestroy(h->ev_d2h);
  for (int k = 0; k < kMaxChunks; ++k)
    if (h->ev_chunk[k]) cudaEventDestroy(h->ev_chunk[k]);
  delete h;
  c->hg = nullptr;
}

cudaError_t hg_configure(glb_ctx* c, uint32_t threads) {
  HostGather* h = c->hg;
  cudaError_t e = cudaSuccess;
  if (!h) {
    h = new (std::nothrow) HostGather();
    if (!h) return cudaErrorMemoryAllocation;
    c->hg = h;
    if (const char* g = getenv("GLB_HOST_GATHER_DMA")) h->dma = atoi(g) != 0;
    if (const char* g = getenv("GLB_HG_STATS")) h->stats = atoi(g) != 0;
    if (const char* g = getenv("GLB_HOST_GATHER_SCATTER_BLOCKS")) h->sblocks = atoi(g) > 0 ? atoi(g) : 0;
    if (const char* g = getenv("GLB_HOST_GATHER_CHUNKS")) {
      const int n = atoi(g);
      h->nch = n < 1 ? 1 : n > kMaxChunks ? kMaxChunks : n;
    }
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    for (int i = 0; i < 2 && e == cudaSuccess; ++i) {
      e = cudaStreamCreateWithPriority(&h->cs[i], cudaStreamNonBlocking,
                                       getenv("GLB_XSTREAM_HIGH") && atoi(getenv("GLB_XSTREAM_HIGH"))
                                           ? hi : lo);
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->ev_end[i], cudaEventDisableTiming);
    }
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->ev_split, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->ev_d2h, cudaEventDisableTiming);
    for (int k = 0; k < kMaxChunks && e == cudaSuccess; ++k)
      e = cudaEventCreateWithFlags(&h->ev_chunk[k], cudaEventDisableTiming);
    if (e != cudaSuccess) return e;
  }
  if (!h->pool || h->pool->size() != (int)threads) {
    for (int i = 0; i < 2; ++i) cudaStreamSynchronize(h->cs[i]);
    delete h->pool;
    h->pool = new (std::nothrow) HostPool((int)threads);
    if (!h->pool) return cudaErrorMemoryAllocation;
  }
  h->nm_est = 0;
  return e;
}

cudaError_t hg_sync(glb_ctx* c) {
  if (!c->hg) return cudaSuccess;
  for (int i = 0; i < 2; ++i) {
    cudaError_t e = c->hg->cs[i] ? cudaStreamSynchronize(c->hg->cs[i]) : cudaSuccess;
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

bool hg_active(const glb_ctx* c) {
  return c->hg && c->hg->pool && c->hg_permille > 0 && c->h_features && c->C < c->V &&
         c->st == c->sts[c->cur];  // a sample of this ctx (not a handoff ring slot)
}

// Size the host part's buffers (pinned work lists and staging, device counts) for the
// current sampler config: the host part of the largest possible miss list.  Called when the
// host-assisted share or the sampler changes (so the first extract does not pay the pinned
// allocations) and again, as a no-op, by every hg_enqueue.
cudaError_t hg_reserve(glb_ctx* c) {
  HostGather* h = c->hg;
  if (!h || !c->hg_permille || !c->D) return cudaSuccess;
  const uint64_t ub = c->sb.ub[c->sb.L] > c->sb.cap_batch ? c->sb.ub[c->sb.L] : c->sb.cap_batch;
  if (!ub) return cudaSuccess;  // no sampler yet
  const uint64_t cap = (ub * c->hg_permille + 999) / 1000;
  cudaError_t e;
  if (h->cap < cap || h->D != c->D) {
    for (int i = 0; i < 2; ++i)
      if ((e = cudaStreamSynchronize(h->cs[i])) != cudaSuccess) return e;
    if ((e = cudaStreamSynchronize(c->stream)) != cudaSuccess) return e;
    hg_free_bufs(h);
    for (int k = 0; k < kSlots; ++k) {
      if ((e = cudaMalloc(&h->dcnt[k], 4 * sizeof(uint32_t))) != cudaSuccess ||
          (e = cudaMemset(h->dcnt[k], 0, 4 * sizeof(uint32_t))) != cudaSuccess ||
          (e = cudaMalloc(&h->ent_dev[k], cap * sizeof(uint2))) != cudaSuccess ||
          (h->dma && (e = cudaMalloc(&h->dstage[k], cap * 4ull * c->D)) != cudaSuccess) ||
          (e = cudaMallocHost((void**)&h->cnt[k], 4 * sizeof(uint32_t))) != cudaSuccess ||
          (e = cudaMallocHost((void**)&h->ent[k], cap * sizeof(uint2))) != cudaSuccess ||
          (e = cudaHostAlloc((void**)&h->stage[k], cap * 4ull * c->D,
                             cudaHostAllocMapped | cudaHostAllocPortable)) != cudaSuccess ||
          (e = cudaHostGetDevicePointer((void**)&h->stage_dev[k], h->stage[k], 0)) != cudaSuccess)
        return e;
      memset(h->cnt[k], 0, 4 * sizeof(uint32_t));
    }
    h->cap = cap;
    h->D = c->D;
  }
  return cudaSuccess;
}

// Enqueue the host part of the current sample's extract (rows of the tail of
// `miss_sorted`) and return the device counts {nh, n_zc, ...} the extract kernel takes.
cudaError_t hg_enqueue(glb_ctx* c, float* out, const uint2* miss_sorted, uint32_t** dcnt_out) {
  HostGather* h = c->hg;
  const int s = c->cur;
  cudaError_t e = hg_reserve(c);
  if (e != cudaSuccess) return e;
  // misses per batch from the pinned counts of recent batches (completed, or a benign
  // race with the copy that is writing them: either value is a miss count)
  for (int k = 0; k < kSlots; ++k) {
    const uint32_t nm = h->cnt[k][3];
    if (nm) h->nm_est = h->nm_est > 0 ? 0.5 * h->nm_est + 0.5 * nm : (double)nm;
  }
  uint64_t target = (uint64_t)(h->nm_est * c->hg_permille / 1000.0);
  if (target > h->cap) target = h->cap;
  k_hg_split<<<c->num_sms, kThreads, 0, c->stream>>>(c->st, (uint32_t)target, miss_sorted,
                                                     h->dcnt[s], h->ent_dev[s]);
  count_launch(c);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  if ((e = cudaEventRecord(h->ev_split, c->stream)) != cudaSuccess) return e;
  // counts (always: they feed the estimate) and the host part's work list -> pinned memory
  if ((e = cudaStreamWaitEvent(h->cs[0], h->ev_split, 0)) != cudaSuccess) return e;
  if ((e = cudaMemcpyAsync(h->cnt[s], h->dcnt[s], 4 * sizeof(uint32_t), cudaMemcpyDeviceToHost,
                           h->cs[0])) != cudaSuccess)
    return e;
  *dcnt_out = h->dcnt[s];
  if (target == 0) return cudaSuccess;  // no estimate yet: the extract kernel takes every miss
  if ((e = cudaMemcpyAsync(h->ent[s], h->ent_dev[s], target * sizeof(uint2),
                           cudaMemcpyDeviceToHost, h->cs[0])) != cudaSuccess)
    return e;
  if ((e = cudaEventRecord(h->ev_d2h, h->cs[0])) != cudaSuccess) return e;
  if ((e = cudaStreamWaitEvent(h->cs[1], h->ev_d2h, 0)) != cudaSuccess) return e;
  const bool vec = (c->D % 4) == 0;
  const uint32_t U = vec ? c->D / 4 : c->D;
  const size_t rb = 4ull * c->D;
  // The host functions run back to back on cs[0] (the host gathers without waiting for any
  // scatter); chunk k's copy-out and scatter run on cs[1] once its host function is done
  // (ev_chunk[k]), so the staged rows cross the link while the host gathers the next chunk.
  for (int k = 0; k < h->nch; ++k) {  // gather chunk k on the host, move it, scatter it
    cudaStream_t q = h->cs[1];
    const uint64_t lo = chunk_lo(target, k, h->nch), hi = chunk_lo(target, k + 1, h->nch);
    if (hi <= lo) continue;
    HgJob* j = &h->job[h->njobs++ % kJobRing];
    while (!j->done.load(std::memory_order_acquire)) std::this_thread::yield();  // ring full
    j->c = c;
    j->slot = s;
    j->k = k;
    j->nch = h->nch;
    j->target = target;
    j->done.store(0, std::memory_order_relaxed);
    if ((e = cudaLaunchHostFunc(h->cs[0], hg_host_fn, j)) != cudaSuccess) {
      j->done.store(1);
      return e;
    }
    if ((e = cudaEventRecord(h->ev_chunk[k], h->cs[0])) != cudaSuccess ||
        (e = cudaStreamWaitEvent(q, h->ev_chunk[k], 0)) != cudaSuccess)
      return e;
    const uint8_t* src = h->stage_dev[s];
    if (h->dma) {
      if ((e = cudaMemcpyAsync(h->dstage[s] + lo * rb, h->stage[s] + lo * rb, (hi - lo) * rb,
                               cudaMemcpyHostToDevice, q)) != cudaSuccess)
        return e;
      src = h->dstage[s];
    }
    const int sg = h->sblocks ? h->sblocks : c->num_sms;
    if (vec)
      k_hg_scatter<float4><<<sg, kThreads, 0, q>>>(
          (float4*)out, (const float4*)src, h->ent_dev[s], h->dcnt[s], lo, hi, U, U);
    else
      k_hg_scatter<float><<<sg, kThreads, 0, q>>>(
          out, (const float*)src, h->ent_dev[s], h->dcnt[s], lo, hi, U, U);
    count_launch(c);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// The extract stream joins the host part; the extract counters get the full miss count.
cudaError_t hg_join(glb_ctx* c) {
  HostGather* h = c->hg;
  cudaError_t e;
  for (int i = 0; i < 2; ++i) {
    if ((e = cudaEventRecord(h->ev_end[i], h->cs[i])) != cudaSuccess) return e;
    if ((e = cudaStreamWaitEvent(c->stream, h->ev_end[i], 0)) != cudaSuccess) return e;
  }
  k_hg_fix<<<1, 1, 0, c->stream>>>(h->dcnt[c->cur], c->xcount);
  count_launch(c);
  return cudaGetLastError();
}

}  // namespace glb
