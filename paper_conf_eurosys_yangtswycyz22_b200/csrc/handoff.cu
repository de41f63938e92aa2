// handoff.cu -- a8: the factored Sampler -> Trainer handoff over peer memory.
//
// Paper: GNNLab's Samplers put each mini-batch's samples into a global queue
// and Trainers take them out and extract their features (Fig 9,
// "Each Sampler ... puts the samples into a global queue ... the Trainer ...
// dequeues", L250-L252 §5.2).  The paper's queue is in host memory (copy to
// host, Table 5 "C"); here the queue slots live in the TRAINER's HBM and the
// sampler's GPU writes a finished sample straight into one with a single copy
// kernel -- over NVLink/NVSwitch when the two ranks are on different GPUs,
// through CUDA IPC when they are different processes -- so no sample ever
// touches host memory and the trainer's extract reads it locally.
//
// Ordering is device-side and cross-process through interprocess CUDA events:
//   sampler: wait consumed[slot] -> k_push -> record ready[slot]
//   trainer: wait ready[sampler][slot] -> k_mark (its own cache map) -> extract
//            -> (consumer) -> record consumed[slot] (glb_handoff_release)
// The host control plane (which batch goes to which slot, "ready"/"released"
// notices) stays with the caller (parallel.py, over the process group's store):
// a wait is only enqueued after the matching record was, which that plane orders.
#include <cuda_runtime.h>
#include <unistd.h>

#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>

#include "glb_internal.cuh"

using namespace glb;

namespace {

constexpr uint32_t kMagicTrainer = 0x474C4254u;  // "GLBT"
constexpr uint32_t kMagicSampler = 0x474C4253u;  // "GLBS"
constexpr uint64_t kAlign = 256;

struct TrainerBlob {
  uint32_t magic, slots;
  int32_t pid, device;
  HandoffLayout lay;
  uint64_t ring_ptr;                          // same-process peers use these directly
  uint64_t consumed_ptr[kHandoffMaxSlots];
  cudaIpcMemHandle_t mem;
  cudaIpcEventHandle_t consumed[kHandoffMaxSlots];
};
struct SamplerBlob {
  uint32_t magic, slots;
  int32_t pid, device;
  uint64_t ready_ptr[kHandoffMaxSlots];
  cudaIpcEventHandle_t ready[kHandoffMaxSlots];
};
static_assert(sizeof(TrainerBlob) <= GLB_HANDOFF_BLOB_BYTES, "trainer blob size");
static_assert(sizeof(SamplerBlob) <= GLB_HANDOFF_BLOB_BYTES, "sampler blob size");
static_assert(sizeof(DevState) + sizeof(uint64_t) <= kAlign, "slot header");

glb_status ho_err(glb_ctx* c, glb_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  c->err = buf;
  return s;
}

glb_status ho_fail(glb_ctx* c, cudaError_t e, const char* what) {
  c->poisoned = true;
  return ho_err(c, GLB_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define HK(expr)                                          \
  do {                                                    \
    cudaError_t e_ = (expr);                              \
    if (e_ != cudaSuccess) return ho_fail(c, e_, #expr);  \
  } while (0)

#define HENTER(c)                                                                     \
  do {                                                                                \
    if (!(c)) return GLB_EINVAL;                                                      \
    if ((c)->poisoned) return ho_err(c, GLB_ECUDA, "ctx poisoned: %s", (c)->err.c_str()); \
    cudaError_t e0_ = cudaSetDevice((c)->device);                                     \
    if (e0_ != cudaSuccess) return ho_fail(c, e0_, "cudaSetDevice");                  \
  } while (0)

uint64_t align_up(uint64_t x) { return (x + kAlign - 1) / kAlign * kAlign; }

// Slot layout from this ctx's sampler capacities (the sizes glb_set_sampler allocated).
HandoffLayout make_layout(const glb_ctx* c) {
  HandoffLayout L = {};
  const SampleBufs& b = c->sbs[0];
  L.L = b.L;
  L.weighted = c->kind == GLB_RANDOM_WALK;
  L.off_tag = sizeof(DevState);
  uint64_t o = kAlign;  // header: DevState, then the u64 tag
  L.cap_uniq = b.ub[b.L] > b.cap_batch ? b.ub[b.L] : b.cap_batch;
  L.off_uniq = o;
  o = align_up(o + 4 * L.cap_uniq);
  for (uint32_t l = 0; l < b.L; ++l) {
    L.cap_indptr[l] = b.ub[l] + 1;
    L.cap_nnz[l] = b.ub[l] * b.k[l];
    L.off_indptr[l] = o;
    o = align_up(o + 4 * L.cap_indptr[l]);
    L.off_indices[l] = o;
    o = align_up(o + 4 * L.cap_nnz[l]);
    if (L.weighted) {
      L.off_weights[l] = o;
      o = align_up(o + 4 * L.cap_nnz[l]);
    }
  }
  L.slot_bytes = o;
  return L;
}

// ---------------------------------------------------------------- push kernel
// One launch copies a finished sample into a trainer slot: the header (sizes), uniq,
// and every block's indptr / indices / weights.  Counts come from the sampler's
// device state (no host sync).  Arrays are 256-byte aligned on both sides, so the
// body moves in 16-byte vectors (NVLink / HBM stores of whole sectors), the < 4-word
// tail in words.
constexpr int kMaxSegs = 1 + 3 * GLB_MAX_HOPS;
struct PushArgs {
  const uint32_t* src[kMaxSegs];
  uint32_t* dst[kMaxSegs];
  uint32_t nseg, L, weighted;
};

__device__ __forceinline__ uint32_t seg_len(const DevState& st, uint32_t s, uint32_t L, uint32_t w) {
  if (s == 0) return st.n[L];
  const uint32_t k = (s - 1) / L, l = (s - 1) % L;  // k: 0 indptr, 1 indices, 2 weights
  if (k == 0) return st.n[l] + 1;
  return (k == 1 || w) ? st.nnz[l] : 0;
}

__global__ void __launch_bounds__(kThreads)
    k_push(PushArgs a, const DevState* __restrict__ st_src, DevState* st_dst, uint64_t* tag_dst,
           uint64_t tag) {
  const DevState st = *st_src;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    *st_dst = st;
    *tag_dst = tag;
  }
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint32_t s = 0; s < a.nseg; ++s) {
    const uint32_t n = seg_len(st, s, a.L, a.weighted);
    const uint32_t nv = n / 4;
    const uint4* src4 = reinterpret_cast<const uint4*>(a.src[s]);
    uint4* dst4 = reinterpret_cast<uint4*>(a.dst[s]);
    for (uint64_t i = tid; i < nv; i += stride) dst4[i] = __ldg(src4 + i);
    for (uint64_t i = 4ull * nv + tid; i < n; i += stride) a.dst[s][i] = __ldg(a.src[s] + i);
  }
}

void free_recv(HandoffRecv* r) {
  if (!r) return;
  for (int p = 0; p < kHandoffMaxPeers; ++p)
    if (r->ready_opened[p])
      for (int s = 0; s < kHandoffMaxSlots; ++s)
        if (r->ready[p][s]) cudaEventDestroy(r->ready[p][s]);
  for (int s = 0; s < kHandoffMaxSlots; ++s) {
    if (r->consumed[s]) cudaEventDestroy(r->consumed[s]);
    if (r->lidslot[s]) cudaFree(r->lidslot[s]);
    if (r->hit[s]) cudaFree(r->hit[s]);
    if (r->miss[s]) cudaFree(r->miss[s]);
    if (r->miss_sorted[s]) cudaFree(r->miss_sorted[s]);
  }
  if (r->ring) cudaFree(r->ring);
  delete r;
}

void free_send(HandoffSend* h) {
  if (!h) return;
  for (int s = 0; s < kHandoffMaxSlots; ++s) {
    if (h->ready[s]) cudaEventDestroy(h->ready[s]);
    if (h->consumed_opened && h->consumed[s]) cudaEventDestroy(h->consumed[s]);
  }
  if (h->ring_ipc && h->ring) cudaIpcCloseMemHandle(h->ring);
  delete h;
}

cudaError_t enable_peer(int dev, int peer_dev) {
  if (dev == peer_dev) return cudaSuccess;
  int ok = 0;
  cudaError_t e = cudaDeviceCanAccessPeer(&ok, dev, peer_dev);
  if (e != cudaSuccess) return e;
  if (!ok) return cudaErrorPeerAccessUnsupported;
  e = cudaDeviceEnablePeerAccess(peer_dev, 0);
  if (e == cudaErrorPeerAccessAlreadyEnabled) {
    cudaGetLastError();
    e = cudaSuccess;
  }
  return e;
}

}  // namespace

namespace glb {
void handoff_free(glb_ctx* c) {
  free_recv(c->ho_recv);
  c->ho_recv = nullptr;
  for (int p = 0; p < kHandoffMaxPeers; ++p) {
    free_send(c->ho_send[p]);
    c->ho_send[p] = nullptr;
  }
}
}  // namespace glb

extern "C" {

glb_status glb_handoff_create(glb_ctx* c, uint32_t slots, void* blob_out) {
  HENTER(c);
  if (!blob_out) return ho_err(c, GLB_EINVAL, "null blob");
  if (slots == 0 || slots > (uint32_t)kHandoffMaxSlots)
    return ho_err(c, GLB_EINVAL, "slots %u not in [1,%d]", slots, kHandoffMaxSlots);
  if (!c->sampler_set) return ho_err(c, GLB_ESTATE, "handoff_create before set_sampler");
  HK(cudaStreamSynchronize(c->stream));
  free_recv(c->ho_recv);
  c->ho_recv = nullptr;
  HandoffRecv* r = new (std::nothrow) HandoffRecv();
  if (!r) return ho_err(c, GLB_ENOMEM, "host alloc");
  r->slots = slots;
  r->lay = make_layout(c);
  const uint64_t cap = r->lay.cap_uniq;
  cudaError_t e = cudaMalloc((void**)&r->ring, r->lay.slot_bytes * slots);
  for (uint32_t s = 0; s < slots && e == cudaSuccess; ++s) {
    if (e == cudaSuccess) e = cudaMalloc((void**)&r->lidslot[s], 4 * cap);
    if (e == cudaSuccess) e = cudaMalloc((void**)&r->hit[s], 8 * cap);
    if (e == cudaSuccess) e = cudaMalloc((void**)&r->miss[s], 8 * cap);
    if (e == cudaSuccess) e = cudaMalloc((void**)&r->miss_sorted[s], 8 * cap);
    if (e == cudaSuccess)
      e = cudaEventCreateWithFlags(&r->consumed[s], cudaEventDisableTiming | cudaEventInterprocess);
  }
  if (e == cudaSuccess) e = cudaMemset(r->ring, 0, r->lay.slot_bytes * slots);
  TrainerBlob b;
  memset(&b, 0, sizeof(b));
  if (e == cudaSuccess) e = cudaIpcGetMemHandle(&b.mem, r->ring);
  for (uint32_t s = 0; s < slots && e == cudaSuccess; ++s)
    e = cudaIpcGetEventHandle(&b.consumed[s], r->consumed[s]);
  if (e != cudaSuccess) {
    free_recv(r);
    if (e == cudaErrorMemoryAllocation) {
      cudaGetLastError();
      return ho_err(c, GLB_ENOMEM, "handoff ring: %s", cudaGetErrorString(e));
    }
    return ho_fail(c, e, "glb_handoff_create");
  }
  b.magic = kMagicTrainer;
  b.slots = slots;
  b.pid = (int32_t)getpid();
  b.device = c->device;
  b.lay = r->lay;
  b.ring_ptr = (uint64_t)(uintptr_t)r->ring;
  for (uint32_t s = 0; s < slots; ++s) b.consumed_ptr[s] = (uint64_t)(uintptr_t)r->consumed[s];
  memset(blob_out, 0, GLB_HANDOFF_BLOB_BYTES);
  memcpy(blob_out, &b, sizeof(b));
  c->ho_recv = r;
  return GLB_OK;
}

glb_status glb_handoff_attach(glb_ctx* c, uint32_t trainer, const void* trainer_blob, void* blob_out) {
  HENTER(c);
  if (!trainer_blob || !blob_out) return ho_err(c, GLB_EINVAL, "null blob");
  if (trainer >= (uint32_t)kHandoffMaxPeers) return ho_err(c, GLB_EINVAL, "trainer id %u >= %d", trainer, kHandoffMaxPeers);
  if (!c->sampler_set) return ho_err(c, GLB_ESTATE, "handoff_attach before set_sampler");
  TrainerBlob b;
  memcpy(&b, trainer_blob, sizeof(b));
  if (b.magic != kMagicTrainer || b.slots == 0 || b.slots > (uint32_t)kHandoffMaxSlots)
    return ho_err(c, GLB_EINVAL, "not a trainer handoff blob");
  // the trainer's slots must hold any sample this ctx can produce
  const HandoffLayout mine = make_layout(c);
  if (b.lay.L != mine.L || b.lay.weighted != mine.weighted)
    return ho_err(c, GLB_EINVAL, "trainer ring has %u hops (weighted %u), sampler %u (%u)",
                  b.lay.L, b.lay.weighted, mine.L, mine.weighted);
  bool fits = b.lay.cap_uniq >= mine.cap_uniq;
  for (uint32_t l = 0; l < mine.L; ++l)
    fits = fits && b.lay.cap_indptr[l] >= mine.cap_indptr[l] && b.lay.cap_nnz[l] >= mine.cap_nnz[l];
  if (!fits) return ho_err(c, GLB_EINVAL, "trainer ring slots are smaller than this sampler's capacity");
  HK(cudaStreamSynchronize(c->stream));
  free_send(c->ho_send[trainer]);
  c->ho_send[trainer] = nullptr;
  HandoffSend* h = new (std::nothrow) HandoffSend();
  if (!h) return ho_err(c, GLB_ENOMEM, "host alloc");
  h->slots = b.slots;
  h->lay = b.lay;
  cudaError_t e = cudaSuccess;
  if (b.pid == (int32_t)getpid()) {  // same process: borrow the pointers (peer access if another GPU)
    e = enable_peer(c->device, b.device);
    h->ring = (uint8_t*)(uintptr_t)b.ring_ptr;
    for (uint32_t s = 0; s < b.slots; ++s) h->consumed[s] = (cudaEvent_t)(uintptr_t)b.consumed_ptr[s];
  } else {
    void* p = nullptr;
    e = cudaIpcOpenMemHandle(&p, b.mem, cudaIpcMemLazyEnablePeerAccess);
    if (e == cudaSuccess) {
      h->ring = (uint8_t*)p;
      h->ring_ipc = true;
    }
    h->consumed_opened = true;
    for (uint32_t s = 0; s < b.slots && e == cudaSuccess; ++s)
      e = cudaIpcOpenEventHandle(&h->consumed[s], b.consumed[s]);
  }
  SamplerBlob o;
  memset(&o, 0, sizeof(o));
  for (uint32_t s = 0; s < b.slots && e == cudaSuccess; ++s) {
    e = cudaEventCreateWithFlags(&h->ready[s], cudaEventDisableTiming | cudaEventInterprocess);
    if (e == cudaSuccess) e = cudaIpcGetEventHandle(&o.ready[s], h->ready[s]);
    o.ready_ptr[s] = (uint64_t)(uintptr_t)h->ready[s];
  }
  if (e != cudaSuccess) {
    free_send(h);
    return ho_fail(c, e, "glb_handoff_attach");
  }
  o.magic = kMagicSampler;
  o.slots = b.slots;
  o.pid = (int32_t)getpid();
  o.device = c->device;
  memset(blob_out, 0, GLB_HANDOFF_BLOB_BYTES);
  memcpy(blob_out, &o, sizeof(o));
  c->ho_send[trainer] = h;
  return GLB_OK;
}

glb_status glb_handoff_connect(glb_ctx* c, uint32_t sampler, const void* sampler_blob) {
  HENTER(c);
  if (!sampler_blob) return ho_err(c, GLB_EINVAL, "null blob");
  if (sampler >= (uint32_t)kHandoffMaxPeers) return ho_err(c, GLB_EINVAL, "sampler id %u >= %d", sampler, kHandoffMaxPeers);
  HandoffRecv* r = c->ho_recv;
  if (!r) return ho_err(c, GLB_ESTATE, "handoff_connect before handoff_create");
  SamplerBlob b;
  memcpy(&b, sampler_blob, sizeof(b));
  if (b.magic != kMagicSampler || b.slots != r->slots)
    return ho_err(c, GLB_EINVAL, "not a sampler blob for this ring (%u slots)", r->slots);
  HK(cudaStreamSynchronize(c->stream));
  if (r->ready_opened[sampler])
    for (int s = 0; s < kHandoffMaxSlots; ++s)
      if (r->ready[sampler][s]) cudaEventDestroy(r->ready[sampler][s]);
  for (int s = 0; s < kHandoffMaxSlots; ++s) r->ready[sampler][s] = nullptr;
  r->ready_opened[sampler] = false;
  if (b.pid == (int32_t)getpid()) {
    for (uint32_t s = 0; s < r->slots; ++s) r->ready[sampler][s] = (cudaEvent_t)(uintptr_t)b.ready_ptr[s];
    return GLB_OK;
  }
  r->ready_opened[sampler] = true;
  for (uint32_t s = 0; s < r->slots; ++s) HK(cudaIpcOpenEventHandle(&r->ready[sampler][s], b.ready[s]));
  return GLB_OK;
}

glb_status glb_handoff_send(glb_ctx* c, uint32_t trainer, uint32_t slot, uint64_t tag) {
  HENTER(c);
  if (trainer >= (uint32_t)kHandoffMaxPeers || !c->ho_send[trainer])
    return ho_err(c, GLB_ESTATE, "trainer %u not attached", trainer);
  HandoffSend* h = c->ho_send[trainer];
  if (slot >= h->slots) return ho_err(c, GLB_EINVAL, "slot %u >= %u", slot, h->slots);
  if (!c->have_sample) return ho_err(c, GLB_ESTATE, "handoff_send without a current sample");
  if (c->last_L != h->lay.L) return ho_err(c, GLB_EINVAL, "sample has %u hops, ring %u", c->last_L, h->lay.L);
  if (c->ho_recv && c->ho_recv->cur >= 0 && c->st != c->sts[c->cur])
    return ho_err(c, GLB_ESTATE, "current sample is a received one");
  uint8_t* base = h->ring + (uint64_t)slot * h->lay.slot_bytes;
  PushArgs a = {};
  a.L = h->lay.L;
  a.weighted = h->lay.weighted;
  a.nseg = 1 + (a.weighted ? 3 : 2) * a.L;
  a.src[0] = c->sb.uniq;
  a.dst[0] = (uint32_t*)(base + h->lay.off_uniq);
  for (uint32_t l = 0; l < a.L; ++l) {
    a.src[1 + l] = c->sb.bindptr[l];
    a.dst[1 + l] = (uint32_t*)(base + h->lay.off_indptr[l]);
    a.src[1 + a.L + l] = c->sb.bindices[l];
    a.dst[1 + a.L + l] = (uint32_t*)(base + h->lay.off_indices[l]);
    if (a.weighted) {
      a.src[1 + 2 * a.L + l] = c->sb.bweights[l];
      a.dst[1 + 2 * a.L + l] = (uint32_t*)(base + h->lay.off_weights[l]);
    }
  }
  // the trainer must be done with the slot's previous sample (no-op before its first release)
  HK(cudaStreamWaitEvent(c->stream, h->consumed[slot], 0));
  k_push<<<c->num_sms * 2, kThreads, 0, c->stream>>>(a, c->st, (DevState*)base,
                                                     (uint64_t*)(base + h->lay.off_tag), tag);
  count_launch(c);
  HK(cudaGetLastError());
  HK(cudaEventRecord(h->ready[slot], c->stream));
  return GLB_OK;
}

glb_status glb_handoff_recv(glb_ctx* c, uint32_t sampler, uint32_t slot) {
  HENTER(c);
  HandoffRecv* r = c->ho_recv;
  if (!r) return ho_err(c, GLB_ESTATE, "handoff_recv before handoff_create");
  if (slot >= r->slots) return ho_err(c, GLB_EINVAL, "slot %u >= %u", slot, r->slots);
  if (sampler >= (uint32_t)kHandoffMaxPeers || !r->ready[sampler][0])
    return ho_err(c, GLB_ESTATE, "sampler %u not connected", sampler);
  if (!c->slot) return ho_err(c, GLB_ESTATE, "no graph loaded");
  const HandoffLayout& L = r->lay;
  uint8_t* base = r->ring + (uint64_t)slot * L.slot_bytes;
  DevState* st = (DevState*)base;
  HK(cudaStreamWaitEvent(c->stream, r->ready[sampler][slot], 0));
  // a4 against THIS ctx's cache (samplers need not hold one): hit / miss lists + marks
  HK(cudaMemsetAsync(&st->nhit, 0, 2 * sizeof(uint32_t), c->stream));
  HK(launch_mark_to(c, (const uint32_t*)(base + L.off_uniq), L.cap_uniq, &st->n[L.L], st,
                    r->hit[slot], r->miss[slot], r->lidslot[slot]));
  SampleBufs v = c->sbs[0];  // capacities; pointers redirected to the slot
  v.uniq = (uint32_t*)(base + L.off_uniq);
  v.lidslot = r->lidslot[slot];
  for (uint32_t l = 0; l < L.L; ++l) {
    v.bindptr[l] = (uint32_t*)(base + L.off_indptr[l]);
    v.bindices[l] = (uint32_t*)(base + L.off_indices[l]);
    v.bweights[l] = L.weighted ? (uint32_t*)(base + L.off_weights[l]) : nullptr;
  }
  v.hit_list = r->hit[slot];
  v.miss_list = r->miss[slot];
  v.miss_sorted = r->miss_sorted[slot];
  c->sb = v;
  c->st = st;
  r->cur = (int)slot;
  c->have_sample = true;
  c->last_L = L.L;
  c->last_kind = L.weighted ? GLB_RANDOM_WALK : c->kind;
  return GLB_OK;
}

glb_status glb_handoff_tag(glb_ctx* c, uint64_t* out) {
  HENTER(c);
  HandoffRecv* r = c->ho_recv;
  if (!out) return ho_err(c, GLB_EINVAL, "null out");
  if (!r || r->cur < 0) return ho_err(c, GLB_ESTATE, "no received sample");
  const uint8_t* base = r->ring + (uint64_t)r->cur * r->lay.slot_bytes;
  HK(cudaMemcpyAsync(out, base + r->lay.off_tag, sizeof(uint64_t), cudaMemcpyDeviceToHost, c->stream));
  HK(cudaStreamSynchronize(c->stream));
  return GLB_OK;
}

glb_status glb_handoff_release(glb_ctx* c, uint32_t slot) {
  HENTER(c);
  HandoffRecv* r = c->ho_recv;
  if (!r) return ho_err(c, GLB_ESTATE, "handoff_release before handoff_create");
  if (slot >= r->slots) return ho_err(c, GLB_EINVAL, "slot %u >= %u", slot, r->slots);
  // after everything enqueued so far on the ctx stream, and the extract (pipeline depth 2
  // runs it on the extract stream)
  if (c->nslots == 2) {
    HK(cudaEventRecord(c->ev_mark, c->xstream));
    HK(cudaStreamWaitEvent(c->stream, c->ev_mark, 0));
  }
  HK(cudaEventRecord(r->consumed[slot], c->stream));
  if (r->cur == (int)slot) {  // the slot's sample is no longer the current one
    r->cur = -1;
    c->sb = c->sbs[c->cur];
    c->st = c->sts[c->cur];
    c->have_sample = false;
  }
  return GLB_OK;
}

}  // extern "C"
