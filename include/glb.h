/*
 * glb.h -- C-ABI of the B200-native GNNLab sample+extract hot path.
 *
 * Paper: GNNLab: A Factored System for Sample-based GNN Training over GPUs
 * (EuroSys'22), text at PAPER.md.  Citations "L<n> §<s>" point into it;
 * "reading Qn" points at DESIGN.md "Readings" (ambiguities resolved).
 *
 * One glb_ctx per (process, GPU).  Plain pointers and sizes only, no torch
 * types.  All functions return a glb_status (0 = OK, < 0 = error) and never
 * throw or abort; glb_last_error() returns a detail string.  Unless stated,
 * calls are asynchronous on the ctx stream (glb_set_stream) and a device
 * pointer argument must stay valid until the stream reaches the call.
 * Calls on one ctx are not re-entrant.  After GLB_ECUDA the ctx is poisoned
 * (every later call returns GLB_ECUDA); destroy it.
 *
 * Device memory owned by the ctx (topology copy, relabel tables, cache,
 * sample buffers) is allocated with cudaMalloc on ctx->device and freed by
 * glb_destroy.  Host feature memory is BORROWED: glb_load_graph registers it
 * (cudaHostRegisterMapped|Portable) and glb_destroy unregisters it; the
 * caller keeps it alive until then.
 */
#ifndef GLB_H
#define GLB_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct glb_ctx glb_ctx;
typedef int32_t glb_status;

enum {
  GLB_OK = 0,
  GLB_EINVAL = -1,  /* bad argument: bad CSR, duplicate seed, id >= V, fanout 0, alpha not in [0,1] */
  GLB_ENOMEM = -2,  /* allocation failed, or a batch exceeds the capacity set by glb_set_sampler */
  GLB_ECUDA = -3,   /* CUDA runtime error (ctx poisoned) */
  GLB_ESTATE = -4,  /* call out of order (e.g. sample before load_graph) */
  GLB_ERANGE = -5   /* epoch >= 2^16 or hop >= 2^8 (RNG counter field widths, reading Q4) */
};

/* sampler kinds */
enum {
  GLB_KHOP_UNIFORM = 0, /* k-hop uniform neighbourhood sampling (L67, Fig 7) */
  GLB_RANDOM_WALK = 1,  /* PinSAGE random walks: "5 neighbors from 4 paths of length 3" (L353) */
  GLB_KHOP_WEIGHTED = 2 /* k-hop weighted: k draws with replacement, P(edge) = w / row sum
                           (L81 fn1, L148 fn5, L136; reading Q19); needs glb_load_edge_weights */
};

/* visit-count recording targets (glb_set_count_mode) */
enum {
  GLB_COUNT_NONE = 0,
  GLB_COUNT_PRESAMPLE = 1, /* PreSC hotness counts h_v (L333 §6.3) */
  GLB_COUNT_ACCESS = 2     /* measured-epoch accesses, for hit rate / Optimal (L148 fn4) */
};

#define GLB_MAX_HOPS 8

/* ------------------------------------------------------------------ ctx */
const char* glb_last_error(const glb_ctx* ctx); /* ctx may be NULL (creation errors) */
glb_status glb_create(int device, glb_ctx** out);
glb_status glb_destroy(glb_ctx* ctx);
/* Run every later call on this stream (cudaStream_t; e.g. torch.cuda.current_stream().cuda_stream).
 * NULL = the legacy default stream.  A new ctx starts on its own non-blocking stream; callers
 * that hand device buffers produced on another stream must set that stream (or synchronise). */
glb_status glb_set_stream(glb_ctx* ctx, void* cuda_stream);
glb_status glb_sync(glb_ctx* ctx); /* cudaStreamSynchronize + deferred device error check */

/* --------------------------------------------------------------- load(dev, graph) (Fig 9)
 * indptr: host u64[V+1], indptr[0]=0, non-decreasing, indptr[V]=E.
 * indices: host u32[E], each < V.  Topology is COPIED into HBM (D1: CSR in GPU
 * memory, L222/L250).  features: host f32[V][feat_dim] row-major, BORROWED and
 * registered as mapped pinned memory (D2); may be NULL (sample-only ctx).
 * Synchronous.  Errors: EINVAL (shape/monotonicity/range), ENOMEM, ECUDA. */
glb_status glb_load_graph(glb_ctx* ctx, uint64_t num_vertices, uint64_t num_edges,
                          const uint64_t* indptr, const uint32_t* indices,
                          const void* features, uint32_t feat_dim);

/* Edge weights for GLB_KHOP_WEIGHTED: host u32[E] parallel to `indices` (e.g. the
 * target's "year registered", L136).  Copied; their inclusive u64 prefix over all edges
 * is kept in HBM (8 B per edge).  Synchronous. */
glb_status glb_load_edge_weights(glb_ctx* ctx, const uint32_t* weights);

/* Sampler used by glb_sample_batch / glb_presample, and the capacity of the
 * per-batch buffers.  kind GLB_KHOP_UNIFORM: fanouts[0..num_hops-1] (hop order
 * from the seeds, reading Q1).  kind GLB_RANDOM_WALK: num_hops layers, each
 * keeping rw_topk of rw_walks walks of rw_len steps (fanouts ignored).
 * max_batch: largest seed count a batch may have.  Synchronous (allocates). */
glb_status glb_set_sampler(glb_ctx* ctx, int kind, const uint32_t* fanouts, uint32_t num_hops,
                           uint32_t rw_walks, uint32_t rw_len, uint32_t rw_topk,
                           uint32_t max_batch);

/* Relabel table used by the next glb_set_sampler (dedup/relabel, L230 "remap(dedup(samples))"):
 * 1 = dense direct-address table (16 B per vertex), 2 = open-addressing hash table sized
 * from the batch's unique-vertex bound (L2-resident for large graphs), 0 = auto (dense unless
 * V > 2x the hash capacity).  Results are identical in both modes.  glb_relabel_mode reports
 * the mode in use (1 or 2). */
glb_status glb_set_relabel_mode(glb_ctx* ctx, int mode);
glb_status glb_relabel_mode(const glb_ctx* ctx, int* out);
/* Bytes of the relabel table covered by a persisting-L2 access-policy window on the sampler's
 * kernels (0 = none).  Set by glb_set_sampler: by default only when the whole table fits in
 * a third of L2 (it then stays resident while the pipelined gather streams through L2);
 * environment GLB_L2_PIN=0 / 1 forces it off / on. */
glb_status glb_relabel_l2_window(const glb_ctx* ctx, uint64_t* bytes_out);

/* Training set T (host u32[n], distinct -- a duplicate is EINVAL -- each < V) and mini-batch size B
 * (L305 §6.2: shuffle T each epoch and divide it; last batch partial).
 * seed keys every draw of the ctx (shuffle and sampling).  Synchronous. */
glb_status glb_set_train_set(glb_ctx* ctx, const uint32_t* train, uint64_t n, uint32_t batch_size,
                             uint64_t seed);
/* number of mini-batches per epoch = ceil(n / B) */
glb_status glb_num_batches(const glb_ctx* ctx, uint32_t* out);
/* a1: device-side epoch permutation (Philox keys + stable radix sort; reading Q9/§8(c).2).
 * Later glb_sample_batch(epoch, b) calls use it. */
glb_status glb_shuffle(glb_ctx* ctx, uint32_t epoch);
/* copy the current epoch permutation to host u32[n] (synchronous; tests) */
glb_status glb_get_permutation(glb_ctx* ctx, uint32_t* host_out);

/* ---------------------------------------------------------------- samples (a2-a4)
 * Per-hop blocks, DGL style (reading Q3): block l has dst = lids 0..n_l-1 and
 * src = lids 0..n_{l+1}-1; uniq[lid] = gid and the first n_l lids are the
 * frontier of hop l (seeds first, in input order; new vertices in
 * first-occurrence order, reading Q5).  Device pointers are OWNED BY THE CTX
 * and valid until the next sample call. */
typedef struct {
  uint32_t num_hops;
  uint32_t num_seeds;
  const uint32_t* uniq;                   /* device u32[sizes[num_hops]] */
  uint64_t sizes[GLB_MAX_HOPS + 1];       /* n_0..n_L (host values) */
  uint64_t nnz[GLB_MAX_HOPS];             /* edges of block l */
  const uint32_t* indptr[GLB_MAX_HOPS];   /* device u32[n_l+1] */
  const uint32_t* indices[GLB_MAX_HOPS];  /* device u32[nnz_l], src lids, slot order */
  const uint32_t* weights[GLB_MAX_HOPS];  /* device u32[nnz_l] visit counts (random walk), else NULL */
  const int32_t* cache_slot;              /* device i32[sizes[L]]: slot of uniq[i] or -1 (a4 "mark") */
} glb_blocks;

/* Sample one mini-batch.  seeds: host or device u32[num_seeds] (distinct, < V).
 * The sampler is the one set by glb_set_sampler; kind GLB_KHOP_UNIFORM may
 * override its fanouts with (fanouts, num_hops) -- pass NULL/0 to keep them.
 * Draws are keyed by (seed, epoch, batch, hop, vertex, slot) (reading Q4).
 * Synchronous: one device->host copy of the sizes.  Errors: EINVAL (dup seed,
 * id >= V), ENOMEM (num_seeds > max_batch), ERANGE, ESTATE. */
glb_status glb_sample(glb_ctx* ctx, const uint32_t* seeds, uint32_t num_seeds,
                      const uint32_t* fanouts, uint32_t num_hops, uint64_t seed, uint32_t epoch,
                      uint32_t batch, glb_blocks* out);

/* Sample mini-batch `batch` of the current epoch permutation (glb_shuffle) with
 * the ctx sampler.  ASYNCHRONOUS: no host sync; sizes stay on the device.
 * Visit counts are recorded per the count mode.  Use glb_sample_result to read
 * sizes (synchronises), or glb_extract_sample to gather features directly. */
glb_status glb_sample_batch(glb_ctx* ctx, uint32_t epoch, uint32_t batch);
/* Sample caller-provided seeds with the ctx sampler, ASYNCHRONOUSLY (no host sync): a host
 * `seeds` buffer is copied to the device on the ctx stream (truly asynchronous when it is
 * pinned; it must stay unchanged until the stream reaches the copy), a device buffer is
 * read in place.  Errors found on the device (duplicate seed, id >= V) surface at the next
 * glb_sync / glb_sample_result.  Errors: ESTATE, EINVAL, ENOMEM (n > max_batch), ERANGE. */
glb_status glb_sample_async(glb_ctx* ctx, const uint32_t* seeds, uint32_t num_seeds,
                            uint64_t seed, uint32_t epoch, uint32_t batch);
glb_status glb_sample_result(glb_ctx* ctx, glb_blocks* out);

/* ---------------------------------------------------------------- PreSC (a5, a6)
 * GLB_COUNT_PRESAMPLE: every batch-unique vertex of every later sample adds 1 to
 * counts[v] (reading Q8); GLB_COUNT_ACCESS: adds 1 to access[v]. */
glb_status glb_set_count_mode(glb_ctx* ctx, int mode);
glb_status glb_reset_counts(glb_ctx* ctx, int which /* GLB_COUNT_PRESAMPLE | _ACCESS */);
/* PreSC#K (L333-335 §6.3): sample every batch of epochs 0..K-1 of this rank's
 * share (batches b with b % world == rank) with recording into counts.
 * Counts accumulate; allreduce them across ranks before glb_build_cache. */
glb_status glb_presample(glb_ctx* ctx, uint32_t K, uint32_t rank, uint32_t world);
/* device pointer of the u32[V] count array (for NCCL allreduce through torch) */
glb_status glb_counts_device_ptr(glb_ctx* ctx, int which, void** out);
glb_status glb_get_counts(glb_ctx* ctx, int which, uint32_t* host_out /* V */);
/* load_cache(hotness_map, alpha) (L301 §6.1): C = floor(alpha*V); rank vertices by
 * (count desc, gid asc) (reading Q10); slot = rank for the first C; copy their
 * feature rows from host memory into an HBM cache f32[C][D].  hotness: NULL =
 * the PreSC counts, else a device u32[V] hotness map (e.g. degree).  Synchronous. */
glb_status glb_build_cache(glb_ctx* ctx, double alpha, const uint32_t* hotness);
glb_status glb_get_cache_slots(glb_ctx* ctx, int32_t* host_out /* V */);

/* Caching policies compared in the paper (L79, L301, L339-L343, Fig 10/12): fill a
 * device u32[V] hotness map for glb_build_cache.  GLB_POLICY_PRESC copies the PreSC
 * counts; GLB_POLICY_DEGREE = out-degree (PaGraph; saturated to 2^32-1);
 * GLB_POLICY_RANDOM = hi32(draw64(v, 0, 0, c3(0,0,POLICY=7), 0)) under `seed`, a
 * random order of the vertices.  hotness_out: device, caller-owned. */
enum { GLB_POLICY_PRESC = 0, GLB_POLICY_DEGREE = 1, GLB_POLICY_RANDOM = 2 };
glb_status glb_policy_hotness(glb_ctx* ctx, int policy, uint64_t seed, uint32_t* hotness_out);

/* Footprint similarity of epoch i to epoch j (Table 2; reading Q16):
 *   sum_{v in T_i and T_j} min(f_i(v), f_j(v)) / sum_{v in T_j} f_j(v),
 * T_x = the floor(top_frac*V) vertices ranked first by (f_x desc, gid asc).
 * f_i, f_j: device u32[V] per-epoch visit counts.  Exact integer sums (num, den)
 * are returned; out = num/den (0 if den == 0).  Synchronous. */
glb_status glb_footprint_similarity(glb_ctx* ctx, const uint32_t* f_i, const uint32_t* f_j,
                                    double top_frac, uint64_t* num, uint64_t* den, double* out);
glb_status glb_cache_size(const glb_ctx* ctx, uint64_t* out);

/* ------------------------------------------------ NEXT-3: peer-sharded cache over NVLink
 * The paper's GPUs cache the same hot rows each, and a cross-GPU access is "74x slower"
 * than local (L516 §9); NVSwitch gives every B200 ~900 GB/s to every peer, so `world`
 * GPUs can instead cache world x as many distinct rows.
 * glb_build_cache_sharded: C = min(V, world * floor(alpha*V)) global rows, ranked as in
 * glb_build_cache (slot[v] = global rank i, reading Q10); this ctx (shard `rank`) stores
 * the rows i with i % world == rank at local row i / world.  world == 1 is
 * glb_build_cache.  Every ctx of the group must build with the same hotness, alpha and
 * world.  Synchronous.  Errors: EINVAL (world > GLB_MAX_SHARDS, rank >= world),
 * ESTATE (no graph / no features).
 * Until every other shard is attached (glb_attach_peer_cache), extract returns ESTATE. */
#define GLB_MAX_SHARDS 16
#define GLB_IPC_HANDLE_BYTES 64
glb_status glb_build_cache_sharded(glb_ctx* ctx, double alpha, const uint32_t* hotness,
                                   uint32_t rank, uint32_t world);
/* device pointer of this ctx's cache rows f32[rows][D] (rows = its shard's row count) */
glb_status glb_cache_device_ptr(glb_ctx* ctx, void** out, uint64_t* rows);
/* CUDA IPC handle (GLB_IPC_HANDLE_BYTES opaque bytes) of this ctx's shard, for another
 * process (e.g. all-gathered over torch.distributed).  ESTATE if there is no shard. */
glb_status glb_cache_ipc_handle(glb_ctx* ctx, void* handle_out);
/* Map shard `peer`'s rows for reading by this ctx's extract: exactly one of
 *  ipc_handle -- from glb_cache_ipc_handle in another process (opened with
 *                cudaIpcOpenMemHandle; closed on the next build or destroy), or
 *  dev_ptr    -- glb_cache_device_ptr of a ctx in THIS process (same GPU, or another
 *                GPU: peer access is enabled; EINVAL if the GPUs cannot access each other).
 * The peer must keep its shard alive (no rebuild / destroy) while this ctx extracts.
 * Synchronous.  Errors: ESTATE (cache not sharded), EINVAL (peer == own rank, >= world). */
glb_status glb_attach_peer_cache(glb_ctx* ctx, uint32_t peer, const void* ipc_handle,
                                 const void* dev_ptr);
/* Counts of the last extract: out[0] = cache hits (local + peer shards), out[1] = host
 * misses, out[2] = hits served by another GPU's shard (0 unless sharded).  Synchronous. */
glb_status glb_last_extract_counts(glb_ctx* ctx, uint64_t* out3);
/* Device u64[3] (hits, misses, peer hits) that every extract rewrites on the ctx stream:
 * copy it device->host after an extract (stream-ordered) to read that extract's counts
 * without a synchronisation.  Peer hits are valid only for a sharded cache. */
glb_status glb_extract_counts_device_ptr(glb_ctx* ctx, void** out);

/* Hit-rate statistics over the recorded accesses (GLB_COUNT_ACCESS) for the
 * current cache: total accesses, accesses served by the cache (H = hits/total),
 * and the Optimal policy's hits: the C largest access counts (L148 fn4, L339).
 * Synchronous.  Exact integers. */
typedef struct { uint64_t total, hits, optimal_hits, cache_rows; } glb_hit_stats;
glb_status glb_hit_stats_get(glb_ctx* ctx, glb_hit_stats* out);

/* ---------------------------------------------------------------- extract (a7)
 * extract(features, samples) (Fig 9; L252): out[i,:] = features[vertices[i],:]
 * for i < n, bytes exact; cache hits read the HBM cache, misses read the
 * mapped pinned host matrix over PCIe (zero copy).  vertices: device u32[n]
 * (any ids < V, duplicates allowed); out: device f32[n][D], caller-owned.
 * stats (nullable, HOST pointer): filled at the next glb_sync; one extract's stats can be
 * pending at a time -- an extract that asks for stats while another's are pending
 * synchronises first.  At pipeline depth 2 glb_extract is ordered after every extract
 * already enqueued on the extract stream (they share the miss-ordering scratch). */
typedef struct { uint64_t hits, misses; } glb_extract_stats;
glb_status glb_extract(glb_ctx* ctx, const uint32_t* vertices, uint64_t n, void* out,
                       glb_extract_stats* stats);
/* Extract the features of the last sample's uniq (out: device f32[>= n_L][D]),
 * using the marks taken during relabel; no host sync. */
glb_status glb_extract_sample(glb_ctx* ctx, void* out, glb_extract_stats* stats);

/* Pipelining (Extract || Sample, "pipelining mechanism ... to overlap
 * the Extract and Train stages", L217 the Sampler/Trainer queue): depth 2 double-buffers
 * the sample slots; glb_extract_sample then runs on the ctx's extract stream, ordered
 * after everything enqueued on the main stream before the call (the sample it reads,
 * the caller's allocation of `out`), while the next glb_sample_batch proceeds on the
 * main stream (it waits only for the extract that last read its slot).  The caller
 * must order its reads of `out` after the extract stream (glb_extract_stream).  depth 1 (default): all
 * work on the main stream.  Synchronous. */
glb_status glb_set_pipeline(glb_ctx* ctx, int depth);
glb_status glb_extract_stream(glb_ctx* ctx, void** cuda_stream_out);
/* Host-assisted misses (L252: the Trainer extracts "from host memory and the feature cache
 * in GPU memory" simultaneously; L79: Extract is bound by the host link).  glb_extract_sample
 * orders a batch's misses by host address; the extract kernel reads the first (1 - fraction)
 * of them from the mapped host matrix (zero copy), while `threads` host threads copy the rest
 * into a pinned staging buffer that the GPU then reads sequentially and scatters into `out`
 * -- random 512-byte zero-copy reads are bound by per-row address translation, the staged
 * rows are not, and the two streams share the link.  Asynchronous: the host
 * copies run in stream host functions (no host sync in the caller).  Results are identical
 * for every fraction.  fraction 0 = off (default; environment GLB_HOST_GATHER = permille,
 * GLB_HOST_GATHER_THREADS); threads 0 = the usable cores minus two.  Applies to samples of
 * this ctx (not to handoff-received ones) and to caches with C < V.  Synchronous (creates the
 * thread pool and sizes the pinned staging for the sampler config -- again at every
 * glb_set_sampler -- so no extract allocates).  Errors: EINVAL (fraction not in [0,1), threads > 256). */
glb_status glb_set_host_gather(glb_ctx* ctx, uint32_t threads, double fraction);
/* Cold store: at the next glb_build_cache (single-GPU cache), copy the rows NOT cached --
 * ranks C..V-1 of the load_cache order (L301) -- into a pinned host buffer in rank order and
 * read misses from it instead of the caller's gid-ordered matrix: a batch's misses then
 * touch fewer 2 MB host regions, the unit the zero-copy link pays for.  Costs
 * (V - C) x D x 4 bytes of pinned host memory and a host copy at build time (the load_cache
 * phase, Table 6).  Results are identical.  enable 0 drops it.  Environment GLB_COLD_STORE=1.
 * Best effort: when the copy would leave less than 16 GB of MemAvailable, or pinning it fails,
 * no cold store is built (a note on stderr; glb_cold_store_rows reports 0) and the misses read
 * the caller's matrix -- load_cache still returns GLB_OK.
 * glb_cold_store_rows: rows held (0 = none).  Synchronous. */
glb_status glb_set_cold_store(glb_ctx* ctx, int enable);
glb_status glb_cold_store_rows(const glb_ctx* ctx, uint64_t* rows);
glb_status glb_host_gather(const glb_ctx* ctx, uint32_t* threads, double* fraction);

/* Timing of the extract kernel itself: CUDA events around every `period`-th
 * glb_extract_sample launch (period 1 = each; 0 = off), on the stream it runs on -- events
 * between the launches of a pipelined step cost overlap, so a bench samples them.
 * glb_extract_times synchronises, returns the durations in call order (up to max) and
 * resets the record; glb_set_timing restarts the call count (the first call is timed). */
glb_status glb_set_timing(glb_ctx* ctx, int period);
glb_status glb_extract_times(glb_ctx* ctx, float* out_ms, uint64_t max, uint64_t* n);

/* ------------------------------------------ a8: factored Sampler -> Trainer handoff (peer memory)
 * GNNLab's Samplers put each mini-batch's samples into a global queue from which a Trainer
 * takes them and extracts their features (Fig 9 L217-L246, L250-L252 §5.2; Table 5 "C").
 * Here the queue slots live in the TRAINER's HBM: a ring of `slots` receive slots, each sized
 * for the largest sample of the trainer's sampler config (glb_set_sampler; samplers must use
 * the same kind / hops and no larger capacities).  A sampler's GPU writes a finished sample
 * (sizes, uniq, every block's indptr / indices / weights) into a slot with ONE copy kernel --
 * over NVLink when the ranks are on different GPUs, through CUDA IPC when they are different
 * processes -- and the trainer marks and extracts it locally.  Ordering is device-side through
 * interprocess CUDA events (no host sync on either side); the caller's control plane decides
 * which batch goes to which (trainer, slot) and must order:
 *   a sampler's glb_handoff_send(t, s) for a slot's k-th use after the trainer's
 *     glb_handoff_release(s) of its (k-1)-th use was CALLED (host order), and
 *   the trainer's glb_handoff_recv(p, s) after sampler p's glb_handoff_send(t, s) was CALLED.
 * Blobs are GLB_HANDOFF_BLOB_BYTES opaque bytes to exchange between processes (e.g. all-gathered
 * over torch.distributed); a peer in the same process is recognised and used directly.
 * Ids (trainer, sampler) are caller-chosen in [0, GLB_HANDOFF_MAX_PEERS), e.g. ranks.
 * glb_set_sampler and glb_destroy drop the ring and every attachment; a ctx must not be
 * destroyed (or re-configured) while a peer may still use its ring or events -- callers
 * synchronise and barrier first. */
#define GLB_HANDOFF_MAX_SLOTS 8
#define GLB_HANDOFF_MAX_PEERS 16
#define GLB_HANDOFF_BLOB_BYTES 2048
/* trainer: allocate the ring (device) and its "consumed" events; blob_out receives the ring's
 * IPC handle, layout and event handles.  Synchronous.  Errors: EINVAL (slots not in
 * [1, GLB_HANDOFF_MAX_SLOTS]), ESTATE (no sampler config), ENOMEM. */
glb_status glb_handoff_create(glb_ctx* ctx, uint32_t slots, void* blob_out);
/* sampler: map trainer `trainer`'s ring from its blob and create this sampler's "ready"
 * events; blob_out receives their handles for glb_handoff_connect.  Synchronous.  Errors:
 * EINVAL (bad blob; ring smaller than this sampler's capacity or other hop count / kind). */
glb_status glb_handoff_attach(glb_ctx* ctx, uint32_t trainer, const void* trainer_blob,
                              void* blob_out);
/* trainer: open sampler `sampler`'s ready events from the blob glb_handoff_attach returned. */
glb_status glb_handoff_connect(glb_ctx* ctx, uint32_t sampler, const void* sampler_blob);
/* sampler: push the current sample (the last glb_sample*) into slot `slot` of trainer
 * `trainer` after the trainer's last release of that slot; `tag` (e.g. the global batch id)
 * travels in the slot header.  Asynchronous on the ctx stream.  Errors: ESTATE (not attached,
 * no sample), EINVAL (slot out of range, hop count mismatch). */
glb_status glb_handoff_send(glb_ctx* ctx, uint32_t trainer, uint32_t slot, uint64_t tag);
/* trainer: make slot `slot` (filled by sampler `sampler`) the ctx's current sample: wait for
 * the push, mark it against THIS ctx's cache (a4: slot map -> hit / miss lists, cache_slot),
 * so glb_sample_result / glb_extract_sample read it in place.  Asynchronous. */
glb_status glb_handoff_recv(glb_ctx* ctx, uint32_t sampler, uint32_t slot);
/* trainer: the tag of the current received sample (synchronous read). */
glb_status glb_handoff_tag(glb_ctx* ctx, uint64_t* out);
/* trainer: the slot may be overwritten once everything enqueued so far on the ctx stream
 * (and, at pipeline depth 2, its extract stream) has run; if it held the current sample,
 * the ctx has no current sample afterwards.  Asynchronous. */
glb_status glb_handoff_release(glb_ctx* ctx, uint32_t slot);

/* launch counter: number of kernels this ctx launched so far (bench evidence) */
uint64_t glb_kernel_launches(const glb_ctx* ctx);

#ifdef __cplusplus
}
#endif
#endif
