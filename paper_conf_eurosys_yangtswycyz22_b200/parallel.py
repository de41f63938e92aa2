"""Multi-GPU orchestration of the sample+extract path (one process per GPU).

Two modes, both over ``torch.distributed`` (NCCL on GPUs, gloo in CPU tests):

* **DP** (default): mini-batch g of an epoch goes to rank
  g mod N (static) -- every draw is keyed by (epoch, batch), so per-batch
  outputs are identical on any rank.  The only collective is the sum
  all-reduce of the u32 PreSC counts (and of measured-epoch access counts for
  the hit-rate metric): integer sums, bit-identical at every N.

* **Factored** (§5.2-5.3): Ns sampler ranks and
  Nt = N - Ns trainer ranks.  Ns = ceil(N / (K + 1)) with K = Tt / Ts from a
  profiled warm-up (L262-L263; Tt is the trainer's per-batch time, which on
  this path is Extract, L438).  A global scheduler hands batches to samplers
  dynamically without synchronisation (L250): a host-side atomic counter in
  the process group's store.  Batch g is extracted by trainer g mod Nt; the
  sampler that produced it publishes (g -> sampler rank) in the store (the
  "global queue" descriptor, L217) and sends a fixed-size header and one
  flat payload (uniq gids, block CSRs) with point-to-point send/recv.

The sampler/trainer roles talk to a ``ctx`` through a narrow interface so
CPU tests can drive the protocol with a stand-in sampler (tests/test_parallel.py).
"""
from __future__ import annotations

import dataclasses
import math

import torch
import torch.distributed as dist

HEADER_WORDS = 32  # int64: [batch, epoch, L, n_0..n_L, nnz_0..nnz_{L-1}, weighted, ...]


# ----------------------------------------------------------------------------- DP
def dp_batches(num_batches: int, rank: int, world: int):
    """Batches of one epoch owned by ``rank`` (round-robin, L252 data parallelism)."""
    return list(range(rank, num_batches, world))


def dp_step_batch(i: int, rank: int, world: int, num_batches: int, first_epoch: int):
    """(epoch, batch) of this rank's i-th step when epochs are consumed in order."""
    g = i * world + rank
    return first_epoch + g // num_batches, g % num_batches


def allreduce_counts(t: torch.Tensor, group=None):
    """Sum u32 visit counts across ranks (int32 view; sums stay < 2^31).

    On CUDA the host waits for the reduction before returning: the library's
    next call (build_cache ranks the counts) may run on a stream that is not
    ordered after NCCL's, so every rank must see the fully reduced counts."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
        if t.is_cuda:
            torch.cuda.synchronize(t.device)
    return t


def presample_dp(ctx, K: int, rank: int, world: int, group=None):
    """PreSC#K sharded by batch, then the count all-reduce."""
    ctx.presample(K, rank, world)
    allreduce_counts(ctx.counts_tensor(1), group)


def build_sharded_cache(ctx, alpha: float, rank: int, world: int, group=None):
    """NEXT-3: each rank caches floor(alpha*V) distinct rows -- the
    ranks i with i % world == rank of the PreSC order -- and maps every other rank's
    shard through CUDA IPC (over NVLink on a multi-GPU box), so the group caches
    world*alpha*|V| rows instead of alpha*|V| replicated ones.  The handles travel as
    64-byte blobs over the process group; the closing barrier guarantees every shard is
    mapped before anyone extracts.  Callers must barrier again before any rank rebuilds
    or frees its shard (peers may still be reading it)."""
    ctx.build_cache_sharded(alpha, rank, world)
    if world == 1:
        return
    handles = [None] * world
    dist.all_gather_object(handles, ctx.cache_ipc_handle(), group=group)
    for p, h in enumerate(handles):
        if p != rank:
            ctx.attach_peer_cache(p, ipc_handle=h)
    dist.barrier(group=group)


# ----------------------------------------------------------------------------- factored
def num_samplers(n_gpus: int, t_sample: float, t_train: float) -> int:
    """Ns = ceil(Ng / (K + 1)), K = Tt / Ts; at least one of each
    role when n_gpus >= 2."""
    if n_gpus <= 1:
        return n_gpus
    K = t_train / max(t_sample, 1e-12)
    ns = math.ceil(n_gpus / (K + 1.0))
    return min(max(ns, 1), n_gpus - 1)


@dataclasses.dataclass
class Roles:
    n_samplers: int
    world: int

    @property
    def n_trainers(self):
        return self.world - self.n_samplers

    def is_sampler(self, rank):
        return rank < self.n_samplers

    def trainer_rank(self, g: int) -> int:
        """Trainer (global rank) that extracts batch g."""
        return self.n_samplers + g % self.n_trainers

    def trainer_batches(self, rank: int, total: int):
        t = rank - self.n_samplers
        return list(range(t, total, self.n_trainers))


def pack_header(g: int, epoch: int, sizes, nnz, weighted: bool, device) -> torch.Tensor:
    h = torch.zeros(HEADER_WORDS, dtype=torch.int64)
    L = len(nnz)
    assert 4 + 2 * L + 1 <= HEADER_WORDS
    h[0], h[1], h[2], h[3] = g, epoch, L, int(weighted)
    h[4:5 + L] = torch.tensor(sizes, dtype=torch.int64)
    h[5 + L:5 + 2 * L] = torch.tensor(nnz, dtype=torch.int64)
    return h.to(device)


def unpack_header(h: torch.Tensor):
    h = h.cpu().tolist()
    g, epoch, L, weighted = h[0], h[1], h[2], bool(h[3])
    sizes = h[4:5 + L]
    nnz = h[5 + L:5 + 2 * L]
    return g, epoch, sizes, nnz, weighted


def payload_len(sizes, nnz, weighted) -> int:
    L = len(nnz)
    n = sizes[-1] + sum(sizes[l] + 1 for l in range(L)) + sum(nnz)
    return n + (sum(nnz) if weighted else 0)


def pack_payload(blocks) -> torch.Tensor:
    """uniq | indptr_0..L-1 | indices_0..L-1 | (weights_0..L-1), int32, contiguous."""
    parts = [blocks.uniq] + list(blocks.indptr) + list(blocks.indices)
    if blocks.weights is not None:
        parts += list(blocks.weights)
    return torch.cat([p.reshape(-1).to(torch.int32) for p in parts])


def unpack_payload(buf: torch.Tensor, sizes, nnz, weighted):
    L = len(nnz)
    o = 0
    uniq = buf[o:o + sizes[-1]]
    o += sizes[-1]
    indptr = []
    for l in range(L):
        indptr.append(buf[o:o + sizes[l] + 1])
        o += sizes[l] + 1
    indices = []
    for l in range(L):
        indices.append(buf[o:o + nnz[l]])
        o += nnz[l]
    weights = None
    if weighted:
        weights = []
        for l in range(L):
            weights.append(buf[o:o + nnz[l]])
            o += nnz[l]
    return uniq, indptr, indices, weights


class GlobalScheduler:
    """Dynamic batch assignment to samplers without synchronisation (L250): an atomic
    counter in the process group's key-value store."""

    def __init__(self, store, key: str):
        self.store = store
        self.key = key

    def next(self) -> int:
        return int(self.store.add(self.key, 1)) - 1


def run_sampler(sample_fn, roles: Roles, rank: int, total: int, store, tag: str, device):
    """Sampler executor (Fig 9): pull batch ids, sample, publish the
    descriptor, send header + payload to the batch's trainer.  Returns #batches."""
    sched = GlobalScheduler(store, f"{tag}/next")
    done = 0
    while True:
        g = sched.next()
        if g >= total:
            break
        epoch, blocks = sample_fn(g)
        weighted = blocks.weights is not None
        store.set(f"{tag}/src/{g}", str(rank))
        dst = roles.trainer_rank(g)
        dist.send(pack_header(g, epoch, blocks.sizes, blocks.nnz, weighted, device), dst)
        dist.send(pack_payload(blocks).to(device), dst)
        done += 1
    return done


def run_trainer(extract_fn, roles: Roles, rank: int, total: int, store, tag: str, device):
    """Trainer executor (Fig 9): for each batch it owns, find the sampler
    through the global queue, receive the samples, extract.  Returns #batches."""
    n = 0
    for g in roles.trainer_batches(rank, total):
        src = int(store.get(f"{tag}/src/{g}"))  # blocks until the descriptor exists
        h = torch.empty(HEADER_WORDS, dtype=torch.int64, device=device)
        dist.recv(h, src)
        g2, epoch, sizes, nnz, weighted = unpack_header(h)
        assert g2 == g, (g2, g)
        buf = torch.empty(payload_len(sizes, nnz, weighted), dtype=torch.int32, device=device)
        dist.recv(buf, src)
        extract_fn(g, epoch, sizes, nnz, unpack_payload(buf, sizes, nnz, weighted))
        n += 1
    return n


# ----------------------------------------------------- factored, peer-memory handoff (a8)
class PeerHandoff:
    """The factored handoff over peer memory (include/glb.h glb_handoff_*): every trainer
    owns a ring of ``slots`` receive slots in its HBM; a sampler's GPU pushes a finished
    sample into one with a single copy kernel (NVLink between GPUs, CUDA IPC between
    processes) and the trainer extracts it in place -- the B200 replacement of the
    send/recv above (no payload packing, no host staging, no host sync on the sampler).

    Batch g goes to trainer ``roles.trainer_rank(g)``, slot ``(g // Nt) % slots``, so batch
    g reuses the slot of batch g - Nt*slots.  The control plane is the process group's
    store (the paper's global queue, L217): ``{tag}/src/{g}`` = the sampler that pushed g
    (set after its push was enqueued), ``{tag}/rel/{g}`` = g's slot was released (set after
    the trainer's release was enqueued).  Device-side order comes from the library's
    interprocess events; the store only orders the host calls that enqueue them."""

    def __init__(self, ctx, roles: Roles, rank: int, slots: int = 4, group=None):
        self.ctx, self.roles, self.rank, self.slots = ctx, roles, rank, slots
        self.standby = 0  # batches this rank extracted as a standby Trainer (switching)
        world = roles.world
        tblob = ctx.handoff_create(slots) if not roles.is_sampler(rank) else None
        tblobs = [None] * world
        dist.all_gather_object(tblobs, tblob, group=group)
        sblobs = {}
        if roles.is_sampler(rank):
            for t in range(roles.n_samplers, world):
                sblobs[t] = ctx.handoff_attach(t, tblobs[t])
        allsb = [None] * world
        dist.all_gather_object(allsb, sblobs, group=group)
        if not roles.is_sampler(rank):
            for s in range(roles.n_samplers):
                ctx.handoff_connect(s, allsb[s][rank])
        dist.barrier(group=group)

    def slot_of(self, g: int) -> int:
        return (g // self.roles.n_trainers) % self.slots


def switch_profit(m_r: int, t_t: float, n_t: int, t_standby: float) -> float:
    """Dynamic executor switching's profit metric (§5.3):
    P = M_r * T_t / N_t - T_t' if N_t > 0, +inf if N_t == 0 -- whether a standby Trainer
    (on a Sampler's GPU, time T_t' per batch) finishes one task before the N_t normal
    Trainers (T_t per batch) drain the M_r tasks remaining in the global queue."""
    if n_t <= 0:
        return math.inf
    return m_r * t_t / n_t - t_standby


def run_sampler_peer(sample_fn, ho: PeerHandoff, total: int, store, tag: str,
                     standby_fn=None, t_train: float = 0.0, t_standby: float = 0.0):
    """Sampler executor over peer memory: pull batch g from the global scheduler (L250),
    sample it (sample_fn(g) leaves it as the ctx's current sample), and push it into its
    trainer's slot once that slot's previous batch was released.

    Dynamic executor switching (L267-L277): when the slot is still busy -- the Trainers
    are behind and this Sampler would idle -- and a ``standby_fn`` is given, the GPU
    switches to a standby Trainer for this batch if the profit metric is positive
    (switch_profit with M_r = batches pushed but not yet extracted): standby_fn(g)
    extracts the batch locally and the global queue records it as done ("-1"), so its
    trainer skips it.  Returns #batches sampled; ho.standby counts the switched ones."""
    sched = GlobalScheduler(store, f"{tag}/next")
    reuse = ho.roles.n_trainers * ho.slots
    done = 0
    while True:
        g = sched.next()
        if g >= total:
            break
        sample_fn(g)
        done += 1
        if g >= reuse:
            rel = f"{tag}/rel/{g - reuse}"
            if standby_fn is not None and not store.check([rel]):
                m_r = int(store.add(f"{tag}/pushed", 0)) - int(store.add(f"{tag}/trained", 0))
                if switch_profit(m_r, t_train, ho.roles.n_trainers, t_standby) > 0:
                    standby_fn(g)
                    ho.standby += 1
                    store.set(f"{tag}/src/{g}", "-1")
                    continue
            store.get(rel)  # blocks until the slot was released
        ho.ctx.handoff_send(ho.roles.trainer_rank(g), ho.slot_of(g), g)
        store.add(f"{tag}/pushed", 1)
        store.set(f"{tag}/src/{g}", str(ho.rank))
    return done


def run_trainer_peer(extract_fn, ho: PeerHandoff, total: int, store, tag: str):
    """Trainer executor over peer memory: for each batch it owns, find its sampler in the
    global queue, make the pushed sample current (mark against this GPU's cache), let
    extract_fn(g) extract / consume it, release the slot.  A batch a standby Trainer took
    (queue entry "-1") is skipped; its slot was never written.  Returns #batches."""
    n = 0
    for g in ho.roles.trainer_batches(ho.rank, total):
        src = int(store.get(f"{tag}/src/{g}"))
        if src < 0:
            store.set(f"{tag}/rel/{g}", "1")
            continue
        s = ho.slot_of(g)
        ho.ctx.handoff_recv(src, s)
        extract_fn(g)
        ho.ctx.handoff_release(s)
        store.add(f"{tag}/trained", 1)
        store.set(f"{tag}/rel/{g}", "1")
        n += 1
    return n
