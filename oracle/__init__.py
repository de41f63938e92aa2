"""CPU ORACLE for the GNNLab sample+extract hot path -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product path (``paper_conf_eurosys_yangtswycyz22_b200``) never imports it and
shares no code with it.

Layers:
  * ``oracle.c`` -- plain single-threaded C: Philox, bounded, shuffle,
    k-hop Floyd sampling, random walk, first-occurrence relabel, extract.
  * this file -- ctypes marshalling plus the whole-epoch definitions written
    with numpy primitives: PreSC counts (§6.3), the top
    alpha|V| cache ranking (L301 §6.1), hit rate and the Optimal policy's
    hit rate (L148 footnote 4, L339).

Pins (tests/test_oracle_*.py): Random123 KATs, the SURVEY §8(c) worked
example, brute-force enumeration + chi-square of Floyd, BFS closed form at
fanout >= max degree, random-walk closed forms on paths/stars, relabel
invariants, brute-force optimal cache on tiny graphs, closed-form features.
"Parity unpinned" items are listed in DESIGN.md: the relabel order and the
RNG counter layout are this build's conventions (the paper fixes neither).
"""
from __future__ import annotations

import ctypes
import dataclasses
import math
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")
_HDR = os.path.join(_HERE, "oracle.h")

SHUFFLE, KHOP, RWALK = 1, 2, 3
EINVAL, ENOMEM, ERANGE = -1, -2, -5
EMPTY = 0xFFFFFFFF


def build(force: bool = False) -> str:
    newest = max(os.path.getmtime(_SRC), os.path.getmtime(_HDR))
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < newest:
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-o", _SO, _SRC])
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        u64, u32, i32, vp = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int, ctypes.c_void_p
        L.orc_philox.argtypes = [vp, vp, vp]
        L.orc_philox.restype = None
        L.orc_c3.argtypes = [u32, u32, u32]
        L.orc_c3.restype = u32
        L.orc_draw64.argtypes = [u64, u32, u32, u32, u32, i32]
        L.orc_draw64.restype = u64
        L.orc_bounded.argtypes = [u64, u32]
        L.orc_bounded.restype = u32
        L.orc_shuffle.argtypes = [vp, u64, u64, u32, vp]
        L.orc_shuffle.restype = i32
        L.orc_sample_khop.argtypes = [vp, vp, u64, vp, u64, vp, u32, u64, u32, u32, vp,
                                      vp, u64, vp, vp, u64, vp, u64, vp, vp, u64]
        L.orc_sample_khop.restype = i32
        L.orc_sample_rwalk.argtypes = [vp, vp, u64, vp, u64, u32, u32, u32, u32, u64, u32, u32,
                                       vp, vp, u64, vp, vp, u64, vp, vp, u64, vp]
        L.orc_sample_rwalk.restype = i32
        L.orc_extract.argtypes = [vp, u64, u32, vp, u64, vp]
        L.orc_extract.restype = i32
        L.orc_sample_khop_weighted.argtypes = [vp, vp, vp, u64, vp, u64, vp, u32, u64, u32, u32,
                                               vp, vp, u64, vp, vp, u64, vp, u64, vp]
        L.orc_sample_khop_weighted.restype = i32
        L.orc_policy_random.argtypes = [u64, u64, vp]
        L.orc_policy_random.restype = None
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data


# ---------------------------------------------------------------- RNG
def philox(ctr, key):
    c = np.ascontiguousarray(ctr, dtype=np.uint32)
    k = np.ascontiguousarray(key, dtype=np.uint32)
    out = np.empty(4, dtype=np.uint32)
    lib().orc_philox(_p(c), _p(k), _p(out))
    return out


def c3(epoch, hop, domain):
    return lib().orc_c3(epoch, hop, domain)


def draw64(seed, c0, c1, c2, c3_, half):
    return lib().orc_draw64(seed, c0, c1, c2, c3_, half)


def bounded(r, n):
    return lib().orc_bounded(r, n)


def feature_value(seed: int, v: int, d: int) -> np.float32:
    """Closed form of the generator's features (DESIGN.md input recipe):
    f(v,d) = ((draw64(v,d,0,c3(0,0,FEATURES=6),0) >> 40) * 2^-23) - 1, exact in f32."""
    r = draw64(seed, v, d, 0, c3(0, 0, 6), 0)
    return np.float32(np.float32(r >> 40) * np.float32(2.0 ** -23) - np.float32(1.0))


class OracleError(RuntimeError):
    def __init__(self, rc):
        super().__init__(f"oracle rc={rc}")
        self.rc = rc


# ---------------------------------------------------------------- a1
def shuffle(T: np.ndarray, seed: int, epoch: int) -> np.ndarray:
    T = np.ascontiguousarray(T, dtype=np.uint32)
    out = np.empty_like(T)
    rc = lib().orc_shuffle(_p(T), T.shape[0], seed, epoch, _p(out))
    if rc:
        raise OracleError(rc)
    return out


def epoch_batches(T: np.ndarray, batch: int, seed: int, epoch: int):
    """Mini-batches of one epoch: shuffle, then consecutive slices of size
    ``batch``, the last one partial (drop_last = False)."""
    perm = shuffle(T, seed, epoch)
    return [perm[b:b + batch] for b in range(0, perm.shape[0], batch)]


# ---------------------------------------------------------------- samples
@dataclasses.dataclass
class Sample:
    uniq: np.ndarray                # u32[n_L], gid by lid
    sizes: list                     # n_0..n_L
    indptr: list                    # per hop u32[n_l+1]
    indices: list                   # per hop u32[nnz_l] (src lids)
    weights: list | None = None     # per hop u32[nnz_l] (random walk only)
    picks: list | None = None       # per hop u32[n_l*k] CSR positions (k-hop only)


def _caps(n0: int, V: int, fanouts):
    ub = [n0]
    for k in fanouts:
        ub.append(min(ub[-1] * (1 + k), V))
    uniq_cap = max(ub[-1], 1)
    indptr_cap = sum(ub[l] + 1 for l in range(len(fanouts))) + 1
    indices_cap = sum(ub[l] * k for l, k in enumerate(fanouts)) + 1
    return uniq_cap, indptr_cap, indices_cap


class GraphOracle:
    """Holds a graph (host CSR) and the oracle's lid scratch array."""

    def __init__(self, indptr: np.ndarray, indices: np.ndarray, features: np.ndarray | None = None):
        self.indptr = np.ascontiguousarray(indptr, dtype=np.uint64)
        self.indices = np.ascontiguousarray(indices, dtype=np.uint32)
        self.V = self.indptr.shape[0] - 1
        self.features = features
        self.lid = np.full(max(self.V, 1), -1, dtype=np.int32)

    # a2 + a3
    def sample_khop(self, seeds, fanouts, seed, epoch, batch, want_picks=False) -> Sample:
        seeds = np.ascontiguousarray(seeds, dtype=np.uint32)
        fan = np.ascontiguousarray(fanouts, dtype=np.uint32)
        L = fan.shape[0]
        ucap, pcap, icap = _caps(seeds.shape[0], self.V, list(fan))
        uniq = np.empty(ucap, np.uint32)
        sizes = np.zeros(L + 1, np.uint64)
        bptr = np.empty(pcap, np.uint32)
        bidx = np.empty(icap, np.uint32)
        nnz = np.zeros(max(L, 1), np.uint64)
        kcap = sum(min(seeds.shape[0] * int(np.prod(1 + fan[:l])), self.V) * int(fan[l])
                   for l in range(L)) + 1
        picks = np.empty(kcap, np.uint32) if want_picks else None
        rc = lib().orc_sample_khop(_p(self.indptr), _p(self.indices), self.V, _p(seeds),
                                   seeds.shape[0], _p(fan), L, seed, epoch, batch, _p(self.lid),
                                   _p(uniq), ucap, _p(sizes), _p(bptr), pcap, _p(bidx), icap,
                                   _p(nnz), _p(picks) if want_picks else None,
                                   kcap if want_picks else 0)
        if rc:
            raise OracleError(rc)
        return self._split(uniq, sizes, bptr, bidx, nnz, L, None,
                           picks=picks, fanouts=list(fan) if want_picks else None)

    # NEXT-1 weighted k-hop + a3
    def sample_khop_weighted(self, weights, seeds, fanouts, seed, epoch, batch) -> Sample:
        w = np.ascontiguousarray(weights, dtype=np.uint32)
        seeds = np.ascontiguousarray(seeds, dtype=np.uint32)
        fan = np.ascontiguousarray(fanouts, dtype=np.uint32)
        L = fan.shape[0]
        ub = [seeds.shape[0]]
        for k in fan:
            ub.append(min(ub[-1] * (1 + int(k)), self.V))
        ucap = max(ub[-1], 1)
        pcap = sum(ub[l] + 1 for l in range(L)) + 1
        icap = sum(ub[l] * int(k) for l, k in enumerate(fan)) + 1
        uniq = np.empty(ucap, np.uint32)
        sizes = np.zeros(L + 1, np.uint64)
        bptr = np.empty(pcap, np.uint32)
        bidx = np.empty(icap, np.uint32)
        nnz = np.zeros(max(L, 1), np.uint64)
        rc = lib().orc_sample_khop_weighted(_p(self.indptr), _p(self.indices), _p(w), self.V,
                                            _p(seeds), seeds.shape[0], _p(fan), L, seed, epoch,
                                            batch, _p(self.lid), _p(uniq), ucap, _p(sizes),
                                            _p(bptr), pcap, _p(bidx), icap, _p(nnz))
        if rc:
            raise OracleError(rc)
        return self._split(uniq, sizes, bptr, bidx, nnz, L, None)

    # a2' + a3
    def sample_rwalk(self, seeds, layers, seed, epoch, batch, walks=4, walk_len=3,
                     topk=5) -> Sample:
        seeds = np.ascontiguousarray(seeds, dtype=np.uint32)
        ucap, pcap, icap = _caps(seeds.shape[0], self.V, [topk] * layers)
        uniq = np.empty(ucap, np.uint32)
        sizes = np.zeros(layers + 1, np.uint64)
        bptr = np.empty(pcap, np.uint32)
        bidx = np.empty(icap, np.uint32)
        bw = np.empty(icap, np.uint32)
        nnz = np.zeros(max(layers, 1), np.uint64)
        rc = lib().orc_sample_rwalk(_p(self.indptr), _p(self.indices), self.V, _p(seeds),
                                    seeds.shape[0], layers, walks, walk_len, topk, seed, epoch,
                                    batch, _p(self.lid), _p(uniq), ucap, _p(sizes), _p(bptr), pcap,
                                    _p(bidx), _p(bw), icap, _p(nnz))
        if rc:
            raise OracleError(rc)
        return self._split(uniq, sizes, bptr, bidx, nnz, layers, bw)

    @staticmethod
    def _split(uniq, sizes, bptr, bidx, nnz, L, bw, picks=None, fanouts=None):
        sizes = [int(x) for x in sizes]
        ips, ixs, ws, pks = [], [], [], []
        po = io = ko = 0
        for l in range(L):
            n_l = sizes[l]
            ips.append(bptr[po:po + n_l + 1].copy())
            m = int(nnz[l])
            ixs.append(bidx[io:io + m].copy())
            if bw is not None:
                ws.append(bw[io:io + m].copy())
            if picks is not None:
                pks.append(picks[ko:ko + n_l * fanouts[l]].copy())
                ko += n_l * fanouts[l]
            po += n_l + 1
            io += m
        return Sample(uniq[:sizes[-1]].copy(), sizes, ips, ixs, ws if bw is not None else None,
                      pks if picks is not None else None)

    def sample(self, sampler: str, seeds, fanouts, seed, epoch, batch, weights=None) -> Sample:
        if sampler == "khop":
            return self.sample_khop(seeds, fanouts, seed, epoch, batch)
        if sampler == "weighted":
            return self.sample_khop_weighted(weights, seeds, fanouts, seed, epoch, batch)
        return self.sample_rwalk(seeds, len(fanouts), seed, epoch, batch, topk=fanouts[0])

    # a7
    def extract(self, vertices) -> np.ndarray:
        v = np.ascontiguousarray(vertices, dtype=np.uint32)
        F = self.features
        D = F.shape[1]
        out = np.empty((v.shape[0], D), np.float32)
        rc = lib().orc_extract(_p(F), self.V, D, _p(v), v.shape[0], _p(out))
        if rc:
            raise OracleError(rc)
        return out

    # a5: PreSC#K (L333: "records the visit count of the sampled vertices";
    # reading Q8/Q9: one visit per (batch, unique vertex), epochs 0..K-1)
    def visit_counts(self, sampler, train, batch_size, fanouts, seed, epochs,
                     batch_filter=None, weights=None) -> np.ndarray:
        counts = np.zeros(self.V, np.uint32)
        for e in epochs:
            for b, seeds in enumerate(epoch_batches(train, batch_size, seed, e)):
                if batch_filter is not None and not batch_filter(e, b):
                    continue
                s = self.sample(sampler, seeds, fanouts, seed, e, b, weights)
                counts[s.uniq] += 1       # uniq is duplicate-free
        return counts

    def presample(self, sampler, train, batch_size, fanouts, seed, K, weights=None) -> np.ndarray:
        return self.visit_counts(sampler, train, batch_size, fanouts, seed, range(K),
                                 weights=weights)


# ---------------------------------------------------------------- a6
def cache_size(alpha: float, V: int) -> int:
    """C = floor(alpha * |V|) in IEEE double (L301 "top-ranked alpha|V|"; reading Q10)."""
    if not (0.0 <= alpha <= 1.0):
        raise ValueError("alpha must be in [0,1]")
    return int(math.floor(alpha * float(V)))


def cache_rank(counts: np.ndarray) -> np.ndarray:
    """Vertices ordered by hotness: count descending, gid ascending (reading Q10).
    A stable sort of -count over gid order is exactly that order."""
    return np.argsort(-counts.astype(np.int64), kind="stable").astype(np.uint32)


def cache_slots(counts: np.ndarray, alpha: float) -> np.ndarray:
    """load_cache(hotness_map, alpha) (L301): slot[rank[i]] = i for i < C, else -1."""
    V = counts.shape[0]
    C = cache_size(alpha, V)
    slot = np.full(V, -1, np.int32)
    order = cache_rank(counts)
    slot[order[:C]] = np.arange(C, dtype=np.int32)
    return slot


# ---------------------------------------------------------------- NEXT-3 sharded cache
def sharded_cache(counts: np.ndarray, alpha: float, world: int):
    """Peer-sharded load_cache (the paper's cross-GPU access, L516 §9):
    `world` GPUs each hold floor(alpha*V) rows, so C = min(V, world*floor(alpha*V))
    distinct rows are cached; the vertex of rank i < C (ranking of L301, reading Q10) has
    global slot i and lives on shard i % world at row i // world.
    Returns (slot i32[V], [rows of shard r: vertex ids in row order, r < world])."""
    V = counts.shape[0]
    C = min(V, world * cache_size(alpha, V))
    order = cache_rank(counts)
    slot = np.full(V, -1, np.int32)
    slot[order[:C]] = np.arange(C, dtype=np.int32)
    shards = [order[:C][r::world] for r in range(world)]
    return slot, shards


def extract_counts(vertices: np.ndarray, slot: np.ndarray, rank: int = 0, world: int = 1):
    """(hits, misses, peer_hits) of one extract on shard `rank`: a hit is a cached vertex
    (L252); a peer hit is one whose row lives on another GPU's shard."""
    s = slot[np.asarray(vertices, dtype=np.int64)]
    hit = s >= 0
    peer = hit & ((s % world) != rank)
    return int(hit.sum()), int((~hit).sum()), int(peer.sum())


# ---------------------------------------------------------------- policies (Fig 10)
def hotness_degree(indptr: np.ndarray) -> np.ndarray:
    """Degree policy (PaGraph; L79, L301): h_v = out-degree."""
    d = np.diff(indptr.astype(np.uint64))
    return np.minimum(d, np.uint64(0xFFFFFFFF)).astype(np.uint32)


def hotness_random(seed: int, V: int) -> np.ndarray:
    """Random policy (L442): a uniformly random order, one draw per vertex."""
    out = np.empty(V, np.uint32)
    lib().orc_policy_random(seed, V, _p(out))
    return out


def footprint_similarity(f_i: np.ndarray, f_j: np.ndarray, top_frac: float = 0.1):
    """Table 2 (L329, reading Q16): sum_{v in T_i & T_j} min(f_i, f_j) / sum_{v in T_j} f_j,
    T_x = the floor(top_frac*V) vertices ranked first by (f_x desc, gid asc).
    Returns (value, numerator, denominator)."""
    C = cache_size(top_frac, f_i.shape[0])
    ti = np.zeros(f_i.shape[0], bool)
    tj = np.zeros(f_j.shape[0], bool)
    ti[cache_rank(f_i)[:C]] = True
    tj[cache_rank(f_j)[:C]] = True
    both = ti & tj
    num = int(np.minimum(f_i[both], f_j[both]).astype(np.uint64).sum())
    den = int(f_j[tj].astype(np.uint64).sum())
    return (num / den if den else 0.0), num, den


# ---------------------------------------------------------------- metric
def hit_rate(acc: np.ndarray, slot: np.ndarray) -> float:
    """H = accesses served by the cache / all accesses (Table 5 H%, L414)."""
    tot = int(acc.sum(dtype=np.uint64))
    return float(int(acc[slot >= 0].sum(dtype=np.uint64))) / tot if tot else 0.0


def optimal_hit_rate(acc: np.ndarray, C: int) -> float:
    """Optimal policy (L148 footnote 4): cache the C most visited vertices of
    the recorded footprints; H* = their accesses / all accesses."""
    tot = int(acc.sum(dtype=np.uint64))
    if tot == 0 or C == 0:
        return 0.0
    top = np.sort(acc.astype(np.uint64))[::-1][:C]
    return float(int(top.sum())) / tot
