"""B200-native GNNLab sample+extract hot path (PAPER.md, EuroSys'22).

Thin Python binding over the C-ABI in ``include/glb.h`` (``libglb.so``,
sm_100a CUDA).  Argument marshalling only: every step of the path runs in the
library's kernels.  PyTorch is used for device memory of caller-owned outputs,
streams and process groups; ctx-owned device buffers are exposed to torch as
zero-copy views through ``__cuda_array_interface__``.

There is no CPU fallback: importing works anywhere, but creating a
``Context`` requires the compiled library and a CUDA device, and fails loudly
otherwise.
"""
from __future__ import annotations

import ctypes
import dataclasses
import os

import numpy as np

from .build import SO as _SO, build  # noqa: F401

KHOP, RWALK, KHOP_WEIGHTED = 0, 1, 2
POLICY_PRESC, POLICY_DEGREE, POLICY_RANDOM = 0, 1, 2
COUNT_NONE, COUNT_PRESAMPLE, COUNT_ACCESS = 0, 1, 2
MAX_HOPS = 8
OK, EINVAL, ENOMEM, ECUDA, ESTATE, ERANGE = 0, -1, -2, -3, -4, -5
_NAMES = {EINVAL: "EINVAL", ENOMEM: "ENOMEM", ECUDA: "ECUDA", ESTATE: "ESTATE", ERANGE: "ERANGE"}

# every symbol include/glb.h declares
EXPORTS = [
    "glb_last_error", "glb_create", "glb_destroy", "glb_set_stream", "glb_sync",
    "glb_load_graph", "glb_set_sampler", "glb_set_train_set", "glb_num_batches", "glb_shuffle",
    "glb_get_permutation", "glb_sample", "glb_sample_batch", "glb_sample_result",
    "glb_set_count_mode", "glb_reset_counts", "glb_presample", "glb_counts_device_ptr",
    "glb_get_counts", "glb_build_cache", "glb_get_cache_slots", "glb_cache_size",
    "glb_hit_stats_get", "glb_extract", "glb_extract_sample", "glb_kernel_launches",
    "glb_set_pipeline", "glb_extract_stream", "glb_set_timing", "glb_extract_times",
    "glb_set_relabel_mode", "glb_relabel_mode", "glb_policy_hotness", "glb_footprint_similarity",
    "glb_load_edge_weights", "glb_build_cache_sharded", "glb_cache_device_ptr",
    "glb_cache_ipc_handle", "glb_attach_peer_cache", "glb_last_extract_counts",
    "glb_sample_async", "glb_extract_counts_device_ptr",
    "glb_handoff_create", "glb_handoff_attach", "glb_handoff_connect", "glb_handoff_send",
    "glb_handoff_recv", "glb_handoff_tag", "glb_handoff_release", "glb_relabel_l2_window",
    "glb_set_host_gather", "glb_host_gather", "glb_set_cold_store", "glb_cold_store_rows",
]
MAX_SHARDS = 16
IPC_HANDLE_BYTES = 64
HANDOFF_MAX_SLOTS = 8
HANDOFF_MAX_PEERS = 16
HANDOFF_BLOB_BYTES = 2048


class GlbError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"{_NAMES.get(code, code)}: {msg}")
        self.code = code


class _Blocks(ctypes.Structure):
    _fields_ = [
        ("num_hops", ctypes.c_uint32),
        ("num_seeds", ctypes.c_uint32),
        ("uniq", ctypes.c_void_p),
        ("sizes", ctypes.c_uint64 * (MAX_HOPS + 1)),
        ("nnz", ctypes.c_uint64 * MAX_HOPS),
        ("indptr", ctypes.c_void_p * MAX_HOPS),
        ("indices", ctypes.c_void_p * MAX_HOPS),
        ("weights", ctypes.c_void_p * MAX_HOPS),
        ("cache_slot", ctypes.c_void_p),
    ]


class _HitStats(ctypes.Structure):
    _fields_ = [("total", ctypes.c_uint64), ("hits", ctypes.c_uint64),
                ("optimal_hits", ctypes.c_uint64), ("cache_rows", ctypes.c_uint64)]


class _XStats(ctypes.Structure):
    _fields_ = [("hits", ctypes.c_uint64), ("misses", ctypes.c_uint64)]


_lib = None


def lib(auto_build: bool = True):
    """Load libglb.so (building it in-tree if stale).  Raises if unavailable."""
    global _lib
    if _lib is not None:
        return _lib
    so = os.environ.get("GLB_LIBRARY")  # A/B builds (tools/ab_build.sh)
    if so is None:
        if auto_build:
            build()
        so = _SO
    if not os.path.exists(so):
        raise RuntimeError(f"{so} missing: run __graft_entry__.build()")
    L = ctypes.CDLL(so)
    vp, u32, u64, i32, dbl = (ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int,
                              ctypes.c_double)
    sig = {
        "glb_last_error": ([vp], ctypes.c_char_p),
        "glb_create": ([i32, ctypes.POINTER(vp)], i32),
        "glb_destroy": ([vp], i32),
        "glb_set_stream": ([vp, vp], i32),
        "glb_sync": ([vp], i32),
        "glb_load_graph": ([vp, u64, u64, vp, vp, vp, u32], i32),
        "glb_set_sampler": ([vp, i32, vp, u32, u32, u32, u32, u32], i32),
        "glb_set_train_set": ([vp, vp, u64, u32, u64], i32),
        "glb_num_batches": ([vp, ctypes.POINTER(u32)], i32),
        "glb_shuffle": ([vp, u32], i32),
        "glb_get_permutation": ([vp, vp], i32),
        "glb_sample": ([vp, vp, u32, vp, u32, u64, u32, u32, ctypes.POINTER(_Blocks)], i32),
        "glb_sample_batch": ([vp, u32, u32], i32),
        "glb_sample_result": ([vp, ctypes.POINTER(_Blocks)], i32),
        "glb_set_count_mode": ([vp, i32], i32),
        "glb_reset_counts": ([vp, i32], i32),
        "glb_presample": ([vp, u32, u32, u32], i32),
        "glb_counts_device_ptr": ([vp, i32, ctypes.POINTER(vp)], i32),
        "glb_get_counts": ([vp, i32, vp], i32),
        "glb_build_cache": ([vp, dbl, vp], i32),
        "glb_get_cache_slots": ([vp, vp], i32),
        "glb_cache_size": ([vp, ctypes.POINTER(u64)], i32),
        "glb_hit_stats_get": ([vp, ctypes.POINTER(_HitStats)], i32),
        "glb_extract": ([vp, vp, u64, vp, ctypes.POINTER(_XStats)], i32),
        "glb_extract_sample": ([vp, vp, ctypes.POINTER(_XStats)], i32),
        "glb_kernel_launches": ([vp], u64),
        "glb_set_pipeline": ([vp, i32], i32),
        "glb_extract_stream": ([vp, ctypes.POINTER(vp)], i32),
        "glb_set_timing": ([vp, i32], i32),
        "glb_extract_times": ([vp, vp, u64, ctypes.POINTER(u64)], i32),
        "glb_set_relabel_mode": ([vp, i32], i32),
        "glb_relabel_mode": ([vp, ctypes.POINTER(i32)], i32),
        "glb_relabel_l2_window": ([vp, ctypes.POINTER(u64)], i32),
        "glb_policy_hotness": ([vp, i32, u64, vp], i32),
        "glb_load_edge_weights": ([vp, vp], i32),
        "glb_build_cache_sharded": ([vp, dbl, vp, u32, u32], i32),
        "glb_cache_device_ptr": ([vp, ctypes.POINTER(vp), ctypes.POINTER(u64)], i32),
        "glb_cache_ipc_handle": ([vp, vp], i32),
        "glb_attach_peer_cache": ([vp, u32, vp, vp], i32),
        "glb_last_extract_counts": ([vp, ctypes.POINTER(u64)], i32),
        "glb_sample_async": ([vp, vp, u32, u64, u32, u32], i32),
        "glb_extract_counts_device_ptr": ([vp, ctypes.POINTER(vp)], i32),
        "glb_handoff_create": ([vp, u32, vp], i32),
        "glb_handoff_attach": ([vp, u32, vp, vp], i32),
        "glb_handoff_connect": ([vp, u32, vp], i32),
        "glb_handoff_send": ([vp, u32, u32, u64], i32),
        "glb_handoff_recv": ([vp, u32, u32], i32),
        "glb_handoff_tag": ([vp, ctypes.POINTER(u64)], i32),
        "glb_handoff_release": ([vp, u32], i32),
        "glb_set_host_gather": ([vp, u32, dbl], i32),
        "glb_set_cold_store": ([vp, i32], i32),
        "glb_cold_store_rows": ([vp, ctypes.POINTER(u64)], i32),
        "glb_host_gather": ([vp, ctypes.POINTER(u32), ctypes.POINTER(dbl)], i32),
        "glb_footprint_similarity": ([vp, vp, vp, dbl, ctypes.POINTER(u64), ctypes.POINTER(u64),
                                      ctypes.POINTER(dbl)], i32),
    }
    for name, (a, r) in sig.items():
        if os.environ.get("GLB_LIBRARY") and not hasattr(L, name):
            continue  # an older A/B build (tools/ab_build.sh) may predate a symbol
        f = getattr(L, name)
        f.argtypes = a
        f.restype = r
    _lib = L
    return L


class _CAI:
    """Zero-copy device view for torch.as_tensor (__cuda_array_interface__ v3)."""

    def __init__(self, ptr, shape, typestr, owner):
        self._owner = owner
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr,
                                         "data": (int(ptr or 0), False), "version": 3,
                                         "strides": None}


def _view(ptr, n, typestr, owner, device):
    import torch
    if n == 0 or not ptr:
        dt = {"<i4": torch.int32, "<u4": torch.int32, "<f4": torch.float32}[typestr]
        return torch.empty(0, dtype=dt, device=device)
    return torch.as_tensor(_CAI(ptr, (n,), typestr, owner), device=device)


@dataclasses.dataclass
class Blocks:
    """One sampled mini-batch (views into ctx-owned memory, valid until the next sample).

    uniq[lid] = gid (int32); the first sizes[l] lids are frontier l.  Block l:
    CSR with dst = lids 0..sizes[l]-1 and src lids in ``indices[l]``."""
    num_seeds: int
    sizes: list
    nnz: list
    uniq: object
    indptr: list
    indices: list
    weights: list | None
    cache_slot: object


def _np_ptr(a):
    return a.ctypes.data if a is not None else None


class Context:
    """One library context per (process, GPU)."""

    def __init__(self, device: int = 0):
        import torch
        self._lib = lib()
        self.device = torch.device("cuda", device)
        h = ctypes.c_void_p()
        rc = self._lib.glb_create(device, ctypes.byref(h))
        if rc != OK:
            raise GlbError(rc, self._lib.glb_last_error(None).decode())
        self._h = h
        self._keep = []
        self.V = 0
        self.D = 0
        # order every call after torch's work on this device (tensors handed in/out)
        self.set_stream(torch.cuda.current_stream(self.device))

    def _ck(self, rc):
        if rc != OK:
            raise GlbError(rc, self._lib.glb_last_error(self._h).decode())

    def close(self):
        if getattr(self, "_h", None):
            self._lib.glb_destroy(self._h)
            self._h = None
            self._keep = []

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ------------------------------------------------------------------ setup
    def set_stream(self, stream):
        """Run later calls on a torch.cuda.Stream (its handle; 0 = legacy default stream)."""
        self._ck(self._lib.glb_set_stream(self._h, stream.cuda_stream or None))

    def sync(self):
        self._ck(self._lib.glb_sync(self._h))

    def load_graph(self, indptr: np.ndarray, indices: np.ndarray, features: np.ndarray | None):
        indptr = np.ascontiguousarray(indptr, dtype=np.uint64)
        indices = np.ascontiguousarray(indices, dtype=np.uint32)
        V = indptr.shape[0] - 1
        D = 0
        if features is not None:
            assert features.dtype == np.float32 and features.flags.c_contiguous
            assert features.shape[0] == V
            D = features.shape[1]
        self._ck(self._lib.glb_load_graph(self._h, V, indices.shape[0], _np_ptr(indptr),
                                          _np_ptr(indices), _np_ptr(features), D))
        self._keep = [features]  # borrowed host memory must outlive the ctx registration
        self.V, self.D = V, D

    def load_edge_weights(self, weights: np.ndarray):
        """u32 per-edge weights (parallel to indices) for the 'weighted' sampler."""
        w = np.ascontiguousarray(weights, dtype=np.uint32)
        self._ck(self._lib.glb_load_edge_weights(self._h, _np_ptr(w)))

    def set_sampler(self, kind: str = "khop", fanouts=(25, 10), walks=4, walk_len=3, topk=5,
                    layers=None, max_batch=8000):
        k = {"khop": KHOP, "rwalk": RWALK, "weighted": KHOP_WEIGHTED}[kind]
        if k in (KHOP, KHOP_WEIGHTED):
            fan = np.ascontiguousarray(fanouts, dtype=np.uint32)
            L = fan.shape[0]
        else:
            L = layers if layers is not None else len(fanouts)
            fan = np.zeros(max(L, 1), np.uint32)
        self._ck(self._lib.glb_set_sampler(self._h, k, _np_ptr(fan), L, walks, walk_len, topk,
                                           max_batch))
        self.kind, self.L = kind, L

    def set_relabel_mode(self, mode: str):
        """'auto' | 'dense' | 'hash' -- relabel table for the next set_sampler."""
        self._ck(self._lib.glb_set_relabel_mode(self._h, {"auto": 0, "dense": 1, "hash": 2}[mode]))

    @property
    def relabel_mode(self) -> str:
        m = ctypes.c_int()
        self._ck(self._lib.glb_relabel_mode(self._h, ctypes.byref(m)))
        return {1: "dense", 2: "hash"}[m.value]

    @property
    def relabel_l2_window(self) -> int:
        """Bytes of the relabel table pinned in L2 for the sampler's kernels (0 = none)."""
        b = ctypes.c_uint64()
        self._ck(self._lib.glb_relabel_l2_window(self._h, ctypes.byref(b)))
        return b.value

    def set_train_set(self, train: np.ndarray, batch_size: int, seed: int):
        t = np.ascontiguousarray(train, dtype=np.uint32)
        self._ck(self._lib.glb_set_train_set(self._h, _np_ptr(t), t.shape[0], batch_size, seed))

    @property
    def num_batches(self) -> int:
        n = ctypes.c_uint32()
        self._ck(self._lib.glb_num_batches(self._h, ctypes.byref(n)))
        return n.value

    def shuffle(self, epoch: int):
        self._ck(self._lib.glb_shuffle(self._h, epoch))

    def permutation(self, n: int) -> np.ndarray:
        out = np.empty(n, np.uint32)
        self._ck(self._lib.glb_get_permutation(self._h, _np_ptr(out)))
        return out

    # ------------------------------------------------------------------ sample
    def _blocks(self, b: _Blocks) -> Blocks:
        L = b.num_hops
        sizes = [int(b.sizes[i]) for i in range(L + 1)]
        nnz = [int(b.nnz[i]) for i in range(L)]
        dev = self.device
        uniq = _view(b.uniq, sizes[-1], "<i4", self, dev)
        ips = [_view(b.indptr[l], sizes[l] + 1, "<i4", self, dev) for l in range(L)]
        ixs = [_view(b.indices[l], nnz[l], "<i4", self, dev) for l in range(L)]
        ws = None
        if L and b.weights[0]:
            ws = [_view(b.weights[l], nnz[l], "<i4", self, dev) for l in range(L)]
        cs = _view(b.cache_slot, sizes[-1], "<i4", self, dev)
        return Blocks(int(b.num_seeds), sizes, nnz, uniq, ips, ixs, ws, cs)

    def sample(self, seeds, fanouts=None, seed=0, epoch=0, batch=0) -> Blocks:
        """seeds: host numpy u32 array or a CUDA int32 tensor."""
        import torch
        if isinstance(seeds, torch.Tensor):
            assert seeds.is_cuda and seeds.dtype in (torch.int32,) and seeds.is_contiguous()
            ptr, n = seeds.data_ptr(), seeds.numel()
            keep = seeds
        else:
            keep = np.ascontiguousarray(seeds, dtype=np.uint32)
            ptr, n = _np_ptr(keep), keep.shape[0]
        fan = None if fanouts is None else np.ascontiguousarray(fanouts, dtype=np.uint32)
        L = 0 if fan is None else fan.shape[0]
        if fan is not None and L == 0:
            fan = np.zeros(1, np.uint32)  # non-NULL pointer + num_hops 0 = no hops
        b = _Blocks()
        self._ck(self._lib.glb_sample(self._h, ptr, n, _np_ptr(fan), L, seed, epoch,
                                      batch, ctypes.byref(b)))
        del keep
        return self._blocks(b)

    def sample_batch(self, epoch: int, batch: int):
        """Asynchronous: sample batch ``batch`` of epoch ``epoch`` (device-resident shuffle)."""
        self._ck(self._lib.glb_sample_batch(self._h, epoch, batch))

    def sample_async(self, seeds, seed=0, epoch=0, batch=0):
        """Asynchronous sample of caller seeds with the ctx sampler: a pinned CPU int32 tensor
        (H2D copy on the ctx stream; keep it unchanged until the stream has consumed it) or
        a CUDA int32 tensor.  Read the blocks with sample_result() (synchronises)."""
        import torch
        assert isinstance(seeds, torch.Tensor) and seeds.dtype == torch.int32
        assert seeds.is_contiguous() and (seeds.is_cuda or seeds.is_pinned())
        self._ck(self._lib.glb_sample_async(self._h, seeds.data_ptr(), seeds.numel(), seed,
                                            epoch, batch))

    def extract_counts_tensor(self):
        """Zero-copy int64 CUDA view [3] = (hits, misses, peer hits) of the last extract,
        rewritten on the ctx stream by every extract (copy it out stream-ordered)."""
        import torch
        p = ctypes.c_void_p()
        self._ck(self._lib.glb_extract_counts_device_ptr(self._h, ctypes.byref(p)))
        return torch.as_tensor(_CAI(p.value, (3,), "<i8", self), device=self.device)

    def sample_result(self) -> Blocks:
        b = _Blocks()
        self._ck(self._lib.glb_sample_result(self._h, ctypes.byref(b)))
        return self._blocks(b)

    # ------------------------------------------------------------------ PreSC
    def set_count_mode(self, mode: int):
        self._ck(self._lib.glb_set_count_mode(self._h, mode))

    def reset_counts(self, which: int):
        self._ck(self._lib.glb_reset_counts(self._h, which))

    def presample(self, K: int, rank: int = 0, world: int = 1):
        self._ck(self._lib.glb_presample(self._h, K, rank, world))

    def counts_tensor(self, which: int = COUNT_PRESAMPLE):
        """Zero-copy int32 torch view of the ctx's u32[V] count array (for all_reduce)."""
        p = ctypes.c_void_p()
        self._ck(self._lib.glb_counts_device_ptr(self._h, which, ctypes.byref(p)))
        return _view(p.value, self.V, "<i4", self, self.device)

    def get_counts(self, which: int = COUNT_PRESAMPLE) -> np.ndarray:
        out = np.empty(self.V, np.uint32)
        self._ck(self._lib.glb_get_counts(self._h, which, _np_ptr(out)))
        return out

    def build_cache(self, alpha: float, hotness=None):
        """hotness: None (PreSC counts) or a CUDA int32 tensor [V] (e.g. degrees)."""
        hp = None
        if hotness is not None:
            assert hotness.is_cuda and hotness.numel() == self.V and hotness.is_contiguous()
            hp = hotness.data_ptr()
        self._ck(self._lib.glb_build_cache(self._h, float(alpha), hp))

    def policy_hotness(self, policy: str, seed: int = 0):
        """Hotness map of a caching policy ('presc' | 'degree' | 'random'), CUDA int32 [V]
        (u32 values), for build_cache (L79, L301, Fig 10)."""
        import torch
        pid = {"presc": POLICY_PRESC, "degree": POLICY_DEGREE, "random": POLICY_RANDOM}[policy]
        out = torch.empty(self.V, dtype=torch.int32, device=self.device)
        self._ck(self._lib.glb_policy_hotness(self._h, pid, seed, out.data_ptr()))
        return out

    def build_cache_policy(self, alpha: float, policy: str, seed: int = 0):
        self.build_cache(alpha, hotness=self.policy_hotness(policy, seed))

    def footprint_similarity(self, f_i, f_j, top_frac: float = 0.1):
        """Table 2 (L329): similarity of epoch i's footprint to epoch j's; f_*: CUDA int32
        [V] visit counts.  Returns (value, numerator, denominator) -- exact integers."""
        num, den, out = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_double()
        self._ck(self._lib.glb_footprint_similarity(self._h, f_i.data_ptr(), f_j.data_ptr(),
                                                    float(top_frac), ctypes.byref(num),
                                                    ctypes.byref(den), ctypes.byref(out)))
        return out.value, num.value, den.value

    # ---------------------------------------------------- NEXT-3: peer-sharded cache
    def build_cache_sharded(self, alpha: float, rank: int, world: int, hotness=None):
        """Cache world*floor(alpha*V) rows over ``world`` GPUs; this ctx holds shard ``rank``
        (global rank i -> shard i % world, row i // world).  Attach the other shards next."""
        hp = None
        if hotness is not None:
            assert hotness.is_cuda and hotness.numel() == self.V and hotness.is_contiguous()
            hp = hotness.data_ptr()
        self._ck(self._lib.glb_build_cache_sharded(self._h, float(alpha), hp, rank, world))

    def cache_device_ptr(self):
        """(device pointer, rows) of this ctx's own cache rows."""
        p, n = ctypes.c_void_p(), ctypes.c_uint64()
        self._ck(self._lib.glb_cache_device_ptr(self._h, ctypes.byref(p), ctypes.byref(n)))
        return p.value, n.value

    def cache_ipc_handle(self) -> bytes:
        buf = ctypes.create_string_buffer(IPC_HANDLE_BYTES)
        self._ck(self._lib.glb_cache_ipc_handle(self._h, buf))
        return buf.raw

    def attach_peer_cache(self, peer: int, ipc_handle: bytes | None = None,
                          dev_ptr: int | None = None):
        """Map shard ``peer``: an IPC handle from another process, or a device pointer of a
        ctx in this process."""
        h = None
        if ipc_handle is not None:
            assert len(ipc_handle) == IPC_HANDLE_BYTES
            h = ctypes.create_string_buffer(ipc_handle, IPC_HANDLE_BYTES)
        self._ck(self._lib.glb_attach_peer_cache(self._h, peer, h, dev_ptr))

    def last_extract_counts(self) -> dict:
        """Synchronous: hits (local + peer), misses and peer-shard hits of the last extract."""
        a = (ctypes.c_uint64 * 3)()
        self._ck(self._lib.glb_last_extract_counts(self._h, a))
        return {"hits": a[0], "misses": a[1], "peer_hits": a[2]}

    def cache_slots(self) -> np.ndarray:
        out = np.empty(self.V, np.int32)
        self._ck(self._lib.glb_get_cache_slots(self._h, _np_ptr(out)))
        return out

    @property
    def cache_size(self) -> int:
        c = ctypes.c_uint64()
        self._ck(self._lib.glb_cache_size(self._h, ctypes.byref(c)))
        return c.value

    def hit_stats(self) -> dict:
        s = _HitStats()
        self._ck(self._lib.glb_hit_stats_get(self._h, ctypes.byref(s)))
        return {"total": s.total, "hits": s.hits, "optimal_hits": s.optimal_hits,
                "cache_rows": s.cache_rows}

    # ------------------------------------- a8: factored Sampler -> Trainer handoff
    def handoff_create(self, slots: int) -> bytes:
        """Trainer: allocate a ring of ``slots`` receive slots in this GPU's HBM; returns the
        blob samplers attach with (include/glb.h glb_handoff_create)."""
        buf = ctypes.create_string_buffer(HANDOFF_BLOB_BYTES)
        self._ck(self._lib.glb_handoff_create(self._h, slots, buf))
        return buf.raw

    def handoff_attach(self, trainer: int, trainer_blob: bytes) -> bytes:
        """Sampler: map trainer ``trainer``'s ring; returns the blob for handoff_connect."""
        tb = ctypes.create_string_buffer(trainer_blob, HANDOFF_BLOB_BYTES)
        buf = ctypes.create_string_buffer(HANDOFF_BLOB_BYTES)
        self._ck(self._lib.glb_handoff_attach(self._h, trainer, tb, buf))
        return buf.raw

    def handoff_connect(self, sampler: int, sampler_blob: bytes):
        sb = ctypes.create_string_buffer(sampler_blob, HANDOFF_BLOB_BYTES)
        self._ck(self._lib.glb_handoff_connect(self._h, sampler, sb))

    def handoff_send(self, trainer: int, slot: int, tag: int):
        """Sampler: push the current sample into (trainer, slot); asynchronous."""
        self._ck(self._lib.glb_handoff_send(self._h, trainer, slot, tag))

    def handoff_recv(self, sampler: int, slot: int):
        """Trainer: the sample in ``slot`` (pushed by ``sampler``) becomes the current one."""
        self._ck(self._lib.glb_handoff_recv(self._h, sampler, slot))

    def handoff_tag(self) -> int:
        t = ctypes.c_uint64()
        self._ck(self._lib.glb_handoff_tag(self._h, ctypes.byref(t)))
        return t.value

    def handoff_release(self, slot: int):
        self._ck(self._lib.glb_handoff_release(self._h, slot))

    # ------------------------------------------------------------------ extract
    def extract(self, vertices, out=None, stats: bool = False):
        """vertices: CUDA int32 tensor of gids; returns out [n, D] float32 (CUDA)."""
        import torch
        assert vertices.is_cuda and vertices.dtype == torch.int32 and vertices.is_contiguous()
        n = vertices.numel()
        if out is None:
            out = torch.empty((n, self.D), dtype=torch.float32, device=vertices.device)
        st = _XStats()
        self._ck(self._lib.glb_extract(self._h, vertices.data_ptr(), n, out.data_ptr(),
                                       ctypes.byref(st) if stats else None))
        if stats:
            self.sync()
            return out, {"hits": st.hits, "misses": st.misses}
        return out

    def extract_sample(self, out, stats: bool = False):
        """Gather features of the last sample's uniq into ``out`` (CUDA f32 [>=n_L, D])."""
        st = _XStats()
        self._ck(self._lib.glb_extract_sample(self._h, out.data_ptr(),
                                              ctypes.byref(st) if stats else None))
        if stats:
            self.sync()
            return {"hits": st.hits, "misses": st.misses}
        return None

    def set_host_gather(self, fraction: float, threads: int = 0):
        """Host-assisted misses: `fraction` of each sample's (address-ordered) misses are
        copied by `threads` host threads into pinned staging that the GPU reads back
        sequentially (include/glb.h glb_set_host_gather); 0 turns it off."""
        self._ck(self._lib.glb_set_host_gather(self._h, int(threads), float(fraction)))

    @property
    def host_gather(self):
        t, f = ctypes.c_uint32(), ctypes.c_double()
        self._ck(self._lib.glb_host_gather(self._h, ctypes.byref(t), ctypes.byref(f)))
        return {"threads": t.value, "fraction": f.value}

    def set_cold_store(self, enable: bool = True):
        """Misses read a rank-ordered pinned copy of the non-cached rows, built by the next
        build_cache (include/glb.h glb_set_cold_store)."""
        self._ck(self._lib.glb_set_cold_store(self._h, int(bool(enable))))

    @property
    def cold_store_rows(self) -> int:
        n = ctypes.c_uint64()
        self._ck(self._lib.glb_cold_store_rows(self._h, ctypes.byref(n)))
        return n.value

    def set_pipeline(self, depth: int):
        """depth 2: double-buffered samples, extract on its own stream overlapping the
        next sample (see include/glb.h glb_set_pipeline)."""
        self._ck(self._lib.glb_set_pipeline(self._h, depth))

    def extract_stream(self):
        """torch stream the extracts run on (order consumers of ``out`` after it)."""
        import torch
        p = ctypes.c_void_p()
        self._ck(self._lib.glb_extract_stream(self._h, ctypes.byref(p)))
        if not p.value:  # the legacy default stream
            return torch.cuda.default_stream(self.device)
        return torch.cuda.ExternalStream(p.value, device=self.device)

    def set_timing(self, period):
        """Time every ``period``-th extract kernel with CUDA events (True = each, 0 = off)."""
        self._ck(self._lib.glb_set_timing(self._h, int(period)))

    def extract_times(self, max_n: int = 1 << 16) -> list:
        """Durations (ms) of the extract kernels recorded since set_timing(True)."""
        buf = np.zeros(max_n, np.float32)
        n = ctypes.c_uint64()
        self._ck(self._lib.glb_extract_times(self._h, buf.ctypes.data, max_n, ctypes.byref(n)))
        return buf[:min(n.value, max_n)].tolist()

    @property
    def launches(self) -> int:
        return int(self._lib.glb_kernel_launches(self._h))
