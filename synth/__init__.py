"""Seeded synthetic workload generator (inputs only).

Both the oracle (``oracle/``) and the CUDA path read what this module
produces; it holds none of the method's arithmetic (no sampling, relabel,
ranking or gather).  The C source is ``synth/synth.c``; the recipe is in
DESIGN.md ("Input recipe") and SURVEY.md §8(d).

Shapes follow BASELINE.json ``configs`` / PAPER.md Table 3 (L357-362):
V, E, feature dim and training-set size of PR / TW / PA / UK, batch 8000
and the paper's fanouts (L353).  Degree skew (gamma) is this build's choice
(the paper used real graphs).
"""
from __future__ import annotations

import ctypes
import dataclasses
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libsynth.so")
_SRC = os.path.join(_HERE, "synth.c")

BASE_SEED = 20220405


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v3", "-fPIC", "-shared", "-pthread",
                               "-o", _SO, _SRC, "-lm"])
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        u64, u32, i32, dbl, vp = (ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int,
                                  ctypes.c_double, ctypes.c_void_p)
        L.synth_degrees.argtypes = [u64, u64, dbl, u64, u64, vp]
        L.synth_degrees.restype = i32
        L.synth_edges.argtypes = [u64, vp, dbl, u64, vp, i32]
        L.synth_edges.restype = i32
        L.synth_features.argtypes = [u64, u32, u64, vp, i32]
        L.synth_features.restype = i32
        L.synth_trainset.argtypes = [u64, u64, u64, vp]
        L.synth_trainset.restype = i32
        L.synth_perm.argtypes = [u64, u64, u32, u64]
        L.synth_perm.restype = u64
        L.synth_perm_fill.argtypes = [u64, u64, u32, vp]
        L.synth_perm_fill.restype = None
        L.synth_edge_weights.argtypes = [u64, vp, u32, u64, vp, i32]
        L.synth_edge_weights.restype = i32
        _lib = L
    return _lib


@dataclasses.dataclass(frozen=True)
class Shape:
    name: str
    V: int
    E: int
    gamma_out: float
    gamma_in: float
    D: int
    n_train: int
    batch: int
    sampler: str              # "khop" | "rwalk"
    fanouts: tuple            # khop: per hop; rwalk: (topk,)*layers
    K: int = 1                # PreSC#K presample epochs
    alphas: tuple = (0.1,)
    cap_div: int = 16         # degree cap = V // cap_div


# BASELINE.json configs[0..4]; SURVEY.md §8(d).
SHAPES = {
    "tiny": Shape("tiny", 10_000, 100_000, 2.2, 2.2, 32, 1_000, 64, "khop", (10, 5), 1,
                  (0.0, 0.05, 0.1, 0.25, 0.5, 1.0)),
    "PR": Shape("PR", 2_449_029, 123_718_280, 2.5, 2.5, 100, 196_615, 8000, "khop", (25, 10), 1,
                (0.0, 0.01, 0.05, 0.10, 0.25, 0.50, 1.0)),
    "TW": Shape("TW", 41_652_230, 1_468_365_182, 2.1, 2.1, 256, 417_000, 8000, "khop",
                (15, 10, 5), 1, (0.25, 0.10, 1.0)),
    "PA": Shape("PA", 111_059_956, 1_615_685_872, 3.5, 2.5, 128, 1_207_179, 8000, "rwalk",
                (5, 5, 5), 1, (0.22, 0.05, 0.10, 1.0)),
    "UK": Shape("UK", 77_741_046, 2_965_197_340, 3.0, 2.1, 256, 1_000_000, 8000, "khop", (25, 10),
                1, (0.18, 1.0)),
    # NEXT-1 (not a BASELINE config): Twitter with 3-hop WEIGHTED sampling, edge weight =
    # the target's "year registered" (Fig 5(b), Fig 12 "GCN (W.)").
    "TWW": Shape("TWW", 41_652_230, 1_468_365_182, 2.1, 2.1, 256, 417_000, 8000, "weighted",
                 (15, 10, 5), 1, (0.25, 0.10, 1.0)),
    "PRW": Shape("PRW", 2_449_029, 123_718_280, 2.5, 2.5, 100, 196_615, 8000, "weighted",
                 (25, 10), 1, (0.05, 0.10, 0.25, 1.0)),
}
CONFIG_INDEX = {"tiny": 0, "PR": 1, "TW": 2, "PA": 3, "UK": 4, "TWW": 2, "PRW": 1}

# PinSAGE random walk: 4 paths of length 3, keep 5.
RW_WALKS, RW_LEN, RW_TOPK = 4, 3, 5


def seed_for(shape: Shape) -> int:
    return BASE_SEED + CONFIG_INDEX.get(shape.name, 9)


def aligned_empty(n: int, dtype, align: int = 1 << 21, huge: bool = False) -> np.ndarray:
    """Page-aligned host array (so it can be cudaHostRegister'ed whole).  huge: anonymous
    mmap advised MADV_HUGEPAGE (2 MB transparent huge pages where the kernel allows)."""
    dtype = np.dtype(dtype)
    nbytes = max(n * dtype.itemsize, 1)
    if huge:
        import mmap
        m = mmap.mmap(-1, nbytes + align, flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
        try:
            m.madvise(mmap.MADV_HUGEPAGE)
        except (AttributeError, OSError):
            pass
        raw = np.frombuffer(m, dtype=np.uint8)
    else:
        raw = np.empty(nbytes + align, dtype=np.uint8)
    off = (-raw.ctypes.data) % align
    return raw[off:off + nbytes].view(dtype)[:n]


@dataclasses.dataclass
class Graph:
    shape: Shape
    seed: int
    indptr: np.ndarray     # u64[V+1]
    indices: np.ndarray    # u32[E]
    train: np.ndarray      # u32[n_train], sorted
    features: np.ndarray | None  # f32[V, D] (None if not generated)
    weights: np.ndarray | None = None  # u32[E] edge weights (weighted sampler shapes)

    @property
    def V(self):
        return self.indptr.shape[0] - 1

    @property
    def E(self):
        return int(self.indptr[-1])

    @property
    def D(self):
        return self.shape.D


def gen_topology(V: int, E: int, gamma_out: float, gamma_in: float, seed: int, cap: int,
                 threads: int = 0):
    L = lib()
    indptr = np.empty(V + 1, dtype=np.uint64)
    rc = L.synth_degrees(V, E, gamma_out, cap, seed, indptr.ctypes.data)
    if rc != 0:
        raise RuntimeError(f"synth_degrees failed rc={rc}")
    indices = aligned_empty(E, np.uint32)
    rc = L.synth_edges(V, indptr.ctypes.data, gamma_in, seed, indices.ctypes.data, threads)
    if rc != 0:
        raise RuntimeError(f"synth_edges failed rc={rc}")
    return indptr, indices


def gen_features(V: int, D: int, seed: int, threads: int = 0, alloc=None) -> np.ndarray:
    """alloc(nbytes) -> writable uint8 numpy buffer (e.g. CUDA pinned memory); default:
    2 MB-aligned pageable memory that glb_load_graph registers."""
    if alloc is None:
        f = aligned_empty(V * D, np.float32).reshape(V, D)
    else:
        f = alloc(V * D * 4).view(np.float32)[:V * D].reshape(V, D)
    lib().synth_features(V, D, seed, f.ctypes.data, threads)
    return f


def gen_edge_weights(indices: np.ndarray, seed: int, levels: int = 16, threads: int = 0):
    """Per-edge weight = the target's "year registered" (1..levels): weighted sampling
    prefers newer neighbours."""
    w = aligned_empty(indices.shape[0], np.uint32)
    lib().synth_edge_weights(indices.shape[0], indices.ctypes.data, levels, seed,
                             w.ctypes.data, threads)
    return w


def gen_trainset(V: int, n: int, seed: int) -> np.ndarray:
    t = np.empty(n, dtype=np.uint32)
    rc = lib().synth_trainset(V, n, seed, t.ctypes.data)
    if rc != 0:
        raise RuntimeError("synth_trainset failed")
    return t


def make_graph(shape: Shape | str, seed: int | None = None, features: bool = True,
               threads: int = 0, feature_alloc=None) -> Graph:
    if isinstance(shape, str):
        shape = SHAPES[shape]
    seed = seed_for(shape) if seed is None else seed
    cap = max(shape.V // shape.cap_div, 1)
    indptr, indices = gen_topology(shape.V, shape.E, shape.gamma_out, shape.gamma_in, seed, cap,
                                   threads)
    train = gen_trainset(shape.V, shape.n_train, seed)
    feats = gen_features(shape.V, shape.D, seed, threads, feature_alloc) if features else None
    w = gen_edge_weights(indices, seed, threads=threads) if shape.sampler == "weighted" else None
    return Graph(shape, seed, indptr, indices, train, feats, w)


def small_graph(V: int, E: int, gamma: float, D: int, n_train: int, seed: int,
                cap: int | None = None, fanouts=(10, 5), batch: int = 64,
                sampler: str = "khop") -> Graph:
    """An arbitrary small power-law workload (parity tests: ragged tails, edge cases)."""
    sh = Shape(f"small{V}", V, E, gamma, gamma, D, n_train, batch, sampler, tuple(fanouts))
    cap = max(V // 16, 1) if cap is None else cap
    indptr, indices = gen_topology(V, E, gamma, gamma, seed, cap)
    return Graph(sh, seed, indptr, indices, gen_trainset(V, n_train, seed),
                 gen_features(V, D, seed))


def rank_order(V: int, seed: int) -> np.ndarray:
    """rank -> vertex map of the generator's degree ranks (rank 0 = the heaviest vertex;
    in- and out-degree share it).  Tools only (e.g. hot-first renumbering experiments)."""
    out = np.empty(V, np.uint32)
    lib().synth_perm_fill(V, seed, 7, out.ctypes.data)
    return out
