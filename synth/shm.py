"""Node-shared inputs: one copy of a generated graph per host, mapped by every local rank.

SURVEY §8(e): "Host features are registered once and mapped into every GPU."  Local
rank 0 generates the graph (synth.make_graph) with every array -- features written in
place -- in anonymous shared memory (memfd), and publishes (pid, fd, size, dtype, shape)
per array through the process group's store; the other local ranks open the same memfds
through /proc/<pid>/fd and map them MAP_SHARED, so N ranks hold one physical copy (PA:
57 GB of features once, not N times) and each rank's glb_load_graph registers the same
pages for its own GPU.  Inputs only: nothing here computes anything of the method.
"""
from __future__ import annotations

import json
import mmap
import os

import numpy as np

from . import Graph, SHAPES, Shape, make_graph, seed_for


class _Mem:
    """A memfd mapping kept alive for the lifetime of the arrays viewing it."""

    def __init__(self, nbytes: int, name: str = "glb_input", fd: int | None = None):
        self.nbytes = max(int(nbytes), 1)
        if fd is None:
            self.fd = os.memfd_create(name)
            os.ftruncate(self.fd, self.nbytes)
        else:
            self.fd = fd
        self.map = mmap.mmap(self.fd, self.nbytes, flags=mmap.MAP_SHARED,
                             prot=mmap.PROT_READ | mmap.PROT_WRITE)

    def array(self, dtype, shape):
        n = int(np.prod(shape)) if len(shape) else 1
        return np.frombuffer(self.map, dtype=dtype, count=n).reshape(shape)


def _open_peer(pid: int, fd: int, nbytes: int) -> _Mem:
    """Map another process's memfd (the same physical pages)."""
    return _Mem(nbytes, fd=os.open(f"/proc/{pid}/fd/{fd}", os.O_RDWR))


class SharedGraph:
    """A Graph whose arrays live in node-shared memory, plus the mappings behind them."""

    def __init__(self, graph: Graph, mems: list, owner: bool):
        self.graph = graph
        self.mems = mems
        self.owner = owner


def node_cpus(node: int) -> set[int] | None:
    """CPUs of NUMA node `node` (sysfs cpulist), None if the node does not exist."""
    try:
        txt = open(f"/sys/devices/system/node/node{node}/cpulist").read().strip()
    except OSError:
        return None
    cpus = set()
    for part in filter(None, txt.split(",")):
        a, _, b = part.partition("-")
        cpus.update(range(int(a), int(b or a) + 1))
    return cpus or None


def _replicate_features(src: np.ndarray, node: int) -> tuple[_Mem, np.ndarray]:
    """A copy of the feature matrix in a new memfd whose pages sit on NUMA node `node`:
    the copy is written by this thread pinned to the node's CPUs, and first touch places
    each page on the node of the CPU that writes it.  Bytes are copied, never computed."""
    m = _Mem(src.nbytes, f"glb_features_numa{node}")
    dst = m.array(src.dtype, src.shape)
    old = os.sched_getaffinity(0)
    cpus = (node_cpus(node) or set()) & old  # only CPUs this process may run on
    try:
        if cpus:
            os.sched_setaffinity(0, cpus)
        flat_s, flat_d = src.reshape(-1), dst.reshape(-1)
        step = 1 << 26  # 256 MB of f32 per slice
        for i in range(0, flat_s.size, step):
            flat_d[i:i + step] = flat_s[i:i + step]
    finally:
        if cpus:
            os.sched_setaffinity(0, old)
    return m, dst


def make_graph_shared(shape: Shape | str, local_rank: int, local_world: int, store,
                      key: str | None = None, seed: int | None = None,
                      numa_node: int | None = None) -> SharedGraph:
    """Generate (local rank 0) or map (other local ranks) the graph of `shape`.

    store: a torch.distributed Store shared by the local ranks (e.g. the default
    process group's).  Every local rank must call this; ranks != 0 block until rank 0
    has published the arrays.

    numa_node (per-socket replicas): the NUMA node of this rank's GPU, given by every
    local rank or by none.  The feature matrix -- the only input the GPUs read over the
    host link at run time (topology is copied to HBM) -- is then held once per NUMA node
    instead of once per host: the lowest local rank of each node other than rank 0's
    copies rank 0's matrix into memory on its own node, and the ranks of that node map
    that copy, so every GPU's zero-copy misses stay on its own socket."""
    if isinstance(shape, str):
        shape = SHAPES[shape]
    seed = seed_for(shape) if seed is None else seed
    key = key or f"glb_shm/{shape.name}/{seed}"
    if local_world <= 1:
        return SharedGraph(make_graph(shape, seed=seed), [], True)
    nodes = None
    if numa_node is not None:
        store.set(f"{key}/numa/{local_rank}", str(int(numa_node)))
        nodes = [int(store.get(f"{key}/numa/{r}")) for r in range(local_world)]
    sg = _make_graph_shared(shape, local_rank, store, key, seed)
    if nodes is None or nodes[local_rank] == nodes[0]:
        return sg  # rank 0's node: its matrix is the replica
    node = nodes[local_rank]
    fkey = f"{key}/features/numa{node}"
    g = sg.graph
    if local_rank == min(r for r in range(local_world) if nodes[r] == node):
        m, feats = _replicate_features(g.features, node)
        store.set(fkey, json.dumps({"pid": os.getpid(), "fd": m.fd, "nbytes": m.nbytes}))
    else:
        d = json.loads(store.get(fkey))
        m = _open_peer(d["pid"], d["fd"], d["nbytes"])
        feats = m.array(g.features.dtype, g.features.shape)
    mems = [(n, x) for n, x in sg.mems if n != "features"] + [("features", m)]
    g = Graph(shape, seed, g.indptr, g.indices, g.train, feats, g.weights)
    return SharedGraph(g, mems, sg.owner)


def _make_graph_shared(shape: Shape, local_rank: int, store, key: str, seed: int) -> SharedGraph:
    if local_rank == 0:
        mems = []

        def alloc(nbytes):
            m = _Mem(nbytes, "glb_features")
            mems.append(("features", m))
            return m.array(np.uint8, (m.nbytes,))

        g = make_graph(shape, seed=seed, feature_alloc=alloc)
        desc = {"pid": os.getpid(), "arrays": {}}
        fm = mems[0][1]
        desc["arrays"]["features"] = [fm.fd, fm.nbytes, "float32", list(g.features.shape)]
        out = {"features": g.features}
        for name in ("indptr", "indices", "train", "weights"):
            a = getattr(g, name)
            if a is None:
                continue
            m = _Mem(a.nbytes, f"glb_{name}")
            v = m.array(a.dtype, a.shape)
            v[...] = a
            mems.append((name, m))
            out[name] = v
            desc["arrays"][name] = [m.fd, m.nbytes, str(a.dtype), list(a.shape)]
        g = Graph(shape, seed, out["indptr"], out["indices"], out["train"], out["features"],
                  out.get("weights"))
        store.set(key, json.dumps(desc))
        return SharedGraph(g, mems, True)
    desc = json.loads(store.get(key))
    mems, out = [], {}
    for name, (fd, nbytes, dt, shp) in desc["arrays"].items():
        m = _open_peer(desc["pid"], fd, nbytes)
        mems.append((name, m))
        out[name] = m.array(np.dtype(dt), tuple(shp))
    g = Graph(shape, seed, out["indptr"], out["indices"], out["train"], out["features"],
              out.get("weights"))
    return SharedGraph(g, mems, False)
