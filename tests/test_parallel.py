"""Multi-process (gloo, CPU) tests of the N>1 orchestration in
paper_conf_eurosys_yangtswycyz22_b200.parallel: DP sharding + count
all-reduce, the factored sampler->trainer protocol (global scheduler,
global-queue descriptors, header/payload send/recv), and the Ns formula.
The GPU sampler is replaced by the CPU oracle as a stand-in (tests only)."""
import os
import socket
import types

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_eurosys_yangtswycyz22_b200 import parallel as par


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)


def test_num_samplers_formula():
    # Ns = ceil(Ng / (K+1)), K = Tt/Ts
    assert par.num_samplers(8, 1.0, 3.0) == 2
    assert par.num_samplers(8, 1.0, 1.0) == 4
    assert par.num_samplers(8, 2.0, 1.0) == 6
    assert par.num_samplers(8, 1.0, 0.0) == 7      # at least one trainer
    assert par.num_samplers(8, 1.0, 100.0) == 1    # at least one sampler
    assert par.num_samplers(1, 1.0, 1.0) == 1


def test_dp_sharding_covers_every_batch_once():
    for world in [1, 2, 3, 8]:
        nb = 25
        seen = sorted(b for r in range(world) for b in par.dp_batches(nb, r, world))
        assert seen == list(range(nb))
        steps = sorted(par.dp_step_batch(i, r, world, nb, 1) for r in range(world)
                       for i in range(10))
        assert len(set(steps)) == 10 * world
        assert steps[0] == (1, 0)


def _dp_worker(rank, world, port, out):
    import oracle
    import synth
    _init(rank, world, port)
    g = synth.make_graph("tiny")
    sh = g.shape
    go = oracle.GraphOracle(g.indptr, g.indices)
    nb = -(-sh.n_train // sh.batch)
    mine = set(par.dp_batches(nb, rank, world))
    c = go.visit_counts("khop", g.train, sh.batch, sh.fanouts, g.seed, range(2),
                        batch_filter=lambda e, b: b in mine)
    t = torch.from_numpy(c.view(np.int32).copy())
    par.allreduce_counts(t)
    if rank == 0:
        np.save(out, t.numpy())
    dist.destroy_process_group()


def test_dp_presample_allreduce_equals_single_process(tmp_path):
    import oracle
    import synth
    out = str(tmp_path / "c.npy")
    world = 2
    mp.spawn(_dp_worker, args=(world, free_port(), out), nprocs=world, join=True)
    g = synth.make_graph("tiny")
    sh = g.shape
    go = oracle.GraphOracle(g.indptr, g.indices)
    full = go.presample("khop", g.train, sh.batch, sh.fanouts, g.seed, 2)
    assert np.array_equal(np.load(out).view(np.uint32), full)


def _factored_worker(rank, world, port, ns, outdir):
    import oracle
    import synth
    _init(rank, world, port)
    g = synth.make_graph("tiny")
    sh = g.shape
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    roles = par.Roles(ns, world)
    batches = oracle.epoch_batches(g.train, sh.batch, g.seed, 1)
    total = len(batches)
    store = dist.distributed_c10d._get_default_store()
    if roles.is_sampler(rank):
        def sample_fn(gidx):
            s = go.sample_khop(batches[gidx], sh.fanouts, g.seed, 1, gidx)
            t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int32))  # noqa: E731
            return 1, types.SimpleNamespace(
                sizes=s.sizes, nnz=[len(x) for x in s.indices], uniq=t(s.uniq),
                indptr=[t(x) for x in s.indptr], indices=[t(x) for x in s.indices], weights=None)
        n = par.run_sampler(sample_fn, roles, rank, total, store, "t", "cpu")
        np.save(os.path.join(outdir, f"s{rank}.npy"), np.array([n]))
    else:
        got = {}

        def extract_fn(gidx, epoch, sizes, nnz, payload):
            uniq, indptr, indices, _ = payload
            exp = go.sample_khop(batches[gidx], sh.fanouts, g.seed, 1, gidx)
            assert epoch == 1 and sizes == exp.sizes
            assert np.array_equal(uniq.numpy().view(np.uint32), exp.uniq)
            for l in range(len(sh.fanouts)):
                assert np.array_equal(indptr[l].numpy().view(np.uint32), exp.indptr[l])
                assert np.array_equal(indices[l].numpy().view(np.uint32), exp.indices[l])
            feats = go.extract(uniq.numpy().view(np.uint32))
            got[gidx] = float(feats.sum(dtype=np.float64))

        n = par.run_trainer(extract_fn, roles, rank, total, store, "t", "cpu")
        np.save(os.path.join(outdir, f"t{rank}.npy"), np.array(sorted(got)))
        assert n == len(roles.trainer_batches(rank, total))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,ns", [(2, 1), (3, 2), (3, 1)])
def test_factored_handoff_protocol(tmp_path, world, ns):
    mp.spawn(_factored_worker, args=(world, free_port(), ns, str(tmp_path)), nprocs=world,
             join=True)
    total = 16
    trained = sorted(int(x) for r in range(ns, world)
                     for x in np.load(tmp_path / f"t{r}.npy"))
    assert trained == list(range(total))                        # every batch extracted once
    sampled = sum(int(np.load(tmp_path / f"s{r}.npy")[0]) for r in range(ns))
    assert sampled == total                                     # every batch sampled once


def test_header_payload_roundtrip():
    b = types.SimpleNamespace(sizes=[3, 7, 12], nnz=[5, 9], uniq=torch.arange(12, dtype=torch.int32),
                              indptr=[torch.tensor([0, 2, 4, 5], dtype=torch.int32),
                                      torch.arange(8, dtype=torch.int32)],
                              indices=[torch.arange(5, dtype=torch.int32),
                                       torch.arange(9, dtype=torch.int32)],
                              weights=[torch.ones(5, dtype=torch.int32),
                                       torch.full((9,), 2, dtype=torch.int32)])
    h = par.pack_header(41, 3, b.sizes, b.nnz, True, "cpu")
    g, e, sizes, nnz, w = par.unpack_header(h)
    assert (g, e, sizes, nnz, w) == (41, 3, b.sizes, b.nnz, True)
    buf = par.pack_payload(b)
    assert buf.numel() == par.payload_len(sizes, nnz, w)
    uniq, ip, ix, ws = par.unpack_payload(buf, sizes, nnz, w)
    assert torch.equal(uniq, b.uniq) and all(torch.equal(a, c) for a, c in zip(ip, b.indptr))
    assert all(torch.equal(a, c) for a, c in zip(ix, b.indices))
    assert all(torch.equal(a, c) for a, c in zip(ws, b.weights))


class _ShardCtx:
    """Stand-in ctx for parallel.build_sharded_cache: records the build and the attaches."""

    def __init__(self, rank):
        self.rank = rank
        self.built = None
        self.attached = {}

    def build_cache_sharded(self, alpha, rank, world):
        self.built = (alpha, rank, world)

    def cache_ipc_handle(self):
        return bytes([self.rank]) * 64  # a 64-byte opaque blob, unique per rank

    def attach_peer_cache(self, peer, ipc_handle=None, dev_ptr=None):
        assert dev_ptr is None and len(ipc_handle) == 64
        self.attached[peer] = ipc_handle


def _shard_worker(rank, world, port, out):
    _init(rank, world, port)
    c = _ShardCtx(rank)
    par.build_sharded_cache(c, 0.125, rank, world)
    ok = c.built == (0.125, rank, world) and sorted(c.attached) == [p for p in range(world)
                                                                     if p != rank]
    ok = ok and all(h == bytes([p]) * 64 for p, h in c.attached.items())
    t = torch.tensor([1 if ok else 0])
    dist.all_reduce(t)
    if rank == 0:
        torch.save(t, out)
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_cache_handle_exchange(tmp_path, world):
    """NEXT-3: every rank builds its shard and maps every other rank's shard from the
    all-gathered IPC handles (gloo, CPU; the CUDA side is tests/test_gpu_sharded.py)."""
    out = str(tmp_path / "ok.pt")
    mp.spawn(_shard_worker, args=(world, free_port(), out), nprocs=world, join=True)
    assert int(torch.load(out)[0]) == world


# ---------------------------------------------------- factored over peer memory (a8)
class _RingCtx:
    """Stand-in for the library's handoff calls: a trainer's ring is a directory of slot
    files; send writes (tag, payload) into the slot file immediately, so a sampler that
    overwrote a slot before its release would be caught by the trainer's tag check."""

    def __init__(self, rank, ringdir):
        self.rank, self.dir, self.cur = rank, ringdir, None
        self.sample = None

    def handoff_create(self, slots):
        return f"ring{self.rank}:{slots}".encode()

    def handoff_attach(self, trainer, blob):
        assert blob.decode().startswith(f"ring{trainer}:")
        return f"ready{self.rank}->{trainer}".encode()

    def handoff_connect(self, sampler, blob):
        assert blob.decode() == f"ready{sampler}->{self.rank}"

    def handoff_send(self, trainer, slot, tag):
        np.save(os.path.join(self.dir, f"t{trainer}s{slot}.npy"),
                np.array([tag, self.rank] + list(self.sample), dtype=np.int64))

    def handoff_recv(self, sampler, slot):
        a = np.load(os.path.join(self.dir, f"t{self.rank}s{slot}.npy"))
        assert int(a[1]) == sampler
        self.cur = (int(a[0]), a[2:])

    def handoff_release(self, slot):
        self.cur = None


def _peer_worker(rank, world, port, ns, slots, total, outdir):
    import time
    _init(rank, world, port)
    roles = par.Roles(ns, world)
    ctx = _RingCtx(rank, outdir)
    ho = par.PeerHandoff(ctx, roles, rank, slots=slots)
    store = dist.distributed_c10d._get_default_store()
    rng = np.random.default_rng(rank)
    if roles.is_sampler(rank):
        def sample_fn(gidx):
            ctx.sample = [gidx * 7 + i for i in range(3)]
        n = par.run_sampler_peer(sample_fn, ho, total, store, "p")
        np.save(os.path.join(outdir, f"s{rank}.npy"), np.array([n]))
    else:
        got = []

        def extract_fn(gidx):
            time.sleep(float(rng.uniform(0, 0.01)))  # let samplers run ahead
            tag, payload = ctx.cur
            assert tag == gidx, (tag, gidx)
            assert payload.tolist() == [gidx * 7 + i for i in range(3)]
            got.append(gidx)

        par.run_trainer_peer(extract_fn, ho, total, store, "p")
        np.save(os.path.join(outdir, f"t{rank}.npy"), np.array(got))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,ns,slots", [(2, 1, 1), (3, 2, 2), (4, 1, 3), (4, 3, 1)])
def test_factored_peer_handoff_protocol(tmp_path, world, ns, slots):
    """Slot g reuse waits for g - Nt*slots's release; every batch reaches its trainer once
    and intact, whatever the interleaving of samplers."""
    total = 30
    mp.spawn(_peer_worker, args=(world, free_port(), ns, slots, total, str(tmp_path)),
             nprocs=world, join=True)
    trained = sorted(int(x) for r in range(ns, world) for x in np.load(tmp_path / f"t{r}.npy"))
    assert trained == list(range(total))
    assert sum(int(np.load(tmp_path / f"s{r}.npy")[0]) for r in range(ns)) == total
    roles = par.Roles(ns, world)
    for r in range(ns, world):  # each trainer got exactly its batches, in order
        assert np.load(tmp_path / f"t{r}.npy").tolist() == roles.trainer_batches(r, total)


def test_switch_profit_formula():
    # P = M_r * T_t / N_t - T_t'; +inf without trainers
    assert par.switch_profit(10, 2.0, 4, 3.0) == 2.0
    assert par.switch_profit(1, 2.0, 4, 3.0) < 0
    assert par.switch_profit(0, 2.0, 0, 3.0) == float("inf")


def _switch_worker(rank, world, port, ns, slots, total, t_standby, outdir):
    import time
    _init(rank, world, port)
    roles = par.Roles(ns, world)
    ctx = _RingCtx(rank, outdir)
    ho = par.PeerHandoff(ctx, roles, rank, slots=slots)
    store = dist.distributed_c10d._get_default_store()
    if roles.is_sampler(rank):
        local = []

        def sample_fn(gidx):
            ctx.sample = [gidx * 7 + i for i in range(3)]

        def standby_fn(gidx):
            assert ctx.sample == [gidx * 7 + i for i in range(3)]
            local.append(gidx)

        n = par.run_sampler_peer(sample_fn, ho, total, store, "w", standby_fn=standby_fn,
                                 t_train=0.02, t_standby=t_standby)
        assert ho.standby == len(local)
        np.save(os.path.join(outdir, f"s{rank}.npy"), np.array([n]))
        np.save(os.path.join(outdir, f"l{rank}.npy"), np.array(local, dtype=np.int64))
    else:
        got = []

        def extract_fn(gidx):
            time.sleep(0.02)  # trainers 10x+ slower than samplers: the switching case (L265)
            tag, payload = ctx.cur
            assert tag == gidx and payload.tolist() == [gidx * 7 + i for i in range(3)]
            got.append(gidx)

        par.run_trainer_peer(extract_fn, ho, total, store, "w")
        np.save(os.path.join(outdir, f"t{rank}.npy"), np.array(got, dtype=np.int64))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,ns,t_standby,expect_switch", [(2, 1, 0.02, True), (3, 1, 0.02, True),
                                                               (3, 2, 0.02, True),
                                                               (2, 1, 1e9, False)])
def test_dynamic_switching_protocol(tmp_path, world, ns, t_standby, expect_switch):
    """Samplers that would idle behind slow trainers switch to standby trainers when the
    profit metric is positive; every batch is extracted exactly once, either by its
    trainer (in order) or by a standby."""
    total, slots = 24, 2  # M_r <= Nt*slots: one slot per trainer never makes P > 0
    mp.spawn(_switch_worker, args=(world, free_port(), ns, slots, total, t_standby, str(tmp_path)),
             nprocs=world, join=True)
    local = sorted(int(x) for r in range(ns) for x in np.load(tmp_path / f"l{r}.npy"))
    trained = sorted(int(x) for r in range(ns, world) for x in np.load(tmp_path / f"t{r}.npy"))
    assert sorted(local + trained) == list(range(total))
    assert (len(local) > 0) == expect_switch
    roles = par.Roles(ns, world)
    for r in range(ns, world):
        mine = [g for g in roles.trainer_batches(r, total) if g not in set(local)]
        assert np.load(tmp_path / f"t{r}.npy").tolist() == mine
    assert sum(int(np.load(tmp_path / f"s{r}.npy")[0]) for r in range(ns)) == total


# ------------------------------------------------- node-shared host inputs
def _shm_worker(rank, world, port, outdir):
    import synth
    from synth import shm
    _init(rank, world, port)
    store = dist.distributed_c10d._get_default_store()
    sg = shm.make_graph_shared("tiny", rank, world, store)
    g = sg.graph
    ref = synth.make_graph("tiny")
    same = all(np.array_equal(getattr(g, n), getattr(ref, n))
               for n in ("indptr", "indices", "train", "features"))
    dist.barrier()
    if rank == 0:  # a write by the owner is seen by every rank: one physical copy
        g.features[5, 3] = 1234.5
    dist.barrier()
    seen = float(g.features[5, 3])
    with open(os.path.join(outdir, f"r{rank}.txt"), "w") as f:
        f.write(f"{int(same)} {seen} {int(sg.owner)} {g.features.ctypes.data % 4096}")
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_node_shared_graph(tmp_path, world):
    """Local rank 0 generates the graph into memfds; the other ranks map the same pages
    (values equal the private generator's, writes are shared, features page-aligned for
    cudaHostRegister)."""
    mp.spawn(_shm_worker, args=(world, free_port(), str(tmp_path)), nprocs=world, join=True)
    for r in range(world):
        same, seen, owner, align = open(tmp_path / f"r{r}.txt").read().split()
        assert same == "1" and float(seen) == 1234.5 and int(align) == 0
        assert int(owner) == (r == 0)


# ------------------------------------------- per-NUMA-node feature replicas
def _numa_worker(rank, world, port, outdir, nodes):
    import synth
    from synth import shm
    _init(rank, world, port)
    store = dist.distributed_c10d._get_default_store()
    sg = shm.make_graph_shared("tiny", rank, world, store, numa_node=nodes[rank])
    g = sg.graph
    ref = synth.make_graph("tiny")
    same = all(np.array_equal(getattr(g, n), getattr(ref, n))
               for n in ("indptr", "indices", "train", "features"))
    dist.barrier()
    # a write by the first rank of each node is seen by exactly the ranks of that node
    if rank == min(r for r in range(world) if nodes[r] == nodes[rank]):
        g.features[2, 1] = 100.0 + nodes[rank]
    dist.barrier()
    seen = float(g.features[2, 1])
    with open(os.path.join(outdir, f"n{rank}.txt"), "w") as f:
        f.write(f"{int(same)} {seen} {g.features.ctypes.data % 4096}")
    dist.barrier()
    dist.destroy_process_group()


def test_numa_feature_replicas(tmp_path):
    """Four local ranks on two NUMA nodes (0, 1, 0, 1): every rank sees the generator's
    values; the ranks of a node share one feature copy and the two nodes' copies are
    distinct memory (a write on one node's copy is invisible on the other's)."""
    nodes = [0, 1, 0, 1]
    world = len(nodes)
    mp.spawn(_numa_worker, args=(world, free_port(), str(tmp_path), nodes), nprocs=world,
             join=True)
    for r in range(world):
        same, seen, align = open(tmp_path / f"n{r}.txt").read().split()
        assert same == "1" and int(align) == 0
        assert float(seen) == 100.0 + nodes[r]
