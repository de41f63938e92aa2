"""NEXT-3 peer-sharded cache (§9 "cross-GPU access"):
W cache shards, each ctx holding the rows of global rank i % W == rank, extract reading
other shards through mapped device pointers.  gpurun gives one GPU, so the W "peers"
here share cuda:0: in one process through glb_cache_device_ptr, and in two processes
through CUDA IPC handles (the path an 8-GPU box uses over NVLink).  Everything is
bit-exact against the oracle: global slots, shard contents, gathered feature bytes and
the (hits, misses, peer hits) counts."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402


def u32(t):
    return t.cpu().numpy().view(np.uint32)


def make_group(g, world, alpha, kind="khop", mode="auto"):
    sh = g.shape
    ctxs = []
    for r in range(world):
        c = glb.Context(0)
        c.load_graph(g.indptr, g.indices, g.features)
        c.set_relabel_mode(mode)
        c.set_sampler(kind, fanouts=sh.fanouts, max_batch=sh.batch)
        c.set_train_set(g.train, sh.batch, g.seed)
        c.set_count_mode(glb.COUNT_PRESAMPLE)
        c.presample(1)
        c.set_count_mode(glb.COUNT_NONE)
        c.build_cache_sharded(alpha, r, world)
        ctxs.append(c)
    for r, c in enumerate(ctxs):
        for p, o in enumerate(ctxs):
            if p != r:
                c.attach_peer_cache(p, dev_ptr=o.cache_device_ptr()[0])
    return ctxs


@pytest.fixture(scope="module")
def tiny():
    g = synth.make_graph("tiny")
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    counts = go.presample("khop", g.train, g.shape.batch, g.shape.fanouts, g.seed, 1)
    return g, go, counts


@pytest.mark.parametrize("world,alpha", [(2, 0.05), (3, 0.1), (4, 0.3), (8, 0.02), (2, 0.0)])
@pytest.mark.parametrize("mode", ["dense", "hash", "dense_hitlist"])
def test_sharded_extract_sample_bit_exact(tiny, world, alpha, mode, monkeypatch):
    """dense_hitlist: hits gathered from the hit list (GLB_GATHER_LIDORDER=0) instead of in
    lid order from the marks (the default)."""
    if mode.endswith("_hitlist"):
        monkeypatch.setenv("GLB_GATHER_LIDORDER", "0")
        mode = mode[:-8]
    g, go, counts = tiny
    sh = g.shape
    slot, shards = oracle.sharded_cache(counts, alpha, world)
    ctxs = make_group(g, world, alpha, mode=mode)
    for r, c in enumerate(ctxs):
        assert np.array_equal(c.cache_slots(), slot)
        assert c.cache_size == int((slot >= 0).sum())
        ptr, rows = c.cache_device_ptr()
        assert rows == shards[r].shape[0]
        if rows:  # the shard's rows are exactly the oracle's feature rows
            view = glb._view(ptr, rows * g.shape.D, "<f4", c, c.device).view(rows, g.shape.D)
            assert np.array_equal(view.cpu().numpy().view(np.uint32),
                                  go.extract(shards[r]).view(np.uint32))
    e = 1
    batches = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
    for r, c in enumerate(ctxs):
        c.shuffle(e)
        for b in [0, 7, len(batches) - 1]:
            c.sample_batch(e, b)
            s = c.sample_result()
            out = torch.full((s.sizes[-1] + 3, sh.D), float("nan"), device="cuda:0")
            c.extract_sample(out)
            cnt = c.last_extract_counts()
            uniq = go.sample_khop(batches[b], sh.fanouts, g.seed, e, b).uniq
            assert np.array_equal(u32(s.uniq), uniq)
            got = out[: s.sizes[-1]].cpu().numpy()
            assert np.array_equal(got.view(np.uint32), go.extract(uniq).view(np.uint32))
            h, m, p = oracle.extract_counts(uniq, slot, r, world)
            assert (cnt["hits"], cnt["misses"], cnt["peer_hits"]) == (h, m, p)
            if world > 1 and alpha > 0:
                assert p > 0
    for c in ctxs:
        c.close()


def test_sharded_generic_extract_duplicates(tiny):
    g, go, counts = tiny
    world, alpha = 3, 0.1
    slot, _ = oracle.sharded_cache(counts, alpha, world)
    ctxs = make_group(g, world, alpha)
    rng = np.random.default_rng(4)
    ids = rng.integers(0, g.shape.V, 5003).astype(np.uint32)
    ids[100:200] = ids[0]  # duplicates
    dev = torch.from_numpy(ids.view(np.int32)).cuda()
    for r, c in enumerate(ctxs):
        out, st = c.extract(dev, stats=True)
        assert np.array_equal(out.cpu().numpy().view(np.uint32), go.extract(ids).view(np.uint32))
        cnt = c.last_extract_counts()
        assert (cnt["hits"], cnt["misses"], cnt["peer_hits"]) == oracle.extract_counts(ids, slot, r, world)
        assert (st["hits"], st["misses"]) == (cnt["hits"], cnt["misses"])
    for c in ctxs:
        c.close()


def test_sharded_full_coverage_and_world1(tiny):
    """world * alpha >= 1: every row is cached somewhere (no host reads); world 1 equals
    build_cache."""
    g, go, counts = tiny
    ctxs = make_group(g, 4, 0.25)
    assert np.all(ctxs[0].cache_slots() >= 0)
    c = ctxs[2]
    c.shuffle(0)
    c.sample_batch(0, 3)
    s = c.sample_result()
    out = torch.empty((s.sizes[-1], g.shape.D), device="cuda:0")
    c.extract_sample(out)
    cnt = c.last_extract_counts()
    assert cnt["misses"] == 0 and cnt["hits"] == s.sizes[-1]
    for x in ctxs:
        x.close()
    a = make_group(g, 1, 0.1)[0]
    b = glb.Context(0)
    b.load_graph(g.indptr, g.indices, g.features)
    b.set_sampler("khop", fanouts=g.shape.fanouts, max_batch=g.shape.batch)
    b.set_train_set(g.train, g.shape.batch, g.seed)
    b.set_count_mode(glb.COUNT_PRESAMPLE)
    b.presample(1)
    b.build_cache(0.1)
    assert np.array_equal(a.cache_slots(), b.cache_slots())
    assert a.cache_device_ptr()[1] == b.cache_device_ptr()[1] == int(0.1 * g.shape.V)


def test_sharded_errors(tiny):
    g, _, _ = tiny
    c = glb.Context(0)
    c.load_graph(g.indptr, g.indices, g.features)
    c.set_sampler("khop", fanouts=g.shape.fanouts, max_batch=g.shape.batch)
    with pytest.raises(glb.GlbError) as ei:
        c.build_cache_sharded(0.1, 2, 2)
    assert ei.value.code == glb.EINVAL
    with pytest.raises(glb.GlbError):
        c.build_cache_sharded(0.1, 0, glb.MAX_SHARDS + 1)
    with pytest.raises(glb.GlbError) as ei:
        c.attach_peer_cache(1, dev_ptr=1)  # not sharded yet
    assert ei.value.code == glb.ESTATE
    c.build_cache_sharded(0.1, 0, 2)
    ids = torch.arange(10, dtype=torch.int32, device="cuda:0")
    with pytest.raises(glb.GlbError) as ei:
        c.extract(ids)  # shard 1 not attached
    assert ei.value.code == glb.ESTATE
    with pytest.raises(glb.GlbError) as ei:
        c.attach_peer_cache(0, dev_ptr=c.cache_device_ptr()[0])  # own rank
    assert ei.value.code == glb.EINVAL
    with pytest.raises(glb.GlbError):
        c.attach_peer_cache(1)  # neither handle nor pointer
    c.close()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, world, port, alpha, outdir):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = synth.make_graph("tiny")
    sh = g.shape
    c = glb.Context(0)
    c.load_graph(g.indptr, g.indices, g.features)
    c.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    c.set_train_set(g.train, sh.batch, g.seed)
    c.set_count_mode(glb.COUNT_PRESAMPLE)
    c.presample(1, rank, world)           # DP presample + count all-reduce (§8(e))
    cnt = c.counts_tensor(glb.COUNT_PRESAMPLE).cpu()
    dist.all_reduce(cnt)
    c.counts_tensor(glb.COUNT_PRESAMPLE).copy_(cnt.cuda())
    c.set_count_mode(glb.COUNT_NONE)
    c.build_cache_sharded(alpha, rank, world)
    handles = [None] * world
    dist.all_gather_object(handles, c.cache_ipc_handle())
    for p in range(world):
        if p != rank:
            c.attach_peer_cache(p, ipc_handle=handles[p])
    c.shuffle(2)
    res = {}
    for b in range(rank, 16, world):
        c.sample_batch(2, b)
        s = c.sample_result()
        out = torch.empty((s.sizes[-1], sh.D), device="cuda:0")
        c.extract_sample(out)
        k = c.last_extract_counts()
        res[b] = (u32(s.uniq), out.cpu().numpy(), (k["hits"], k["misses"], k["peer_hits"]))
    np.save(os.path.join(outdir, f"r{rank}.npy"), np.array([res], dtype=object), allow_pickle=True)
    dist.barrier()  # peers keep their shards alive until every rank has read them
    c.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_ipc_processes(tiny, tmp_path, world):
    import torch.multiprocessing as mp
    g, go, counts = tiny
    sh = g.shape
    alpha = 0.08
    mp.spawn(_ipc_worker, args=(world, _free_port(), alpha, str(tmp_path)), nprocs=world,
             join=True)
    slot, _ = oracle.sharded_cache(counts, alpha, world)
    batches = oracle.epoch_batches(g.train, sh.batch, g.seed, 2)
    seen = 0
    for r in range(world):
        res = np.load(os.path.join(tmp_path, f"r{r}.npy"), allow_pickle=True)[0]
        for b, (uniq, feats, cnt) in res.items():
            exp = go.sample_khop(batches[b], sh.fanouts, g.seed, 2, b).uniq
            assert np.array_equal(uniq, exp)
            assert np.array_equal(feats.view(np.uint32), go.extract(exp).view(np.uint32))
            assert cnt == oracle.extract_counts(exp, slot, r, world)
            seen += 1
    assert seen == 16
