"""a8 factored Sampler -> Trainer handoff over peer memory (include/glb.h glb_handoff_*;
PAPER.md Fig 9 L217-L246, L250-L252 §5.2).  gpurun gives one GPU, so sampler and trainer
share cuda:0: two ctxs in one process (borrowed pointers / events), and two processes
exchanging real CUDA IPC handles (the path an 8-GPU box takes over NVLink).  Everything the
trainer sees is bit-exact against the oracle: sizes, uniq, every block (and random-walk
weights), the trainer-side marks against ITS cache, the gathered feature bytes, and the
hit/miss counts."""
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


def make(g, kind, fanouts, alpha, layers=None):
    sh = g.shape
    c = glb.Context(0)
    c.load_graph(g.indptr, g.indices, g.features)
    c.set_sampler(kind, fanouts=fanouts, layers=layers, max_batch=sh.batch)
    c.set_train_set(g.train, sh.batch, g.seed)
    if alpha is not None:
        c.set_count_mode(glb.COUNT_PRESAMPLE)
        c.presample(1)
        c.set_count_mode(glb.COUNT_NONE)
        c.build_cache(alpha)
    return c


def expected(go, kind, batches, sh, g, e, b, layers):
    if kind == "khop":
        return go.sample_khop(batches[b], sh.fanouts, g.seed, e, b)
    return go.sample_rwalk(batches[b], layers, g.seed, e, b)


@pytest.fixture(scope="module")
def tiny():
    g = synth.make_graph("tiny")
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    counts = go.presample("khop", g.train, g.shape.batch, g.shape.fanouts, g.seed, 1)
    return g, go, counts


@pytest.mark.parametrize("kind,layers", [("khop", None), ("rwalk", 2)])
@pytest.mark.parametrize("pipeline", [1, 2])
def test_handoff_same_process_bit_exact(tiny, kind, layers, pipeline):
    g, go, counts = tiny
    sh = g.shape
    alpha = 0.3
    trainer = make(g, kind, sh.fanouts, alpha, layers)  # PreSC#1 with its own sampler
    if kind != "khop":
        counts = go.presample("rwalk", g.train, sh.batch, (5,) * layers, g.seed, 1)
    trainer.set_pipeline(pipeline)
    sampler = make(g, kind, sh.fanouts, None, layers)  # samplers hold no cache
    sampler.set_pipeline(pipeline)
    slots = 3
    blob = trainer.handoff_create(slots)
    trainer.handoff_connect(5, sampler.handoff_attach(2, blob))
    slot_map = oracle.cache_slots(counts, alpha)
    assert np.array_equal(trainer.cache_slots(), slot_map)
    e = 1
    batches = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
    order = [0, 1, 2, 3, 7, len(batches) - 1, 4, 5]
    for i, b in enumerate(order):
        s = i % slots
        sampler.sample_batch(e, b)
        sampler.handoff_send(2, s, 1000 + b)
        trainer.handoff_recv(5, s)
        exp = expected(go, kind, batches, sh, g, e, b, layers)
        got = trainer.sample_result()
        assert got.num_seeds == len(batches[b])
        assert got.sizes == exp.sizes
        assert np.array_equal(u32(got.uniq), exp.uniq)
        for l in range(len(exp.indices)):
            assert np.array_equal(u32(got.indptr[l]), exp.indptr[l])
            assert np.array_equal(u32(got.indices[l]), exp.indices[l])
            if kind == "rwalk":
                assert np.array_equal(u32(got.weights[l]), exp.weights[l])
        # a4 on the trainer: its own cache map
        assert np.array_equal(got.cache_slot.cpu().numpy(), slot_map[exp.uniq])
        assert trainer.handoff_tag() == 1000 + b
        out = torch.full((exp.sizes[-1] + 2, sh.D), float("nan"), device="cuda:0")
        st = trainer.extract_sample(out, stats=True)
        assert np.array_equal(out[: exp.sizes[-1]].cpu().numpy().view(np.uint32),
                              go.extract(exp.uniq).view(np.uint32))
        hits = int((slot_map[exp.uniq] >= 0).sum())
        assert (st["hits"], st["misses"]) == (hits, exp.sizes[-1] - hits)
        trainer.handoff_release(s)
    # the sampler's own sample is untouched by the pushes
    sampler.sample_batch(e, 9)
    assert np.array_equal(u32(sampler.sample_result().uniq),
                          expected(go, kind, batches, sh, g, e, 9, layers).uniq)
    sampler.close()
    trainer.close()


def test_handoff_errors(tiny):
    g, _, _ = tiny
    sh = g.shape
    t = make(g, "khop", sh.fanouts, 0.1)
    s = make(g, "khop", sh.fanouts, None)
    with pytest.raises(glb.GlbError):
        t.handoff_create(0)
    with pytest.raises(glb.GlbError):
        t.handoff_create(glb.HANDOFF_MAX_SLOTS + 1)
    with pytest.raises(glb.GlbError):  # not attached
        s.handoff_send(0, 0, 0)
    with pytest.raises(glb.GlbError):  # no ring
        t.handoff_recv(0, 0)
    blob = t.handoff_create(2)
    big = make(g, "khop", (25, 10), None)  # larger capacity than the trainer's slots
    with pytest.raises(glb.GlbError):
        big.handoff_attach(0, blob)
    rw = make(g, "rwalk", sh.fanouts, None, layers=2)
    with pytest.raises(glb.GlbError):  # other sampler kind
        rw.handoff_attach(0, blob)
    with pytest.raises(glb.GlbError):  # not a blob
        s.handoff_attach(0, bytes(glb.HANDOFF_BLOB_BYTES))
    t.handoff_connect(1, s.handoff_attach(0, blob))
    with pytest.raises(glb.GlbError):  # no current sample
        s.handoff_send(0, 0, 0)
    s.shuffle(0)
    s.sample_batch(0, 0)
    with pytest.raises(glb.GlbError):
        s.handoff_send(0, 2, 0)  # slot out of range
    with pytest.raises(glb.GlbError):
        t.handoff_recv(3, 0)  # sampler 3 not connected
    for c in (t, s, big, rw):
        c.close()


# ------------------------------------------------------------------ two processes (IPC)
def free_port():
    so = socket.socket()
    so.bind(("127.0.0.1", 0))
    p = so.getsockname()[1]
    so.close()
    return p


def _worker(rank, world, port, outdir, ns, total, switching=False):
    import torch.distributed as dist

    from paper_conf_eurosys_yangtswycyz22_b200 import parallel as par
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = synth.make_graph("tiny")
    sh = g.shape
    roles = par.Roles(ns, world)
    # samplers hold no cache, unless they may switch to standby trainers (same cache here)
    ctx = make(g, "khop", sh.fanouts, 0.2 if switching or not roles.is_sampler(rank) else None)
    ctx.set_pipeline(2)
    ho = par.PeerHandoff(ctx, roles, rank, slots=2)
    store = dist.distributed_c10d._get_default_store()
    nb = ctx.num_batches
    res = {}

    def extract_fn(gi, tag=None):
        s = ctx.sample_result()
        out = torch.empty((s.sizes[-1], sh.D), dtype=torch.float32, device="cuda:0")
        st = ctx.extract_sample(out, stats=True)
        res[gi] = (ctx.handoff_tag() if tag is None else tag, u32(s.uniq).copy(),
                   [u32(x).copy() for x in s.indptr], [u32(x).copy() for x in s.indices],
                   out.cpu().numpy().view(np.uint32).copy(), st["hits"])
        if switching and tag is None:
            import time
            time.sleep(0.01)  # slow trainers: samplers would idle (the switching case, L265)

    if roles.is_sampler(rank):
        def sample_fn(gi):
            ctx.sample_batch(1 + gi // nb, gi % nb)
        standby = (lambda gi: extract_fn(gi, tag=gi)) if switching else None
        par.run_sampler_peer(sample_fn, ho, total, store, "h", standby_fn=standby,
                             t_train=0.01, t_standby=0.001)
        assert ho.standby == len(res)
    else:
        par.run_trainer_peer(extract_fn, ho, total, store, "h")
    np.save(os.path.join(outdir, f"r{rank}.npy"), np.array([res], dtype=object), allow_pickle=True)
    torch.cuda.synchronize()
    dist.barrier()
    ctx.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,ns,switching", [(2, 1, False), (3, 2, False), (3, 1, False),
                                                (2, 1, True), (3, 1, True)])
def test_handoff_two_processes_ipc_bit_exact(tiny, tmp_path, world, ns, switching):
    """...and with dynamic executor switching: batches a sampler
    extracted as a standby trainer are bit-exact too, and every batch is extracted once."""
    import torch.multiprocessing as mp
    g, go, counts = tiny
    sh = g.shape
    total = 21  # crosses an epoch boundary (16 batches per epoch), reuses every slot
    mp.spawn(_worker, args=(world, free_port(), str(tmp_path), ns, total, switching),
             nprocs=world, join=True)
    slot_map = oracle.cache_slots(counts, 0.2)
    nb = (len(g.train) + sh.batch - 1) // sh.batch
    seen = set()
    n_standby = 0
    for r in range(world):
        res = np.load(os.path.join(tmp_path, f"r{r}.npy"), allow_pickle=True)[0]
        for gi, (tag, uniq, indptr, indices, feats, hits) in res.items():
            e, b = 1 + gi // nb, gi % nb
            assert tag == gi
            exp = go.sample_khop(oracle.epoch_batches(g.train, sh.batch, g.seed, e)[b],
                                 sh.fanouts, g.seed, e, b)
            assert np.array_equal(uniq, exp.uniq)
            for l in range(len(exp.indices)):
                assert np.array_equal(indptr[l], exp.indptr[l])
                assert np.array_equal(indices[l], exp.indices[l])
            assert np.array_equal(feats, go.extract(exp.uniq).view(np.uint32).reshape(-1, sh.D))
            assert hits == int((slot_map[exp.uniq] >= 0).sum())
            assert gi not in seen
            seen.add(gi)
            n_standby += r < ns
    assert seen == set(range(total))
    assert (n_standby > 0) == switching
