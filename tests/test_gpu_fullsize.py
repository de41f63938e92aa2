"""Full-size parity for BASELINE configs[2..4] (TW 3-hop GCN, PA PinSAGE random
walk with PreSC#K, UK GraphSAGE): PreSC counts over all K presample epochs
(oracle sharded by batch over host threads, summed exactly), cache slots at
the config's alphas, every output of four measured batches (first, second, a
random one, the last partial one) and sampled extracted rows, all in the
launch configuration bench.py uses.  Host RAM: TW ~50 GB, PA ~65 GB,
UK ~95 GB (features in pinned memory)."""
import concurrent.futures as cf
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu, pytest.mark.slow]

import oracle  # noqa: E402
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402

THREADS = min(32, os.cpu_count() or 1)


def u32(t):
    return t.cpu().numpy().view(np.uint32)


def oracle_sample(go, sh, seeds, seed, e, b):
    if sh.sampler == "khop":
        return go.sample_khop(seeds, sh.fanouts, seed, e, b)
    return go.sample_rwalk(seeds, len(sh.fanouts), seed, e, b, synth.RW_WALKS, synth.RW_LEN,
                           sh.fanouts[0])


def oracle_counts_parallel(g, sh, epochs):
    """Oracle visit counts, batches sharded over threads (each with its own scratch)."""
    jobs = [(e, b, s) for e in epochs
            for b, s in enumerate(oracle.epoch_batches(g.train, sh.batch, g.seed, e))]
    shards = [jobs[i::THREADS] for i in range(THREADS)]

    def run(shard):
        go = oracle.GraphOracle(g.indptr, g.indices)
        c = np.zeros(g.V, np.uint32)
        for e, b, s in shard:
            c[oracle_sample(go, sh, s, g.seed, e, b).uniq] += 1
        return c

    with cf.ThreadPoolExecutor(THREADS) as ex:
        return sum(ex.map(run, shards)).astype(np.uint32)


def make_sampler_ctx(g, sh, features=True):
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features if features else None)
    if sh.sampler == "khop":
        ctx.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    else:
        ctx.set_sampler("rwalk", layers=len(sh.fanouts), walks=synth.RW_WALKS,
                        walk_len=synth.RW_LEN, topk=sh.fanouts[0], max_batch=sh.batch)
    ctx.set_train_set(g.train, sh.batch, g.seed)
    return ctx


def check_handoff(g, sh, go, trainer, slot_map, e):
    """a8 at full size (config 5's factored split): a topology-only sampler ctx pushes
    batches into the trainer ctx's HBM ring (glb_handoff_*); the trainer marks them against
    its cache and extracts.  Bit-exact samples, sampled rows and hit counts."""
    sampler = make_sampler_ctx(g, sh, features=False)  # samplers hold no features / cache
    trainer.handoff_connect(0, sampler.handoff_attach(1, trainer.handoff_create(2)))
    ob = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
    nb = len(ob)
    rng = np.random.default_rng(1)
    ub = sh.batch
    for k in sh.fanouts:
        ub = min(ub * (1 + k), sh.V)
    out = torch.empty((ub, sh.D), dtype=torch.float32, device="cuda")
    for i, b in enumerate([0, 1, int(rng.integers(2, nb - 1)), nb - 1]):
        sampler.sample_batch(e, b)
        sampler.handoff_send(1, i % 2, b)
        trainer.handoff_recv(0, i % 2)
        s = trainer.sample_result()
        os_ = oracle_sample(go, sh, ob[b], g.seed, e, b)
        assert s.sizes == os_.sizes, b
        assert np.array_equal(u32(s.uniq), os_.uniq)
        for l in range(len(sh.fanouts)):
            assert np.array_equal(u32(s.indptr[l]), os_.indptr[l]), (b, l)
            assert np.array_equal(u32(s.indices[l]), os_.indices[l]), (b, l)
        assert np.array_equal(s.cache_slot.cpu().numpy(), slot_map[os_.uniq])
        st = trainer.extract_sample(out, stats=True)
        idx = rng.integers(0, s.sizes[-1], 2048)
        got = out[torch.from_numpy(idx).cuda()].cpu().numpy()
        assert np.array_equal(got.view(np.uint32), g.features[os_.uniq[idx]].view(np.uint32))
        assert st["hits"] == int((slot_map[os_.uniq] >= 0).sum())
        assert trainer.handoff_tag() == b
        trainer.handoff_release(i % 2)
    sampler.close()


def check_config(name, Ks=None, handoff=False):
    sh = synth.SHAPES[name]
    g = synth.make_graph(sh)
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features)
    if sh.sampler == "khop":
        ctx.set_sampler("khop", fanouts=sh.fanouts, max_batch=sh.batch)
    else:
        ctx.set_sampler("rwalk", layers=len(sh.fanouts), walks=synth.RW_WALKS,
                        walk_len=synth.RW_LEN, topk=sh.fanouts[0], max_batch=sh.batch)
    ctx.set_train_set(g.train, sh.batch, g.seed)
    for K in (Ks or [sh.K]):
        ctx.reset_counts(glb.COUNT_PRESAMPLE)
        ctx.presample(K)
        counts = oracle_counts_parallel(g, sh, range(K))
        assert np.array_equal(ctx.get_counts(glb.COUNT_PRESAMPLE), counts), f"PreSC#{K}"
        for a in sh.alphas:
            ctx.build_cache(a)
            assert np.array_equal(ctx.cache_slots(), oracle.cache_slots(counts, a)), (K, a)
    e = max(Ks or [sh.K])
    ob = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
    nb = len(ob)
    rng = np.random.default_rng(0)
    ub = sh.batch
    for k in sh.fanouts:
        ub = min(ub * (1 + k), sh.V)
    out = torch.empty((ub, sh.D), dtype=torch.float32, device="cuda")
    for b in [0, 1, int(rng.integers(2, nb - 1)), nb - 1]:
        ctx.sample_batch(e, b)
        s = ctx.sample_result()
        os_ = oracle_sample(go, sh, ob[b], g.seed, e, b)
        assert s.sizes == os_.sizes, b
        assert np.array_equal(u32(s.uniq), os_.uniq)
        for l in range(len(sh.fanouts)):
            assert np.array_equal(u32(s.indptr[l]), os_.indptr[l]), (b, l)
            assert np.array_equal(u32(s.indices[l]), os_.indices[l]), (b, l)
            if sh.sampler == "rwalk":
                assert np.array_equal(u32(s.weights[l]), os_.weights[l]), (b, l)
        st = ctx.extract_sample(out, stats=True)
        idx = rng.integers(0, s.sizes[-1], 2048)
        got = out[torch.from_numpy(idx).cuda()].cpu().numpy()
        assert np.array_equal(got.view(np.uint32), g.features[os_.uniq[idx]].view(np.uint32))
        slot = ctx.cache_slots()
        assert st["hits"] == int((slot[os_.uniq] >= 0).sum())
    if handoff:
        check_handoff(g, sh, go, ctx, oracle.cache_slots(counts, sh.alphas[-1]), e)
    ctx.close()


def test_tw_fullsize():
    check_config("TW")


def test_pa_fullsize_presc_k123():
    check_config("PA", Ks=[1, 2, 3])


def test_uk_fullsize():
    """configs[4]: also the factored sampler -> trainer handoff at full size."""
    check_config("UK", handoff=True)
