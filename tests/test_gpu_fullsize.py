"""Full-size parity for BASELINE configs[2..4] (TW 3-hop GCN, PA PinSAGE random
walk with PreSC#K, UK GraphSAGE) and the weighted TWW: PreSC counts over all K
presample epochs (oracle sharded by batch over host threads, summed exactly),
cache slots at the config's alphas, every output of four measured batches
(first, second, a random one, the last partial one) at the paper's R% -- so
the PCIe miss path runs -- and one at alpha = 1, with EVERY extracted byte
compared, all in the launch configuration bench.py uses.  Host RAM: TW ~50 GB, PA ~65 GB,
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


def oracle_sample(go, sh, seeds, seed, e, b, weights=None):
    if sh.sampler == "khop":
        return go.sample_khop(seeds, sh.fanouts, seed, e, b)
    if sh.sampler == "weighted":
        return go.sample_khop_weighted(weights, seeds, sh.fanouts, seed, e, b)
    return go.sample_rwalk(seeds, len(sh.fanouts), seed, e, b, synth.RW_WALKS, synth.RW_LEN,
                           sh.fanouts[0])


CHUNK = 1 << 18  # rows per host compare


def assert_rows_exact(go, out, uniq):
    """EVERY gathered byte of out[:n] against the oracle's extract (a7: memcpy of row
    uniq[i] of the host matrix), in chunks of CHUNK rows (device->host copy + compare)."""
    n = uniq.shape[0]
    for a in range(0, n, CHUNK):
        b = min(n, a + CHUNK)
        got = out[a:b].cpu().numpy().view(np.uint32)
        want = go.extract(uniq[a:b]).view(np.uint32)
        if not np.array_equal(got, want):
            bad = np.nonzero((got != want).any(axis=1))[0]
            raise AssertionError(f"{bad.size} rows differ in [{a}, {b}), first lid {a + bad[0]}")


def oracle_counts_parallel(g, sh, epochs):
    """Oracle visit counts, batches sharded over threads (each with its own scratch)."""
    jobs = [(e, b, s) for e in epochs
            for b, s in enumerate(oracle.epoch_batches(g.train, sh.batch, g.seed, e))]
    shards = [jobs[i::THREADS] for i in range(THREADS)]

    def run(shard):
        go = oracle.GraphOracle(g.indptr, g.indices)
        c = np.zeros(g.V, np.uint32)
        for e, b, s in shard:
            c[oracle_sample(go, sh, s, g.seed, e, b, g.weights).uniq] += 1
        return c

    with cf.ThreadPoolExecutor(THREADS) as ex:
        return sum(ex.map(run, shards)).astype(np.uint32)


def make_sampler_ctx(g, sh, features=True, relabel="auto"):
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features if features else None)
    ctx.set_relabel_mode(relabel)
    if g.weights is not None:
        ctx.load_edge_weights(g.weights)
    if sh.sampler in ("khop", "weighted"):
        ctx.set_sampler(sh.sampler, fanouts=sh.fanouts, max_batch=sh.batch)
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
        assert_rows_exact(go, out, os_.uniq)
        assert st["hits"] == int((slot_map[os_.uniq] >= 0).sum())
        assert trainer.handoff_tag() == b
        trainer.handoff_release(i % 2)
    sampler.close()


def check_batches(ctx, g, sh, go, e, batches, out, slot_map):
    """Every output of the given batches of epoch e: sizes, uniq, every block (and RW
    weights), the a4 marks, hit count, and every extracted byte."""
    ob = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
    for b in batches:
        ctx.sample_batch(e, b)
        s = ctx.sample_result()
        os_ = oracle_sample(go, sh, ob[b], g.seed, e, b, g.weights)
        assert s.sizes == os_.sizes, b
        assert np.array_equal(u32(s.uniq), os_.uniq)
        for l in range(len(sh.fanouts)):
            assert np.array_equal(u32(s.indptr[l]), os_.indptr[l]), (b, l)
            assert np.array_equal(u32(s.indices[l]), os_.indices[l]), (b, l)
            if sh.sampler == "rwalk":
                assert np.array_equal(u32(s.weights[l]), os_.weights[l]), (b, l)
        assert np.array_equal(s.cache_slot.cpu().numpy(), slot_map[os_.uniq]), b
        st = ctx.extract_sample(out, stats=True)
        assert st["hits"] == int((slot_map[os_.uniq] >= 0).sum())
        assert st["misses"] == int((slot_map[os_.uniq] < 0).sum())
        assert_rows_exact(go, out, os_.uniq)


def check_config(name, Ks=None, handoff=False, relabel_modes=("auto",)):
    """PreSC#K counts in full (every K), cache slots at every alpha of the config, then
    four measured batches (first, second, a random one, the last partial one) at the
    paper's R% (sh.alphas[0]: misses over PCIe) and one at alpha = 1 (all HBM hits), every
    output and every extracted byte; optionally again in other relabel modes."""
    sh = synth.SHAPES[name]
    g = synth.make_graph(sh)
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    counts_by_K = {}
    ub = sh.batch
    for k in sh.fanouts:
        ub = min(ub * (1 + k), sh.V)
    out = torch.empty((ub, sh.D), dtype=torch.float32, device="cuda")
    ctx = None
    for mode in relabel_modes:
        ctx = make_sampler_ctx(g, sh, relabel=mode)
        ctx.set_pipeline(2)  # bench.py's launch configuration (extract stream, misses first)
        if 4 * sh.D <= 512:  # ... and its host-assisted misses for <= 512-byte rows
            ctx.set_host_gather(0.15, threads=4)
        if mode != "auto":
            assert ctx.relabel_mode == mode
        for K in (Ks or [sh.K]):
            ctx.reset_counts(glb.COUNT_PRESAMPLE)
            ctx.presample(K)
            if K not in counts_by_K:
                counts_by_K[K] = oracle_counts_parallel(g, sh, range(K))
            counts = counts_by_K[K]
            assert np.array_equal(ctx.get_counts(glb.COUNT_PRESAMPLE), counts), (mode, K)
            if mode == relabel_modes[0]:
                for a in sh.alphas:
                    ctx.build_cache(a)
                    assert np.array_equal(ctx.cache_slots(), oracle.cache_slots(counts, a)), (K, a)
        e = max(Ks or [sh.K])
        nb = -(-len(g.train) // sh.batch)
        rng = np.random.default_rng(0)
        a0 = sh.alphas[0]
        ctx.set_cold_store(4 * sh.D <= 512)  # the bench's cold store for <= 512-byte rows
        ctx.build_cache(a0)
        slot_map = oracle.cache_slots(counts, a0)
        assert a0 < 1.0
        check_batches(ctx, g, sh, go, e, [0, 1, int(rng.integers(2, nb - 1)), nb - 1], out,
                      slot_map)
        ctx.set_cold_store(False)
        ctx.build_cache(1.0)
        check_batches(ctx, g, sh, go, e, [int(rng.integers(0, nb))], out,
                      oracle.cache_slots(counts, 1.0))
        if mode != relabel_modes[-1]:
            ctx.close()
    if handoff:
        ctx.build_cache(a0)
        check_handoff(g, sh, go, ctx, oracle.cache_slots(counts, a0), e)
    ctx.close()


def test_tw_fullsize():
    """configs[2]; also in hash relabel mode (bit-identical by construction)."""
    check_config("TW", relabel_modes=("auto", "hash"))


def test_tww_weighted_fullsize():
    """NEXT-1 at Twitter size: 3-hop weighted k-hop (edge weight = target year)."""
    check_config("TWW")


def test_pa_fullsize_presc_k123():
    check_config("PA", Ks=[1, 2, 3])


def test_uk_fullsize():
    """configs[4]: also the factored sampler -> trainer handoff at full size."""
    check_config("UK", handoff=True)
