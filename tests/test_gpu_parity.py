"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle,
element by element, bit-exact (integer ids, counts, slots; feature bytes).

Sizes: the tiny config (BASELINE configs[0]) everywhere, small power-law
graphs for ragged tails / wide fanouts / random walks, and the full PR config
(configs[1]) in the launch configuration bench.py times, on sampled batches
(first, second, a random one, the last partial one) plus full PreSC counts.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
import paper_conf_eurosys_yangtswycyz22_b200 as glb  # noqa: E402
import synth  # noqa: E402


def u32(t):
    return t.cpu().numpy().view(np.uint32)


def assert_same_sample(gs, os_, weighted=False):
    assert gs.sizes == os_.sizes
    assert np.array_equal(u32(gs.uniq), os_.uniq)
    for l in range(len(os_.indices)):
        assert np.array_equal(u32(gs.indptr[l]), os_.indptr[l]), f"indptr hop {l}"
        assert np.array_equal(u32(gs.indices[l]), os_.indices[l]), f"indices hop {l}"
        if weighted:
            assert np.array_equal(u32(gs.weights[l]), os_.weights[l]), f"weights hop {l}"


MODES = ["dense", "hash"]


def make_ctx(g, kind="khop", fanouts=(10, 5), max_batch=None, layers=None, mode="auto"):
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features)
    ctx.set_relabel_mode(mode)
    ctx.set_sampler(kind, fanouts=fanouts, layers=layers,
                    max_batch=max_batch or g.shape.batch)
    if mode != "auto":
        assert ctx.relabel_mode == mode
    ctx.set_train_set(g.train, g.shape.batch, g.seed)
    return ctx


@pytest.fixture(scope="module")
def tiny():
    g = synth.make_graph("tiny")
    return g, oracle.GraphOracle(g.indptr, g.indices, g.features)


def test_worked_example_on_gpu():
    import json
    import os
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden",
                                       "survey_worked_example.json")))
    indptr = np.array(gold["graph"]["indptr"], np.uint64)
    indices = np.array(gold["graph"]["indices"], np.uint32)
    feats = synth.gen_features(8, 32, 42)
    ctx = glb.Context(0)
    ctx.load_graph(indptr, indices, feats)
    ctx.set_sampler("khop", fanouts=(3, 2), max_batch=8)
    s = ctx.sample(np.array([0, 5], np.uint32), seed=42, epoch=0, batch=0)
    assert u32(s.uniq).tolist() == gold["khop"]["uniq"]
    for l, b in enumerate(gold["khop"]["blocks"]):
        assert u32(s.indptr[l]).tolist() == b["indptr"]
        assert u32(s.indices[l]).tolist() == b["indices"]
    s = ctx.sample(np.array([0, 5], np.uint32), seed=42, epoch=0, batch=1)
    assert u32(s.uniq).tolist() == gold["khop"]["uniq_batch1"]
    ctx.set_sampler("rwalk", layers=2, max_batch=8)
    s = ctx.sample(np.array([0, 5], np.uint32), seed=42, epoch=0, batch=0)
    assert u32(s.uniq).tolist() == gold["rwalk"]["uniq"]
    for l, b in enumerate(gold["rwalk"]["blocks"]):
        assert u32(s.indptr[l]).tolist() == b["indptr"]
        assert u32(s.indices[l]).tolist() == b["indices"]
        assert u32(s.weights[l]).tolist() == b["weights"]
    ctx.set_train_set(np.arange(8, dtype=np.uint32), 3, 42)
    ctx.shuffle(0)
    assert ctx.permutation(8).tolist() == gold["shuffle"]["epoch0"]
    ctx.shuffle(1)
    assert ctx.permutation(8).tolist() == gold["shuffle"]["epoch1"]


DEDUP_MODES = ["dense_dedup1", "hash_dedup1", "dense_dedup2", "hash_dedup2"]


def _dedup(mode, monkeypatch):
    """'<mode>_dedup<n>': GLB_RELABEL_DEDUP=n (1 warp-level, 2 block smem-staged pre-dedup
    of picks before the relabel-table insert); returns the relabel mode."""
    if "_dedup" in mode:
        mode, n = mode.split("_dedup")
        monkeypatch.setenv("GLB_RELABEL_DEDUP", n)
    return mode


@pytest.mark.parametrize("mode", MODES + ["dense_dedup1", "hash_dedup1", "dense_dedup2",
                                          "hash_dedup2"])
def test_tiny_every_batch_bit_exact(tiny, mode, monkeypatch):
    if "_dedup" in mode:
        mode, n = mode.split("_dedup")
        monkeypatch.setenv("GLB_RELABEL_DEDUP", n)
    g, go = tiny
    sh = g.shape
    ctx = make_ctx(g, fanouts=sh.fanouts, mode=mode)
    for e in [0, 1]:
        ob = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
        ctx.shuffle(e)
        assert np.array_equal(ctx.permutation(g.train.shape[0]), np.concatenate(ob))
        for b, seeds in enumerate(ob):
            ctx.sample_batch(e, b)
            assert_same_sample(ctx.sample_result(), go.sample_khop(seeds, sh.fanouts, g.seed, e, b))


def test_host_and_device_seed_paths(tiny):
    g, go = tiny
    ctx = make_ctx(g, fanouts=(10, 5))
    seeds = g.train[100:164]
    exp = go.sample_khop(seeds, (10, 5), 7, 3, 9)
    assert_same_sample(ctx.sample(seeds, seed=7, epoch=3, batch=9), exp)
    dev = torch.from_numpy(seeds.view(np.int32)).cuda()
    assert_same_sample(ctx.sample(dev, seed=7, epoch=3, batch=9), exp)
    # fanout override within capacity
    assert_same_sample(ctx.sample(seeds, fanouts=(4, 2), seed=7, epoch=3, batch=9),
                       go.sample_khop(seeds, (4, 2), 7, 3, 9))


@pytest.mark.parametrize("fanouts", [(25, 10), (15, 10, 5), (3,), (1, 1, 1), (32, 2), (40, 33)])
@pytest.mark.parametrize("mode", MODES + DEDUP_MODES)
def test_fanout_variants_power_law(fanouts, mode, monkeypatch):
    """*_dedup*: picks pre-deduplicated (warp / block) before the relabel-table insert; a
    small graph with hubs (gamma 2.1), so duplicate picks within a warp / block are common."""
    mode = _dedup(mode, monkeypatch)
    g = synth.small_graph(6000, 90000, 2.1, 8, 700, seed=11)
    go = oracle.GraphOracle(g.indptr, g.indices)
    ctx = make_ctx(g, fanouts=fanouts, max_batch=300, mode=mode)
    for b, n0 in enumerate([1, 37, 300]):
        seeds = g.train[b * 200:b * 200 + n0]
        assert_same_sample(ctx.sample(seeds, seed=5, epoch=b, batch=b),
                           go.sample_khop(seeds, fanouts, 5, b, b))


def test_empty_batch_zero_hops_and_degree_zero():
    # vertex 3 and 4 have no out-edges
    indptr = np.array([0, 2, 4, 5, 5, 5], np.uint64)
    indices = np.array([1, 3, 0, 4, 2], np.uint32)
    go = oracle.GraphOracle(indptr, indices)
    ctx = glb.Context(0)
    ctx.load_graph(indptr, indices, None)
    ctx.set_sampler("khop", fanouts=(2, 2), max_batch=4)
    s = ctx.sample(np.array([], np.uint32), seed=1)
    assert s.sizes == [0, 0, 0]
    for seeds in ([3], [3, 4], [0, 3], [4, 0, 1, 2]):
        assert_same_sample(ctx.sample(np.array(seeds, np.uint32), seed=1),
                           go.sample_khop(seeds, (2, 2), 1, 0, 0))
    s = ctx.sample(np.array([2, 1], np.uint32), fanouts=(), seed=1)
    assert s.sizes == [2] and u32(s.uniq).tolist() == [2, 1]


@pytest.mark.parametrize("mode", MODES)
def test_errors(mode):
    g = synth.small_graph(500, 3000, 2.2, 4, 50, seed=8)
    ctx = make_ctx(g, fanouts=(3, 2), max_batch=16, mode=mode)
    with pytest.raises(glb.GlbError) as e:
        ctx.sample(np.array([1, 2, 1], np.uint32))
    assert e.value.code == glb.EINVAL
    with pytest.raises(glb.GlbError) as e:
        ctx.sample(np.array([1, 500], np.uint32))
    assert e.value.code == glb.EINVAL
    with pytest.raises(glb.GlbError) as e:
        ctx.sample(np.arange(17, dtype=np.uint32))
    assert e.value.code == glb.ENOMEM
    with pytest.raises(glb.GlbError) as e:
        ctx.sample(np.array([1], np.uint32), epoch=1 << 16)
    assert e.value.code == glb.ERANGE
    with pytest.raises(glb.GlbError) as e:
        ctx.build_cache(1.5)
    assert e.value.code == glb.EINVAL
    # T is a set (L305; reading Q6): a duplicate training id is rejected up front
    with pytest.raises(glb.GlbError) as e:
        ctx.set_train_set(np.array([3, 7, 3], np.uint32), 2, 1)
    assert e.value.code == glb.EINVAL
    # device-side errors are sticky: a bad asynchronous batch followed by a good one still
    # reports at the next sync (an earlier batch's error is not lost)
    ctx.set_pipeline(2)
    ctx.sample_async(torch.tensor([4, 5, 4], dtype=torch.int32).pin_memory(), seed=1)
    ctx.sample_async(torch.tensor([6, 8], dtype=torch.int32).pin_memory(), seed=1)
    with pytest.raises(glb.GlbError) as e:
        ctx.sync()
    assert e.value.code == glb.EINVAL
    ctx.sync()  # reported once, then cleared
    ctx.set_pipeline(1)
    # the ctx still works after errors
    go = oracle.GraphOracle(g.indptr, g.indices)
    assert_same_sample(ctx.sample(np.array([1, 2], np.uint32), seed=3),
                       go.sample_khop([1, 2], (3, 2), 3, 0, 0))
    bad = glb.Context(0)
    with pytest.raises(glb.GlbError) as e:
        bad.load_graph(np.array([0, 2, 1], np.uint64), np.array([0, 1], np.uint32), None)
    assert e.value.code == glb.EINVAL
    with pytest.raises(glb.GlbError) as e:
        bad.load_graph(np.array([0, 1, 2], np.uint64), np.array([0, 7], np.uint32), None)
    assert e.value.code == glb.EINVAL


@pytest.mark.parametrize("layers,walks,length,topk", [(3, 4, 3, 5), (2, 4, 3, 5), (1, 2, 5, 3),
                                                      (2, 8, 2, 7)])
@pytest.mark.parametrize("mode", MODES)
def test_random_walk_parity(layers, walks, length, topk, mode):
    g = synth.small_graph(8000, 60000, 2.5, 8, 600, seed=21)
    go = oracle.GraphOracle(g.indptr, g.indices)
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, None)
    ctx.set_relabel_mode(mode)
    ctx.set_sampler("rwalk", layers=layers, walks=walks, walk_len=length, topk=topk, max_batch=200)
    for b, n0 in enumerate([1, 64, 200]):
        seeds = g.train[b * 200:b * 200 + n0]
        gs = ctx.sample(seeds, seed=9, epoch=1, batch=b)
        os_ = go.sample_rwalk(seeds, layers, 9, 1, b, walks, length, topk)
        assert_same_sample(gs, os_, weighted=True)


@pytest.mark.parametrize("mode", MODES)
def test_presample_cache_and_hit_stats(tiny, mode):
    g, go = tiny
    sh = g.shape
    ctx = make_ctx(g, fanouts=sh.fanouts, mode=mode)
    for K in [1, 2]:
        ctx.reset_counts(glb.COUNT_PRESAMPLE)
        ctx.presample(K)
        exp = go.presample("khop", g.train, sh.batch, sh.fanouts, g.seed, K)
        assert np.array_equal(ctx.get_counts(glb.COUNT_PRESAMPLE), exp)
    counts = go.presample("khop", g.train, sh.batch, sh.fanouts, g.seed, 2)
    # access recording over the measured epochs 2..3
    ctx.reset_counts(glb.COUNT_ACCESS)
    ctx.set_count_mode(glb.COUNT_ACCESS)
    for e in [2, 3]:
        for b in range(ctx.num_batches):
            ctx.sample_batch(e, b)
    ctx.set_count_mode(glb.COUNT_NONE)
    ctx.sync()
    acc = go.visit_counts("khop", g.train, sh.batch, sh.fanouts, g.seed, [2, 3])
    assert np.array_equal(ctx.get_counts(glb.COUNT_ACCESS), acc)
    for a in sh.alphas:
        ctx.build_cache(a)
        slot = oracle.cache_slots(counts, a)
        assert np.array_equal(ctx.cache_slots(), slot), a
        hs = ctx.hit_stats()
        C = oracle.cache_size(a, g.V)
        assert hs["cache_rows"] == C
        tot = int(acc.sum())
        assert hs["total"] == tot
        assert hs["hits"] == int(acc[slot >= 0].sum())
        assert hs["optimal_hits"] / tot == pytest.approx(oracle.optimal_hit_rate(acc, C), abs=0)
        assert hs["hits"] <= hs["optimal_hits"]


GATHER_ENV = {"warp": {"GLB_GATHER_WARP": "1"}, "block": {"GLB_GATHER_WARP": "0"},
              "nobins": {"GLB_MISS_BIN_LOG2": "0"},
              "finebins": {"GLB_MISS_BIN_LOG2": "7"},  # one bin per row: the device-scan path
              "warp_finebins": {"GLB_GATHER_WARP": "1", "GLB_MISS_BIN_LOG2": "7"},
              # host-assisted misses (glb_set_host_gather): 40 % / 90 % of them by host threads
              "host400": {"GLB_HOST_GATHER": "400", "GLB_HOST_GATHER_THREADS": "4"},
              "host900_nobins": {"GLB_HOST_GATHER": "900", "GLB_HOST_GATHER_THREADS": "3",
                                 "GLB_MISS_BIN_LOG2": "0"},
              "missblocks3": {"GLB_MISS_BLOCKS": "3"},  # 3 blocks take every host miss
              # hits gathered in lid order from the marks (the default) / from the hit list
              "lidorder": {"GLB_GATHER_LIDORDER": "1"},
              "hitlist": {"GLB_GATHER_LIDORDER": "0"},
              # the miss-taking blocks start on the misses (GLB_MISSES_FIRST)
              "missesfirst": {"GLB_MISSES_FIRST": "1", "GLB_MISS_BLOCKS": "3"},
              # misses read from the rank-ordered cold store (glb_set_cold_store)
              "coldstore": {"GLB_COLD_STORE": "1"},
              "coldstore_host_nobins": {"GLB_COLD_STORE": "1", "GLB_HOST_GATHER": "400",
                                        "GLB_HOST_GATHER_THREADS": "2", "GLB_MISS_BIN_LOG2": "0"},
              "missesfirst_host": {"GLB_MISSES_FIRST": "1", "GLB_HOST_GATHER": "300",
                                   "GLB_HOST_GATHER_THREADS": "2"},
              "lidorder_host": {"GLB_GATHER_LIDORDER": "1", "GLB_HOST_GATHER": "400",
                                "GLB_HOST_GATHER_THREADS": "2"},
              "dedup2_host": {"GLB_RELABEL_DEDUP": "2", "GLB_HOST_GATHER": "500"}}


@pytest.mark.parametrize("mode", MODES + ["bulk", "bulkmiss", "bulkboth"] + list(GATHER_ENV))
@pytest.mark.parametrize("alpha", [0.0, 0.1, 0.5, 1.0])
def test_extract_sample_bytes(tiny, alpha, mode, monkeypatch):
    """mode 'bulk': hits through the cp.async.bulk gather (GLB_GATHER_BULK=1, off by
    default), misses through the LSU gather; GATHER_ENV: the block / warp-independent
    gathers and the miss orderings (none, 2 MB bins, one bin per row)."""
    g, go = tiny
    sh = g.shape
    if mode in ("bulk", "bulkboth"):
        monkeypatch.setenv("GLB_GATHER_BULK", "1")
    if mode in ("bulkmiss", "bulkboth"):
        monkeypatch.setenv("GLB_MISS_BULK", "1")
    for k, v in GATHER_ENV.get(mode, {}).items():
        monkeypatch.setenv(k, v)
    ctx = make_ctx(g, fanouts=sh.fanouts, mode=mode if mode in MODES else "auto")
    ctx.presample(1)
    ctx.build_cache(alpha)
    slot = ctx.cache_slots()
    for e, b in [(1, 0), (1, 15)]:
        ctx.sample_batch(e, b)
        s = ctx.sample_result()
        out = torch.full((s.sizes[-1] + 3, g.D), float("nan"), device="cuda")
        st = ctx.extract_sample(out, stats=True)
        seeds = oracle.epoch_batches(g.train, sh.batch, g.seed, e)[b]
        os_ = go.sample_khop(seeds, sh.fanouts, g.seed, e, b)
        exp = go.extract(os_.uniq)
        got = out[:s.sizes[-1]].cpu().numpy()
        assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))
        assert torch.isnan(out[s.sizes[-1]:]).all()          # nothing written past n_L
        assert st["hits"] == int((slot[os_.uniq] >= 0).sum())
        assert st["hits"] + st["misses"] == s.sizes[-1]
        assert np.array_equal(s.cache_slot.cpu().numpy(), slot[os_.uniq])


@pytest.mark.parametrize("variant", ["default"] + list(GATHER_ENV))
@pytest.mark.parametrize("D", [7, 32, 64, 100, 128, 256])
def test_extract_generic_ids_dims(D, variant, monkeypatch):
    for k, v in GATHER_ENV.get(variant, {}).items():
        monkeypatch.setenv(k, v)
    V = 3000
    g = synth.small_graph(V, 20000, 2.2, D, 300, seed=D)
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    ctx = make_ctx(g, fanouts=(5,), max_batch=64)
    ctx.presample(1)
    ctx.build_cache(0.3)
    rng = np.random.default_rng(D)
    for n in [0, 1, 33, 5000]:
        ids = rng.integers(0, V, n).astype(np.uint32)
        if n > 3:
            ids[1] = ids[0]                                   # duplicates allowed
        out, st = ctx.extract(torch.from_numpy(ids.view(np.int32)).cuda(), stats=True)
        assert np.array_equal(out.cpu().numpy().view(np.uint32), go.extract(ids).view(np.uint32))
        assert st["hits"] == int((ctx.cache_slots()[ids] >= 0).sum()) and st["hits"] + st["misses"] == n
    with pytest.raises(glb.GlbError):
        ctx.extract(torch.tensor([0, V], dtype=torch.int32, device="cuda"))
        ctx.sync()


def test_degree_hotness_cache():
    g = synth.small_graph(4000, 40000, 2.2, 16, 200, seed=3)
    ctx = make_ctx(g, fanouts=(5,), max_batch=64)
    deg = np.diff(g.indptr).astype(np.uint32)
    ctx.build_cache(0.1, hotness=torch.from_numpy(deg.view(np.int32)).cuda())
    assert np.array_equal(ctx.cache_slots(), oracle.cache_slots(deg, 0.1))


# ----------------------------------------------------------------------------- full PR size
@pytest.fixture(scope="module")
def pr():
    g = synth.make_graph("PR")
    return g, oracle.GraphOracle(g.indptr, g.indices, g.features)


@pytest.mark.slow
def test_pr_full_size_parity(pr):
    """configs[1] at full size, bench launch configuration: PreSC#1 counts in
    full, cache slots at the sweep's alphas, and every output of four batches --
    every extracted byte -- at alpha = 1 (all HBM hits) and at alpha = 0.05 (most rows
    over PCIe from the pinned host matrix)."""
    g, go = pr
    sh = g.shape
    ctx = make_ctx(g, fanouts=sh.fanouts)
    ctx.presample(sh.K)
    counts = go.presample("khop", g.train, sh.batch, sh.fanouts, g.seed, sh.K)
    assert np.array_equal(ctx.get_counts(glb.COUNT_PRESAMPLE), counts)
    for a in (0.05, 0.25):
        ctx.build_cache(a)
        assert np.array_equal(ctx.cache_slots(), oracle.cache_slots(counts, a))
    e = sh.K
    ob = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
    nb = len(ob)
    rng = np.random.default_rng(0)
    out = torch.empty((sh.batch * 26 * 11, g.D), device="cuda")
    for a in (1.0, 0.05):
        ctx.build_cache(a)
        slot = oracle.cache_slots(counts, a)
        for b in [0, 1, int(rng.integers(2, nb - 1)), nb - 1]:
            ctx.sample_batch(e, b)
            s = ctx.sample_result()
            os_ = go.sample_khop(ob[b], sh.fanouts, g.seed, e, b)
            assert_same_sample(s, os_)
            st = ctx.extract_sample(out, stats=True)
            assert st["hits"] == int((slot[os_.uniq] >= 0).sum())
            n = s.sizes[-1]
            got = out[:n].cpu().numpy().view(np.uint32)
            assert np.array_equal(got, go.extract(os_.uniq).view(np.uint32)), (a, b)


@pytest.mark.parametrize("alpha", [1.0, 0.3])
@pytest.mark.parametrize("mode", MODES)
def test_pipeline_depth2_bit_exact(tiny, alpha, mode):
    """Pipelined Extract || Sample (two streams, double-buffered slots) gives the
    same bytes as the oracle for every batch of an epoch."""
    g, go = tiny
    sh = g.shape
    ctx = make_ctx(g, fanouts=sh.fanouts, mode=mode)
    ctx.presample(1)
    ctx.build_cache(alpha)
    ctx.set_pipeline(2)
    e = 1
    ob = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
    outs, sizes = [], []
    for b in range(len(ob)):
        ctx.sample_batch(e, b)
        outs.append(torch.full((64 * 11 * 6, g.D), float("nan"), device="cuda"))
        ctx.extract_sample(outs[-1])
    ctx.sync()
    for b, seeds in enumerate(ob):
        exp = go.sample_khop(seeds, sh.fanouts, g.seed, e, b)
        n = exp.sizes[-1]
        got = outs[b][:n].cpu().numpy()
        assert np.array_equal(got.view(np.uint32), go.extract(exp.uniq).view(np.uint32)), b
        assert torch.isnan(outs[b][n:]).all()
    # the current sample is still readable after the pipeline drained
    assert_same_sample(ctx.sample_result(),
                       go.sample_khop(ob[-1], sh.fanouts, g.seed, e, len(ob) - 1))


def test_policies_and_similarity(tiny):
    g, go = tiny
    sh = g.shape
    ctx = make_ctx(g, fanouts=sh.fanouts)
    deg = ctx.policy_hotness("degree")
    assert np.array_equal(u32(deg), oracle.hotness_degree(g.indptr))
    rnd = ctx.policy_hotness("random", seed=77)
    assert np.array_equal(u32(rnd), oracle.hotness_random(77, g.V))
    for pol, h in [("degree", oracle.hotness_degree(g.indptr)),
                   ("random", oracle.hotness_random(77, g.V))]:
        for a in [0.05, 0.3]:
            ctx.build_cache_policy(a, pol, seed=77)
            assert np.array_equal(ctx.cache_slots(), oracle.cache_slots(h, a)), (pol, a)
    # footprint similarity between epochs 1 and 2 (Table 2 analog)
    fs = []
    for e in [1, 2]:
        ctx.reset_counts(glb.COUNT_ACCESS)
        ctx.set_count_mode(glb.COUNT_ACCESS)
        for b in range(ctx.num_batches):
            ctx.sample_batch(e, b)
        ctx.set_count_mode(glb.COUNT_NONE)
        ctx.sync()
        fs.append(ctx.counts_tensor(glb.COUNT_ACCESS).clone())
    got = ctx.footprint_similarity(fs[0], fs[1], 0.1)
    f1 = go.visit_counts("khop", g.train, sh.batch, sh.fanouts, g.seed, [1])
    f2 = go.visit_counts("khop", g.train, sh.batch, sh.fanouts, g.seed, [2])
    assert got[1:] == oracle.footprint_similarity(f1, f2, 0.1)[1:]


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("fanouts", [(10, 5), (15, 10, 5), (40,)])
def test_weighted_khop_parity(fanouts, mode):
    g = synth.small_graph(6000, 90000, 2.1, 8, 700, seed=13)
    w = synth.gen_edge_weights(g.indices, 13)
    w[::7] = 0                                              # some zero-weight edges
    go = oracle.GraphOracle(g.indptr, g.indices)
    ctx = glb.Context(0)
    ctx.load_graph(g.indptr, g.indices, g.features)
    ctx.load_edge_weights(w)
    ctx.set_relabel_mode(mode)
    ctx.set_sampler("weighted", fanouts=fanouts, max_batch=300)
    for b, n0 in enumerate([1, 37, 300]):
        seeds = g.train[b * 200:b * 200 + n0]
        assert_same_sample(ctx.sample(seeds, seed=5, epoch=b, batch=b),
                           go.sample_khop_weighted(w, seeds, fanouts, 5, b, b))
    # PreSC with the weighted sampler (Fig 11(a)/Table 2 "3-hop weighted" analog)
    ctx.set_sampler("weighted", fanouts=fanouts, max_batch=64)
    ctx.set_train_set(g.train, 64, g.seed)
    ctx.presample(1)
    exp = go.presample("weighted", g.train, 64, fanouts, g.seed, 1, weights=w)
    assert np.array_equal(ctx.get_counts(glb.COUNT_PRESAMPLE), exp)


def test_sample_async_pinned_seeds_and_device_counts(tiny):
    """glb_sample_async (pinned host or device seeds, no host sync) gives the oracle's
    sample; glb_extract_counts_device_ptr holds each extract's (hits, misses) in stream
    order (the e2e bench path)."""
    g, go = tiny
    sh = g.shape
    ctx = make_ctx(g, fanouts=sh.fanouts)
    ctx.set_count_mode(glb.COUNT_PRESAMPLE)
    ctx.presample(1)
    ctx.set_count_mode(glb.COUNT_NONE)
    ctx.build_cache(0.2)
    slot = ctx.cache_slots()
    cnt = ctx.extract_counts_tensor()
    host = torch.zeros((3, 3), dtype=torch.int64).pin_memory()
    outs = []
    batches = oracle.epoch_batches(g.train, sh.batch, g.seed, 4)
    for j, b in enumerate([0, 5, len(batches) - 1]):
        seeds = torch.from_numpy(batches[b].view(np.int32).copy())
        seeds = seeds.pin_memory() if j != 1 else seeds.cuda()
        ctx.sample_async(seeds, seed=g.seed, epoch=4, batch=b)
        s = ctx.sample_result()
        exp = go.sample_khop(batches[b], sh.fanouts, g.seed, 4, b)
        assert_same_sample(s, exp)
        out = torch.empty((s.sizes[-1], sh.D), device="cuda")
        ctx.extract_sample(out)
        host[j].copy_(cnt, non_blocking=True)
        outs.append((exp.uniq, out))
    torch.cuda.synchronize()
    for j, (uniq, out) in enumerate(outs):
        hits = int((slot[uniq] >= 0).sum())
        assert host[j].tolist() == [hits, len(uniq) - hits, 0]
        assert np.array_equal(out.cpu().numpy().view(np.uint32), go.extract(uniq).view(np.uint32))
    with pytest.raises(AssertionError):
        ctx.sample_async(torch.from_numpy(batches[0].view(np.int32).copy()))  # pageable


@pytest.mark.parametrize("D", [7, 100])
@pytest.mark.parametrize("depth", [1, 2])
@pytest.mark.parametrize("fraction", [0.3, 0.75])
def test_host_gather_every_batch(D, depth, fraction):
    """Host-assisted misses (glb_set_host_gather): every batch of an epoch, pipelined or not,
    gives the oracle's bytes and counts; fraction 0 turns it off again."""
    g = synth.small_graph(6000, 60000, 2.2, D, 500, seed=11 + D)
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    sh = g.shape
    ctx = make_ctx(g, fanouts=sh.fanouts, max_batch=sh.batch)
    ctx.presample(1)
    ctx.build_cache(0.2)
    ctx.set_host_gather(fraction, threads=3)
    assert ctx.host_gather["threads"] == 3 and abs(ctx.host_gather["fraction"] - fraction) < 1e-9
    ctx.set_pipeline(depth)
    slot = ctx.cache_slots()
    e = 1
    ob = oracle.epoch_batches(g.train, sh.batch, g.seed, e)
    outs = []
    for b in range(len(ob)):
        ctx.sample_batch(e, b)
        out = torch.full((sh.batch * 11 * 6 + 1, D), float("nan"), device="cuda")
        st = ctx.extract_sample(out, stats=(depth == 1))  # depth 2: batches stay in flight
        outs.append((b, out, st))
    torch.cuda.synchronize()
    for b, out, st in outs:
        os_ = go.sample_khop(ob[b], sh.fanouts, g.seed, e, b)
        n = os_.uniq.shape[0]
        assert np.array_equal(out[:n].cpu().numpy().view(np.uint32),
                              go.extract(os_.uniq).view(np.uint32)), b
        assert torch.isnan(out[n:]).all()
        if st is not None:
            assert st["hits"] == int((slot[os_.uniq] >= 0).sum())
            assert st["misses"] == n - st["hits"]
    ctx.set_host_gather(0.0)
    assert ctx.host_gather["fraction"] == 0.0


@pytest.mark.parametrize("alpha", [0.0, 0.3, 1.0])
def test_cold_store(alpha):
    """glb_set_cold_store: the non-cached rows copied in rank order into pinned host memory;
    samples' and generic extracts give the oracle's bytes (pipelined, host-assisted too)."""
    g = synth.small_graph(5000, 50000, 2.2, 24, 400, seed=21)
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    sh = g.shape
    ctx = make_ctx(g, fanouts=sh.fanouts, max_batch=sh.batch)
    ctx.set_cold_store(True)
    ctx.presample(1)
    ctx.build_cache(alpha)
    V = g.indptr.shape[0] - 1
    assert ctx.cold_store_rows == (V - int(np.floor(alpha * V)) if alpha < 1.0 else 0)
    ctx.set_host_gather(0.3, threads=2)
    ctx.set_pipeline(2)
    ob = oracle.epoch_batches(g.train, sh.batch, g.seed, 1)
    for b in range(len(ob)):
        ctx.sample_batch(1, b)
        s = ctx.sample_result()
        out = torch.full((s.sizes[-1], sh.D), float("nan"), device="cuda")
        ctx.extract_sample(out, stats=True)
        exp = go.sample_khop(ob[b], sh.fanouts, g.seed, 1, b)
        assert np.array_equal(out.cpu().numpy().view(np.uint32), go.extract(exp.uniq).view(np.uint32))
    ids = np.random.default_rng(3).integers(0, V, 3000).astype(np.uint32)
    o, st = ctx.extract(torch.from_numpy(ids.view(np.int32)).cuda(), stats=True)
    assert np.array_equal(o.cpu().numpy().view(np.uint32), go.extract(ids).view(np.uint32))
    ctx.set_cold_store(False)
    assert ctx.cold_store_rows == 0


@pytest.mark.parametrize("D", [7, 100])
def test_cold_store_rebuild(D):
    """The cold store follows the cache: load_cache at another alpha (and with another
    hotness map) replaces it; scalar (D % 4 != 0) and vector rows; depth 1 and 2; every
    batch's bytes equal the oracle's after each rebuild."""
    g = synth.small_graph(4000, 40000, 2.2, D, 500, seed=23)
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    sh = g.shape
    V = g.indptr.shape[0] - 1
    ctx = make_ctx(g, fanouts=sh.fanouts, max_batch=sh.batch)
    ctx.set_cold_store(True)
    ctx.presample(1)
    ob = oracle.epoch_batches(g.train, sh.batch, g.seed, 1)
    for alpha, depth, degree in ((0.2, 1, False), (0.6, 2, False), (0.35, 2, True)):
        if degree:
            ctx.build_cache_policy(alpha, "degree")
        else:
            ctx.build_cache(alpha)
        assert ctx.cold_store_rows == V - int(np.floor(alpha * V))
        ctx.set_pipeline(depth)
        for b in range(len(ob)):
            ctx.sample_batch(1, b)
            s = ctx.sample_result()
            out = torch.full((s.sizes[-1], sh.D), float("nan"), device="cuda")
            st = ctx.extract_sample(out, stats=True)
            exp = go.sample_khop(ob[b], sh.fanouts, g.seed, 1, b)
            assert np.array_equal(out.cpu().numpy().view(np.uint32),
                                  go.extract(exp.uniq).view(np.uint32))
            assert st["hits"] + st["misses"] == exp.uniq.shape[0]
