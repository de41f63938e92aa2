"""Pins for the oracle's epoch shuffle, PreSC counts, cache ranking, hit rate
and Optimal hit rate (PAPER.md L148 fn4, L301, L305, L329-339), and extract
(closed-form features)."""
import itertools

import numpy as np
import pytest

import oracle
import synth


def test_shuffle_is_permutation_and_batches():
    T = np.sort(np.random.default_rng(0).choice(10000, 1000, replace=False)).astype(np.uint32)
    p0 = oracle.shuffle(T, 5, 0)
    p1 = oracle.shuffle(T, 5, 1)
    assert sorted(p0.tolist()) == T.tolist() and sorted(p1.tolist()) == T.tolist()
    assert not np.array_equal(p0, p1)
    bs = oracle.epoch_batches(T, 64, 5, 0)
    assert len(bs) == 16 and len(bs[-1]) == 1000 - 15 * 64       # last batch partial (40)
    assert np.array_equal(np.concatenate(bs), p0)


def test_presample_count_invariants():
    g = synth.make_graph("tiny")
    go = oracle.GraphOracle(g.indptr, g.indices)
    sh = g.shape
    tot_nl = 0
    for b, seeds in enumerate(oracle.epoch_batches(g.train, sh.batch, g.seed, 0)):
        tot_nl += go.sample_khop(seeds, sh.fanouts, g.seed, 0, b).sizes[-1]
    c1 = go.presample("khop", g.train, sh.batch, sh.fanouts, g.seed, 1)
    assert int(c1.sum()) == tot_nl                                  # one per (batch, unique v)
    assert c1.max() <= 16
    c2 = go.presample("khop", g.train, sh.batch, sh.fanouts, g.seed, 2)
    assert np.all(c2 >= c1) and c2.max() <= 32                     # K=2 adds epoch 1
    assert np.all(c1[g.train] >= 1)                                # every seed is visited


def brute_rank(counts):
    return [v for _, v in sorted((-int(c), v) for v, c in enumerate(counts))]


def test_cache_rank_and_slots():
    rng = np.random.default_rng(3)
    counts = rng.integers(0, 5, 200).astype(np.uint32)
    assert oracle.cache_rank(counts).tolist() == brute_rank(counts)
    prev = set()
    for a in [0.0, 0.01, 0.1, 0.33, 0.5, 0.999, 1.0]:
        slot = oracle.cache_slots(counts, a)
        C = oracle.cache_size(a, 200)
        members = set(np.nonzero(slot >= 0)[0].tolist())
        assert len(members) == C and prev <= members                # nested in alpha
        assert sorted(slot[slot >= 0].tolist()) == list(range(C))    # slots 0..C-1
        assert [int(slot[v]) for v in brute_rank(counts)[:C]] == list(range(C))
        prev = members
    for bad in [-0.1, 1.1, float("nan")]:
        with pytest.raises(ValueError):
            oracle.cache_size(bad, 10)
    assert oracle.cache_size(0.29, 100) == 28                       # floor in IEEE double


def test_hit_rate_bounds_and_bruteforce_optimal():
    rng = np.random.default_rng(9)
    for trial in range(30):
        V = int(rng.integers(3, 12))
        acc = rng.integers(0, 6, V).astype(np.uint32)
        counts = rng.integers(0, 6, V).astype(np.uint32)
        for C in range(0, V + 1):
            a = C / V
            slot = oracle.cache_slots(counts, a)
            C2 = int(np.sum(slot >= 0))
            H = oracle.hit_rate(acc, slot)
            Hs = oracle.optimal_hit_rate(acc, C2)
            tot = acc.sum()
            best = max(sum(int(acc[v]) for v in sub)
                       for sub in itertools.combinations(range(V), C2)) if tot else 0
            assert Hs == pytest.approx(best / tot if tot else 0.0)
            assert H <= Hs + 1e-12
        if acc.sum():
            assert oracle.hit_rate(acc, oracle.cache_slots(counts, 1.0)) == 1.0
            assert oracle.hit_rate(acc, oracle.cache_slots(counts, 0.0)) == 0.0
        # caching by the true access counts reaches the optimum
        assert oracle.hit_rate(acc, oracle.cache_slots(acc, 0.5)) == pytest.approx(
            oracle.optimal_hit_rate(acc, oracle.cache_size(0.5, V)))


def test_presc_hit_rate_close_to_optimal_tiny():
    """Sanity (not a pin of exact values): PreSC#1 on the tiny config beats a
    random cache and stays below Optimal (L339: PreSC is 'almost as good as
    the Optimal policy')."""
    g = synth.make_graph("tiny")
    go = oracle.GraphOracle(g.indptr, g.indices)
    sh = g.shape
    counts = go.presample("khop", g.train, sh.batch, sh.fanouts, g.seed, 1)
    acc = go.visit_counts("khop", g.train, sh.batch, sh.fanouts, g.seed, [1, 2])
    for a in [0.05, 0.1, 0.25]:
        slot = oracle.cache_slots(counts, a)
        H = oracle.hit_rate(acc, slot)
        Hs = oracle.optimal_hit_rate(acc, oracle.cache_size(a, g.V))
        rnd = np.full(g.V, -1, np.int32)
        pick = np.random.default_rng(0).choice(g.V, oracle.cache_size(a, g.V), replace=False)
        rnd[pick] = 0
        assert oracle.hit_rate(acc, rnd) < H <= Hs


def test_extract_matches_closed_form_features():
    g = synth.make_graph("tiny")
    go = oracle.GraphOracle(g.indptr, g.indices, g.features)
    seeds = oracle.epoch_batches(g.train, 64, g.seed, 0)[3]
    s = go.sample_khop(seeds, [10, 5], g.seed, 0, 3)
    out = go.extract(s.uniq)
    rng = np.random.default_rng(0)
    for i in rng.integers(0, s.uniq.shape[0], 200):
        d = int(rng.integers(0, g.D))
        exp = oracle.feature_value(g.seed, int(s.uniq[i]), d)
        assert out[i, d].view(np.uint32) == np.float32(exp).view(np.uint32)
    # duplicates allowed: one row per entry
    out2 = go.extract(np.array([5, 5, 0], np.uint32))
    assert np.array_equal(out2[0], out2[1])


def test_footprint_similarity_pins():
    # identical footprints -> 1; disjoint top sets -> 0
    f = np.array([5, 0, 3, 9, 1, 0, 7, 2, 0, 4], np.uint32)
    assert oracle.footprint_similarity(f, f, 0.3)[0] == 1.0
    g = np.array([0, 6, 0, 0, 0, 8, 0, 0, 5, 0], np.uint32)
    assert oracle.footprint_similarity(f, g, 0.3)[0] == 0.0
    # hand-computed (L329): T_i = {3, 6, 0} (9, 7, 5), T_j = {0, 3, 1} (8, 6, 5 with tie -> gid)
    h = np.array([8, 5, 0, 6, 0, 0, 2, 0, 0, 5], np.uint32)
    v, num, den = oracle.footprint_similarity(f, h, 0.3)
    assert (num, den) == (min(5, 8) + min(9, 6), 8 + 6 + 5) and v == pytest.approx(11 / 19)
    # brute force against the definition on random small inputs
    rng = np.random.default_rng(4)
    for _ in range(50):
        V = int(rng.integers(2, 15))
        fi = rng.integers(0, 6, V).astype(np.uint32)
        fj = rng.integers(0, 6, V).astype(np.uint32)
        frac = float(rng.choice([0.1, 0.3, 0.5, 1.0]))
        C = oracle.cache_size(frac, V)
        ti = set(brute_rank(fi)[:C])
        tj = set(brute_rank(fj)[:C])
        num = sum(min(int(fi[v]), int(fj[v])) for v in ti & tj)
        den = sum(int(fj[v]) for v in tj)
        assert oracle.footprint_similarity(fi, fj, frac)[1:] == (num, den)


def test_policy_hotness_pins():
    indptr = np.array([0, 3, 3, 7, 8], np.uint64)
    assert oracle.hotness_degree(indptr).tolist() == [3, 0, 4, 1]
    r1 = oracle.hotness_random(5, 20000)
    assert np.array_equal(r1, oracle.hotness_random(5, 20000))
    assert not np.array_equal(r1, oracle.hotness_random(6, 20000))
    # high words of the draw: roughly uniform over 16 buckets
    from scipy import stats
    assert stats.chisquare(np.bincount(r1 >> 28, minlength=16)).pvalue > 1e-3
    # equals the definition for a few vertices
    for v in [0, 7, 19999]:
        assert r1[v] == oracle.draw64(5, v, 0, 0, oracle.c3(0, 0, 7), 0) >> 32


def test_presc_vs_degree_and_random_on_tiny():
    """Fig 10 / L339-L343 shape check at alpha = 10% (properties of these seeded
    inputs, not paper values): PreSC far above Random, and on this power-law graph
    with correlated in/out degrees Degree comes close to PreSC (L339-L341: Degree
    is competitive only on power-law graphs)."""
    g = synth.make_graph("tiny")
    go = oracle.GraphOracle(g.indptr, g.indices)
    sh = g.shape
    counts = go.presample("khop", g.train, sh.batch, sh.fanouts, g.seed, 1)
    acc = go.visit_counts("khop", g.train, sh.batch, sh.fanouts, g.seed, [1, 2])
    h = {p: oracle.hit_rate(acc, oracle.cache_slots(x, 0.1)) for p, x in
         [("presc", counts), ("degree", oracle.hotness_degree(g.indptr)),
          ("random", oracle.hotness_random(g.seed, g.V))]}
    assert h["presc"] > 2 * h["random"]
    assert h["presc"] > 0.95 * h["degree"]


def test_sharded_cache_pins():
    """NEXT-3: world shards of floor(alpha*V) rows each hold exactly the
    world*floor(alpha*V) top-ranked vertices (a brute-force sort), disjointly, shard r
    holding the ranks i = r, r+world, ... in row order; world = 1 is load_cache itself."""
    rng = np.random.default_rng(9)
    counts = rng.integers(0, 7, 150).astype(np.uint32)
    ranked = brute_rank(counts)
    for alpha in [0.0, 0.02, 0.1, 0.2, 0.5, 1.0]:
        slot1, sh1 = oracle.sharded_cache(counts, alpha, 1)
        assert np.array_equal(slot1, oracle.cache_slots(counts, alpha))
        for world in [2, 3, 8]:
            slot, shards = oracle.sharded_cache(counts, alpha, world)
            C = min(150, world * int(alpha * 150))
            members = [v for s in shards for v in s.tolist()]
            assert sorted(members) == sorted(ranked[:C])            # the top C, disjoint
            assert sorted(slot[slot >= 0].tolist()) == list(range(C))
            for r, s in enumerate(shards):
                assert s.tolist() == [ranked[i] for i in range(r, C, world)]
                assert all(int(slot[v]) % world == r for v in s.tolist())
            if world * alpha >= 1.0:
                assert C == 150 and np.all(slot >= 0)               # every row cached somewhere


def test_extract_counts_pins():
    slot = np.array([-1, 0, 1, 2, 3, -1, 4], np.int32)              # 5 cached rows over 2 shards
    ids = np.array([0, 1, 2, 3, 4, 5, 6, 6, 1], np.uint32)
    assert oracle.extract_counts(ids, slot) == (7, 2, 0)
    # shard 0 holds slots 0, 2, 4 (vertices 1, 3, 6); shard 1 slots 1, 3 (vertices 2, 4)
    assert oracle.extract_counts(ids, slot, 0, 2) == (7, 2, 2)      # vertices 2 and 4
    assert oracle.extract_counts(ids, slot, 1, 2) == (7, 2, 5)      # 1, 3, 6, 6, 1
