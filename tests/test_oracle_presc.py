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
