"""Pins for the oracle's weighted k-hop sampler (NEXT-1; PAPER.md L81 fn1, L148 fn5,
L136; reading Q19: k draws with replacement, inverse CDF over the row's weights)."""
import numpy as np
import pytest
from scipy import stats

import oracle
import synth


def star(weights):
    n = len(weights)
    indptr = np.array([0, n] + [n] * n, np.uint64)
    indices = np.arange(1, n + 1, dtype=np.uint32)
    return oracle.GraphOracle(indptr, indices), np.array(weights, np.uint32)


def test_pick_frequency_proportional_to_weight():
    go, w = star([1, 2, 3, 4, 0, 6])
    cnt = np.zeros(len(w))
    for b in range(3000):
        s = go.sample_khop_weighted(w, [0], [4], 9, 0, b)
        assert len(s.indices[0]) == 4                      # with replacement: always k
        for lid in s.indices[0]:
            cnt[int(s.uniq[lid]) - 1] += 1
    assert cnt[4] == 0                                     # zero weight never drawn
    p = w / w.sum()
    nz = p > 0
    chi2, pval = stats.chisquare(cnt[nz], cnt.sum() * p[nz])
    assert pval > 1e-3, (cnt, pval)


def test_unit_weights_uniform_over_positions():
    go, w = star([1] * 7)
    cnt = np.zeros(7)
    for b in range(4000):
        s = go.sample_khop_weighted(w, [0], [3], 4, 1, b)
        for lid in s.indices[0]:
            cnt[int(s.uniq[lid]) - 1] += 1
    assert stats.chisquare(cnt).pvalue > 1e-3


def test_zero_total_weight_and_empty_rows():
    # 0 -> {1, 2} with weights 0, 0; 1 -> {} ; 2 -> {0} weight 5
    indptr = np.array([0, 2, 2, 3], np.uint64)
    indices = np.array([1, 2, 0], np.uint32)
    w = np.array([0, 0, 5], np.uint32)
    go = oracle.GraphOracle(indptr, indices)
    s = go.sample_khop_weighted(w, [0, 1, 2], [3], 1, 0, 0)
    assert s.indptr[0].tolist() == [0, 0, 0, 3]
    assert s.uniq[s.indices[0]].tolist() == [0, 0, 0]


def test_invariants_power_law():
    g = synth.small_graph(3000, 30000, 2.2, 4, 200, seed=6)
    w = synth.gen_edge_weights(g.indices, 6)
    go = oracle.GraphOracle(g.indptr, g.indices)
    seeds = g.train[:64]
    s = go.sample_khop_weighted(w, seeds, [10, 5], 3, 0, 0)
    assert len(set(s.uniq.tolist())) == len(s.uniq) and s.uniq[:64].tolist() == seeds.tolist()
    for l, k in enumerate([10, 5]):
        n_l = s.sizes[l]
        first_new = []
        seen = set()
        for d in range(n_l):
            v = int(s.uniq[d])
            lo, hi = int(g.indptr[v]), int(g.indptr[v + 1])
            row = s.indices[l][s.indptr[l][d]:s.indptr[l][d + 1]]
            W = int(w[lo:hi].sum())
            assert len(row) == (k if W > 0 else 0)
            allowed = {int(g.indices[q]) for q in range(lo, hi) if w[q] > 0}
            assert {int(s.uniq[x]) for x in row} <= allowed      # positive-weight CSR edges
            for x in row.tolist():
                if x >= n_l and x not in seen:
                    seen.add(x)
                    first_new.append(x)
        assert first_new == list(range(n_l, s.sizes[l + 1]))


def test_newer_neighbours_preferred():
    """L136: weights = target's year; heavier targets are sampled more often."""
    g = synth.small_graph(3000, 60000, 2.2, 4, 500, seed=7)
    w = synth.gen_edge_weights(g.indices, 7)
    go = oracle.GraphOracle(g.indptr, g.indices)
    tot = np.zeros(17)
    for b in range(5):
        s = go.sample_khop_weighted(w, g.train[b * 100:(b + 1) * 100], [10], 2, 0, b)
        # weight of each picked target (year of the target vertex: same for all its in-edges)
        year = np.zeros(g.V, np.uint32)
        year[g.indices] = w
        tot += np.bincount(year[s.uniq[s.indices[0]]], minlength=17)
    assert tot[13:].sum() > 2 * tot[1:5].sum()
