"""Pins for the oracle's k-hop sampler + relabel (PAPER.md L67, L169-185,
L230, L410; readings Q2, Q3, Q5-Q7).

* brute-force enumeration of all C(n,k) subsets + chi-square (uniform k-subset)
* BFS closed form when fanout >= max degree (BFS layers == hop discoveries)
* relabel invariants on random power-law graphs
"""
import itertools
import math

import numpy as np
import pytest
from scipy import stats

import oracle
import synth


def star(n, extra_edges=()):
    """vertex 0 -> 1..n; vertices 1..n have no out-edges."""
    indptr = np.zeros(n + 2, np.uint64)
    indptr[1:] = n
    indices = np.arange(1, n + 1, dtype=np.uint32)
    return oracle.GraphOracle(indptr, indices)


@pytest.mark.parametrize("n,k", [(4, 2), (5, 3), (6, 2), (7, 5), (8, 3), (8, 4)])
def test_floyd_uniform_subsets_chi2(n, k):
    g = star(n)
    subsets = {frozenset(c): i for i, c in enumerate(itertools.combinations(range(n), k))}
    cnt = np.zeros(len(subsets))
    trials = 12000
    for b in range(trials):
        s = g.sample_khop([0], [k], 7, 0, b, want_picks=True)
        p = s.picks[0].tolist()
        assert len(set(p)) == k and all(0 <= x < n for x in p)     # without replacement
        # the picked CSR positions are what the block holds (vertex p+1, lid order)
        assert sorted(int(s.uniq[x]) - 1 for x in s.indices[0]) == sorted(p)
        cnt[subsets[frozenset(p)]] += 1
    chi2, pval = stats.chisquare(cnt)
    assert pval > 1e-3, (chi2, pval)


def test_small_degree_takes_whole_row_in_csr_order():
    g = star(5)
    for k in [5, 6, 25]:
        s = g.sample_khop([0], [k], 1, 0, 0, want_picks=True)
        assert s.picks[0][:5].tolist() == [0, 1, 2, 3, 4]
        assert s.uniq.tolist() == [0, 1, 2, 3, 4, 5]
        assert s.indices[0].tolist() == [1, 2, 3, 4, 5]


def test_marginal_inclusion_probability():
    # each of n positions is chosen with probability k/n
    n, k, trials = 20, 6, 6000
    g = star(n)
    hits = np.zeros(n)
    for b in range(trials):
        s = g.sample_khop([0], [k], 3, 2, b, want_picks=True)
        hits[s.picks[0]] += 1
    p = k / n
    z = (hits - trials * p) / math.sqrt(trials * p * (1 - p))
    assert np.abs(z).max() < 5.0


def bfs_layers(indptr, indices, seeds, L):
    V = len(indptr) - 1
    dist = np.full(V, -1)
    dist[seeds] = 0
    frontier = list(seeds)
    for l in range(1, L + 1):
        nxt = []
        for v in frontier:
            for u in indices[indptr[v]:indptr[v + 1]]:
                if dist[u] < 0:
                    dist[u] = l
                    nxt.append(u)
        frontier = nxt
    return dist


def test_bfs_closed_form_when_fanout_exceeds_degree():
    g = synth.small_graph(3000, 12000, 2.3, 8, 100, seed=5, cap=40)
    go = oracle.GraphOracle(g.indptr, g.indices)
    maxdeg = int(np.diff(g.indptr).max())
    seeds = g.train[:20]
    L = 3
    s = go.sample_khop(seeds, [maxdeg] * L, 11, 0, 0)
    dist = bfs_layers(g.indptr.astype(np.int64), g.indices, seeds.astype(np.int64), L)
    # vertices with lid in [n_l, n_{l+1}) are exactly the BFS layer l+1
    for l in range(L + 1):
        lo = 0 if l == 0 else s.sizes[l - 1]
        got = set(s.uniq[lo:s.sizes[l]].tolist())
        assert got == set(np.nonzero(dist == l)[0].tolist())
    # each block row is the full CSR row, in CSR order
    for l in range(L):
        for d in range(s.sizes[l]):
            v = s.uniq[d]
            row = g.indices[g.indptr[v]:g.indptr[v + 1]]
            blk = s.uniq[s.indices[l][s.indptr[l][d]:s.indptr[l][d + 1]]]
            assert blk.tolist() == row.tolist()


def check_relabel_invariants(s, indptr, indices, seeds, fanouts):
    uniq = s.uniq
    assert len(set(uniq.tolist())) == len(uniq)                      # dedup
    assert uniq[:len(seeds)].tolist() == list(seeds)                # seeds are the prefix
    for l, k in enumerate(fanouts):
        n_l, n_next = s.sizes[l], s.sizes[l + 1]
        ip, ix = s.indptr[l], s.indices[l]
        assert ip.shape[0] == n_l + 1 and ip[0] == 0 and ip[-1] == ix.shape[0]
        assert np.all(np.diff(ip.astype(np.int64)) >= 0)
        assert ix.shape[0] == 0 or ix.max() < n_next
        first_new = []
        seen = set()
        for d in range(n_l):
            v = int(uniq[d])
            deg = int(indptr[v + 1] - indptr[v])
            row = ix[ip[d]:ip[d + 1]]
            assert row.shape[0] == min(deg, k)
            nbrs = indices[indptr[v]:indptr[v + 1]]
            gids = uniq[row]
            # each emitted edge is a CSR edge; multiplicities within the row's multiset
            vals, cnts = np.unique(gids, return_counts=True)
            nv, nc = np.unique(nbrs, return_counts=True)
            m = dict(zip(nv.tolist(), nc.tolist()))
            for a, c in zip(vals.tolist(), cnts.tolist()):
                assert m.get(a, 0) >= c
            for x in row.tolist():
                if x >= n_l and x not in seen:
                    seen.add(x)
                    first_new.append(x)
        # first appearances of new lids are exactly n_l, n_l+1, ... (first-occurrence order)
        assert first_new == list(range(n_l, n_next))


@pytest.mark.parametrize("fanouts", [(10, 5), (25, 10), (15, 10, 5), (3,), (1, 1, 1, 1)])
def test_relabel_invariants_power_law(fanouts):
    g = synth.small_graph(5000, 60000, 2.2, 4, 500, seed=3)
    go = oracle.GraphOracle(g.indptr, g.indices)
    for b in range(3):
        seeds = g.train[b * 64:(b + 1) * 64]
        s = go.sample_khop(seeds, fanouts, 99, 1, b)
        check_relabel_invariants(s, g.indptr, g.indices, seeds.tolist(), fanouts)


def test_self_loops_and_multi_edges():
    # 0 -> {0, 1, 1, 2}; self loop maps to own lid, duplicate picks give two edges
    indptr = np.array([0, 4, 4, 4], np.uint64)
    indices = np.array([0, 1, 1, 2], np.uint32)
    go = oracle.GraphOracle(indptr, indices)
    s = go.sample_khop([0], [4], 1, 0, 0)
    assert s.uniq.tolist() == [0, 1, 2]
    assert s.indices[0].tolist() == [0, 1, 1, 2]


def test_edge_cases_and_errors():
    g = synth.small_graph(500, 3000, 2.2, 4, 50, seed=8)
    go = oracle.GraphOracle(g.indptr, g.indices)
    s = go.sample_khop(g.train[:5], [], 1, 0, 0)                   # num_hops = 0
    assert s.uniq.tolist() == g.train[:5].tolist() and s.sizes == [5]
    s = go.sample_khop(np.array([], np.uint32), [3, 2], 1, 0, 0)    # empty batch
    assert s.sizes == [0, 0, 0] and s.uniq.shape[0] == 0
    with pytest.raises(oracle.OracleError) as e:
        go.sample_khop([1, 2, 1], [3], 1, 0, 0)                     # duplicate seed (Q6)
    assert e.value.rc == oracle.EINVAL
    with pytest.raises(oracle.OracleError) as e:
        go.sample_khop([1, 500], [3], 1, 0, 0)                      # id >= V
    assert e.value.rc == oracle.EINVAL
    with pytest.raises(oracle.OracleError) as e:
        go.sample_khop([1], [3], 1, 1 << 16, 0)                     # epoch field width
    assert e.value.rc == oracle.ERANGE
    with pytest.raises(oracle.OracleError) as e:
        go.sample_khop([1], [0], 1, 0, 0)                           # fanout 0
    assert e.value.rc == oracle.EINVAL
    # the scratch map is restored after errors and successes
    assert np.all(go.lid == -1)


def test_rng_keys_change_the_draw():
    g = synth.small_graph(2000, 40000, 2.2, 4, 200, seed=4)
    go = oracle.GraphOracle(g.indptr, g.indices)
    seeds = g.train[:64]
    base = go.sample_khop(seeds, [10, 5], 1, 0, 0).uniq
    assert np.array_equal(base, go.sample_khop(seeds, [10, 5], 1, 0, 0).uniq)   # deterministic
    for args in [(2, 0, 0), (1, 1, 0), (1, 0, 1)]:                                # seed/epoch/batch
        assert not np.array_equal(base, go.sample_khop(seeds, [10, 5], *args).uniq)
