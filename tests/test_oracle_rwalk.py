"""Pins for the oracle's PinSAGE random-walk selection (
reading Q13): closed forms on paths and stars, dead ends, and the exact
expected visit counts 4 * sum_t P^t[v,u] on a 6-vertex graph."""
import numpy as np

import oracle


def csr(adj, V):
    indptr = np.zeros(V + 1, np.uint64)
    for v in range(V):
        indptr[v + 1] = indptr[v] + len(adj.get(v, []))
    indices = np.array([u for v in range(V) for u in adj.get(v, [])], np.uint32)
    return oracle.GraphOracle(indptr, indices)


def test_path_graph_closed_form():
    # 0 -> 1 -> 2 -> 3 -> 4 -> 5 (deterministic walks): every walk visits 1,2,3
    g = csr({i: [i + 1] for i in range(5)}, 6)
    s = g.sample_rwalk([0], 1, 5, 0, 0)
    assert s.uniq.tolist() == [0, 1, 2, 3]
    assert s.indices[0].tolist() == [1, 2, 3]
    assert s.weights[0].tolist() == [4, 4, 4]


def test_dead_end_and_start_exclusion():
    # 0 -> 1 -> 0 (cycle): walks from 0 visit 1, 0(excluded), 1  -> count(1) = 8
    g = csr({0: [1], 1: [0]}, 3)
    s = g.sample_rwalk([0, 2], 1, 5, 0, 0)           # vertex 2 has no out-edges
    assert s.indptr[0].tolist() == [0, 1, 1]
    assert s.uniq[s.indices[0]].tolist() == [1]
    assert s.weights[0].tolist() == [8]


def test_star_topk_and_tiebreak():
    # hub 0 -> leaves 1..8 (each leaf -> 0): per walk two leaf visits, 8 in total
    adj = {0: list(range(1, 9))}
    adj.update({i: [0] for i in range(1, 9)})
    g = csr(adj, 9)
    for b in range(50):
        s = g.sample_rwalk([0], 1, 17, 3, b)
        w = s.weights[0].tolist()
        gids = s.uniq[s.indices[0]].tolist()
        assert len(w) <= 5 and sum(w) <= 8
        # sorted by (count desc, gid asc)
        keys = [(-c, x) for c, x in zip(w, gids)]
        assert keys == sorted(keys)


def test_expected_visits_match_matrix_powers():
    adj = {0: [1, 2, 2], 1: [3, 0], 2: [4, 5], 3: [5], 4: [], 5: [1, 4, 0]}
    V = 6
    g = csr(adj, V)
    P = np.zeros((V, V))
    for v, nb in adj.items():
        for u in nb:
            P[v, u] += 1.0 / len(nb)
    Pt = np.eye(V)
    expect = np.zeros(V)
    for _ in range(3):
        Pt = Pt @ P
        expect += 4 * Pt[0]
    expect[0] = 0.0
    trials = 8000
    tot = np.zeros(V)
    sq = np.zeros(V)
    for b in range(trials):
        s = g.sample_rwalk([0], 1, 23, 0, b)
        c = np.zeros(V)
        c[s.uniq[s.indices[0]]] = s.weights[0]     # <=5 other vertices: nothing truncated
        tot += c
        sq += c * c
    mean = tot / trials
    sd = np.sqrt(np.maximum(sq / trials - mean ** 2, 1e-12) / trials)
    assert np.all(np.abs(mean - expect) < 5 * sd + 1e-9), (mean, expect)
