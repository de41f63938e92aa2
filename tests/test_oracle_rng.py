"""Pins for the oracle's RNG layer and the SURVEY §8(c) worked example.

Philox: Random123 known-answer vectors (external standard).  bounded():
exact boundary points of floor(r*n/2^64).  Worked example: an independent
implementation of the same conventions (tests/golden/survey_worked_example.json).
"""
import json
import os

import numpy as np
import pytest

import oracle

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden",
                                   "survey_worked_example.json")))


def h(x):
    return int(x, 16)


@pytest.mark.parametrize("kat", GOLD["philox_kat"])
def test_philox_random123_kat(kat):
    out = oracle.philox([h(x) for x in kat["ctr"]], [h(x) for x in kat["key"]])
    assert [int(x) for x in out] == [h(x) for x in kat["out"]]


def test_draw64_halves_and_c3():
    # c3 layout (reading Q4): epoch<<16 | hop<<8 | domain
    assert oracle.c3(0, 0, oracle.KHOP) == 0x2
    assert oracle.c3(3, 2, oracle.RWALK) == (3 << 16) | (2 << 8) | 3
    assert oracle.c3(0x1FFFF, 0x1FF, 0x1FF) == 0xFFFFFFFF  # fields are masked
    for d in GOLD["draw64"]:
        assert oracle.draw64(GOLD["seed"], *d["args"]) == h(d["value"])
    # half 0 = w1:w0, half 1 = w3:w2 of the same Philox block
    w = oracle.philox([7, 8, 9, 10], [42, 0])
    assert oracle.draw64(42, 7, 8, 9, 10, 0) == (int(w[1]) << 32) | int(w[0])
    assert oracle.draw64(42, 7, 8, 9, 10, 1) == (int(w[3]) << 32) | int(w[2])
    # the seed's high word is the second key word
    w = oracle.philox([1, 2, 3, 4], [5, 6])
    assert oracle.draw64((6 << 32) | 5, 1, 2, 3, 4, 0) == (int(w[1]) << 32) | int(w[0])


def test_bounded_boundaries():
    """bounded(r,n) = floor(r n / 2^64): value t is produced exactly by
    r in [ceil(t 2^64/n), ceil((t+1) 2^64/n)).  Check both sides of every
    boundary for several n, plus the extremes."""
    for d in GOLD["bounded"]:
        assert oracle.bounded(h(d["r"]), d["n"]) == d["value"]
    rng = np.random.default_rng(1)
    for n in [1, 2, 3, 5, 7, 10, 25, 1000, 153064, 2**31 + 11, 2**32 - 1]:
        ts = sorted(set([1, n - 1] + [int(x) for x in rng.integers(1, max(n, 2), 20)]))
        for t in ts:
            if not (0 < t < n):
                continue
            lo = -(-(t << 64) // n)          # ceil(t 2^64 / n)
            assert oracle.bounded(lo, n) == t
            assert oracle.bounded(lo - 1, n) == t - 1
        assert oracle.bounded(0, n) == 0
        assert oracle.bounded(2**64 - 1, n) == n - 1


def test_bounded_uniform_small_n():
    # every value of [0,n) is hit by r = top bits sweep, counts differ by <= 1
    for n in [3, 5, 6, 7, 11]:
        M = 4096
        vals = [oracle.bounded((i << 52) + 12345, n) for i in range(M)]
        c = np.bincount(vals, minlength=n)
        assert c.max() - c.min() <= 1


def test_worked_example_khop():
    g = GOLD["graph"]
    go = oracle.GraphOracle(np.array(g["indptr"], np.uint64), np.array(g["indices"], np.uint32))
    k = GOLD["khop"]
    s = go.sample_khop(k["seeds"], k["fanouts"], GOLD["seed"], k["epoch"], k["batch"],
                       want_picks=True)
    assert s.uniq.tolist() == k["uniq"]
    for l, b in enumerate(k["blocks"]):
        assert s.indptr[l].tolist() == b["indptr"]
        assert s.indices[l].tolist() == b["indices"]
        exp = [0xFFFFFFFF if x is None else x for x in k["picks"][l]]
        assert s.picks[l].tolist() == exp
    s1 = go.sample_khop(k["seeds"], k["fanouts"], GOLD["seed"], k["epoch"], 1)
    assert s1.uniq.tolist() == k["uniq_batch1"]


def test_worked_example_rwalk():
    g = GOLD["graph"]
    go = oracle.GraphOracle(np.array(g["indptr"], np.uint64), np.array(g["indices"], np.uint32))
    r = GOLD["rwalk"]
    s = go.sample_rwalk(r["seeds"], r["layers"], GOLD["seed"], r["epoch"], r["batch"],
                        r["walks"], r["walk_len"], r["topk"])
    assert s.uniq.tolist() == r["uniq"]
    for l, b in enumerate(r["blocks"]):
        assert s.indptr[l].tolist() == b["indptr"]
        assert s.indices[l].tolist() == b["indices"]
        assert s.weights[l].tolist() == b["weights"]


def test_worked_example_shuffle_and_features():
    sh = GOLD["shuffle"]
    assert oracle.shuffle(np.array(sh["T"]), GOLD["seed"], 0).tolist() == sh["epoch0"]
    assert oracle.shuffle(np.array(sh["T"]), GOLD["seed"], 1).tolist() == sh["epoch1"]
    for f in GOLD["features"]:
        val = oracle.feature_value(GOLD["seed"], f["v"], f["d"])
        assert int(np.float32(val).view(np.uint32)) == h(f["bits"])
        assert abs(float(val) - f["value"]) < 1e-8
