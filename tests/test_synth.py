"""Input generator checks (inputs only; not part of the method)."""
import numpy as np

import synth


def test_thread_count_invariance_and_shape():
    a = synth.gen_topology(20000, 300000, 2.2, 2.2, 77, 20000 // 16, threads=1)
    b = synth.gen_topology(20000, 300000, 2.2, 2.2, 77, 20000 // 16, threads=7)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    indptr, indices = a
    assert indptr[0] == 0 and indptr[-1] == 300000 and np.all(np.diff(indptr.astype(np.int64)) >= 0)
    assert indices.max() < 20000
    assert np.diff(indptr).max() <= 20000 // 16 + 1
    f1 = synth.gen_features(100, 8, 3, threads=1)
    f2 = synth.gen_features(100, 8, 3, threads=4)
    assert np.array_equal(f1, f2) and f1.min() >= -1.0 and f1.max() < 1.0


def test_trainset_distinct_sorted():
    t = synth.gen_trainset(10000, 1000, 5)
    assert np.all(np.diff(t.astype(np.int64)) > 0) and t.max() < 10000


def test_perm_is_bijection():
    n = 1000
    p = [synth.lib().synth_perm(n, 9, 7, x) for x in range(n)]
    assert sorted(p) == list(range(n))
