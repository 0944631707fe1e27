"""The shared input generator: deterministic, thread-count independent, row-addressable."""
import numpy as np

import gen


def test_rows_thread_independent_and_addressable():
    a = gen.make_rows(3, 500, nthreads=1)
    b = gen.make_rows(3, 500, nthreads=4)
    assert np.array_equal(a, b)
    c = gen.make_rows(3, 100, row0=200)
    assert np.array_equal(a[200:300], c)
    idx = np.array([5, 77, 499])
    assert np.array_equal(gen.make_rows_idx(3, idx), a[idx])


def test_forest_deterministic_and_valid():
    f1 = gen.make_forest(2, n_trees=30, nthreads=1)
    f2 = gen.make_forest(2, n_trees=30, nthreads=3)
    for k in ("root", "feature", "threshold", "left", "right", "leaf_value", "default_left"):
        assert np.array_equal(f1[k], f2[k])
    f = f1
    internal = f["feature"] >= 0
    assert (f["feature"][internal] < 28).all()
    assert (f["left"][internal] > np.arange(len(internal))[internal]).all()  # BFS: children later
    # dyadic leaves k/256, |k| <= 256
    lv = f["leaf_value"][~internal] * 256
    assert np.array_equal(lv, np.round(lv)) and np.abs(lv).max() <= 256


def test_covtype_shape_one_hot():
    X = gen.make_rows(3, 200)
    assert (X[:, 10:14].sum(1) == 1).all() and (X[:, 14:54].sum(1) == 1).all()
    assert np.array_equal(X[:, :10], np.round(X[:, :10]))


def test_subsample_sorted_distinct():
    s = gen.subsample(1, 10_000, 500)
    assert len(np.unique(s)) == 500 and (np.diff(s) > 0).all() and s.max() < 10_000
