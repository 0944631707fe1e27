"""Pins of the CPU oracle against things other than itself (SURVEY §8(c) "What pins each part").

Each test fixes the oracle to a value the paper or the mathematics determines:
  * hand-worked forests (tests/golden/handbuilt_forest.json): the node test, ties, signed zero,
    NaN defaults, infinities (readings Z1-Z3);
  * brute-force path boxes for random trees of depth <= 3 (every sample lies in exactly one box);
  * a complete single-feature BST reaches leaf bisect_right(thresholds, x) (textbook reduction);
  * a forest of stumps equals a searchsorted/suffix-sum closed form;
  * dyadic leaf values make every sum exact, so fp32 outputs equal exact rational arithmetic;
  * argmax / vote / binary tie rules (reading Z14);
  * invariants: one leaf per (sample, tree), visits = sum of leaf depths.
"""
import bisect
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import gen
import oracle
from tlib import GOLDEN


def _hand():
    g = json.load(open(os.path.join(GOLDEN, "handbuilt_forest.json")))
    f = {k: np.array(v) for k, v in g["forest"].items()}
    forest = dict(root=f["root"].astype(np.int32), feature=f["feature"].astype(np.int32),
                  threshold=f["threshold"].astype(np.float32), left=f["left"].astype(np.int32),
                  right=f["right"].astype(np.int32), leaf_value=f["leaf_value"].astype(np.float32),
                  default_left=f["default_left"].astype(np.uint8), tree_class=None,
                  n_classes=1, agg=oracle.AGG_SUM)
    X = np.array([[float(v) for v in r] for r in g["rows"]], np.float32)
    return g, forest, X


def test_handbuilt_worked_answers():
    g, forest, X = _hand()
    assert np.signbit(X[2, 0]) and X[2, 0] == 0.0  # the -0.0 row really is negative zero
    r = oracle.predict(forest, X, want_leaf=True)
    assert r["leaf"].tolist() == g["expected_leaf"]
    assert r["out"][:, 0].tolist() == g["expected_sum"]
    assert r["visits"].tolist() == g["expected_visits"]
    r2 = oracle.predict(forest, X, want_leaf=True, use_default_left=False)
    assert r2["leaf"].tolist() == g["expected_leaf_no_default"]
    assert r2["out"][:, 0].tolist() == g["expected_sum_no_default"]


def test_handbuilt_base_average_binary():
    g, forest, X = _hand()
    exp = np.array(g["expected_sum"])
    r = oracle.predict(forest, X, agg=oracle.AGG_SUM, base_score=0.5)
    assert r["out"][:, 0].tolist() == (exp + 0.5).tolist()
    r = oracle.predict(forest, X, agg=oracle.AGG_AVERAGE, base_score=-1.0)
    assert r["out"][:, 0].tolist() == (exp / 2 - 1.0).tolist()
    r = oracle.predict(forest, X, agg=oracle.AGG_BINARY, base_score=-8.25)
    # margin exactly 0 => class 0 (reading Z14); positive => 1
    assert r["cls"].tolist() == [int(v - 8.25 > 0) for v in exp]
    assert (exp - 8.25 == 0).sum() == 3


# ----------------------------------------------------------------- random small forests
def random_forest(rng, n_trees, max_depth, d, p_split=0.8, n_classes=1, vote=False,
                  dyadic=True, thr_grid=None):
    """Random binary trees in plain Python (independent of gen/), node ids global, BFS-free."""
    feature, thr, left, right, val, dl, root = [], [], [], [], [], [], []

    def new():
        feature.append(-1); thr.append(0.0); left.append(-1); right.append(-1)
        val.append(0.0); dl.append(0)
        return len(feature) - 1

    def grow(k, depth):
        if depth < max_depth and (depth == 0 or rng.random() < p_split):
            feature[k] = int(rng.integers(d))
            thr[k] = float(rng.choice(thr_grid)) if thr_grid is not None else float(rng.normal())
            dl[k] = int(rng.integers(2))
            L, R = new(), new()
            left[k], right[k] = L, R
            grow(L, depth + 1)
            grow(R, depth + 1)
        else:
            if vote:
                val[k] = float(rng.integers(n_classes))
            elif dyadic:
                val[k] = float(rng.integers(-256, 257)) / 256.0
            else:
                val[k] = float(np.float32(rng.normal() * 0.1))

    for _ in range(n_trees):
        r = new()
        root.append(r)
        grow(r, 0)
    return dict(root=np.array(root, np.int32), feature=np.array(feature, np.int32),
                threshold=np.array(thr, np.float32), left=np.array(left, np.int32),
                right=np.array(right, np.int32), leaf_value=np.array(val, np.float32),
                default_left=np.array(dl, np.uint8),
                tree_class=np.arange(n_trees, dtype=np.int32) % n_classes,
                n_classes=n_classes, agg=oracle.AGG_SUM)


def path_boxes(forest, t, d):
    """Every root->leaf path of tree t as a box {feature: [lo, hi)} (left: x < b => hi = b)."""
    out = []
    stack = [(int(forest["root"][t]), [(-np.inf, np.inf)] * d)]
    while stack:
        k, box = stack.pop()
        if forest["feature"][k] < 0:
            out.append((k, box))
            continue
        f, b = int(forest["feature"][k]), float(forest["threshold"][k])
        lb = list(box); lo, hi = lb[f]; lb[f] = (lo, min(hi, b))
        rb = list(box); lo, hi = rb[f]; rb[f] = (max(lo, b), hi)
        stack.append((int(forest["left"][k]), lb))
        stack.append((int(forest["right"][k]), rb))
    return out


@pytest.mark.parametrize("seed", range(6))
def test_brute_force_path_boxes_depth3(seed):
    rng = np.random.default_rng(seed)
    d = 4
    grid = np.array([-1.0, -0.5, 0.0, 0.25, 1.0], np.float32)
    forest = random_forest(rng, 12, 3, d, thr_grid=grid)
    # include values equal to thresholds so ties are exercised
    X = rng.choice(np.concatenate([grid, rng.normal(size=20).astype(np.float32)]),
                   size=(300, d)).astype(np.float32)
    r = oracle.predict(forest, X, want_leaf=True)
    for t in range(len(forest["root"])):
        boxes = path_boxes(forest, t, d)
        for i in range(X.shape[0]):
            hits = [k for k, box in boxes
                    if all(lo <= X[i, j] < hi for j, (lo, hi) in enumerate(box))]
            assert len(hits) == 1, "exactly one box holds each sample"
            assert r["leaf"][i, t] == hits[0]


def _complete_bst(thresholds):
    """Complete BST over one feature; leaves carry their in-order index."""
    feature, thr, left, right, val = [], [], [], [], []

    # balanced over indices [0, m) with m = 2^D - 1 internal nodes
    def build(lo, hi, leaf_base):  # internal thresholds thresholds[lo:hi]
        k = len(feature)
        feature.append(-1); thr.append(0.0); left.append(-1); right.append(-1); val.append(0.0)
        if lo >= hi:
            val[k] = float(leaf_base)
            return k, leaf_base + 1
        mid = (lo + hi) // 2
        feature[k] = 0
        thr[k] = float(thresholds[mid])
        L, nb = build(lo, mid, leaf_base)
        R, nb = build(mid + 1, hi, nb)
        left[k], right[k] = L, R
        return k, nb

    build(0, len(thresholds), 0)
    return dict(root=np.array([0], np.int32), feature=np.array(feature, np.int32),
                threshold=np.array(thr, np.float32), left=np.array(left, np.int32),
                right=np.array(right, np.int32), leaf_value=np.array(val, np.float32),
                default_left=None, tree_class=None, n_classes=1, agg=oracle.AGG_SUM)


@pytest.mark.parametrize("D", [1, 2, 3, 4, 5, 6])
def test_bst_equals_bisect_right(D):
    rng = np.random.default_rng(D)
    m = 2 ** D - 1
    u = np.sort(rng.choice(np.arange(-500, 500), size=m, replace=False)).astype(np.float32) / 8
    forest = _complete_bst(u)
    xs = np.concatenate([u, u - 0.0625, u + 0.0625, [-1e9, 1e9, -np.inf, np.inf]]).astype(np.float32)
    r = oracle.predict(forest, xs[:, None])
    exp = [bisect.bisect_right(list(u), float(x)) for x in xs]
    assert r["out"][:, 0].tolist() == [float(e) for e in exp]
    assert r["visits"].tolist() == [D] * len(xs)  # a complete tree: every path has D tests


def test_stumps_equal_searchsorted_closed_form():
    rng = np.random.default_rng(7)
    T = 1000
    b = (rng.integers(-200, 200, size=T) / 16).astype(np.float32)  # many ties
    Lv = (rng.integers(-256, 257, size=T) / 256).astype(np.float32)
    Rv = (rng.integers(-256, 257, size=T) / 256).astype(np.float32)
    n_nodes = 3 * T
    forest = dict(root=np.arange(0, n_nodes, 3, dtype=np.int32),
                  feature=np.tile(np.array([0, -1, -1], np.int32), T),
                  threshold=np.repeat(b, 3).astype(np.float32) * np.tile([1, 0, 0], T).astype(np.float32),
                  left=np.array([[3 * t + 1, -1, -1] for t in range(T)], np.int32).ravel(),
                  right=np.array([[3 * t + 2, -1, -1] for t in range(T)], np.int32).ravel(),
                  leaf_value=np.array([[0, Lv[t], Rv[t]] for t in range(T)], np.float32).ravel(),
                  default_left=None, tree_class=None, n_classes=1, agg=oracle.AGG_SUM)
    xs = np.concatenate([b[:200], rng.normal(size=200) * 8]).astype(np.float32)
    r = oracle.predict(forest, xs[:, None])
    # closed form: pred(x) = sum_t R_t + sum_{t: b_t > x} (L_t - R_t)
    order = np.argsort(b, kind="stable")
    bs = b[order]
    diff = (Lv - Rv).astype(np.float64)[order]
    suffix = np.concatenate([np.cumsum(diff[::-1])[::-1], [0.0]])
    exp = Rv.astype(np.float64).sum() + suffix[np.searchsorted(bs, xs, side="right")]
    assert np.array_equal(r["raw"][:, 0], exp)  # dyadic => exact in any order


@pytest.mark.parametrize("agg", [oracle.AGG_SUM, oracle.AGG_AVERAGE, oracle.AGG_BINARY])
def test_dyadic_sums_exact_rational(agg):
    rng = np.random.default_rng(11 + agg)
    forest = random_forest(rng, 37, 5, 6)
    X = rng.normal(size=(200, 6)).astype(np.float32)
    X[rng.random(X.shape) < 0.05] = np.nan
    base = 0.375
    r = oracle.predict(forest, X, agg=agg, base_score=base, want_leaf=True)
    T = len(forest["root"])
    for i in range(X.shape[0]):
        s = sum(Fraction(float(forest["leaf_value"][r["leaf"][i, t]])) for t in range(T))
        if agg == oracle.AGG_AVERAGE:
            s = s / T
        s = s + Fraction(base)
        assert r["out"][i, 0] == np.float32(float(s))
        if agg == oracle.AGG_BINARY:
            assert r["cls"][i] == int(s > 0)


def test_class_sum_argmax_ties_lowest():
    rng = np.random.default_rng(3)
    C = 4
    base_forest = random_forest(rng, 5, 4, 3)
    # duplicate the 5 trees into every class => all class sums tie => class 0
    T0 = len(base_forest["root"])
    nn = len(base_forest["feature"])
    parts = {k: [] for k in ("root", "feature", "threshold", "left", "right", "leaf_value",
                             "default_left")}
    for c in range(C):
        off = c * nn
        parts["root"].append(base_forest["root"] + off)
        parts["feature"].append(base_forest["feature"])
        parts["threshold"].append(base_forest["threshold"])
        parts["left"].append(np.where(base_forest["left"] >= 0, base_forest["left"] + off, -1))
        parts["right"].append(np.where(base_forest["right"] >= 0, base_forest["right"] + off, -1))
        parts["leaf_value"].append(base_forest["leaf_value"])
        parts["default_left"].append(base_forest["default_left"])
    forest = {k: np.concatenate(v).astype(base_forest[k].dtype) for k, v in parts.items()}
    forest["tree_class"] = np.repeat(np.arange(C, dtype=np.int32), T0)
    X = rng.normal(size=(50, 3)).astype(np.float32)
    r = oracle.predict(forest, X, agg=oracle.AGG_CLASS_SUM, n_classes=C)
    assert (r["cls"] == 0).all()
    assert (r["out"] == r["out"][:, :1]).all()
    # make class 2 strictly larger by adding a constant-leaf stump tree to class 2
    k0 = len(forest["feature"])
    f2 = {k: np.concatenate([forest[k], np.array(v, forest[k].dtype)]) for k, v in dict(
        feature=[-1], threshold=[0], left=[-1], right=[-1], leaf_value=[0.5],
        default_left=[0]).items()}
    f2["root"] = np.concatenate([forest["root"], np.array([k0], np.int32)])
    f2["tree_class"] = np.concatenate([forest["tree_class"], np.array([2], np.int32)])
    r = oracle.predict(f2, X, agg=oracle.AGG_CLASS_SUM, n_classes=C)
    assert (r["cls"] == 2).all()


def test_vote_counts_and_ties():
    rng = np.random.default_rng(5)
    C = 3
    forest = random_forest(rng, 30, 4, 5, n_classes=C, vote=True)
    X = rng.normal(size=(100, 5)).astype(np.float32)
    r = oracle.predict(forest, X, agg=oracle.AGG_VOTE, n_classes=C, want_leaf=True)
    for i in range(X.shape[0]):
        v = np.bincount(forest["leaf_value"][r["leaf"][i]].astype(int), minlength=C)
        assert r["out"][i].tolist() == v.astype(np.float32).tolist()
        assert r["cls"][i] == int(np.flatnonzero(v == v.max())[0])


def _depths(forest):
    dep = np.zeros(len(forest["feature"]), np.int64)
    for r in forest["root"]:
        stack = [(int(r), 0)]
        while stack:
            k, dd = stack.pop()
            dep[k] = dd
            if forest["feature"][k] >= 0:
                stack += [(int(forest["left"][k]), dd + 1), (int(forest["right"][k]), dd + 1)]
    return dep


def test_invariants_on_generated_c1():
    f = gen.make_forest(1)
    X = gen.make_rows(1, 1000)
    r = oracle.predict(f, X, want_leaf=True)
    T = len(f["root"])
    # exactly one leaf per (sample, tree), inside that tree's node range
    bounds = np.append(f["root"], len(f["feature"]))
    for t in range(T):
        lt = r["leaf"][:, t]
        assert ((lt >= bounds[t]) & (lt < bounds[t + 1])).all()
        assert (f["feature"][lt] < 0).all()
    dep = _depths(f)
    assert (dep[r["leaf"]].sum(1) == r["visits"].astype(np.int64)).all()


def test_oracle_thread_count_independent():
    f = gen.make_forest(2, n_trees=40, leaf_mode="normal")
    X = gen.make_rows(2, 3000)
    a = oracle.predict(f, X, nthreads=1)
    b = oracle.predict(f, X, nthreads=0)
    assert np.array_equal(a["raw"], b["raw"]) and np.array_equal(a["fp"], b["fp"])


def test_oracle_rows_subset_matches_full():
    f = gen.make_forest(2, n_trees=20)
    X = gen.make_rows(2, 500)
    idx = gen.subsample(9, 500, 60)
    a = oracle.predict(f, X, want_leaf=True)
    b = oracle.predict(f, X, rows=idx, want_leaf=True)
    assert np.array_equal(a["leaf"][idx], b["leaf"]) and np.array_equal(a["raw"][idx], b["raw"])


# ----------------------------------------------------------------- fingerprint
_M64 = (1 << 64) - 1


def _mix64(z: int) -> int:
    """splitmix64's output finaliser, restated in plain Python integers."""
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def test_mix64_known_answers():
    """The restated finaliser reproduces the published splitmix64 stream of seed 0 (state advanced
    by the golden gamma 0x9E3779B97F4A7C15 before each output): 0xE220A8397B1DCDAF,
    0x6E789E6AA1B965F4, 0x06C45D188009454F."""
    s, got = 0, []
    for _ in range(3):
        s = (s + 0x9E3779B97F4A7C15) & _M64
        got.append(_mix64(s))
    assert got == [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]


def _fp_from_leaves(leaf: np.ndarray, tree_ids) -> np.ndarray:
    out = np.zeros(leaf.shape[0], np.uint64)
    for i in range(leaf.shape[0]):
        acc = 0
        for j, t in enumerate(tree_ids):
            acc = (acc + _mix64(((int(t) << 32) | (int(leaf[i, j]) & 0xFFFFFFFF)) & _M64)) & _M64
        out[i] = acc
    return out


def test_fingerprint_restated_from_leaf_ids():
    """fp[i] = sum_t mix64((t << 32) | leaf[i][t]) mod 2^64, restated from the
    oracle's own leaf ids (not from its fingerprint code)."""
    rng = np.random.default_rng(5)
    f = random_forest(rng, 23, 5, 6)
    X = rng.normal(size=(257, 6)).astype(np.float32)
    r = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1, want_leaf=True)
    assert np.array_equal(r["fp"], _fp_from_leaves(r["leaf"], range(23)))


def test_fingerprint_single_leaf_trees_closed_form():
    """Trees that are single leaves: every row reaches the root, so fp is the same closed-form
    constant for every row."""
    T = 9
    roots = np.arange(100, 100 + T, dtype=np.int32)
    n = 110
    f = dict(root=roots, feature=np.full(n, -1, np.int32), threshold=np.zeros(n, np.float32),
             left=np.full(n, -1, np.int32), right=np.full(n, -1, np.int32),
             leaf_value=np.zeros(n, np.float32), default_left=None, tree_class=None)
    X = np.zeros((5, 2), np.float32)
    r = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1)
    want = 0
    for t in range(T):
        want = (want + _mix64((t << 32) | (100 + t))) & _M64
    assert r["fp"].tolist() == [want] * 5


def test_fingerprint_tree_sharded_sum_equals_full():
    """Invariant: splitting the trees into shards and summing the shards'
    fingerprints (each tree keeping its global index t) gives the full forest's fingerprint.
    The shard fingerprints are restated from the oracle's leaf ids of each sub-forest."""
    rng = np.random.default_rng(9)
    f = random_forest(rng, 31, 6, 5)
    X = rng.normal(size=(123, 5)).astype(np.float32)
    full = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1)
    perm = rng.permutation(31)
    tot = np.zeros(X.shape[0], np.uint64)
    for shard in np.array_split(perm, 4):
        sub = dict(f, root=f["root"][shard])
        rs = oracle.predict(sub, X, agg=oracle.AGG_SUM, n_classes=1, want_leaf=True)
        tot = tot + _fp_from_leaves(rs["leaf"], shard)   # uint64 wraps mod 2^64
    assert np.array_equal(tot, full["fp"])
