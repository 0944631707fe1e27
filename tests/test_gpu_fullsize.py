"""SURVEY §8(d) parity set at BASELINE.json's full sizes, in the launch configurations bench.py times.

Parity set (SURVEY §8(d) "The CPU oracle beside it"):
  * scores and classes: every row of C2 (1M) and C4 (500K), a seeded 10 % of C3 (400K of 4M),
    a seeded 1 % of C5 (100K of 10M, full 4000-tree forest through the fused reduce, world 1);
    scores within max(1e-5 |ref|, 1e-6) of the oracle's fp64 value (north_star), classes exact
    outside the fp64 rounding window of reading R3 (tlib.margin_bound; the rows inside it are
    counted and must stay a negligible fraction);
  * fingerprints (sum_t mix64((t << 32) | leaf)): the GPU's for ALL n rows, compared on every
    parity row; for C5 also the invariant that the 8 tree shards' fingerprints sum to the
    unsharded one on all 10M rows;
  * leaf ids as full n x T arrays on the first 64K rows, from the LEAF instantiation of the
    production kernel (same schedule, walk and launch plan);
  * leaf ids from the production instantiation itself ("marked trees"): the forest is rebuilt with
    every leaf value zero except those of a few marked trees, whose leaves carry their preorder
    ordinal shifted into disjoint bit fields; the layout is checked to be unchanged, the raw fp64
    sums (tahoe_predict_partial, the same kernel instantiation as the bench's multi-slice launch)
    are exact integers, and decoding them gives each marked tree's leaf for every one of the n rows.
"""
import numpy as np
import pytest

import gen
import oracle
from tlib import margin_bound

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402

LEAF_ROWS = 65536


def _tree_leaves(f, t):
    """Leaves of tree t in preorder (left child first), as caller node ids."""
    out, st = [], [int(f["root"][t])]
    while st:
        k = st.pop()
        if f["feature"][k] < 0:
            out.append(k)
        else:
            st.append(int(f["right"][k]))
            st.append(int(f["left"][k]))
    return out


def _check_rows(out, cls, ref, agg, bound, what):
    tol = np.maximum(1e-5 * np.abs(ref["out"]), 1e-6)
    err = np.abs(out - ref["out"])
    assert (err <= tol).all(), f"{what}: max err {err.max()}"
    window = 0
    if agg == oracle.AGG_BINARY:
        sure = np.abs(ref["raw"][:, 0]) > bound
    elif agg == oracle.AGG_CLASS_SUM:
        srt = np.sort(ref["raw"], axis=1)
        sure = (srt[:, -1] - srt[:, -2]) > bound
    else:
        sure = None
    if sure is not None:
        assert np.array_equal(cls[sure], ref["cls"][sure]), f"{what}: classes differ"
        window = int((~sure).sum())
        assert window <= max(1, len(sure) // 10000), f"{what}: {window} rows in the fp64 window"
    print(f"[parity] {what}: {len(out)} rows, max rel err "
          f"{float((err / np.maximum(np.abs(ref['out']), 1e-30)).max()):.3e}, "
          f"R3 window bound {bound:.2e}, rows in window {window}")


def _marked_trees_check(f, cid, Xd, X, calib, dev, trees_per_run=4, runs=2, seed=0):
    """Leaf ids of marked trees through the production kernel instantiation over all rows."""
    rng = np.random.default_rng(seed + cid)
    C = f["n_classes"]
    tc = f["tree_class"] if f.get("tree_class") is not None else np.arange(len(f["root"])) % C
    Fr = T.Forest(f, device=0).layout(calib)
    er = Fr.export_sliced()
    for run in range(runs):
        c = int(rng.integers(C)) if C > 1 else 0
        cand = np.flatnonzero(tc == c)
        trees = rng.choice(cand, size=min(trees_per_run, len(cand)), replace=False)
        lv = {int(t): _tree_leaves(f, int(t)) for t in trees}
        nmax = max(len(v) for v in lv.values())
        bits = int(np.ceil(np.log2(nmax + 2)))
        trees = trees[: max(1, 52 // bits)]
        g = dict(f)
        g["leaf_value"] = np.zeros_like(f["leaf_value"])
        for k, t in enumerate(trees):
            for o, node in enumerate(lv[int(t)]):
                g["leaf_value"][node] = np.float32((o + 1) * 2.0 ** (bits * k))
        G = T.Forest(g, device=0).layout(calib)
        eg = G.export_sliced()
        assert (er is None) == (eg is None)
        if er is not None:   # the layout does not depend on leaf values
            assert np.array_equal(er["leaf_meta"], eg["leaf_meta"])
            assert np.array_equal(er["nodes"][..., 1], eg["nodes"][..., 1])
            internal = er["leaf_meta"][..., 0] < 0
            assert np.array_equal(er["nodes"][..., 0][internal], eg["nodes"][..., 0][internal])
        assert G.select_strategy(X.shape[0], X.shape[1]) == Fr.select_strategy(X.shape[0], X.shape[1])
        part = G.predict_partial(Xd)
        torch.cuda.synchronize()
        v = part[:, c].cpu().numpy()
        assert np.array_equal(v, np.floor(v)), "marked sums are exact integers"
        vi = v.astype(np.int64)
        sub = dict(f, root=f["root"][trees], tree_class=np.zeros(len(trees), np.int32))
        ref = oracle.predict(sub, X, agg=oracle.AGG_SUM, n_classes=1, want_leaf=True)
        for k, t in enumerate(trees):
            ords = ((vi >> (bits * k)) & ((1 << bits) - 1)) - 1
            lut = np.full(len(f["feature"]), -1, np.int64)
            lut[lv[int(t)]] = np.arange(len(lv[int(t)]))
            assert np.array_equal(ords, lut[ref["leaf"][:, k]]), f"tree {t}: leaf ids differ"
        G.close()
        del part
    Fr.close()
    print(f"[parity] C{cid}: marked-tree leaf ids equal on all {X.shape[0]} rows ({runs} runs)")


def _sample_config(cid, parity_rows=None, marked=True):
    """Scores/classes on the parity set, fingerprints on all rows (checked on the parity set), leaf
    ids on the first 64K rows, marked-tree leaf ids on all rows."""
    cfg = gen.CONFIGS[cid]
    n = cfg.n_samples
    f = gen.make_forest(cid, leaf_mode="normal")
    calib = gen.make_calibration(cid)
    F = T.Forest(f, device=0).layout(calib)
    X = gen.make_rows(cid, n)
    dev = torch.device("cuda", 0)
    Xd = torch.from_numpy(X).to(dev)
    # the bench launch: the strategy the cost model picks for n rows, forced as bench.py does
    strat = F.select_strategy(n, cfg.n_features)
    out = torch.empty((n, F.n_out), dtype=torch.float32, device=dev)
    cls = torch.empty(n, dtype=torch.int32, device=dev)
    F.predict(Xd, out=out, out_class=cls, force_strategy=strat)
    fp = torch.empty(n, dtype=torch.int64, device=dev)
    F.predict(Xd, out=torch.empty_like(out), out_fingerprint=fp, force_strategy=strat)
    torch.cuda.synchronize()
    idx = np.arange(n) if parity_rows is None else gen.subsample(4000 + cid, n, parity_rows)
    ref = oracle.predict(f, X, rows=idx)
    _check_rows(out.cpu().numpy()[idx], cls.cpu().numpy()[idx], ref, f["agg"], margin_bound(f),
                f"C{cid} strategy {strat}")
    assert np.array_equal(fp.cpu().numpy().view(np.uint64)[idx], ref["fp"]), "fingerprints differ"
    del fp
    m = min(LEAF_ROWS, n)
    leaf = torch.full((m, F.n_trees), -1, dtype=torch.int32, device=dev)
    fpl = torch.empty(m, dtype=torch.int64, device=dev)
    o2 = torch.empty((m, F.n_out), dtype=torch.float32, device=dev)
    F.predict(Xd[:m], out=o2, out_leaf=leaf, out_fingerprint=fpl, force_strategy=strat)
    torch.cuda.synchronize()
    refl = oracle.predict(f, X[:m], want_leaf=True)
    assert np.array_equal(leaf.cpu().numpy(), refl["leaf"]), "leaf ids differ"
    assert np.array_equal(fpl.cpu().numpy().view(np.uint64), refl["fp"])
    del leaf
    if marked:
        _marked_trees_check(f, cid, Xd, X, calib, dev)
    F.close()
    del Xd


def test_fullsize_c2_all_rows():
    _sample_config(2)


def test_fullsize_c3_ten_percent():
    _sample_config(3, parity_rows=gen.CONFIGS[3].n_samples // 10)


def test_fullsize_c4_all_rows():
    _sample_config(4)


def test_fullsize_c5_one_percent_fused_reduce_and_shard_fingerprints():
    """C5 in bench.py's N=1 launch configuration: the full 4000-tree forest (direct image in
    L2-sized chunks) over all 10M rows through the fused reduce (world-1 NCCL communicator);
    scores on a seeded 1 % (100K rows); GPU fingerprints of all 10M rows checked on those rows;
    the 8 tree shards' fingerprints sum to the unsharded one on every row; marked-tree leaf ids
    from the production (chunked, non-fused) direct kernel on all rows."""
    cfg = gen.CONFIGS[5]
    n = cfg.n_samples
    f = gen.make_forest(5, leaf_mode="normal")
    calib = gen.make_calibration(5)
    full = T.Forest(f, device=-1).layout(calib)
    S = full.shard(0, 1, device=0)
    assert S.stats()["direct_chunks"] > 1
    try:
        comm = T.Comm(T.tahoe_comm_unique_id(), 1, 0, 0)
    except T.TahoeError as e:  # pragma: no cover
        pytest.skip(f"NCCL device API unavailable: {e}")
    X = gen.make_rows(5, n)
    dev = torch.device("cuda", 0)
    Xd = torch.from_numpy(X).to(dev)
    out = S.predict_reduce(comm, Xd, mode=T.REDUCE_ALL)
    fp = torch.empty(n, dtype=torch.int64, device=dev)
    S.predict(Xd, out=torch.empty((n, 1), dtype=torch.float32, device=dev), out_fingerprint=fp)
    torch.cuda.synchronize()
    idx = gen.subsample(4005, n, n // 100)
    ref = oracle.predict(f, X, rows=idx)
    _check_rows(out.cpu().numpy()[idx], np.zeros(len(idx), np.int32), ref, f["agg"],
                margin_bound(f), "C5 full forest, fused reduce")
    fph = fp.cpu().numpy().view(np.uint64)
    assert np.array_equal(fph[idx], ref["fp"]), "fingerprints differ"
    tot = torch.zeros(n, dtype=torch.int64, device=dev)
    shard_fp = torch.empty(n, dtype=torch.int64, device=dev)
    o = torch.empty((n, 1), dtype=torch.float32, device=dev)
    for r in range(8):
        Sr = full.shard(r, 8, device=0)
        Sr.predict(Xd, out=o, out_fingerprint=shard_fp)
        tot += shard_fp          # int64 adds wrap: the sum mod 2^64
        Sr.close()
    torch.cuda.synchronize()
    assert np.array_equal(tot.cpu().numpy().view(np.uint64), fph), "shard fingerprints must sum to the full one"
    comm.close()
    del out, o, tot, shard_fp, fp
    # marked trees through the production direct kernel (chunked image, eight threads per row)
    _marked_trees_check_direct(f, full, Xd, X, calib)
    S.close()


def _marked_trees_check_direct(f, full, Xd, X, calib, runs=2):
    rng = np.random.default_rng(55)
    for run in range(runs):
        trees = rng.choice(len(f["root"]), size=4, replace=False)
        lv = {int(t): _tree_leaves(f, int(t)) for t in trees}
        bits = int(np.ceil(np.log2(max(len(v) for v in lv.values()) + 2)))
        trees = trees[: max(1, 52 // bits)]
        g = dict(f)
        g["leaf_value"] = np.zeros_like(f["leaf_value"])
        for k, t in enumerate(trees):
            for o, node in enumerate(lv[int(t)]):
                g["leaf_value"][node] = np.float32((o + 1) * 2.0 ** (bits * k))
        G = T.Forest(g, device=-1).layout(calib).shard(0, 1, device=0)
        assert G.stats()["direct_chunks"] > 1
        part = G.predict_partial(Xd)
        torch.cuda.synchronize()
        v = part[:, 0].cpu().numpy()
        assert np.array_equal(v, np.floor(v))
        vi = v.astype(np.int64)
        sub = dict(f, root=f["root"][trees], tree_class=np.zeros(len(trees), np.int32))
        ref = oracle.predict(sub, X, agg=oracle.AGG_SUM, n_classes=1, want_leaf=True)
        for k, t in enumerate(trees):
            ords = ((vi >> (bits * k)) & ((1 << bits) - 1)) - 1
            lut = np.full(len(f["feature"]), -1, np.int64)
            lut[lv[int(t)]] = np.arange(len(lv[int(t)]))
            assert np.array_equal(ords, lut[ref["leaf"][:, k]]), f"tree {t}: leaf ids differ"
        G.close()
        del part
    print(f"[parity] C5: marked-tree leaf ids equal on all {X.shape[0]} rows ({runs} runs)")
