"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the same seeded inputs.

Bars (BASELINE.json north_star):
  * leaf ids (caller node ids, n x T) and fingerprints: bit-exact;
  * classes: bit-exact (dyadic runs) / exact wherever the fp64 decision margin exceeds the fp64
    rounding bound (random-leaf runs);
  * scores: bit-exact with dyadic leaves; |gpu - ref| <= max(1e-5 |ref|, 1e-6) with N(0, 0.1) leaves.
Every strategy is forced in turn; sizes span many tiles and a ragged tail.
"""
import numpy as np
import pytest

import gen
import oracle
from tlib import margin_bound

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402

STRATS = [T.STRATEGY_DIRECT, T.STRATEGY_SLICED, T.STRATEGY_SLICED_CODED, T.STRATEGY_ROWS]


def _usable(F, s):
    st = F.stats()
    if s == T.STRATEGY_ROWS:
        return st["rows_ok"]
    if s == T.STRATEGY_SLICED:
        return st["sliced_valid"]
    if s == T.STRATEGY_SLICED_CODED:
        return st["sliced_valid"] and st["coded_valid"]
    return True


def _strats(F):
    return [s for s in STRATS if _usable(F, s)]


def _gpu_run(F, X, strategy, want_leaf=True):
    """Predict through the C ABI with `strategy` forced (leaf ids and fingerprints come from the
    LEAF instantiation of the strategy's kernel)."""
    dev = torch.device("cuda", 0)
    Xd = torch.from_numpy(X).to(dev)
    n = X.shape[0]
    out = torch.empty((n, F.n_out), dtype=torch.float32, device=dev)
    cls = torch.full((n,), -7, dtype=torch.int32, device=dev)
    leaf = torch.full((n, F.n_trees), -7, dtype=torch.int32, device=dev) if want_leaf else None
    fp = torch.empty(n, dtype=torch.int64, device=dev) if want_leaf else None
    F.predict(Xd, out=out, out_class=cls, out_leaf=leaf, out_fingerprint=fp, force_strategy=strategy)
    torch.cuda.synchronize()
    res = dict(out=out.cpu().numpy(), cls=cls.cpu().numpy())
    if want_leaf:
        res["leaf"] = leaf.cpu().numpy()
        res["fp"] = fp.cpu().numpy().view(np.uint64)
    return res


def _check(res, ref, agg, exact, want_leaf=True, bound=None):
    """Compare GPU results with the oracle's; returns the number of rows whose class decision lies
    inside the fp64 rounding window (reading R3; `bound` from tlib.margin_bound, either class
    accepted there)."""
    if want_leaf and "leaf" in res:
        assert np.array_equal(res["leaf"], ref["leaf"]), "leaf ids differ"
        assert np.array_equal(res["fp"], ref["fp"]), "fingerprints differ"
    window = 0
    if exact:
        assert np.array_equal(res["out"], ref["out"]), "dyadic scores must be bit-exact"
        if agg in (oracle.AGG_BINARY, oracle.AGG_CLASS_SUM, oracle.AGG_VOTE):
            assert np.array_equal(res["cls"], ref["cls"])
    else:
        tol = np.maximum(1e-5 * np.abs(ref["out"]), 1e-6)
        assert (np.abs(res["out"] - ref["out"]) <= tol).all(), \
            f"max err {np.abs(res['out'] - ref['out']).max()}"
        assert bound is not None, "random-leaf class checks need the fp64 window"
        if agg == oracle.AGG_BINARY:
            sure = np.abs(ref["raw"][:, 0]) > bound
        elif agg == oracle.AGG_CLASS_SUM:
            srt = np.sort(ref["raw"], axis=1)
            sure = (srt[:, -1] - srt[:, -2]) > bound
        else:
            sure = np.ones(len(ref["cls"]), bool)
        if agg in (oracle.AGG_BINARY, oracle.AGG_CLASS_SUM):
            assert np.array_equal(res["cls"][sure], ref["cls"][sure])
            window = int((~sure).sum())
    return window


CASES = [  # (config, n_trees override, n rows, leaf mode)
    (1, None, 1000, "dyadic"),
    (1, None, 1000, "normal"),
    (2, None, 20011, "dyadic"),
    (2, None, 6007, "normal"),
    (3, None, 8009, "dyadic"),
    (4, 200, 3001, "dyadic"),
]


@pytest.mark.parametrize("cid,ntrees,n,mode", CASES)
@pytest.mark.parametrize("layout", [False, True])
def test_parity_configs(cid, ntrees, n, mode, layout):
    f = gen.make_forest(cid, n_trees=ntrees, leaf_mode=mode)
    X = gen.make_rows(cid, n)
    F = T.Forest(f, device=0)
    if layout:
        F.layout(gen.make_calibration(cid, 4096))
    ref = oracle.predict(f, X, want_leaf=True)
    for s in _strats(F):
        _check(_gpu_run(F, X, s), ref, f["agg"], mode == "dyadic", bound=margin_bound(f))


def test_parity_c4_full_forest_subsample():
    f = gen.make_forest(4)
    X = gen.make_rows(4, 2003)
    F = T.Forest(f, device=0).layout(gen.make_calibration(4, 4096))
    ref = oracle.predict(f, X, want_leaf=True)
    for s in _strats(F):
        _check(_gpu_run(F, X, s), ref, f["agg"], True)


def test_parity_c5_subsample_direct_and_shards():
    f = gen.make_forest(5, n_trees=600)
    X = gen.make_rows(5, 1500)
    F = T.Forest(f, device=0).layout(gen.make_calibration(5, 8192))
    ref = oracle.predict(f, X, want_leaf=True)
    _check(_gpu_run(F, X, -1), ref, f["agg"], True)
    # fake multi-rank tree sharding on one GPU: sum of shard partials -> finalize == full
    dev = torch.device("cuda", 0)
    Xd = torch.from_numpy(X).to(dev)
    tot = torch.zeros((X.shape[0], 1), dtype=torch.float64, device=dev)
    for r in range(4):
        S = F.shard(r, 4)
        tot += S.predict_partial(Xd)
    out = F.finalize(tot)
    assert np.array_equal(out.cpu().numpy(), ref["out"])


def test_edge_cases_nan_misaligned_wide_d_and_tiny_batches():
    f = gen.make_forest(2, n_trees=64)
    F = T.Forest(f, device=0).layout(gen.make_calibration(2, 2048))
    X = gen.make_rows(2, 4099)
    X[::5, 3] = np.nan
    X[::11, :] = np.nan
    ref = oracle.predict(f, X, want_leaf=True)
    for s in _strats(F):
        _check(_gpu_run(F, X, s), ref, f["agg"], True)
    # misaligned X (offset by one float => no TMA) and wider rows than the forest needs
    dev = torch.device("cuda", 0)
    Xw = np.concatenate([X, np.full((X.shape[0], 5), 9.0, np.float32)], axis=1)
    buf = torch.empty(Xw.size + 1, dtype=torch.float32, device=dev)
    buf[1:] = torch.from_numpy(Xw.ravel()).to(dev)
    Xm = buf[1:].view(Xw.shape)
    for s in _strats(F):
        out = torch.empty((X.shape[0], 1), dtype=torch.float32, device=dev)
        F.predict(Xm, out=out, force_strategy=s)
        torch.cuda.synchronize()
        assert np.array_equal(out.cpu().numpy(), ref["out"])
    for n in (0, 1, 31, 33, 64, 65):
        for s in _strats(F):
            Xd = torch.from_numpy(X[:n].copy()).to(dev)
            out = torch.full((n, 1), -1.0, dtype=torch.float32, device=dev)
            F.predict(Xd, out=out, force_strategy=s)
            torch.cuda.synchronize()
            assert np.array_equal(out.cpu().numpy(), ref["out"][:n])


def test_aggregations_average_base_vote():
    from test_oracle_pins import random_forest
    rng = np.random.default_rng(21)
    f = random_forest(rng, 45, 6, 5)
    X = rng.normal(size=(3001, 5)).astype(np.float32)
    for agg, base in ((oracle.AGG_AVERAGE, 0.625), (oracle.AGG_SUM, -2.0), (oracle.AGG_BINARY, 0.25)):
        F = T.Forest(f, n_features=5, n_classes=1, agg=agg, base_score=base, device=0)
        ref = oracle.predict(f, X, agg=agg, base_score=base, want_leaf=True)
        for s in _strats(F):
            _check(_gpu_run(F, X, s), ref, agg, True)
    C = 4
    fv = random_forest(rng, 40, 5, 5, n_classes=C, vote=True)
    F = T.Forest(fv, n_features=5, n_classes=C, agg=oracle.AGG_VOTE, device=0)
    ref = oracle.predict(fv, X, agg=oracle.AGG_VOTE, n_classes=C, want_leaf=True)
    _check(_gpu_run(F, X, -1), ref, oracle.AGG_VOTE, True)


def test_layout_never_changes_results():
    f = gen.make_forest(3, n_trees=140)
    X = gen.make_rows(3, 3000)
    ref = oracle.predict(f, X, want_leaf=True)
    F = T.Forest(f, device=0)
    outs = []
    for kw in (dict(), dict(node_reorder=0, tree_group=0), dict(node_reorder=1, tree_group=0),
               dict(t_nodes=2, l_hash=64, m_chunks=16)):
        F.layout(gen.make_calibration(3, 3000), **kw)
        for s in _strats(F):
            r = _gpu_run(F, X, s)
            _check(r, ref, f["agg"], True)
            outs.append(r["out"])
    assert all(np.array_equal(o, outs[0]) for o in outs)


def test_predict_host_end_to_end():
    f = gen.make_forest(2, n_trees=100)
    F = T.Forest(f, device=0).layout(gen.make_calibration(2, 2048))
    X = gen.make_rows(2, 300_001)
    Xh = torch.from_numpy(X).pin_memory()
    out = torch.empty((X.shape[0], 1), dtype=torch.float32).pin_memory()
    cls = torch.empty(X.shape[0], dtype=torch.int32).pin_memory()
    F.predict_host(Xh, out, cls)
    torch.cuda.synchronize()
    idx = gen.subsample(5, X.shape[0], 3000)
    ref = oracle.predict(f, X, rows=idx)
    assert np.array_equal(out.numpy()[idx], ref["out"])
    assert np.array_equal(cls.numpy()[idx], ref["cls"])


def test_single_leaf_trees_and_stumps():
    """Trees whose root is a leaf (encoded as a 3-node stump in the sliced image) mixed with
    ordinary trees: consecutive nonzero leaves must still be summed exactly."""
    from test_oracle_pins import random_forest
    rng = np.random.default_rng(8)
    base = random_forest(rng, 40, 4, 6)
    nn = len(base["feature"])
    k = 25
    f = {kk: np.concatenate([base[kk], v]).astype(base[kk].dtype) for kk, v in dict(
        feature=np.full(k, -1), threshold=np.zeros(k), left=np.full(k, -1), right=np.full(k, -1),
        leaf_value=(rng.integers(-256, 257, size=k) / 256.0),
        default_left=np.zeros(k)).items()}
    order = rng.permutation(40 + k)
    roots = np.concatenate([base["root"], np.arange(nn, nn + k, dtype=np.int32)])[order]
    f["root"] = roots.astype(np.int32)
    f["tree_class"] = np.zeros(len(roots), np.int32)
    X = rng.normal(size=(2049, 6)).astype(np.float32)
    ref = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1, want_leaf=True)
    F = T.Forest(f, n_features=6, n_classes=1, agg=oracle.AGG_SUM, device=0)
    for s in _strats(F):
        _check(_gpu_run(F, X, s), ref, oracle.AGG_SUM, True)


def test_gpu_visit_counts_equal_oracle_and_drive_layout():
    """Algorithm 1 line 16: visit counts measured by the GPU equal the oracle's path counts, and a
    layout driven by them equals the host-calibrated layout."""
    f = gen.make_forest(3, n_trees=120)
    Xc = gen.make_calibration(3, 5000)
    Xc[::97, 5] = np.nan
    F = T.Forest(f, device=0)
    dev = torch.device("cuda", 0)
    cnt = F.layout_gpu(torch.from_numpy(Xc).to(dev))
    assert np.array_equal(cnt, oracle.node_counts(f, Xc))
    G = T.Forest(f, device=0).layout(Xc)
    ia = T.tahoe_forest_layout_info(F.handle, len(f["feature"]), F.n_trees)
    ib = T.tahoe_forest_layout_info(G.handle, len(f["feature"]), G.n_trees)
    for k in ("count", "hot_left", "order"):
        assert np.array_equal(ia[k], ib[k]), k
    X = gen.make_rows(3, 2000)
    ref = oracle.predict(f, X, want_leaf=True)
    for s in _strats(F):
        _check(_gpu_run(F, X, s), ref, f["agg"], True)


def test_direct_chunked_image_parity(monkeypatch):
    """Reading R4: a direct image walked in L2-sized chunks of trees (one launch per chunk, fp64
    partials accumulated in chunk order) gives the same leaves, fingerprints, classes and dyadic
    scores as the oracle; chunk size forced small through TAHOE_DIRECT_CHUNK_KB at build time."""
    monkeypatch.setenv("TAHOE_DIRECT_CHUNK_KB", "64")
    for cid, ntrees, nrows in ((3, 280, 2500), (5, 120, 700)):
        f = gen.make_forest(cid, n_trees=ntrees)
        F = T.Forest(f, device=0).layout(gen.make_calibration(cid, 4096))
        assert F.stats()["direct_chunks"] > 1
        X = gen.make_rows(cid, nrows)
        X[::9, 2] = np.nan
        ref = oracle.predict(f, X, want_leaf=True)
        _check(_gpu_run(F, X, T.STRATEGY_DIRECT), ref, f["agg"], True)
        res = _gpu_run(F, X, T.STRATEGY_DIRECT, want_leaf=False)   # fused-finalize path
        _check(res, ref, f["agg"], True, want_leaf=False)
        F.close()


@pytest.mark.parametrize("cid,ntrees,variant", [(2, 120, None), (5, 60, None), (2, 120, "4"),
                                                (5, 60, "2"), (5, 60, "1"), (5, 60, "3"),
                                                (2, 120, "6"), (5, 60, "7"), (5, 60, "8"),
                                                (2, 120, "9"), (5, 60, "10"), (2, 120, "11")])
def test_direct_large_batch_variants(cid, ntrees, variant, monkeypatch):
    """Large-batch direct kernels (staged rows; 2, 4, 8 (default) or 16 threads per row for scalar
    outputs, one thread per row free-running or warp-lockstep; the measured-and-rejected tree-head
    (8, 9) and node-group (10, 11) experiments) against the oracle, scores and classes bit-exact with
    dyadic leaves, >= 32K rows with a ragged last tile."""
    if variant is not None:
        monkeypatch.setenv("TAHOE_DIRECT_VARIANT", variant)
    f = gen.make_forest(cid, n_trees=ntrees)
    F = T.Forest(f, base_score=0.5, device=0).layout(gen.make_calibration(cid, 4096))
    n = 40_001
    X = gen.make_rows(cid, n)
    X[::7, 3] = np.nan
    ref = oracle.predict(f, X, base_score=0.5)
    _check(_gpu_run(F, X, T.STRATEGY_DIRECT, want_leaf=False), ref, f["agg"], True, want_leaf=False)
    dev = torch.device("cuda", 0)
    part = F.predict_partial(torch.from_numpy(X).to(dev))   # raw path (no fused finalize)
    torch.cuda.synchronize()
    # partials carry no base score; the oracle's raw margin does (dyadic: both exact)
    assert np.array_equal(part.cpu().numpy(), ref["raw"] - 0.5), "dyadic partial sums are exact"
    F.close()


def test_rank_codes_threshold_ties_signed_zero_inf_nan():
    """Reading R7: the rank-coded slices decide "x < b" exactly.  Rows are built from the forest's
    own thresholds (x == b goes right), their float neighbours, -0.0 / +0.0, +-Inf and NaN (default
    path from the node's default_left); a threshold of 0.0 is planted so signed zeros meet it.
    Scores and classes are bit-exact against the oracle (dyadic leaves), and equal the fp32
    slices and the direct strategy."""
    rng = np.random.default_rng(77)
    f = gen.make_forest(2, n_trees=96)
    f = {k: (v.copy() if isinstance(v, np.ndarray) else v) for k, v in f.items()}
    internal = np.flatnonzero(f["feature"] >= 0)
    f["threshold"][internal[::17]] = 0.0
    f["threshold"][internal[5::41]] = -0.0
    f["default_left"][:] = rng.integers(0, 2, size=len(f["default_left"]))
    F = T.Forest(f, device=0).layout(gen.make_calibration(2, 4096))
    assert F.stats()["coded_valid"], F.stats()["coded_why"]
    n, d = 9001, f["n_features"]
    X = gen.make_rows(2, n)
    thr_by_feat = [f["threshold"][internal[f["feature"][internal] == j]] for j in range(d)]
    pick = rng.random(X.shape)
    for j in range(d):
        t = thr_by_feat[j]
        if len(t) == 0:
            continue
        m = pick[:, j] < 0.35
        v = rng.choice(t, size=m.sum())
        kind = rng.integers(0, 3, size=m.sum())
        v = np.where(kind == 1, np.nextafter(v, np.float32(np.inf)), v)
        v = np.where(kind == 2, np.nextafter(v, np.float32(-np.inf)), v)
        X[m, j] = v.astype(np.float32)
    X[pick > 0.97] = -0.0
    X[(pick > 0.95) & (pick <= 0.97)] = 0.0
    X[(pick > 0.94) & (pick <= 0.95)] = np.inf
    X[(pick > 0.93) & (pick <= 0.94)] = -np.inf
    X[(pick > 0.92) & (pick <= 0.93)] = np.nan
    ref = oracle.predict(f, X, want_leaf=True)
    outs = []
    for s in _strats(F):
        r = _gpu_run(F, X, s)
        _check(r, ref, f["agg"], True)
        outs.append(r["out"])
    assert len(outs) == 4 and all(np.array_equal(o, outs[0]) for o in outs)


def test_rank_codes_eligibility_and_auto_choice():
    """The coded twin exists when the forest qualifies (<= 127 attributes, no subnormal leaf),
    gives leaf ids / fingerprints through its LEAF instantiation, and is refused (E_UNSUPPORTED)
    when forced on a forest that does not qualify."""
    f = gen.make_forest(2, n_trees=32)
    F = T.Forest(f, device=0)
    assert F.stats()["coded_valid"]
    X = torch.from_numpy(gen.make_rows(2, 100)).cuda()
    out = torch.empty((100, 1), dtype=torch.float32, device="cuda")
    leaf = torch.empty((100, F.n_trees), dtype=torch.int32, device="cuda")
    F.predict(X, out=out, out_leaf=leaf, force_strategy=T.STRATEGY_SLICED_CODED)
    torch.cuda.synchronize()
    r0 = oracle.predict(f, X.cpu().numpy(), want_leaf=True)
    assert np.array_equal(leaf.cpu().numpy(), r0["leaf"])
    g = {k: (v.copy() if isinstance(v, np.ndarray) else v) for k, v in f.items()}
    leaves = np.flatnonzero(g["feature"] < 0)
    g["leaf_value"][leaves[3]] = np.float32(1e-40)   # subnormal leaf value
    G = T.Forest(g, device=0)
    assert not G.stats()["coded_valid"]
    with pytest.raises(T.TahoeError):
        G.predict(X, out=out, force_strategy=T.STRATEGY_SLICED_CODED)
    ref = oracle.predict(g, X.cpu().numpy())
    G.predict(X, out=out)                                  # auto: fp32 slices or direct
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), ref["out"])


@pytest.mark.parametrize("banks", ["1", "0"])
@pytest.mark.parametrize("cid,ntrees,n", [(2, 120, 30011), (3, 210, 20011), (1, None, 1000)])
def test_rank_code_prepass_kernels(cid, ntrees, n, banks, monkeypatch):
    """Both row-coding pre-passes (bank-private tables in shared memory; bisection through L2) feed
    the coded slices the same codes: scores and classes bit-exact against the oracle with NaN rows
    and a ragged last tile."""
    monkeypatch.setenv("TAHOE_CODE_BANKS", banks)
    f = gen.make_forest(cid, n_trees=ntrees)
    F = T.Forest(f, device=0).layout(gen.make_calibration(cid, 4096))
    st = F.stats()
    assert st["coded_valid"] and st["code_bank_rows"] > 0
    X = gen.make_rows(cid, n)
    X[::13, 1] = np.nan
    ref = oracle.predict(f, X)
    _check(_gpu_run(F, X, T.STRATEGY_SLICED_CODED, want_leaf=False), ref, f["agg"], True,
           want_leaf=False)


def test_rank_codes_multislice_classes_and_partials(monkeypatch):
    """Multi-slice, multi-class coded launches (partials staged in shared memory, written by the
    warp closing each tile, combined per class in slice order): CLASS_SUM scores and argmax
    bit-exact with dyadic leaves, and the raw per-class partials (tahoe_predict_partial, no base)
    exact too."""
    monkeypatch.setenv("TAHOE_FORCE_STRATEGY", "2")
    f = gen.make_forest(3, n_trees=280)
    F = T.Forest(f, base_score=0.25, device=0).layout(gen.make_calibration(3, 4096))
    st = F.stats()
    assert st["coded_valid"] and st["n_slices"] > 1
    n = 50_003
    X = gen.make_rows(3, n)
    X[::29, 4] = np.nan
    ref = oracle.predict(f, X, base_score=0.25, want_leaf=True)
    res = _gpu_run(F, X, -1, want_leaf=False)
    _check(res, ref, f["agg"], True, want_leaf=False)
    _check(_gpu_run(F, X, -1), ref, f["agg"], True)   # LEAF instantiation, same launch plan
    part = F.predict_partial(torch.from_numpy(X).cuda())
    torch.cuda.synchronize()
    assert np.array_equal(part.cpu().numpy(), ref["raw"] - 0.25), "dyadic partial sums are exact"


@pytest.mark.parametrize("d", [3, 15, 31, 100, 127])
def test_rank_codes_row_widths(d, monkeypatch):
    """Every code-row geometry: 3-15 attributes (64-byte rows, one pass), 31 (64-byte rows, all 32
    slots used, the pad slot is the leaf's), 100 and 127 attributes (256-byte rows, four 32-lane
    passes of the pre-pass; 127 leaves a single pad slot).  Thresholds on a coarse grid make
    x == b frequent.  Dyadic scores bit-exact against the oracle through both pre-passes."""
    from test_oracle_pins import random_forest
    rng = np.random.default_rng(d)
    grid = np.linspace(-2.0, 2.0, 41)
    f = random_forest(rng, 48, 6, d, thr_grid=grid)
    # 20011 rows = 313 code tiles: every CTA of a one-slice forest walks several tiles, so every
    # ring buffer is used (256-byte rows once misaligned the second buffer's row base)
    X = rng.normal(size=(20011, d)).astype(np.float32)
    X[rng.random(X.shape) < 0.3] = rng.choice(grid, size=1)[0]
    X[::37, 0] = np.nan
    F = T.Forest(f, n_features=d, n_classes=1, agg=oracle.AGG_SUM, device=0)
    st = F.stats()
    assert st["sliced_valid"] and st["coded_valid"], st["coded_why"]
    ref = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1)
    for banks in ("1", "0"):
        monkeypatch.setenv("TAHOE_CODE_BANKS", banks)
        _check(_gpu_run(F, X, T.STRATEGY_SLICED_CODED, want_leaf=False), ref, oracle.AGG_SUM, True,
               want_leaf=False)


def test_fingerprint_without_leaf_array_every_strategy():
    """out_fingerprint alone (out_leaf NULL) through every strategy, single and multi-slice,
    direct image chunked or not: fingerprints equal the oracle's."""
    for cid, nt, chunk in ((2, 300, None), (3, 280, None), (5, 80, "64")):
        import os
        if chunk:
            os.environ["TAHOE_DIRECT_CHUNK_KB"] = chunk
        try:
            f = gen.make_forest(cid, n_trees=nt)
            F = T.Forest(f, device=0).layout(gen.make_calibration(cid, 4096))
        finally:
            os.environ.pop("TAHOE_DIRECT_CHUNK_KB", None)
        X = gen.make_rows(cid, 40_003)
        ref = oracle.predict(f, X)
        dev = torch.device("cuda", 0)
        Xd = torch.from_numpy(X).to(dev)
        for s in _strats(F):
            fp = torch.empty(X.shape[0], dtype=torch.int64, device=dev)
            out = torch.empty((X.shape[0], F.n_out), dtype=torch.float32, device=dev)
            F.predict(Xd, out=out, out_fingerprint=fp, force_strategy=s)
            torch.cuda.synchronize()
            assert np.array_equal(fp.cpu().numpy().view(np.uint64), ref["fp"]), (cid, s)
            assert np.array_equal(out.cpu().numpy(), ref["out"]), (cid, s)
        F.close()
