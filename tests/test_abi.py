"""C-ABI tests that need no GPU: the library loads and exports every symbol include/tahoe.h
declares; tahoe_forest_build's validation codes; host-only handles; and the layout introspection
hooks against the layout oracle (Fig. 1 / Fig. 3 of the paper)."""
import ctypes
import hashlib
import json
import os
import re

import numpy as np
import pytest

import gen
import oracle
from oracle import layout_oracle as lo
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
from tlib import GOLDEN, ROOT


def test_library_exports_every_header_symbol():
    hdr = open(os.path.join(ROOT, "include", "tahoe.h")).read()
    names = set(re.findall(r"\b(tahoe_[a-z0-9_]+)\s*\(", hdr))
    assert len(names) >= 20
    L = T.load()
    for nm in sorted(names):
        assert hasattr(L, nm), nm
    assert names == set(T.SYMBOLS)


def _stump_arrays():
    return dict(root=np.array([0], np.int32), feature=np.array([0, -1, -1], np.int32),
                threshold=np.array([0.5, 0, 0], np.float32), left=np.array([1, -1, -1], np.int32),
                right=np.array([2, -1, -1], np.int32),
                leaf_value=np.array([0, 1.0, 2.0], np.float32))


def _build(arrs, n_features=1, n_classes=1, agg=T.AGG_SUM):
    return T.tahoe_forest_build(arrs, n_features, n_classes, agg, 0.0, -1)


def test_build_ok_and_host_only_predict_is_state_error():
    h = _build(_stump_arrays())
    assert T.tahoe_forest_n_outputs(h) == 1 and T.tahoe_forest_n_trees(h) == 1
    L = T.load()
    st = L.tahoe_predict(h, ctypes.c_void_p(16), 1, 1, ctypes.c_void_p(16), None)
    assert st == T.TAHOE_E_STATE
    assert L.tahoe_predict(h, None, 0, 1, None, None) == T.TAHOE_E_STATE
    T.tahoe_forest_free(h)


def test_fused_reduce_host_validation():
    """f4 boundary: row split, argument errors and host-only handles (no GPU needed)."""
    L = T.load()
    for n, w in ((0, 1), (1, 3), (10, 3), (1001, 8), (2**40 + 3, 7)):
        cover = 0
        prev = 0
        for r in range(w):
            lo, hi = T.tahoe_reduce_rows(n, w, r, T.REDUCE_SCATTER)
            assert lo == prev and hi >= lo and hi - lo in (n // w, n // w + 1)
            prev, cover = hi, cover + hi - lo
        assert prev == n and cover == n
    lo, hi = ctypes.c_int64(), ctypes.c_int64()
    assert L.tahoe_reduce_rows(10, 2, 2, 0, ctypes.byref(lo), ctypes.byref(hi)) == T.TAHOE_E_INVAL
    assert L.tahoe_reduce_rows(10, 0, 0, 0, ctypes.byref(lo), ctypes.byref(hi)) == T.TAHOE_E_INVAL
    assert L.tahoe_reduce_rows(10, 2, 0, 7, ctypes.byref(lo), ctypes.byref(hi)) == T.TAHOE_E_INVAL
    assert L.tahoe_reduce_rows(-1, 2, 0, 0, ctypes.byref(lo), ctypes.byref(hi)) == T.TAHOE_E_INVAL
    h = _build(_stump_arrays())
    arr = (ctypes.c_void_p * 1)(16)
    assert L.tahoe_reduce_partials(h, arr, 1, 0, 0, 4, ctypes.c_void_p(16), None, None) == T.TAHOE_E_STATE
    assert L.tahoe_predict_reduce(h, None, None, 4, 1, 0, None, None, None) == T.TAHOE_E_INVAL
    c = ctypes.c_void_p()
    buf = (ctypes.c_uint8 * 128)()
    assert L.tahoe_comm_init(buf, 2, 2, 0, ctypes.byref(c)) == T.TAHOE_E_INVAL
    assert L.tahoe_comm_init(None, 1, 0, 0, ctypes.byref(c)) == T.TAHOE_E_INVAL
    L.tahoe_comm_free(None)
    T.tahoe_forest_free(h)


@pytest.mark.parametrize("mutate,msg", [
    (lambda a: a.update(feature=np.array([3, -1, -1], np.int32)), "n_features"),
    (lambda a: a.update(left=np.array([7, -1, -1], np.int32)), "out of range"),
    (lambda a: a.update(left=np.array([2, -1, -1], np.int32)), "reachable twice"),
    (lambda a: a.update(left=np.array([0, -1, -1], np.int32)), "reachable twice"),
    (lambda a: a.update(threshold=np.array([np.nan, 0, 0], np.float32)), "NaN threshold"),
    (lambda a: a.update(root=np.array([5], np.int32)), "out of range"),
])
def test_build_validation_errors(mutate, msg):
    a = _stump_arrays()
    mutate(a)
    with pytest.raises(T.TahoeError) as e:
        _build(a)
    assert e.value.status == T.TAHOE_E_INVAL and msg in str(e.value)


def test_build_vote_and_class_validation():
    a = _stump_arrays()
    with pytest.raises(T.TahoeError) as e:
        _build(dict(a, leaf_value=np.array([0, 0.5, 1], np.float32)), n_classes=2, agg=T.AGG_VOTE)
    assert e.value.status == T.TAHOE_E_INVAL
    with pytest.raises(T.TahoeError):
        _build(dict(a, tree_class=np.array([3], np.int32)), n_classes=2, agg=T.AGG_CLASS_SUM)
    with pytest.raises(T.TahoeError):
        T.tahoe_forest_build(a, 1, 0, T.AGG_SUM, 0.0, -1)
    h = _build(dict(a, leaf_value=np.array([0, 1, 0], np.float32)), n_classes=2, agg=T.AGG_VOTE)
    assert T.tahoe_forest_n_outputs(h) == 2
    T.tahoe_forest_free(h)


def test_unreachable_nodes_ignored():
    a = _stump_arrays()
    a = {k: np.concatenate([v, v[:1]]) if k != "root" else v for k, v in a.items()}
    a["left"][3] = 99  # garbage in an unreachable node
    h = _build(a)
    assert T.tahoe_forest_stats(h)["nodes"] == 3
    T.tahoe_forest_free(h)


def test_sha1_matches_hashlib():
    for m in [b"", b"abc", bytes(range(200)), b"\x00" * 64, b"tahoe" * 33]:
        assert T.tahoe_sha1(m) == hashlib.sha1(m).digest()


def test_product_simhash_and_lsh_reproduce_fig3():
    g = json.load(open(os.path.join(GOLDEN, "fig3_simhash.json")))
    cs, bits = T.tahoe_simhash(np.array(g["strings"]), np.array(g["weights"]))
    assert np.allclose(cs, g["checksum"], atol=1e-12) and bits.tolist() == g["normalized"]
    reps = np.array([g["reps"][k] for k in ("T1", "T2", "T3")], np.uint8)
    col, order = T.tahoe_lsh_order(reps, g["m_chunks"])
    assert col[0, 1] == 0 and col[1, 2] == 2 and col[0, 2] == 1
    assert ["T1", "T2", "T3"][order[0]] == "T2" and list(order) == [1, 2, 0]


def test_product_lsh_order_equals_oracle_random():
    rng = np.random.default_rng(4)
    for T_ in (5, 17, 60):
        bits = (rng.random((T_, 32)) < 0.5).astype(np.uint8)
        col, order = T.tahoe_lsh_order(bits, 8)
        ocol = lo.lsh_collisions(bits, 8)
        assert np.array_equal(col, ocol)
        assert list(order) == lo.lsh_order(ocol)


def _fig1_product_forest():
    """Fig. 1's three trees with one attribute per internal node, and 100 calibration rows that
    reproduce the edge counts of tests/golden/fig1_reorg.json."""
    g = json.load(open(os.path.join(GOLDEN, "fig1_reorg.json")))
    names = ["V11", "V12", "V13", "V14", "V15", "V16", "V17", "V21", "V22", "V23", "V24", "V25",
             "V31", "V32", "V33", "V34", "V35"]
    idx = {n: i for i, n in enumerate(names)}
    feat_of = {"V11": 0, "V12": 1, "V13": 2, "V21": 7, "V23": 8, "V31": 9, "V32": 10}
    adj = {}
    for t in g["trees"]:
        adj.update({k: v for k, v in t.items() if k != "_root"})
    N = len(names)
    a = dict(root=np.array([0, 7, 12], np.int32), feature=np.full(N, -1, np.int32),
             threshold=np.zeros(N, np.float32), left=np.full(N, -1, np.int32),
             right=np.full(N, -1, np.int32), leaf_value=np.arange(N, dtype=np.float32) / 4)
    for n, (l, r) in adj.items():
        a["feature"][idx[n]] = feat_of[n]
        a["threshold"][idx[n]] = 0.5
        a["left"][idx[n]] = idx[l]
        a["right"][idx[n]] = idx[r]
    X = np.ones((100, 11), np.float32)
    X[:80, 0] = 0; X[:48, 1] = 0; X[80:86, 2] = 0
    X[:30, 7] = 0; X[30:50, 8] = 0; X[:, 9] = 0; X[:, 10] = 0
    return g, names, idx, a, X


def test_product_layout_matches_fig1_fig3_and_oracle():
    g, names, idx, a, X = _fig1_product_forest()
    h = T.tahoe_forest_build(a, 11, 1, T.AGG_SUM, 0.0, -1)
    T.tahoe_forest_layout(h, X)
    info = T.tahoe_forest_layout_info(h, len(names), 3)
    cnt = oracle.node_counts(a, X)
    assert np.array_equal(info["count"], cnt)
    for e, c in g["edge_counts_after_training"].items():
        assert info["count"][idx[e.split("->")[1]]] == c
    assert np.array_equal(info["hot_left"], lo.hot_is_left(a, cnt))
    assert info["hot_left"][idx["V21"]] == 0 and info["hot_left"][idx["V13"]] == 0
    g3 = json.load(open(os.path.join(GOLDEN, "fig3_simhash.json")))
    tok, w = T.tahoe_tree_tokens(h, 0, 2)
    assert [[names[k] for k in t] for t in tok] == g3["tree1_tokens_tnodes2"]
    assert w.tolist() == g3["weights"]
    # expected node reads per tree = sum of node probabilities
    assert info["exp_reads"][0] == pytest.approx(1 + 0.8 + 0.2 + 0.48 + 0.32 + 0.06 + 0.14)
    T.tahoe_forest_free(h)


def test_product_tokens_simhash_equal_oracle_on_generated_forest():
    f = gen.make_forest(2, n_trees=12)
    Xc = gen.make_calibration(2, 3000)
    h = T.tahoe_forest_build(f, f["n_features"], 1, f["agg"], 0.0, -1)
    T.tahoe_forest_layout(h, Xc)
    info = T.tahoe_forest_layout_info(h, len(f["feature"]), 12)
    cnt = oracle.node_counts(f, Xc)
    assert np.array_equal(info["count"], cnt)
    hl = lo.hot_is_left(f, cnt)
    assert np.array_equal(info["hot_left"], hl)
    npb = cnt / len(Xc)
    for t in range(12):
        tok, w = T.tahoe_tree_tokens(h, t, 4)
        otok = lo.tokens(f, t, 4, hl)
        assert [tuple(int(k) for k in row if k >= 0) for row in tok] == otok
        assert np.array_equal(w, np.array([npb[tk[-1]] for tk in otok]))
        cs, bits = T.tahoe_tree_simhash(h, t, 4, 128)
        S = np.stack([lo.token_bits(lo.token_bytes(f, tk), 128).astype(np.int64) * 2 - 1
                      for tk in otok])
        ocs = np.zeros(128)
        for i in range(len(otok)):      # sequential sum in token order
            ocs = ocs + npb[otok[i][-1]] * S[i]
        assert np.allclose(cs, ocs, rtol=0, atol=1e-12)
        assert np.array_equal(bits, (ocs >= 0).astype(np.uint8))
    T.tahoe_forest_free(h)


def decode_sliced(img, X, n_trees, n_classes):
    """Walk the exported SLICED image on the host (test-side decoder, independent of the
    product's kernels): returns leaf[n, T] (caller node ids) and per-class fp64 sums.
    Node words: internal y = off_bytes << (F+3) | default_left << (F+2) | attribute << 2 (left
    child next); leaf y = next_root_bytes << (F+3) | (2^F - 1) << 2; slot rows of slot_bytes."""
    n = X.shape[0]
    F = img["feature_bits"]
    fmask = (1 << F) - 1
    leaf = np.full((n, n_trees), -1, np.int64)
    sums = np.zeros((n, n_classes))
    sb = img["slot_bytes"]
    for s in range(img["n_slices"]):
        c = img["slice_info"][s, 1]
        for lane in range(img["cols"]):
            end = img["col_len"][s, lane]
            x_t, y_t = img["nodes"][s, end, lane]
            assert y_t == fmask << 2 and x_t == 0, "terminal self-loop closes the column"
            for i in range(n):
                k = 0
                while k < end:
                    x, y = (int(v) for v in img["nodes"][s, k, lane])
                    if ((y >> 2) & fmask) == fmask:
                        t, node = img["leaf_meta"][s, k, lane]
                        leaf[i, t] = node
                        sums[i, c] += float(np.uint32(x).view(np.float32))
                        k += (y >> (F + 3)) // sb
                    else:
                        thr = float(np.uint32(x).view(np.float32))
                        v = X[i, (y >> 2) & fmask]
                        go_left = bool((y >> (F + 2)) & 1) if np.isnan(v) else bool(v < thr)
                        k += 1 if go_left else (y >> (F + 3)) // sb
                assert k == end
    return leaf, sums


@pytest.mark.parametrize("cid,ntrees,nrows", [(1, None, 200), (2, 60, 60), (3, 70, 40)])
def test_sliced_image_decodes_to_oracle(cid, ntrees, nrows):
    f = gen.make_forest(cid, n_trees=ntrees)
    X = gen.make_rows(cid, nrows)
    X[::7, 1] = np.nan
    h = T.tahoe_forest_build(f, f["n_features"], f["n_classes"], f["agg"], 0.0, -1)
    for layout in (False, True):
        if layout:
            T.tahoe_forest_layout(h, gen.make_calibration(cid, 2000))
        img = T.tahoe_forest_export_sliced(h)
        assert img is not None
        leaf, sums = decode_sliced(img, X, len(f["root"]), f["n_classes"])
        r = oracle.predict(f, X, want_leaf=True)
        assert np.array_equal(leaf, r["leaf"])
        if f["agg"] == oracle.AGG_CLASS_SUM:
            assert np.array_equal(sums, r["raw"])      # dyadic leaves: exact in any order
        else:
            assert np.array_equal(sums[:, 0], r["raw"][:, 0])
    T.tahoe_forest_free(h)


def test_shards_partition_trees():
    f = gen.make_forest(2, n_trees=50)
    h = T.tahoe_forest_build(f, 28, 1, T.AGG_BINARY, 0.0, -1)
    T.tahoe_forest_layout(h, gen.make_calibration(2, 1000))
    seen = []
    for r in range(4):
        s = T.tahoe_forest_shard(h, r, 4, -1)
        info = T.tahoe_forest_layout_info(s, len(f["feature"]), T.tahoe_forest_n_trees(s))
        seen += list(info["order"])
        st = T.tahoe_forest_stats(s)
        assert st["n_trees_full"] == 50
        T.tahoe_forest_free(s)
    assert sorted(seen) == list(range(50))
    T.tahoe_forest_free(h)


def test_layout_from_counts_equals_layout_from_rows():
    """tahoe_forest_layout_counts (counts measured elsewhere, Algorithm 1 line 16) gives the same
    layout as calibrating on the rows themselves."""
    f = gen.make_forest(2, n_trees=40)
    Xc = gen.make_calibration(2, 2048)
    a = T.tahoe_forest_build(f, 28, 1, T.AGG_BINARY, 0.0, -1)
    b = T.tahoe_forest_build(f, 28, 1, T.AGG_BINARY, 0.0, -1)
    T.tahoe_forest_layout(a, Xc)
    T.tahoe_forest_layout_counts(b, oracle.node_counts(f, Xc), len(Xc), Xc)
    ia = T.tahoe_forest_layout_info(a, len(f["feature"]), 40)
    ib = T.tahoe_forest_layout_info(b, len(f["feature"]), 40)
    for k in ("count", "hot_left", "exp_reads", "order"):
        assert np.array_equal(ia[k], ib[k]), k
    ea, eb = T.tahoe_forest_export_sliced(a), T.tahoe_forest_export_sliced(b)
    assert np.array_equal(ea["nodes"], eb["nodes"])
    T.tahoe_forest_free(a)
    T.tahoe_forest_free(b)


def test_pack_refine_improves_simulated_lockstep(monkeypatch):
    """Reading R6: the measured-path local search never makes the packing's simulated cost worse
    than the expected-work packing it starts from, and the image still decodes to the oracle."""
    f = gen.make_forest(3, n_trees=140)
    effs = {}
    monkeypatch.setenv("TAHOE_SLOT_BUDGET", "600")   # host-only handle: give it a budget
    for flag in ("0", "1"):
        monkeypatch.setenv("TAHOE_PACK_REFINE", flag)
        h = T.tahoe_forest_build(f, f["n_features"], f["n_classes"], f["agg"], 0.0, -1)
        T.tahoe_forest_layout(h, gen.make_calibration(3, 4096))
        st = T.tahoe_forest_stats(h)
        assert st["sliced_valid"], st["sliced_why"]
        effs[flag] = st["lockstep_eff_sim"]
        if flag == "1":
            X = gen.make_rows(3, 40)
            img = T.tahoe_forest_export_sliced(h)
            leaf, _ = decode_sliced(img, X, len(f["root"]), f["n_classes"])
            assert np.array_equal(leaf, oracle.predict(f, X, want_leaf=True)["leaf"])
        T.tahoe_forest_free(h)
    assert effs["1"] >= effs["0"] - 1e-12, effs


def test_wide_code_layout_host():
    """Reading R8 on a host-only handle: a forest over 2000 attributes gets the wide codes; its
    virtual attributes number sum_j ceil(K_j / 127) over the distinct thresholds K_j of each
    attribute (counted here with numpy), the code row is the smallest power of two above them
    (the all-ones byte is the leaf's pad), the slices are packed for the room the 3-tile code ring
    leaves, and the (shared) sliced image still decodes to the oracle's leaves."""
    f = gen.make_forest(4, n_trees=120)
    h = T.tahoe_forest_build(f, f["n_features"], f["n_classes"], f["agg"], 0.0, -1)
    T.tahoe_forest_layout(h, gen.make_calibration(4, 2048))
    st = T.tahoe_forest_stats(h)
    assert st["sliced_valid"] and st["coded_valid"] and st["code8"], st["coded_why"]
    feat, thr = f["feature"], f["threshold"]
    k = [len(np.unique(thr[feat == j])) for j in range(f["n_features"])]
    nv = int(sum((x + 126) // 127 for x in k))
    assert st["code8_virtual"] == nv
    V = st["code8_vfbits"]
    assert (1 << V) - 1 >= nv and (1 << (V - 1)) - 1 < nv
    ring = 6 * 8 * (1 << V) + (1 << V) + 6 * 16 + 6 * 8 * 8 + 256
    assert ((st["slots_max"] * 128 + 1023) // 1024) * 1024 + ring <= 232448
    X = gen.make_rows(4, 24)
    img = T.tahoe_forest_export_sliced(h)
    leaf, _ = decode_sliced(img, X, len(f["root"]), f["n_classes"])
    assert np.array_equal(leaf, oracle.predict(f, X, want_leaf=True)["leaf"])
    T.tahoe_forest_free(h)


def test_layout_state_export_import_roundtrip():
    """tahoe_forest_layout_export / _import: a second build of the same arrays that imports the
    first handle's layout state has the same counts, hot children, expected reads, tree order and
    the same encoded sliced image; blobs from another forest or garbage are refused (E_INVAL)."""
    import gen
    from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
    f = gen.make_forest(3, n_trees=60)
    a = T.Forest(f, device=-1).layout(gen.make_calibration(3, 3000))
    blob = a.layout_state()
    b = T.Forest(f, device=-1).apply_layout_state(blob)
    ia = T.tahoe_forest_layout_info(a.handle, len(f["feature"]), a.n_trees)
    ib = T.tahoe_forest_layout_info(b.handle, len(f["feature"]), b.n_trees)
    for k in ("count", "hot_left", "exp_reads", "order"):
        assert np.array_equal(ia[k], ib[k]), k
    ea, eb = a.export_sliced(), b.export_sliced()
    for k in ("nodes", "leaf_meta", "col_len", "slice_info"):
        assert np.array_equal(ea[k], eb[k]), k
    assert a.stats()["lockstep_eff_sim"] == b.stats()["lockstep_eff_sim"]
    other = T.Forest(gen.make_forest(3, n_trees=61), device=-1)
    with pytest.raises(T.TahoeError):
        other.apply_layout_state(blob)
    with pytest.raises(T.TahoeError):
        b.apply_layout_state(b"not a layout blob at all")
    with pytest.raises(T.TahoeError):
        b.apply_layout_state(blob[:-3])


def test_microbenchmark_and_profile_walk_argument_checks():
    """tahoe_measure_visit_rate refuses bad variants / step counts before touching a device;
    tahoe_profile_walk on a host-only handle is E_STATE (no CPU prediction path)."""
    r = ctypes.c_double()
    L = T.load()
    for variant, steps, reps in ((3, 256, 10), (-1, 256, 10), (0, 1, 10), (0, 255, 10), (0, 258, 10), (1, 260, 10),
                                 (0, 256, 0), (2, 10_000, 1)):
        assert L.tahoe_measure_visit_rate(0, variant, steps, reps, ctypes.byref(r), None) == T.TAHOE_E_INVAL
    h = _build(_stump_arrays())
    st = np.zeros(8, np.float64)
    rc = L.tahoe_profile_walk(h, ctypes.c_void_p(1), 4, 1, ctypes.c_void_p(1), st.ctypes.data, None)
    assert rc == T.TAHOE_E_STATE
    T.tahoe_forest_free(h)


def _slot_collision(f, slot, fbits, cal=None):
    """Estimated probability that some shared-memory bank sees two code words in one warp-wide code
    load (reading R10): lanes read the word of their node's attribute (weight: calibrated
    internal visits, or 2^-depth) or, at a leaf, the pad word of slot 2^F - 1; the second half's row
    holds slot j at j ^ 32.  Python restatement of the objective, for the test only."""
    feat = np.asarray(f["feature"])
    left = np.asarray(f["left"])
    root = np.asarray(f["root"])
    nf = f["n_features"]
    depth = np.full(len(feat), -1)
    for r in root:
        st = [(int(r), 0)]
        while st:
            k, dep = st.pop()
            depth[k] = dep
            if left[k] >= 0:
                st.append((int(left[k]), dep + 1))
                st.append((int(f["right"][k]), dep + 1))
    w = np.zeros(nf)
    internal = (left >= 0) & (depth >= 0)
    pk = cal if cal is not None else np.ldexp(1.0, -np.minimum(depth, 60))
    np.add.at(w, feat[internal], pk[internal])
    visits = w.sum()
    pl = len(root) / (visits + len(root))
    w = w / visits * (1 - pl)
    nw = (1 << fbits) // 2
    M = np.zeros(nw)
    np.add.at(M, np.asarray(slot) // 2, w)
    M[((1 << fbits) - 1) // 2] += pl
    ok = 1.0
    for b in range(32):
        none, one = 1.0, 0.0
        for h in range(2):
            for pw in range(b, nw, 32):
                u = 1 - (1 - M[pw ^ (16 * h)]) ** 16
                one = one * (1 - u) + none * u
                none *= 1 - u
        ok *= none + one
    return 1 - ok


def test_code_slot_assignment():
    """Reading R10: the u16 code slots are a bijection of the attributes onto slots below the
    leaves' pad slot 2^F - 1, deterministic, the identity for 64-byte rows (C2), and for C3's
    128-byte rows they lower the estimated bank-collision probability below the identity's."""
    for cid, fbits in ((2, 5), (3, 6)):
        f = gen.make_forest(cid, n_trees=200)
        slots = []
        for _ in range(2):
            h = T.tahoe_forest_build(f, f["n_features"], f["n_classes"], f["agg"], 0.0, -1)
            st = T.tahoe_forest_stats(h)
            assert st["coded_valid"] and st["sliced_fbits"] == fbits, st["coded_why"]
            slots.append(st["code_slot"])
            T.tahoe_forest_free(h)
        s = slots[0]
        assert s == slots[1], "deterministic"
        assert len(s) == f["n_features"] and len(set(s)) == len(s)
        assert all(0 <= j < (1 << fbits) - 1 for j in s)
        if fbits == 5:
            assert s == list(range(f["n_features"]))
        else:
            ident = _slot_collision(f, list(range(f["n_features"])), fbits)
            mine = _slot_collision(f, s, fbits)
            assert mine < ident - 0.05, (mine, ident)


def test_prepass_lane_plan_covers_every_slot_once():
    """The row-coding pre-pass plan (encode.cpp build_code_banks, kernels.cu k_encode_rows_banks):
    replaying the kernel's assignment from the exported lane descriptors ({slot, attribute, table
    offset, stride | K}, slot < 0: idle lane; every lane codes all rows), every code slot of every
    row is written exactly once — by a lane of the slot's attribute, or with the pad code for the
    slots no attribute owns — for C1, C2, C3 and random forests of 3-127 attributes."""
    from test_oracle_pins import random_forest
    forests = [gen.make_forest(cid) for cid in (1, 2, 3)]
    for d, grid in ((3, None), (40, None), (54, 7), (100, None), (127, 41)):
        rng = np.random.default_rng(d)
        thr_grid = None if grid is None else np.linspace(-2.0, 2.0, grid)
        forests.append(dict(random_forest(rng, 60, 7, d, thr_grid=thr_grid), n_features=d))
    for f in forests:
        cid = f.get("config", f["n_features"])
        h = T.tahoe_forest_build(f, f["n_features"], f["n_classes"], f["agg"], 0.0, -1)
        st = T.tahoe_forest_stats(h)
        T.tahoe_forest_free(h)
        assert st["coded_valid"] and st["code_bank_passes"] > 0
        desc = np.array(st["code_bank_desc"], np.int64).reshape(-1, 4)
        nslots = max(32, 1 << st["sliced_fbits"])
        owner = {s: a for a, s in enumerate(st["code_slot"])}
        writes = np.zeros((32, nslots), np.int64)
        for dx, feat, _base, _w in desc:
            if dx < 0:
                continue                                     # idle lane
            slot, ph, r = dx & 255, (dx >> 8) & 15, 1 << ((dx >> 12) & 3)
            assert ph < r
            assert (feat == -1 and slot not in owner) or owner.get(slot) == feat, (slot, feat)
            for s in range(4 // r):
                for q in range(8):
                    writes[ph + r * (8 * s + q), slot] += 1
        assert (writes == 1).all(), (cid, np.argwhere(writes != 1)[:5])


def test_cost_model_picks_for_the_bench_workloads():
    """The shipped cost-model constants (costmodel_b200.json, fitted on the B200) pick the measured
    fastest strategy for the bench's launch configurations (profiles/r02_costmodel.md): the
    rank-coded slices for C2 (1M rows), C3 (4M) and C4 (500K), ROWS for a C2 batch of 100."""
    picks = {}
    for cid, n in ((2, 1_000_000), (3, 4_000_000), (4, 500_000), (2, 100)):
        f = gen.make_forest(cid)
        h = T.tahoe_forest_build(f, f["n_features"], f["n_classes"], f["agg"], 0.0, -1)
        T.tahoe_forest_layout(h, gen.make_calibration(cid, 4096))
        picks[(cid, n)] = T.tahoe_select_strategy(h, n, f["n_features"])
        T.tahoe_forest_free(h)
    assert picks[(2, 1_000_000)] == T.STRATEGY_SLICED_CODED, picks
    assert picks[(3, 4_000_000)] == T.STRATEGY_SLICED_CODED, picks
    assert picks[(4, 500_000)] == T.STRATEGY_SLICED_CODED, picks
    assert picks[(2, 100)] == T.STRATEGY_ROWS, picks
