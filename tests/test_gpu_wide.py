"""GPU parity of the wide rank codes (reading R8): rows of more than 127 attributes coded
as u8 over virtual attributes (an attribute with K distinct thresholds split into ceil(K / 127)
pieces), staged in shared memory next to slices packed for the room the code-tile ring leaves.

The decisions at piece boundaries are the new arithmetic, so rows are built from the forest's own
thresholds — in particular the first and last threshold of every piece — and their float
neighbours, plus -0.0 / +0.0, +-Inf and NaN (default path).  Scores and classes must be bit-exact
against the CPU oracle with dyadic leaves, and equal the fp32 slices and the direct strategy.
"""
import numpy as np
import pytest

import oracle
from test_gpu_parity import _check, _gpu_run, _strats
from test_oracle_pins import random_forest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402


def _wide_forest(seed, d, n_trees, depth, grid_n, n_classes=1):
    rng = np.random.default_rng(seed)
    grid = np.sort(rng.normal(size=grid_n)).astype(np.float32)
    grid[grid_n // 2] = 0.0
    f = random_forest(rng, n_trees, depth, d, p_split=0.9, n_classes=n_classes, thr_grid=grid)
    if n_classes > 1:
        f["agg"] = oracle.AGG_CLASS_SUM
    return f, rng


def _boundary_rows(f, rng, n, d):
    """Rows whose values sit on thresholds (piece boundaries first), next to them, on signed zeros,
    infinities and NaN."""
    internal = np.flatnonzero(f["feature"] >= 0)
    X = rng.normal(size=(n, d)).astype(np.float32)
    pick = rng.random(X.shape)
    for j in range(d):
        t = np.unique(f["threshold"][internal[f["feature"][internal] == j]])
        if len(t) == 0:
            continue
        bounds = t[np.unique(np.concatenate([np.arange(0, len(t), 127), np.arange(126, len(t), 127),
                                             [len(t) - 1]]))]
        m = pick[:, j] < 0.45
        half = rng.random(m.sum()) < 0.5
        v = np.where(half, rng.choice(bounds, size=m.sum()), rng.choice(t, size=m.sum()))
        kind = rng.integers(0, 3, size=m.sum())
        v = np.where(kind == 1, np.nextafter(v, np.float32(np.inf)), v)
        v = np.where(kind == 2, np.nextafter(v, np.float32(-np.inf)), v)
        X[m, j] = v.astype(np.float32)
    X[pick > 0.985] = -0.0
    X[(pick > 0.975) & (pick <= 0.985)] = 0.0
    X[(pick > 0.97) & (pick <= 0.975)] = np.inf
    X[(pick > 0.965) & (pick <= 0.97)] = -np.inf
    X[(pick > 0.96) & (pick <= 0.965)] = np.nan
    return X


def test_wide_codes_piece_boundaries_ties_signed_zero_inf_nan():
    d = 160
    f, rng = _wide_forest(8, d, 420, 9, 600)
    F = T.Forest(f, n_features=d, n_classes=1, agg=oracle.AGG_SUM, device=0)
    st = F.stats()
    assert st["coded_valid"] and st["code8"], st["coded_why"]
    assert st["code8_virtual"] > d, "some attribute must span several pieces"
    X = _boundary_rows(f, rng, 20011, d)
    ref = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1, want_leaf=True)
    outs = []
    for s in _strats(F):
        r = _gpu_run(F, X, s)          # leaf ids + fingerprints (LEAF instantiations)
        _check(r, ref, oracle.AGG_SUM, True)
        outs.append(r["out"])
    assert len(outs) == len(_strats(F)) >= 3 and all(np.array_equal(o, outs[0]) for o in outs)


@pytest.mark.parametrize("tma", ["1", "0"])
@pytest.mark.parametrize("d", [130, 255, 600, 1500])
def test_wide_codes_row_geometries(d, tma, monkeypatch):
    """Code rows of 256 B .. 2 KB (V = 8 .. 11), one or several pre-pass bands, ragged last
    tile; NaN rows take their default paths.  Both pre-pass kernels: rows staged by TMA (d % 4 ==
    0) and rows through L1 ($TAHOE_CODE8_TMA=0, and every d % 4 != 0)."""
    monkeypatch.setenv("TAHOE_CODE8_TMA", tma)
    f, rng = _wide_forest(d, d, 160, 8, 300)
    F = T.Forest(f, n_features=d, n_classes=1, agg=oracle.AGG_SUM, device=0)
    st = F.stats()
    assert st["coded_valid"] and st["code8"], st["coded_why"]
    assert (1 << st["code8_vfbits"]) > st["code8_virtual"]
    X = rng.normal(size=(7001, d)).astype(np.float32)
    X[::23, 0] = np.nan
    X[5::31, :] = np.nan
    ref = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1, want_leaf=True)
    _check(_gpu_run(F, X, T.STRATEGY_SLICED_CODED, want_leaf=False), ref, oracle.AGG_SUM, True,
           want_leaf=False)
    _check(_gpu_run(F, X, T.STRATEGY_SLICED_CODED), ref, oracle.AGG_SUM, True)


def test_wide_codes_multiclass_partials_and_slice_switching(monkeypatch):
    """Many slices over fewer CTAs than slices on a small batch and the full GPU on a large one
    (dynamic tile claiming, CTAs moving between slices): CLASS_SUM scores, argmax and the raw
    per-class partials (tahoe_predict_partial, no base) bit-exact."""
    monkeypatch.setenv("TAHOE_FORCE_STRATEGY", "2")
    d = 300
    f, rng = _wide_forest(11, d, 900, 8, 400, n_classes=5)
    F = T.Forest(f, n_features=d, n_classes=5, agg=oracle.AGG_CLASS_SUM, base_score=0.5, device=0)
    st = F.stats()
    assert st["code8"] and st["n_slices"] > 5, st
    for n in (333, 60_017):
        X = rng.normal(size=(n, d)).astype(np.float32)
        X[::41, 7] = np.nan
        ref = oracle.predict(f, X, agg=oracle.AGG_CLASS_SUM, n_classes=5, base_score=0.5,
                             want_leaf=True)
        _check(_gpu_run(F, X, -1, want_leaf=False), ref, oracle.AGG_CLASS_SUM, True, want_leaf=False)
        _check(_gpu_run(F, X, -1), ref, oracle.AGG_CLASS_SUM, True)
        part = F.predict_partial(torch.from_numpy(X).cuda())
        torch.cuda.synchronize()
        assert np.array_equal(part.cpu().numpy(), ref["raw"] - 0.5), "dyadic partial sums are exact"


def test_wide_codes_unused_attributes_take_no_bytes_and_fallback():
    """Attributes no node tests get no code byte (0 pieces): 4000 attributes of which ~1970 are
    used code into 2 KB rows.  With more than 4095 used attributes (4 KB rows would leave no
    room for a slice next to the ring) the forest keeps the fp32 slices, rows read from global
    memory; both stay exact."""
    for d, trees, depth, wide in ((4000, 64, 6, True), (6000, 300, 8, False)):
        f, rng = _wide_forest(5, d, trees, depth, 200)
        F = T.Forest(f, n_features=d, n_classes=1, agg=oracle.AGG_SUM, device=0)
        st = F.stats()
        used = len(np.unique(f["feature"][f["feature"] >= 0]))
        assert st["code8"] == wide and st["coded_valid"] == wide, (d, st["code8_virtual"], used)
        if wide:
            assert st["code8_virtual"] == used   # <= 127 thresholds each: one piece per used attribute
        X = rng.normal(size=(3001, d)).astype(np.float32)
        ref = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1)
        for s in _strats(F):
            _check(_gpu_run(F, X, s, want_leaf=False), ref, oracle.AGG_SUM, True, want_leaf=False)


def _chunked_case():
    """Body of test_wide_codes_chunked_launches (run in a child with $TAHOE_CODE8_CHUNK_MB set:
    the chunk size is read once per process)."""
    d = 600
    f, rng = _wide_forest(77, d, 160, 8, 300)
    F = T.Forest(f, n_features=d, n_classes=1, agg=oracle.AGG_SUM, device=0)
    assert F.stats()["code8"]
    X = rng.normal(size=(9001, d)).astype(np.float32)
    X[::29, 3] = np.nan
    ref = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1, want_leaf=True)
    _check(_gpu_run(F, X, T.STRATEGY_SLICED_CODED, want_leaf=False), ref, oracle.AGG_SUM, True,
           want_leaf=False)
    _check(_gpu_run(F, X, T.STRATEGY_SLICED_CODED), ref, oracle.AGG_SUM, True)


@pytest.mark.parametrize("tma", ["1", "0"])
def test_wide_codes_chunked_launches(tma):
    """Batches coded and walked in several launches of whole tiles (1 MB of code rows each: the
    pre-pass's tensor map starts at each chunk's first row), both pre-pass kernels."""
    import os
    import subprocess
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    root = os.path.dirname(here)
    env = dict(os.environ, TAHOE_CODE8_CHUNK_MB="1", TAHOE_CODE8_TMA=tma,
               PYTHONPATH=os.pathsep.join([root, here, os.environ.get("PYTHONPATH", "")]))
    r = subprocess.run([sys.executable, "-c", "import test_gpu_wide as t; t._chunked_case()"],
                       cwd=here, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]


@pytest.mark.parametrize("n_trees,depth", [(1, 3), (1, 6), (3, 6), (5, 6)])
def test_wide_codes_small_rows_half_warp_swizzle(n_trees, depth):
    """Wide codes whose used attributes fit rows of 32 .. 256 bytes (V = 5 .. 8; few trees over 1000
    attributes): the second half-warp's rows keep byte v at v ^ min(64, row / 2) — the swizzle
    must stay inside the row (a first version XORed 64 into 32-byte rows).  Leaf ids, scores and
    fingerprints bit-exact against the oracle, NaN rows and a ragged last tile included."""
    d = 1000
    f, rng = _wide_forest(7 + n_trees + depth, d, n_trees, depth, 300)
    F = T.Forest(f, n_features=d, n_classes=1, agg=oracle.AGG_SUM, device=0)
    st = F.stats()
    assert st["coded_valid"] and st["code8"], st["coded_why"]
    assert st["code8_vfbits"] <= 8, st["code8_vfbits"]
    X = rng.normal(size=(3003, d)).astype(np.float32)
    X[::17, :] = np.nan
    ref = oracle.predict(f, X, agg=oracle.AGG_SUM, n_classes=1, want_leaf=True)
    _check(_gpu_run(F, X, T.STRATEGY_SLICED_CODED), ref, oracle.AGG_SUM, True)
    _check(_gpu_run(F, X, T.STRATEGY_SLICED_CODED, want_leaf=False), ref, oracle.AGG_SUM, True,
           want_leaf=False)
