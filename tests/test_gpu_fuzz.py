"""GPU parity fuzz: seeded random forests of every shape the strategies branch on, through every
usable strategy, bit-exact against the CPU oracle (dyadic leaves).

Shapes vary the attribute count across every code-row geometry (3 .. 3000 attributes, with the
row-size boundaries 31/32/33, 127/128, 255, 2047: u16 codes, wide u8 codes, rows too wide for
either), tree count and depth (stumps, single leaves, deep trees), classes and every aggregation
(sum, average, binary, class sums, vote), NaN density and default paths, thresholds drawn from a coarse
grid (ties x == b) or continuous values, and batch sizes across the small- and large-batch
kernel variants with ragged tails.
"""
import numpy as np
import pytest

import oracle
from test_gpu_parity import _check, _gpu_run, _strats
from test_oracle_pins import random_forest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402

N_CASES = 48


def _case(seed):
    rng = np.random.default_rng(1000 + seed)
    d = int(rng.choice([3, 17, 31, 32, 33, 64, 127, 128, 255, 300, 1000, 2047, 3000]))
    n_trees = int(rng.choice([1, 7, 40, 150]))
    depth = int(rng.choice([1, 3, 6, 10]))
    n_classes = int(rng.choice([1, 1, 3]))
    vote = n_classes > 1 and rng.random() < 0.3
    grid = np.linspace(-1.5, 1.5, int(rng.choice([9, 61, 400]))) if rng.random() < 0.6 else None
    f = random_forest(rng, n_trees, depth, d, p_split=float(rng.choice([0.5, 0.8, 0.95])),
                      n_classes=n_classes, vote=vote, thr_grid=grid)
    if n_classes == 1:
        agg = int(rng.choice([oracle.AGG_SUM, oracle.AGG_AVERAGE, oracle.AGG_BINARY]))
    else:
        agg = oracle.AGG_VOTE if vote else oracle.AGG_CLASS_SUM
    n = int(rng.choice([1, 63, 2049, 40_001]))
    n = min(n, 12_000_000 // (d * 4) + 1)   # keep X under ~12 MB
    X = rng.normal(size=(n, d)).astype(np.float32)
    if grid is not None:
        m = rng.random(X.shape) < 0.3
        X[m] = rng.choice(grid, size=int(m.sum())).astype(np.float32)
    X[rng.random(X.shape) < float(rng.choice([0.0, 0.01, 0.2]))] = np.nan
    base = float(rng.choice([0.0, 0.25]))
    return f, d, n_classes, agg, base, X


@pytest.mark.parametrize("seed", range(N_CASES))
def test_fuzz_all_strategies_bit_exact(seed):
    f, d, n_classes, agg, base, X = _case(seed)
    F = T.Forest(f, n_features=d, n_classes=n_classes, agg=agg, base_score=base, device=0)
    ref = oracle.predict(f, X, agg=agg, n_classes=n_classes, base_score=base, want_leaf=True)
    outs = []
    for s in _strats(F):
        r = _gpu_run(F, X, s)
        _check(r, ref, agg, True)
        outs.append(r["out"])
    r = _gpu_run(F, X, -1, want_leaf=False)   # the cost model's own choice
    _check(r, ref, agg, True, want_leaf=False)
    assert all(np.array_equal(o, outs[0]) for o in outs)
    F.close()
