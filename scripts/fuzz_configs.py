"""Seeded sweep over the BASELINE-shaped generators (not part of the test suite): random tree
subsets of C1-C5, random batch sizes (1 .. 150K rows, ragged), NaN rows, layout on / off, every
usable strategy and the cost model's choice, bit-exact against the oracle (dyadic leaves)."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np
import gen, oracle
from test_gpu_parity import _gpu_run, _strats
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
s0, s1 = int(sys.argv[1]), int(sys.argv[2])
fails = 0
for seed in range(s0, s1):
    rng = np.random.default_rng(seed)
    cid = int(rng.integers(1, 6))
    cfg = gen.CONFIGS[cid]
    nt = int(rng.integers(1, min(cfg.n_trees, 300 if cid != 5 else 40) + 1))
    f = gen.make_forest(cid, n_trees=nt)
    n = int(rng.choice([1, 65, 4097, 33_000, 150_001 if cid not in (4,) else 20_001]))
    X = gen.make_rows(cid, n, row0=int(rng.integers(0, 10**6)))
    X[rng.random(n) < 0.05, int(rng.integers(0, cfg.n_features))] = np.nan
    F = T.Forest(f, device=0)
    if rng.random() < 0.5:
        F.layout(gen.make_calibration(cid, 2048))
    ref = oracle.predict(f, X, want_leaf=True)
    msg = []
    for s in _strats(F) + [-1]:
        r = _gpu_run(F, X, s, want_leaf=(s in (0, 1)))
        if not np.array_equal(r["out"], ref["out"]):
            msg.append(f"out s={s} ({int((r['out'] != ref['out']).sum())})")
        if f["agg"] in (oracle.AGG_BINARY, oracle.AGG_CLASS_SUM, oracle.AGG_VOTE) and not np.array_equal(r["cls"], ref["cls"]):
            msg.append(f"cls s={s}")
        if "leaf" in r and not np.array_equal(r["leaf"], ref["leaf"]):
            msg.append(f"leaf s={s}")
    if msg:
        fails += 1
        print("FAIL seed", seed, "C", cid, "trees", nt, "n", n, F.stats()["n_slices"], msg, flush=True)
    F.close()
print("done", s0, s1, "fails", fails, flush=True)
