"""Debug fuzz case 5 (u16 coded slices): vary pre-pass, NaN, batch size."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np, torch
import oracle
from test_gpu_fuzz import _case
from test_gpu_parity import _gpu_run
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
f, d, nc, agg, base, X0 = _case(5)
for banks in ("1", "0"):
    os.environ["TAHOE_CODE_BANKS"] = banks
    for nan in (True, False):
        for n in (9472, 9536, 23623):
            X = X0[:n].copy()
            if not nan:
                X[np.isnan(X)] = 0.5
            F = T.Forest(f, n_features=d, n_classes=nc, agg=agg, base_score=base, device=0)
            ref = oracle.predict(f, X, agg=agg, n_classes=nc, base_score=base)
            r = _gpu_run(F, X, 2, want_leaf=False)
            bad = np.argwhere(r["out"] != ref["out"])
            print("banks", banks, "nan", nan, "n", n, "mismatches", len(bad), "first", bad[:1].tolist(), flush=True)
            F.close()
