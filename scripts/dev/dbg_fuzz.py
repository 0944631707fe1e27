"""Debug one fuzz case: per strategy, where the GPU result differs from the oracle."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np, torch
import oracle
from test_gpu_fuzz import _case
from test_gpu_parity import _gpu_run, _strats
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
seed = int(sys.argv[1])
f, d, nc, agg, base, X = _case(seed)
F = T.Forest(f, n_features=d, n_classes=nc, agg=agg, base_score=base, device=0)
st = F.stats()
print({k: st[k] for k in ("n_slices", "sliced_valid", "coded_valid", "code8", "slots_max")}, "agg", agg, "base", base, "n", X.shape, flush=True)
ref = oracle.predict(f, X, agg=agg, n_classes=nc, base_score=base, want_leaf=True)
for s in _strats(F) + [-1]:
    r = _gpu_run(F, X, s, want_leaf=(s != -1))
    bad = np.argwhere(r["out"] != ref["out"])
    print("strategy", s, "mismatches", len(bad), flush=True)
    for i, c in bad[:5]:
        print("   row", i, "class", c, "gpu", r["out"][i, c], "ref", ref["out"][i, c], "raw", ref["raw"][i], "nan", np.isnan(X[i]).sum(), flush=True)
    if "leaf" in r:
        lb = np.argwhere(r["leaf"] != ref["leaf"])
        print("   leaf mismatches", len(lb), lb[:3].tolist())
