"""Small runs of the coded kernels (R7 u16 and R8 wide) for compute-sanitizer."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "both"
dev = torch.device("cuda", 0)
cases = []
if which in ("both", "u16"):
    cases.append((2, 64, 3001))
if which in ("both", "wide"):
    cases.append((4, 200, 2001))
for cid, ntrees, n in cases:
    f = gen.make_forest(cid, n_trees=ntrees)
    F = T.Forest(f, device=0)
    X = gen.make_rows(cid, n)
    X[::17, 1] = np.nan
    Xd = torch.from_numpy(X).to(dev)
    out = torch.empty((n, F.n_out), device=dev)
    F.predict(Xd, out=out, force_strategy=2)
    torch.cuda.synchronize()
    print(cid, F.stats()["n_slices"], "ok", flush=True)
