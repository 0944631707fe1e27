"""Debug: C4-shaped forest, each sliced strategy forced, synchronize after each (sanitizer target)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402

ntrees = int(sys.argv[1]) if len(sys.argv) > 1 else 40
n = int(sys.argv[2]) if len(sys.argv) > 2 else 301
strats = [int(s) for s in sys.argv[3].split(",")] if len(sys.argv) > 3 else [2, 1]
dev = torch.device("cuda", 0)
f = gen.make_forest(4, n_trees=ntrees)
F = T.Forest(f, device=0)
st = F.stats()
print({k: st[k] for k in ("n_slices", "slots_max", "code8", "code8_vfbits", "code8_virtual", "code8_bands")}, flush=True)
X = gen.make_rows(4, n)
X[::17, 1] = np.nan
ref = oracle.predict(f, X)
Xd = torch.from_numpy(X).to(dev)
for s in strats:
    out = torch.empty((n, F.n_out), device=dev)
    cls = torch.empty(n, dtype=torch.int32, device=dev)
    F.predict(Xd, out=out, out_class=cls, force_strategy=s)
    torch.cuda.synchronize()
    o = out.cpu().numpy()
    print("strategy", s, "exact", np.array_equal(o, ref["out"]), "maxdiff", float(np.abs(o - ref["out"]).max()), flush=True)
