import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gen, oracle
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
f = gen.make_forest(3, n_trees=280)
F = T.Forest(f, device=0).layout(gen.make_calibration(3, 4096))
print(F.stats()["n_slices"], F.stats()["cta_split"])
n = int(sys.argv[1]) if len(sys.argv) > 1 else 50003
X = gen.make_rows(3, n)
Xd = torch.from_numpy(X).cuda()
out = torch.empty((n, F.n_out), device="cuda")
cls = torch.empty(n, dtype=torch.int32, device="cuda")
F.predict(Xd, out=out, out_class=cls, force_strategy=2)
torch.cuda.synchronize()
ref = oracle.predict(f, X[:2000])
print("match", np.array_equal(out.cpu().numpy()[:2000], ref["out"]))
