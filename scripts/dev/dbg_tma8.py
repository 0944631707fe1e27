import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))), "tests"))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import oracle
from test_gpu_wide import _wide_forest, _boundary_rows
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
d = int(sys.argv[1]) if len(sys.argv) > 1 else 160
f, rng = _wide_forest(8, d, 420, 9, 600)
F = T.Forest(f, n_features=d, n_classes=1, agg=oracle.AGG_SUM, device=0)
st = F.stats(); print({k: st[k] for k in ("code8", "code8_virtual", "code8_vfbits", "code8_bands", "n_slices")})
X = torch.from_numpy(_boundary_rows(f, rng, 2001, d)).cuda()
out = F.predict(X, force_strategy=T.STRATEGY_SLICED_CODED)
torch.cuda.synchronize(); print("ok", out[:4])
