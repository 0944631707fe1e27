"""Experiment: does walking a C5 tree shard in groups of trees (all SMs on one group at a time, so
each SM's L1 holds only that group's hot nodes) beat walking all of the shard's trees per row?
Times the direct walk over the 500-tree shard (F.shard(0, 8)) and over its 1/k parts
(F.shard(g, 8k), g < k) on the same rows; the sum over the parts is what a grouped kernel would
cost if its only change were the L1 working set."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import gen
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T

n = int(sys.argv[1]) if len(sys.argv) > 1 else 300_000
f = gen.make_forest(5, leaf_mode="normal")
F = T.Forest(f, device=0)
F.layout(gen.make_calibration(5, 16384))
X = torch.from_numpy(gen.make_rows(5, n)).cuda()
part = torch.empty((n, 1), dtype=torch.float64, device="cuda")


def tm(H, reps=5):
    for _ in range(2):
        H.predict_partial(X, part)
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); H.predict_partial(X, part); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


S = F.shard(0, 8)
print(f"shard 0/8 ({S.n_trees if hasattr(S, 'n_trees') else '?'} trees): {tm(S):.3f} ms", flush=True)
for k in (2, 4, 8, 16):
    parts = [F.shard(g, 8 * k) for g in range(k)]
    ts = [tm(P) for P in parts]
    print(f"k={k}: parts {['%.3f' % t for t in ts]} sum {sum(ts):.3f} ms", flush=True)
    for P in parts:
        P.close()
