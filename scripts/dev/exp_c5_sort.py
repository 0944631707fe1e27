"""Experiment: does ordering rows by their top-of-tree decisions speed up the direct walk (C5 shard)?"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gen
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
f = gen.make_forest(5, n_trees=500, leaf_mode="normal")
F = T.Forest(f, device=0).layout(gen.make_calibration(5, 16384))
n = int(sys.argv[1]) if len(sys.argv) > 1 else 300_000
Xn = gen.make_rows(5, n)
root = f["root"]; feat = f["feature"]; thr = f["threshold"]; left = f["left"]; right = f["right"]

def decisions(X, t, levels):
    k = np.full(X.shape[0], root[t]); key = np.zeros(X.shape[0], np.int64)
    for _ in range(levels):
        fk = feat[k]; internal = fk >= 0
        go = np.where(internal, X[np.arange(X.shape[0]), np.maximum(fk, 0)] < thr[k], False)
        key = key * 2 + go
        k = np.where(internal, np.where(go, left[k], right[k]), k)
    return key

def timeit(X):
    Xd = torch.from_numpy(np.ascontiguousarray(X)).cuda()
    part = torch.empty((n, 1), dtype=torch.float64, device="cuda")
    for _ in range(2):
        F.predict_partial(Xd, part)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); F.predict_partial(Xd, part); e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1)

print("unsorted", round(timeit(Xn), 3), "ms", flush=True)
for ntr, lev in ((8, 2), (16, 3), (4, 6)):
    keys = [decisions(Xn, t, lev) for t in range(ntr)]
    order = np.lexsort(keys[::-1])
    print(f"sorted by {ntr} trees x {lev} levels", round(timeit(Xn[order]), 3), "ms", flush=True)
order = np.argsort(Xn[:, 0], kind="stable")
print("sorted by column 0", round(timeit(Xn[order]), 3), "ms", flush=True)
