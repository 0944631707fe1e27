"""Timing diagnostic for C5 (4000 trees, depth <= 20): one tree shard of 8 on one GPU."""
import os, sys, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gen
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
t = time.time()
f = gen.make_forest(5, leaf_mode="normal")
print("gen forest %.1fs" % (time.time() - t), flush=True)
t = time.time()
F = T.Forest(f, device=0)
print("build %.1fs" % (time.time() - t), flush=True)
t = time.time()
F.layout(gen.make_calibration(5, 16384))
print("layout %.1fs" % (time.time() - t), json.dumps(F.stats()), flush=True)
S = F.shard(0, 8)
print("shard stats", json.dumps(S.stats()), flush=True)
n = int(sys.argv[1]) if len(sys.argv) > 1 else 200_000
X = torch.from_numpy(gen.make_rows(5, n)).cuda()
part = torch.empty((n, 1), dtype=torch.float64, device="cuda")
for _ in range(2):
    S.predict_partial(X, part)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(); S.predict_partial(X, part); e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1)
print(f"C5 shard 0/8 n={n}: {ms:.2f} ms -> {n/ms*1e3/1e6:.2f} M samples/s per shard; "
      f"full 10M x 8 shards on 8 GPUs est {10e6/n*ms/1e3:.2f} s", flush=True)
