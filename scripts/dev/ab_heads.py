"""A/B diagnostic: k_direct_tlp (variant 5) vs tree heads in shared memory (variants 8 / 9) on a
C5 tree shard and on the full C5 forest; outputs compared bit for bit with variant 5."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gen
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
n = int(sys.argv[1]) if len(sys.argv) > 1 else 300_000
f = gen.make_forest(5, leaf_mode="normal")
F = T.Forest(f, device=0)
F.layout(gen.make_calibration(5, 16384))
S = F.shard(0, 8)
X = torch.from_numpy(gen.make_rows(5, n)).cuda()
cases = [(v, None) for v in (sys.argv[2].split(",") if len(sys.argv) > 2 else ["5"])] if len(sys.argv) > 2 else \
    [("5", None), ("8", "4"), ("8", "8"), ("8", "16"), ("9", "8"), ("9", "16"), ("5", None)]
for name, H in ((f"shard0/8", S), ("full", F)):
    part = torch.empty((n, 1), dtype=torch.float64, device="cuda")
    ref = None
    for v, kh in cases:
        os.environ["TAHOE_DIRECT_VARIANT"] = v
        if kh: os.environ["TAHOE_DIRECT_HEADS"] = kh
        for _ in range(2): H.predict_partial(X, part)
        torch.cuda.synchronize()
        ts = []
        for _ in range(3):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); H.predict_partial(X, part); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        out = part.cpu().numpy().copy()
        if ref is None: ref = out
        same = np.array_equal(out.view(np.uint64), ref.view(np.uint64))
        print(f"{name} n={n} variant={v} kh={kh}: {np.median(ts):.3f} ms  bit-equal={same}", flush=True)
