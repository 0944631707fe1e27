# C5 500-tree shard over 300K rows (the per-GPU work of the 8-way tree shard): direct variants
python - <<'PY'
import os, sys, time, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch, gen
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
import oracle
f = gen.make_forest(5, leaf_mode="normal")
full = T.Forest(f, device=-1).layout(gen.make_calibration(5))
S = full.shard(3, 8, device=0)
X = gen.make_rows(5, 300_000)
Xd = torch.from_numpy(X).cuda()
part = torch.empty((300_000, 1), dtype=torch.float64, device="cuda")
ref = None
for v in ["5", "12", "13", "14", "5", "12", "13", "14"]:
    os.environ["TAHOE_DIRECT_VARIANT"] = v
    for _ in range(2): S.predict_partial(Xd, part)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(5): S.predict_partial(Xd, part)
    b.record(); torch.cuda.synchronize()
    got = part.cpu().numpy()
    if ref is None: ref = got.copy()
    print("variant", v, round(a.elapsed_time(b) / 5, 3), "ms", "max|diff| vs v5", float(np.abs(got - ref).max()))
PY
