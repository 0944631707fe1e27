"""Large seeded fuzz sweep (not part of the test suite): the test_gpu_fuzz shapes with many more
seeds, optionally after layout() on calibration rows, plus predict_partial and the host
end-to-end call, all against the oracle."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np, torch
import oracle
from test_gpu_fuzz import _case
from test_gpu_parity import _gpu_run, _strats
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
s0, s1 = int(sys.argv[1]), int(sys.argv[2])
fails = 0
for seed in range(s0, s1):
    f, d, nc, agg, base, X = _case(seed)
    rng = np.random.default_rng(seed)
    F = T.Forest(f, n_features=d, n_classes=nc, agg=agg, base_score=base, device=0)
    if seed % 2:
        cal = rng.normal(size=(min(2048, 4_000_000 // (4 * d) + 1), d)).astype(np.float32)
        F.layout(cal)
    ref = oracle.predict(f, X, agg=agg, n_classes=nc, base_score=base, want_leaf=True)
    msg = []
    for s in _strats(F) + [-1]:
        r = _gpu_run(F, X, s, want_leaf=(s >= 0))   # every strategy has leaf ids (round 2)
        if not np.array_equal(r["out"], ref["out"]):
            msg.append(f"out s={s} ({int((r['out'] != ref['out']).sum())})")
        if agg != oracle.AGG_SUM and agg != oracle.AGG_AVERAGE and not np.array_equal(r["cls"], ref["cls"]):
            msg.append(f"cls s={s}")
        if "leaf" in r and not np.array_equal(r["leaf"], ref["leaf"]):
            msg.append(f"leaf s={s}")
        if "fp" in r and not np.array_equal(r["fp"], ref["fp"]):
            msg.append(f"fp s={s}")
    if agg != oracle.AGG_VOTE:   # raw sums: no base, no average
        rsum = oracle.predict(f, X, agg=oracle.AGG_SUM if nc == 1 else oracle.AGG_CLASS_SUM, n_classes=nc)["raw"]
        part = F.predict_partial(torch.from_numpy(X).cuda())
        torch.cuda.synchronize()
        if not np.array_equal(part.cpu().numpy(), rsum):
            msg.append("partial")
    out_h = torch.empty(ref["out"].shape, dtype=torch.float32)
    F.predict_host(torch.from_numpy(np.ascontiguousarray(X)), out_h)
    torch.cuda.synchronize()
    if not np.array_equal(out_h.numpy(), ref["out"]):
        msg.append("host")
    st = F.stats()
    if msg:
        fails += 1
        print("FAIL seed", seed, "d", d, "trees", len(f["root"]), "n", X.shape[0], "classes", nc, "agg", agg,
              "slices", st["n_slices"], "code8", st["code8"], msg, flush=True)
    F.close()
print("done", s0, s1, "fails", fails, flush=True)
