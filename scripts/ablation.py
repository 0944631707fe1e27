"""Layout-technique ablation (the paper's Fig. 8):
kernel time of both strategies with probability-based node rearrangement and
similarity-based tree rearrangement switched on/off, plus the packing's simulated
lockstep efficiency.  python scripts/ablation.py [configs...]"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402

ROWS = {2: 1_000_000, 3: 1_000_000, 4: 100_000, 5: 100_000}


def kernel_ms(F, X, strat, reps=5):
    out = torch.empty((X.shape[0], F.n_out), device=X.device)
    for _ in range(2):
        F.predict(X, out=out, force_strategy=strat)
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        F.predict(X, out=out, force_strategy=strat)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def main():
    cids = [int(c) for c in sys.argv[1:]] or [2, 3, 4]
    res = []
    for cid in cids:
        f = gen.make_forest(cid, n_trees=500 if cid == 5 else None, leaf_mode="normal")
        Xc = gen.make_calibration(cid, 8192)
        X = torch.from_numpy(gen.make_rows(cid, ROWS[cid])).cuda()
        F = T.Forest(f, device=0)
        for nr in (0, 1):
            for tg in (0, 1):
                F.layout(Xc, node_reorder=nr, tree_group=tg)
                st = F.stats()
                rec = dict(config=cid, n=ROWS[cid], node_reorder=nr, tree_group=tg,
                           direct_ms=kernel_ms(F, X, T.STRATEGY_DIRECT),
                           sliced_ms=kernel_ms(F, X, T.STRATEGY_SLICED) if st["sliced_valid"] else None,
                           coded_ms=kernel_ms(F, X, T.STRATEGY_SLICED_CODED) if st["coded_valid"] and st["sliced_valid"] else None,
                           n_slices=st["n_slices"], eff_sim=st["lockstep_eff_sim"])
                res.append(rec)
                print(json.dumps(rec), flush=True)
        F.close()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    json.dump(res, open(os.path.join(ROOT, "gpurun_out", "ablation.json"), "w"), indent=1)
    out = ["# Round 2 layout ablation (SURVEY §8(f) f3; the paper's Fig. 8, P:1732-1739)", "",
           "`python scripts/ablation.py 2 3 4 5` on one B200 (round-2 final kernels): kernel time (CUDA events, "
           "median of 5) of every strategy with probability-based node rearrangement (node_reorder, P:616-628) and "
           "similarity-based tree rearrangement (tree_group, P:773-806) switched off/on; C5 uses one 500-tree shard "
           "(the sliced strategies do not apply: its trees exceed a lane column).", "",
           "| config | rows | node_reorder | tree_group | direct ms | fp32 sliced ms | rank-coded ms | slices | simulated lockstep eff. |",
           "|---|---|---|---|---|---|---|---|---|"]
    f3 = lambda v: "–" if v is None else f"{v:.3f}"
    for r in res:
        out.append(f"| C{r['config']} | {r['n']} | {r['node_reorder']} | {r['tree_group']} | {f3(r['direct_ms'])} | "
                   f"{f3(r['sliced_ms'])} | {f3(r.get('coded_ms'))} | {r['n_slices']} | {r['eff_sim']:.3f} |")
    open(os.path.join(ROOT, "gpurun_out", "ablation.md"), "w").write("\n".join(out) + "\n")


if __name__ == "__main__":
    main()
