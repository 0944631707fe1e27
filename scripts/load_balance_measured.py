"""Load balance MEASURED on the B200 (Table 3 "A.C.V." = average coefficient of
variation of execution time across threads; Fig. 2(c)): the rank-coded
walk runs through tahoe_profile_walk, an instrumented copy that reads the SM clock every loop
iteration, so each lane's span (walk start -> its last iteration) is measured per work unit.
Reported per config and packing: the mean CV of lane spans per unit (the lockstep-relevant
variation), the mean lockstep efficiency (mean/max span per unit) and the CV of the lanes' total
spans over the launch (the paper's per-thread execution-time CV).  Packings: the product layout
(similarity order + expected-work packing + measured-path refinement, R6) against plain
round-robin dealing of the trees in input order (TAHOE_PACK=rr, no grouping / reorder: FIL's
assignment).  Each packing runs in its own process (the packer reads its environment
once).  Prints one JSON line per run."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def one(cid, n, pack):
    sys.path.insert(0, ROOT)
    import torch
    import gen
    from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
    f = gen.make_forest(cid, leaf_mode="normal")
    F = T.Forest(f, device=0)
    if pack == "product":
        F.layout(gen.make_calibration(cid))
    else:
        F.layout(gen.make_calibration(cid), node_reorder=0, tree_group=0)
    X = torch.from_numpy(gen.make_rows(cid, n, row0=7_000_000)).cuda()   # held-out rows
    out = torch.empty((n, F.n_out), device="cuda")
    T.tahoe_profile_walk(F.handle, X, n, X.shape[1], out)   # warm-up
    r = T.tahoe_profile_walk(F.handle, X, n, X.shape[1], out)
    st = F.stats()
    r.update(config=f"C{cid}", n=n, packing=pack, n_slices=st["n_slices"],
             lockstep_eff_sim=st["lockstep_eff_sim"])
    print(json.dumps(r), flush=True)


def main():
    if len(sys.argv) > 1 and sys.argv[1] == "--one":
        one(int(sys.argv[2]), int(sys.argv[3]), sys.argv[4])
        return
    for cid, n in ((2, 1_000_000), (3, 1_000_000)):
        for pack in ("product", "round-robin"):
            env = dict(os.environ)
            if pack == "round-robin":
                env["TAHOE_PACK"] = "rr"
            subprocess.run([sys.executable, __file__, "--one", str(cid), str(n), pack], env=env,
                           check=True)


if __name__ == "__main__":
    main()
