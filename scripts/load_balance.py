"""Load balance across threads — the Table 3 / Fig. 2c analog (P:566-574,
P:2092-2155): "A.C.V." = average coefficient of variation of per-thread execution time.

In k_sliced a lane walks one lane column for the two rows of its chains; lanes of a warp run in
lockstep, so a lane's *work* (useful node steps) is what differs between threads, and the warp's
time is set by its slowest lane.  The per-lane step counts are exact: they are obtained by walking
the library's exported sliced image (tahoe_forest_export_sliced) for real rows with the kernel's
row-to-lane mapping (unit u of a 64-row tile: half h walks rows u+16h and u+32+16h).  For the
direct strategy (lane = sample) a thread's work is the sample's total visits.

Variants: "tahoe" = the product layout (LPT / round-robin packing, similarity grouping, hot-first
order); "fil" = FIL's assignment (trees dealt round-robin, no grouping, no node
reordering).  Each variant runs in its own process (TAHOE_PACK is read once per process).

    python scripts/load_balance.py [--rows 2048] [--configs 2,3,4]
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def lane_steps(img, X):
    """steps[row, slice, column] of the exported image (useful steps before the terminal)."""
    import numpy as np
    m = X.shape[0]
    F = img["feature_bits"]
    fm = (1 << F) - 1
    sb = img["slot_bytes"]
    C = img["cols"]
    S = img["n_slices"]
    steps = np.zeros((m, S, C), np.int64)
    for s in range(S):
        for c in range(C):
            end = img["col_len"][s, c]
            xs = img["nodes"][s, :end + 1, c, 0].astype(np.uint32)
            ys = img["nodes"][s, :end + 1, c, 1].astype(np.int64)
            thr = xs.view(np.float32)
            att = (ys >> 2) & fm
            off = (ys >> (F + 3)) // sb
            dl = (ys >> (F + 2)) & 1
            k = np.zeros(m, np.int64)
            cnt = np.zeros(m, np.int64)
            act = k < end
            while act.any():
                rows = np.nonzero(act)[0]
                kk = k[act]
                a = att[kk]
                leaf = a == fm
                v = X[rows, np.where(leaf, 0, a)]
                gl = np.where(np.isnan(v), dl[kk] == 1, v < thr[kk]) & ~leaf
                k[act] = kk + np.where(gl, 1, off[kk])
                cnt[act] += 1
                act = k < end
            steps[:, s, c] = cnt
    return steps


def measure(cid, rows, variant):
    import numpy as np
    import gen
    from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
    f = gen.make_forest(cid)
    h = T.tahoe_forest_build(f, f["n_features"], f["n_classes"], f["agg"], 0.0, -1)
    opts = None
    if variant == "fil":
        opts = T.LayoutOpts(0, 0, 0, 0, 0, 0, 0)      # no node reorder, no tree grouping
    T.tahoe_forest_layout(h, gen.make_calibration(cid, 8192), opts)
    img = T.tahoe_forest_export_sliced(h)
    X = gen.make_rows(cid, rows)
    st = lane_steps(img, X)                 # [m, S, 16]
    m = (rows // 64) * 64
    cvs, useful, issued = [], 0, 0
    for t0 in range(0, m, 64):
        for u in range(16):
            for s in range(st.shape[1]):
                # lane (h, c): chain A row t0+u+16h, chain B row t0+u+32+16h
                A = np.stack([st[t0 + u, s], st[t0 + u + 16, s]])        # [2 halves, 16]
                B = np.stack([st[t0 + u + 32, s], st[t0 + u + 48, s]])
                work = (A + B).ravel().astype(np.float64)             # 32 lanes
                if work.mean() > 0:
                    cvs.append(work.std() / work.mean())
                mx = max(A.max(), B.max())
                useful += int(A.sum() + B.sum())
                issued += 64 * 2 * ((int(mx) + 1) // 2)
    # direct strategy: thread = sample, work = total visits; CV across a 256-thread block
    per_row = st.sum(axis=(1, 2))[:m].astype(np.float64)
    blocks = per_row.reshape(-1, 256) if m >= 256 else per_row.reshape(1, -1)
    dcv = float(np.mean(blocks.std(axis=1) / blocks.mean(axis=1)))
    T.tahoe_forest_free(h)
    return dict(config=cid, variant=variant, rows=m, slices=int(st.shape[1]),
                acv_sliced=float(np.mean(cvs)), lockstep_eff=useful / issued,
                acv_direct=dcv)


def main():
    rows = 2048
    configs = [2, 3, 4]
    if "--rows" in sys.argv:
        rows = int(sys.argv[sys.argv.index("--rows") + 1])
    if "--configs" in sys.argv:
        configs = [int(c) for c in sys.argv[sys.argv.index("--configs") + 1].split(",")]
    if "--one" in sys.argv:
        cid, variant = sys.argv[sys.argv.index("--one") + 1].split(":")
        print(json.dumps(measure(int(cid), rows, variant)))
        return
    res = []
    for cid in configs:
        for variant in ("fil", "tahoe"):
            env = dict(os.environ)
            env.pop("TAHOE_PACK", None)
            if variant == "fil":
                env["TAHOE_PACK"] = "rr"
            out = subprocess.run([sys.executable, __file__, "--rows", str(rows), "--one",
                                  f"{cid}:{variant}"], env=env, capture_output=True, text=True,
                                 check=True).stdout
            res.append(json.loads(out.strip().splitlines()[-1]))
            print(json.dumps(res[-1]), flush=True)
    print()
    print("| config | assignment | slices | A.C.V. of lane work (sliced) | lockstep eff. | A.C.V. per-sample work (direct, 256-thread blocks) |")
    print("|---|---|---|---|---|---|")
    for r in res:
        name = "FIL round-robin, no grouping/reorder" if r["variant"] == "fil" else "Tahoe layout (product)"
        print(f"| C{r['config']} | {name} | {r['slices']} | {100 * r['acv_sliced']:.1f} % | "
              f"{r['lockstep_eff']:.3f} | {100 * r['acv_direct']:.1f} % |")


if __name__ == "__main__":
    main()
