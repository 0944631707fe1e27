"""Write profiles/r01_costmodel.md from a fit (gpurun_out/costmodel_fit.json by default) and install
its constants as paper_conf_eurosys_xiedlll21_b200/costmodel_b200.json."""
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
src = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "costmodel_fit.json")
d = json.load(open(src))
p, rows = d["params"], d["rows"]
json.dump(p, open(os.path.join(ROOT, "paper_conf_eurosys_xiedlll21_b200", "costmodel_b200.json"), "w"), indent=1)
json.dump(d, open(os.path.join(ROOT, "profiles", "r01_costmodel_fit.json"), "w"), indent=1)


def f(v):
    return "–" if v is None or (isinstance(v, float) and (math.isinf(v) or math.isnan(v))) else f"{v:.4g}"


out = ["# Round 1 cost-model fit (B200, `python scripts/fit_costmodel.py`)", "",
       "Model (csrc/costmodel.cpp, Eq. 1 of the paper re-targeted):", "",
       "* sliced: `T = a_s + b_s * U_s * (rows in global ? g_s : 1)`, "
       "`U_s = ceil(tiles/cps) * 64 * V / (slices * eff_sim)`",
       "* coded (rank-coded slices, reading R7): `T = a_c + b_c * U_s + e_c * ceil(n/64) * 64 * passes / SMs`",
       "* wide codes (reading R8, > 127 attributes): `T = a_w + b_w * U_s + e_w * ceil(n/64) * 64 * passes / SMs`",
       "* direct: `T = a_d + (d > 256 ? g_d : 1) * max(l_d * V, b_d * V * n / SMs)`", "",
       "Kernels: the 16-lane-column `k_sliced`, the rank-coded `k_sliced_codes` with its row-coding "
       "pre-pass, the wide-code `k_sliced_codes8` with its pre-pass (C4), and the staged-row direct "
       "kernels (eight threads per row over 64-row tiles for scalar outputs) for batches >= 32K rows.", "",
       f"Fitted constants (microseconds): a_s = {p['a_s']:.3g}, b_s = {p['b_s']:.4g}, "
       f"g_s = {p['g_s']:.3g}, a_c = {p['a_c']:.3g}, b_c = {p['b_c']:.4g}, e_c = {p['e_c']:.4g}, "
       f"a_w = {p.get('a_w', float('nan')):.3g}, b_w = {p.get('b_w', float('nan')):.4g}, e_w = {p.get('e_w', float('nan')):.4g}, "
       f"a_d = {p['a_d']:.4g}, l_d = {p['l_d']:.4g}, b_d = {p['b_d']:.4g}, g_d = {p['g_d']:.4g}", "",
       f"Rank accuracy (model picks the measured-fastest strategy): **{p['rank_accuracy']}** "
       "(paper: 87/90, P:2413-2422).", "",
       "| config | n | direct ms | sliced ms | coded ms | model direct | model sliced | model coded | measured best | model best |",
       "|---|---|---|---|---|---|---|---|---|---|"]
miss = []
for r in rows:
    c = f"C{r['config']}" + (" (500-tree shard)" if r["config"] == 5 else "")
    meas = {"direct": r["direct_ms"]}
    pred = {"direct": r["pred_direct_us"]}
    if r["sliced_ms"] is not None:
        meas["sliced"] = r["sliced_ms"]
        pred["sliced"] = r["pred_sliced_us"]
    if r.get("coded_ms") is not None:
        meas["coded"] = r["coded_ms"]
        pred["coded"] = r["pred_coded_us"]
    mb, pb = min(meas, key=meas.get), min(pred, key=pred.get)
    if r["sliced_ms"] is not None and mb != pb:
        miss.append(f"C{r['config']} n={r['n']} ({mb} measured fastest, model picks {pb}: "
                    + ", ".join(f"{k} {v:.3g} ms" for k, v in meas.items()) + ")")
    sl = f(r["sliced_ms"]) if r["sliced_ms"] is not None else "n/a (trees exceed a lane column)"
    out.append(f"| {c} | {r['n']} | {f(r['direct_ms'])} | {sl} | {f(r.get('coded_ms'))} | "
               f"{f(r['pred_direct_us'] / 1000)} | {f(r.get('pred_sliced_us', math.inf) / 1000)} | "
               f"{f(r.get('pred_coded_us', math.inf) / 1000)} | {mb} | {pb} |")
out.append("")
out.append("Misses: " + "; ".join(miss) + "." if miss else "Every ordering on this sweep is predicted correctly.")
out.append("The model's job is the choice, not the absolute time: the direct term is loose at large n. "
           "Small batches stay on the fp32 slices: the coded path pays a second launch and a "
           "shared-memory table load per CTA.")
open(os.path.join(ROOT, "profiles", "r01_costmodel.md"), "w").write("\n".join(out) + "\n")
print(p)
