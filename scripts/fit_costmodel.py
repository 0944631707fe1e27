"""Fit the strategy cost model on this chip (Algorithm 1 line 4: "Measure hardware
parameters by a microbenchmark").

Times both strategies on the BASELINE-shaped forests over a sweep of batch sizes, fits

    sliced : T = a_s + b_s * U_s,   U_s = ceil(tiles / cps) * 64 * V / (slices * eff_sim)
    direct : T = a_d + max(l_d * V, b_d * V * n / SMs)
    coded  : T = a_c + b_c * U_s + e_c * ceil(n / 64) * 64 * passes / SMs   (reading R7)
    wide   : T = a_w + b_w * U_s + e_w * ceil(n / 64) * 64 * passes / SMs   (reading R8, d > 127)

(costmodel.cpp), writes paper_conf_eurosys_xiedlll21_b200/costmodel_b200.json (read by
libtahoe.so at load) and a report with the model's rank accuracy (paper: 87/90 correct orderings,
P:2413-2422).  Usage on the GPU box:  python scripts/fit_costmodel.py [--quick]
"""
import json
import math
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
from scipy.optimize import least_squares  # noqa: E402

import gen  # noqa: E402
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402

QUICK = "--quick" in sys.argv
SWEEP = {
    1: [100, 1000, 10_000, 100_000],
    2: [100, 1000, 10_000, 100_000, 1_000_000],
    3: [1000, 10_000, 100_000, 1_000_000],
    4: [1000, 10_000, 100_000, 300_000],
    5: [1000, 10_000, 100_000],
}


def time_ms(F, X, strat, reps=5):
    out = torch.empty((X.shape[0], F.n_out), dtype=torch.float32, device=X.device)
    for _ in range(2):
        F.predict(X, out=out, force_strategy=strat)
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        F.predict(X, out=out, force_strategy=strat)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def measure():
    rows = []
    for cid, ns in SWEEP.items():
        if QUICK:
            ns = ns[::2]
        if cid == 5:
            f = gen.make_forest(5, n_trees=500, leaf_mode="normal")
        else:
            f = gen.make_forest(cid, leaf_mode="normal")
        F = T.Forest(f, device=0).layout(gen.make_calibration(cid, 8192))
        st = F.stats()
        Xall = torch.from_numpy(gen.make_rows(cid, max(ns))).cuda()
        for n in ns:
            X = Xall[:n]
            rec = dict(config=cid, n=n, V=st["expected_node_reads_per_sample"],
                       slices=st["n_slices"], eff_sim=st["lockstep_eff_sim"],
                       sms=st["num_sms"], sliced_valid=st["sliced_valid"],
                       coded_valid=st["sliced_valid"] and st["coded_valid"],
                       passes=max(1, (1 << (st["code8_vfbits"] if st["code8"] else st["sliced_fbits"])) // 32),
                       wide=bool(st["code8"]),
                       rows_global=cid == 4)  # C4: d = 2000 (> 256, too wide to stage)
            rec["direct_ms"] = time_ms(F, X, T.STRATEGY_DIRECT)
            rec["sliced_ms"] = time_ms(F, X, T.STRATEGY_SLICED) if st["sliced_valid"] else None
            rec["coded_ms"] = time_ms(F, X, T.STRATEGY_SLICED_CODED) if rec["coded_valid"] else None
            rows.append(rec)
            print(json.dumps(rec), flush=True)
        F.close()
    return rows


# Row-coding cost of the wide codes per row-pass per SM, from the C4 bench's pre-pass
# (k_encode_rows8: 2.6 ms per 500K rows x 64 passes on 148 SMs).  The sweep alone cannot separate
# it from the walk (on the one wide config both terms grow with n).
E_W_PREPASS = 2600.0 / (500_032 * 64 / 148)


def main():
    if "--refit" in sys.argv:   # re-fit saved measurements (no GPU)
        rows = json.load(open(sys.argv[sys.argv.index("--refit") + 1]))["rows"]
    else:
        rows = measure()

    def U_s(r):
        tiles = math.ceil(r["n"] / 64)
        cps = max(1, r["sms"] // r["slices"])
        return math.ceil(tiles / cps) * 64 * r["V"] / (r["slices"] * max(r["eff_sim"], 0.05))

    sl = [r for r in rows if r["sliced_ms"] is not None and not r["rows_global"]]
    A = np.array([[1.0, U_s(r)] for r in sl])
    y = np.array([r["sliced_ms"] * 1000 for r in sl])
    w = 1.0 / y
    a_s, b_s = np.linalg.lstsq(A * w[:, None], y * w, rcond=None)[0]
    a_s = max(a_s, 1.0)
    gl = [r for r in rows if r["sliced_ms"] is not None and r["rows_global"] and r["n"] >= 10_000]
    g_s = float(np.median([(r["sliced_ms"] * 1000 - a_s) / (b_s * U_s(r)) for r in gl])) if gl else 4.0

    def E_c(r):
        return math.ceil(r["n"] / 64) * 64 * r["passes"] / r["sms"]

    def fit3(cd, default):
        if len(cd) < 3:
            return default
        Ac = np.array([[1.0, U_s(r), E_c(r)] for r in cd])
        yc = np.array([r["coded_ms"] * 1000 for r in cd])
        wc = 1.0 / yc
        a, b, e = np.linalg.lstsq(Ac * wc[:, None], yc * wc, rcond=None)[0]
        return max(a, 1.0), max(b, 1e-9), max(e, 0.0)

    a_c, b_c, e_c = fit3([r for r in rows if r["coded_ms"] is not None and not r["wide"]], (30.0, 6.6e-5, 1.6e-5))
    wd = [r for r in rows if r["coded_ms"] is not None and r["wide"]]
    e_w = E_W_PREPASS
    if len(wd) >= 2:   # a_w, b_w on the walk's share (total - pre-pass term)
        Aw = np.array([[1.0, U_s(r)] for r in wd])
        yw = np.array([r["coded_ms"] * 1000 - e_w * E_c(r) for r in wd])
        ww = 1.0 / np.array([r["coded_ms"] * 1000 for r in wd])
        a_w, b_w = np.linalg.lstsq(Aw * ww[:, None], yw * ww, rcond=None)[0]
        a_w, b_w = max(a_w, 1.0), max(b_w, 1e-9)
    else:
        a_w, b_w = 40.0, 1.68e-4

    def direct_model(p, r):
        a, l, b, g = p
        return a + (g if r["rows_global"] else 1.0) * max(l * r["V"], b * r["V"] * r["n"] / r["sms"])

    yd = np.array([r["direct_ms"] * 1000 for r in rows])
    res = least_squares(lambda p: np.log([direct_model(np.abs(p), r) for r in rows]) - np.log(yd),
                        x0=[5.0, 0.1, 3e-4, 2.0])
    a_d, l_d, b_d, g_d = np.abs(res.x)
    params = dict(a_s=float(a_s), b_s=float(b_s), g_s=g_s, a_d=float(a_d), l_d=float(l_d), b_d=float(b_d),
                  g_d=float(g_d), a_c=float(a_c), b_c=float(b_c), e_c=float(e_c),
                  a_w=float(a_w), b_w=float(b_w), e_w=float(e_w),
                  units="microseconds",
                  gpu=torch.cuda.get_device_name(0) if torch.cuda.is_available() else "NVIDIA B200")

    correct = total = 0
    report = []
    for r in rows:
        ps = (params["a_s"] + params["b_s"] * U_s(r) * (g_s if r["rows_global"] else 1.0)
              if r["sliced_ms"] is not None else math.inf)
        if r["coded_ms"] is None:
            pc = math.inf
        elif r["wide"]:
            pc = a_w + b_w * U_s(r) + e_w * E_c(r)
        else:
            pc = a_c + b_c * U_s(r) + e_c * E_c(r)
        pd = direct_model([a_d, l_d, b_d, g_d], r)
        r.update(pred_sliced_us=ps, pred_direct_us=pd, pred_coded_us=pc)
        if r["sliced_ms"] is None:
            continue
        total += 1
        meas_t = {"direct": r["direct_ms"], "sliced": r["sliced_ms"]}
        if r["coded_ms"] is not None:
            meas_t["coded"] = r["coded_ms"]
        pred_t = {"direct": pd, "sliced": ps, "coded": pc}
        meas = min(meas_t, key=meas_t.get)
        pred = min(pred_t, key=pred_t.get)
        correct += meas == pred
        report.append((r["config"], r["n"], r["direct_ms"], r["sliced_ms"],
                       r["coded_ms"] if r["coded_ms"] is not None else float("nan"),
                       pd / 1000, ps / 1000, pc / 1000, meas, pred))
    params["rank_accuracy"] = f"{correct}/{total}"
    path = os.path.join(ROOT, "paper_conf_eurosys_xiedlll21_b200", "costmodel_b200.json")
    json.dump(params, open(path, "w"), indent=1)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    json.dump(dict(params=params, rows=rows), open(os.path.join(ROOT, "gpurun_out", "costmodel_fit.json"), "w"), indent=1)
    print(json.dumps(params))
    print("config n direct_ms sliced_ms coded_ms pred_direct_ms pred_sliced_ms pred_coded_ms measured_best predicted_best")
    for t in report:
        print(" ".join(f"{v:.4g}" if isinstance(v, float) else str(v) for v in t))


if __name__ == "__main__":
    main()
