"""Low-parallelism latency workload (the paper's batch-100 "low parallelism"
runs): per-batch latency p50/p99 for batch 100 / 1K / 10K, for the cost
model's choice and every usable strategy, with plain launches and CUDA-graph replay (plus the
L2-persisting window on the auto choice).  Device-resident batches; host-observed latency per
call (launch + kernels + synchronize, 2000 calls after 50 warm-ups) and the device time of a
graph replay (CUDA events).  Prints one JSON line per (config, batch, strategy)."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402

NAMES = {0: "direct", 1: "sliced", 2: "sliced-coded", 3: "rows"}


def measure(fn, reps=2000):
    for _ in range(50):
        fn()
    torch.cuda.synchronize()
    lat = np.empty(reps)
    for r in range(reps):
        t = time.perf_counter()
        fn()
        torch.cuda.synchronize()
        lat[r] = (time.perf_counter() - t) * 1e6
    return dict(p50_us=float(np.percentile(lat, 50)), p99_us=float(np.percentile(lat, 99)),
                mean_us=float(lat.mean()))


def device_us(g, reps=500):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s = torch.cuda.current_stream()
    a.record(s)
    for _ in range(reps):
        g.replay()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) * 1000.0 / reps


def run(cid, out_lines):
    f = gen.make_forest(cid, leaf_mode="normal")
    F = T.Forest(f, device=0).layout(gen.make_calibration(cid))
    st = F.stats()
    for n in (100, 1000, 10_000):
        X = torch.from_numpy(gen.make_rows(cid, n)).cuda()
        out = torch.empty((n, F.n_out), device="cuda")
        auto = F.select_strategy(n, X.shape[1])
        strats = [-1] + [s for s in (0, 1, 2, 3) if (s != 1 or st["sliced_valid"]) and
                         (s != 2 or st["coded_valid"]) and (s != 3 or st["rows_ok"])]
        for strat in strats:
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                F.predict(X, out=out, force_strategy=strat, stream=s)
            torch.cuda.synchronize()
            plain = measure(lambda: F.predict(X, out=out, force_strategy=strat))
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=s):
                F.predict(X, out=out, force_strategy=strat, stream=s)
            graph = measure(g.replay)
            rec = dict(config=f"C{cid}", n=n, strategy=NAMES[auto if strat < 0 else strat],
                       auto=strat < 0, plain=plain, graph=graph, graph_device_us=device_us(g),
                       predicted_us=F.predict_cost_us(auto if strat < 0 else strat, n))
            if strat < 0:
                T.tahoe_forest_l2_persist(F.handle, torch.cuda.current_stream(), 1.0)
                rec["l2_persist_plain"] = measure(lambda: F.predict(X, out=out))
                T.tahoe_forest_l2_persist(F.handle, torch.cuda.current_stream(), 0.0)
            out_lines.append(rec)
            print(json.dumps(rec), flush=True)
    F.close()


def main():
    cfgs = [int(a) for a in sys.argv[1:]] or [2, 3]
    lines = []
    for cid in cfgs:
        run(cid, lines)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    json.dump(lines, open(os.path.join(ROOT, "gpurun_out", "latency.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
