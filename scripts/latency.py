"""Low-parallelism latency workload (the paper's batch-100 "low parallelism"
runs): per-batch latency p50/p99 for batch 100 / 1K / 10K on C2, with
plain launches, CUDA-graph replay, and the L2-persisting forest window.  Device-resident batches;
each call's latency is host-observed (launch + kernel + sync), not a throughput number."""
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


def main():
    cid = int(sys.argv[1]) if len(sys.argv) > 1 else 2
    f = gen.make_forest(cid, leaf_mode="normal")
    F = T.Forest(f, device=0).layout(gen.make_calibration(cid))
    res = dict(config=cid, results=[])
    for n in (100, 1000, 10_000):
        X = torch.from_numpy(gen.make_rows(cid, n)).cuda()
        out = torch.empty((n, F.n_out), device="cuda")
        strat = F.select_strategy(n, X.shape[1])
        plain = measure(lambda: F.predict(X, out=out))
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            F.predict(X, out=out)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            F.predict(X, out=out)
        graph = measure(g.replay)
        T.tahoe_forest_l2_persist(F.handle, torch.cuda.current_stream(), 1.0)
        persist = measure(lambda: F.predict(X, out=out))
        T.tahoe_forest_l2_persist(F.handle, torch.cuda.current_stream(), 0.0)
        rec = dict(n=n, strategy={0: "direct", 1: "sliced"}[strat], plain=plain, graph=graph,
                   l2_persist=persist)
        res["results"].append(rec)
        print(json.dumps(rec), flush=True)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    json.dump(res, open(os.path.join(ROOT, "gpurun_out", f"latency_c{cid}.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
