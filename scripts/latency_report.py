"""profiles/r02_latency.md from gpurun_out/latency.json (scripts/latency.py)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
src = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "latency.json")
recs = json.load(open(src))
out = ["# Round 2 latency workload (SURVEY §8(f) f1; the paper's batch-100 'low parallelism', P:1714-1722)", "",
       "`python scripts/latency.py 2 3` on one B200 (round-2 final kernels and cost model): device-resident batches; "
       "host-observed latency per call (launch + kernels + synchronize, Python/ctypes call included), 2000 calls after 50 "
       "warm-ups; `device` = CUDA-event time of one graph replay (mean of 500); `model` = the cost model's prediction "
       "(tahoe_predict_cost_us).  Raw records: `profiles/r02_latency.json`.", "",
       "| config | batch | strategy | auto | plain p50 / p99 (us) | CUDA graph p50 / p99 (us) | device (us) | model (us) |",
       "|---|---|---|---|---|---|---|---|"]
for r in recs:
    out.append(f"| {r['config']} | {r['n']} | {r['strategy']} | {'yes' if r['auto'] else ''} | "
               f"{r['plain']['p50_us']:.1f} / {r['plain']['p99_us']:.1f} | {r['graph']['p50_us']:.1f} / {r['graph']['p99_us']:.1f} | "
               f"{r['graph_device_us']:.1f} | {r['predicted_us']:.1f} |")
l2 = [r for r in recs if "l2_persist_plain" in r]
if l2:
    out += ["", "L2-persisting window on the forest image (`tahoe_forest_l2_persist`, hit ratio 1.0), the cost model's pick, plain calls:", "",
            "| config | batch | strategy | plain p50 (us) | with L2 persist p50 (us) |", "|---|---|---|---|---|"]
    for r in l2:
        out.append(f"| {r['config']} | {r['n']} | {r['strategy']} | {r['plain']['p50_us']:.1f} | {r['l2_persist_plain']['p50_us']:.1f} |")
open(os.path.join(ROOT, "profiles", "r02_latency.md"), "w").write("\n".join(out) + "\n")
print("\n".join(out[:14]))
