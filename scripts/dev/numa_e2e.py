"""Experiment: e2e (tahoe_predict_host) with the pinned buffers first-touched on the GPU's NUMA node
(process affinity = NVML's CPU affinity of the GPU) vs the default placement."""
import os, sys, time, json
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import numpy as np, torch, pynvml
import gen
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T

pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
ncpu = os.cpu_count()
words = (ncpu + 63) // 64
mask = pynvml.nvmlDeviceGetCpuAffinity(h, words)
local = [c for c in range(ncpu) if (mask[c // 64] >> (c % 64)) & 1]
print("cpus", ncpu, "gpu-local", len(local), local[:8], "...", flush=True)
try:
    print(open("/sys/devices/system/node/online").read().strip(), flush=True)
except Exception:
    pass
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
f = gen.make_forest(cfg)
F = T.Forest(f, device=0).layout(gen.make_calibration(cfg))
X = gen.make_rows(cfg, 1_000_000 if cfg == 2 else 4_000_000)
allc = sorted(os.sched_getaffinity(0))
for mode in ("default", "local", "default", "local"):
    os.sched_setaffinity(0, local if mode == "local" else allc)
    Xh = torch.from_numpy(X).pin_memory()
    oh = torch.empty((X.shape[0], F.n_out), dtype=torch.float32).pin_memory()
    for _ in range(3):
        F.predict_host(Xh, oh)
    torch.cuda.synchronize()
    ts = []
    for _ in range(20):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); F.predict_host(Xh, oh); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    print(mode, round(X.shape[0] / (np.mean(ts) / 1e3) / 1e6, 1), "M samples/s", flush=True)
    del Xh, oh
    os.sched_setaffinity(0, allc)
