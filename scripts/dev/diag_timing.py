"""Timing diagnostic: per-stage CUDA-event times of one C2 predict (not a bench number)."""
import os, sys, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gen
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T

cid = int(sys.argv[1]) if len(sys.argv) > 1 else 2
n = int(sys.argv[2]) if len(sys.argv) > 2 else gen.CONFIGS[cid].n_samples
f = gen.make_forest(cid, leaf_mode="normal")
F = T.Forest(f, device=0).layout(gen.make_calibration(cid))
st = F.stats()
print(json.dumps(st))
print(f"C{cid} slices={st['n_slices']} eff_sim={st['lockstep_eff_sim']:.3f} V={st['expected_node_reads_per_sample']:.1f}")
X = torch.from_numpy(gen.make_rows(cid, n)).cuda()
out = torch.empty((n, F.n_out), device="cuda")
cls = torch.empty(n, dtype=torch.int32, device="cuda")
s = torch.cuda.current_stream()
for strat in (2, 1, 0):
    if (strat == 1 and not st["sliced_valid"]) or (strat == 2 and not st.get("coded_valid")):
        continue
    for _ in range(3):
        F.predict(X, out=out, out_class=cls, force_strategy=strat)
    torch.cuda.synchronize()
    res = []
    for _ in range(5):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        for x in e: x.record(s)
        torch.cuda.synchronize()
        h0 = time.perf_counter()
        e[0].record(s)
        F.predict(X, out=out, out_class=cls, force_strategy=strat, ev_main_begin=e[2], ev_main_end=e[3])
        e[1].record(s)
        h1 = time.perf_counter()
        torch.cuda.synchronize()
        res.append((e[0].elapsed_time(e[1]), e[2].elapsed_time(e[3]), e[0].elapsed_time(e[2]), e[3].elapsed_time(e[1]), (h1 - h0) * 1e3))
    r = np.array(res)
    print(f"C{cid} n={n} strategy={strat}: step {r[:,0].mean():.3f} ms kernel {r[:,1].mean():.3f} ms pre {r[:,2].mean():.3f} post {r[:,3].mean():.3f} host-call {r[:,4].mean():.3f} ms")
