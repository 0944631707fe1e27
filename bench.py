#!/usr/bin/env python
"""Benchmark of the hot path: batched decision-tree-ensemble prediction (Tahoe, EuroSys '21).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config 3]
    python -m torch.distributed.run --nnodes=1 --nproc-per-node N --master-addr 127.0.0.1 \
        --master-port P bench.py --gpus N ...

Workload (BASELINE.json metric "samples/sec per forest at 1/2/4/8 B200"; the one config quoted over
1/2/4/8 GPUs is configs[2]): C3, a covtype-shaped 7-class forest of 7 x 200 random post-pruned
trees (depth <= 12, 54 attributes) over 4M synthetic samples, split contiguously over the N ranks
(rank r predicts rows [r n / N, (r + 1) n / N): the paper's even partition; strong
scaling, no data-path collective).  --weak gives every rank its own 4M rows.  --config 2 / 4 / 5
run the other BASELINE configs (C5: tree-sharded, fused NVLink reduce).  A step = one tahoe_predict
of the rank's rows (all §8(a) rows: row coding, traversal, combine, finalize).  Rank 0 prints one
JSON line.

--impl reference: the CPU oracle (oracle/, the "reference arm" of this tier) timed on the box's
host cores on a bounded sample of the same workload per step (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import gen  # noqa: E402

METRIC = "samples/sec per forest"
UNIT = "samples/s"


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return dict(hbm_gbs=float(d["hbm_gbs"]), sm_max_mhz=float(d.get("sm_max_mhz", 1965.0)),
                    source="measured (MEASURED_PEAKS.json)")
    return dict(hbm_gbs=6650.0, sm_max_mhz=1965.0, source="fallback (B200_PROFILING.md)")


class ClockSampler:
    """SM clocks and clock-event (throttle) reasons sampled DURING the timed region
    (B200_PROFILING.md clocks line): NVML every 10 ms in a thread (the device is found by PCI bus
    id, so CUDA and NVML orderings cannot disagree); nvidia-smi -lms 50 if NVML is unavailable."""

    _REASONS = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
                ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
                ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
                ("hw_power_brake", "nvmlClocksEventReasonHwPowerBrakeSlowdown"),
                ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"))

    def __init__(self, index: int):
        self.index = index
        self.sm, self.mx, self.reasons = [], [], set()
        self.proc = None
        self.thread = None
        self.stop_flag = threading.Event()
        self.nvml = None

    def _handle(self):
        import pynvml
        pynvml.nvmlInit()
        try:
            import torch
            pr = torch.cuda.get_device_properties(self.index)
            bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
            return pynvml, pynvml.nvmlDeviceGetHandleByPciBusId(bus.encode())
        except Exception:
            return pynvml, pynvml.nvmlDeviceGetHandleByIndex(self.index)

    def start(self):
        try:
            nv, h = self._handle()
            self.nvml = (nv, h)
            self.mx.append(float(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)))
        except Exception:
            self.nvml = None
        if self.nvml:
            self.thread = threading.Thread(target=self._poll_nvml, daemon=True)
            self.thread.start()
            return
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read_smi, daemon=True)
        self.thread.start()

    def _poll_nvml(self):
        nv, h = self.nvml
        while not self.stop_flag.is_set():
            try:
                self.sm.append(float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)))
                bits = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                for name, attr in self._REASONS:
                    if bits & getattr(nv, attr, 0):
                        self.reasons.add(name)
            except Exception:
                pass
            self.stop_flag.wait(0.01)

    def _read_smi(self):
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.proc.stdout:
            r = [p.strip() for p in line.split(",")]
            if len(r) >= 7 and r[0].replace(".", "").isdigit():
                self.sm.append(float(r[0]))
                if r[1].replace(".", "").isdigit():
                    self.mx.append(float(r[1]))
                self.reasons.update(names[j] for j in range(4) if r[3 + j] == "Active")

    def stop(self) -> dict | None:
        self.stop_flag.set()
        if self.proc:
            time.sleep(0.06)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()
        if self.thread:
            self.thread.join(timeout=2)
        if not self.sm:
            return None
        return {"sm_mhz": statistics.median(self.sm), "sm_max_mhz": max(self.mx) if self.mx else None,
                "reasons": sorted(self.reasons), "samples": len(self.sm),
                "source": "nvml 10 ms" if self.nvml else "nvidia-smi 50 ms"}


def rank_rows(cfg, n: int, rank: int, world: int, weak: bool) -> tuple[int, int]:
    """Rows [lo, hi) of the config's seeded test matrix that `rank` predicts: a contiguous 1/world
    of n (strong scaling), or its own n rows with --weak."""
    if weak:
        return rank * n, (rank + 1) * n
    return (n * rank) // world, (n * (rank + 1)) // world


def host_cores() -> int:
    """The box's host cores available to this process (torchrun sets OMP_NUM_THREADS=1 per rank,
    so the oracle is given its thread count explicitly)."""
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def oracle_rate(f, X, target_s: float, max_rows: int):
    """Oracle (as it stands) on a bounded seeded sample of X, all host cores.  Returns (rows/s,
    rows, seconds, mean visits, sample indices, oracle result)."""
    import oracle
    probe = min(2000, X.shape[0])
    t = time.perf_counter()
    oracle.predict(f, X[:probe], nthreads=host_cores())
    dt = max(time.perf_counter() - t, 1e-6)
    rows = int(min(max_rows, X.shape[0], max(probe, probe / dt * target_s)))
    idx = gen.subsample(4242, X.shape[0], rows)
    t = time.perf_counter()
    r = oracle.predict(f, X, rows=idx, nthreads=host_cores())
    dt = time.perf_counter() - t
    return rows / dt, rows, dt, float(r["visits"].mean()), idx, r


def oracle_single_core(f, X, rows: int = 10_000):
    """Single-core oracle rate on the first `rows` rows (SURVEY §8(d) "two numbers per config")."""
    import oracle
    m = min(rows, X.shape[0])
    t = time.perf_counter()
    oracle.predict(f, X[:m], nthreads=1)
    return m / (time.perf_counter() - t), m


def parity_record(f, out_rows: np.ndarray, cls_rows: np.ndarray, ref: dict) -> dict:
    """GPU outputs on the oracle's sample rows against the oracle (north_star bars): scores within
    max(1e-5 |ref|, 1e-6); classes exact outside the fp64 rounding window of reading R3 (bound
    4 gamma_T T max|v|), rows inside it counted."""
    import oracle
    tol = np.maximum(1e-5 * np.abs(ref["out"]), 1e-6)
    err = np.abs(out_rows - ref["out"])
    bad = (err > tol).any(axis=1)
    leaves = f["feature"] < 0
    T = len(f["root"])
    u = 2.0 ** -53
    bound = 4.0 * (T * u / (1 - T * u)) * T * float(np.abs(f["leaf_value"][leaves]).max())
    agg = f["agg"]
    window = 0
    cls_bad = 0
    if agg in (oracle.AGG_BINARY, oracle.AGG_CLASS_SUM):
        if agg == oracle.AGG_BINARY:
            sure = np.abs(ref["raw"][:, 0]) > bound
        else:
            srt = np.sort(ref["raw"], axis=1)
            sure = (srt[:, -1] - srt[:, -2]) > bound
        window = int((~sure).sum())
        cls_bad = int((cls_rows[sure] != ref["cls"][sure]).sum())
    rel = err / np.maximum(np.abs(ref["out"]), 1e-30)
    return dict(rows=int(len(out_rows)), mismatches=int(bad.sum()) + cls_bad,
                score_mismatches=int(bad.sum()), class_mismatches=cls_bad,
                max_abs_err=float(err.max()) if err.size else 0.0,
                max_rel_err=float(rel.max()) if rel.size else 0.0,
                classes_in_R3_window=window, r3_bound=bound,
                tolerance="max(1e-5 |ref|, 1e-6) vs the oracle's fp64 sum rounded once")


def visit_peak(device: int, variant: int) -> dict | None:
    """Live microbenchmark (Algorithm 1 line 4): node reads per second of the production coded walk
    on ideal data, plus raw shared-memory bytes per SM clock (tahoe_measure_visit_rate)."""
    from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
    try:
        T.tahoe_measure_visit_rate(device, variant, 256, 200)   # warm clocks
        best = 0.0
        bw = None
        for _ in range(3):
            r, b = T.tahoe_measure_visit_rate(device, variant, 256, 2000)
            if r > best:
                best, bw = r, b
        return dict(node_reads_per_s=best, smem_bytes_per_clk_sm=bw, variant=variant)
    except Exception as e:  # pragma: no cover
        return dict(error=str(e))


def run_reference(args, cfg):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    n = cfg.n_samples
    f = gen.make_forest(cfg, leaf_mode="normal")
    X = gen.make_rows(cfg, min(n, 200_000))
    cores = host_cores()
    rate0 = oracle_rate(f, X, 1.0, 20000)[0]
    rows = int(min(X.shape[0], max(1000, rate0 * 4.0)))   # ~4 s of oracle work per step
    idx = gen.subsample(99, X.shape[0], rows)
    for _ in range(args.warmup):
        oracle.predict(f, X, rows=idx[: max(1, rows // 8)], nthreads=cores)
    times = []
    for _ in range(args.steps):
        t = time.perf_counter()
        oracle.predict(f, X, rows=idx, nthreads=cores)
        times.append(time.perf_counter() - t)
    ms = 1000.0 * statistics.mean(times)
    value = rows / (ms / 1000.0)
    sample = f"{rows} seeded rows per step of the {cfg.name} workload ({n} rows)"
    line = dict(metric=METRIC, value=value, unit=UNIT, n_gpus=args.gpus, steps=args.steps,
                warmup=args.warmup, ms_per_step=ms, ms_median=1000.0 * statistics.median(times),
                ms_min=1000.0 * min(times), higher_is_better=True,
                scaling="weak" if args.weak else "strong",
                vs_baseline=None, dtype="f32", data="synthetic", impl="reference",
                config=_config(cfg, n, None, args.gpus, args.weak),
                cpu_baseline=dict(value=value, unit=UNIT, cores=cores, kind="oracle",
                                  sample=sample),
                e2e=dict(value=value, unit=UNIT, h2d_bytes_per_step=0, d2h_bytes_per_step=0))
    print(json.dumps(line), flush=True)
    return 0


def run_tree_sharded(args, cfg):
    """BASELINE C5 launch configuration: the forest's trees are split over the ranks
    (tahoe_forest_shard), every rank predicts fp64 partials of its trees for ALL rows.
    --reduce fused (default): the partials land in an NCCL symmetric window and one
    kernel per rank sums the peers' partials of its row block over NVLink (LSA barrier, rank-order
    fp64 sum) and finalises them (tahoe_predict_reduce).  --reduce nccl: one ncclReduce onto
    rank 0, which finalises all rows.  Strong scaling (total work fixed) unless --weak."""
    import torch
    import torch.distributed as dist
    from paper_conf_eurosys_xiedlll21_b200 import dist as D
    from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    T.load(build_if_missing=(rank == 0 and world == 1))
    args.warmup = max(args.warmup, 3)
    # --weak: the paper's weak-scaling setup, "duplicate the set N_G times": every
    # GPU walks its 1/G of the trees over G copies of the rows, so per-GPU work stays fixed
    reps = world if args.weak else 1
    n = cfg.n_samples * reps
    f = gen.make_forest(cfg, leaf_mode="normal")
    t0 = time.perf_counter()
    # rank 0 lays the full forest out once; the other ranks apply its layout state (dist.shared_layout)
    full = D.shared_layout(T.Forest(f, device=-1), gen.make_calibration(cfg) if rank == 0 else None)
    S = full.shard(rank, world, device=local)
    layout_s = time.perf_counter() - t0
    Xh = gen.make_rows(cfg, cfg.n_samples)
    Xd = torch.from_numpy(Xh).to(dev).repeat(reps, 1)
    stream = torch.cuda.current_stream()
    fused = args.reduce == "fused"
    if fused:
        comm = D.init_comm(local)
        lo, hi = T.tahoe_reduce_rows(n, world, rank, T.REDUCE_SCATTER)
        out = torch.empty((hi - lo, S.n_out), dtype=torch.float32, device=dev)
    else:
        part = torch.empty((n, S.n_out), dtype=torch.float64, device=dev)
        out = torch.empty((n, S.n_out), dtype=torch.float32, device=dev)

    def step():
        if fused:
            S.predict_reduce(comm, Xd, mode=T.REDUCE_SCATTER, out=out)
            return
        S.predict_partial(Xd, part)
        if world > 1:
            D.reduce_partials(part, dst=0)
        if rank == 0:
            S.finalize(part, out)   # the shard carries the full forest's aggregation and tree count

    for _ in range(args.warmup):
        step()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    sampler = ClockSampler(local)
    sampler.start()
    for e in ev:
        e[0].record(stream)
        step()
        e[1].record(stream)
    torch.cuda.synchronize()
    clocks = sampler.stop()
    ms = sum(a.elapsed_time(b) for a, b in ev) / args.steps
    if world > 1:
        ms = D.max_over_ranks(ms, device=dev)
    # end to end through the public API with pinned HOST buffers (one GPU: the whole forest on
    # this rank, tahoe_predict_host: chunked H2D of the rows / traversal / D2H of the outputs)
    e2e = None
    if world == 1 and not args.weak:
        Xp = torch.from_numpy(Xh).pin_memory()
        oh = torch.empty((n, S.n_out), dtype=torch.float32).pin_memory()
        S.predict_host(Xp, oh)
        torch.cuda.synchronize()
        e2e_ms = []
        for _ in range(max(2, min(args.steps, 3))):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            S.predict_host(Xp, oh)
            b.record(stream)
            torch.cuda.synchronize()
            e2e_ms.append(a.elapsed_time(b))
        e2e = dict(value=n / (sum(e2e_ms) / len(e2e_ms) / 1000.0), unit=UNIT,
                   h2d_bytes_per_step=int(Xp.numel() * 4), d2h_bytes_per_step=int(oh.numel() * 4))
        del Xp, oh
    if rank == 0:
        st = S.stats()
        # the oracle (as it stands) on a bounded sample of the same rows and the FULL forest
        cpu = None
        parity = None
        visits = st["expected_visits_per_sample"]   # this rank's shard, calibration estimate
        if not args.no_cpu and world == 1:
            import oracle
            rate, rows, secs, vis, idx, ref = oracle_rate(f, Xh, 12.0, 200_000)
            r1, m1 = oracle_single_core(f, Xh, 500)
            cpu = dict(value=rate, unit=UNIT, cores=host_cores(), kind="oracle",
                       sample=f"{rows} seeded rows of this workload, full {cfg.n_trees}-tree forest "
                              f"({secs:.1f} s of oracle work)",
                       single_core=dict(value=r1, unit=UNIT, cores=1, sample=f"first {m1} rows"))
            visits = vis
            if not args.weak:
                oh_dev = out.cpu().numpy()
                parity = parity_record(f, oh_dev[idx], np.zeros(len(idx), np.int32), ref)
        # roofline of the traversal (k_direct_tlp over the L2-sized chunks of the shard's image):
        # node reads per sample (internal visits + one leaf read per tree) against the node-read
        # rate of the same direct walk when every node read hits L1 (tahoe_measure_visit_rate
        # variant 2, measured live); the time is the whole step (traversal launches + the
        # reduce/finalize kernel, < 1 % of it)
        n_sms = st["num_sms"]
        reads_per_sample = visits + st["n_trees"]
        achieved = n * reads_per_sample / (ms / 1000.0) / 1e9
        vp = visit_peak(local, 2)
        if vp and "node_reads_per_s" in vp:
            peak, peak_src = vp["node_reads_per_s"] / 1e9, (
                "measured live: tahoe_measure_visit_rate variant 2 (the direct walk, every node read "
                "an L1 hit: 8 threads per row over staged rows, 4 CTAs of 512 threads per SM)")
        else:
            peaks = _peaks()
            peak = 128.0 * n_sms * peaks["sm_max_mhz"] * 1e6 / 12.0 / 1e9
            peak_src = "derived: 128 B/clk/SM / 12 B per node read (microbenchmark unavailable)"
        roofline = dict(bound="alu", pipe="L1/TEX data pipe (node loads) (DESIGN.md §5 Roofline)",
                        kernel="k_direct_tlp", achieved=achieved, peak=peak, unit="G node reads/s",
                        frac=achieved / peak, traffic=None, kernel_ms=ms,
                        units_per_launch=f"{n} samples x {reads_per_sample:.0f} node reads ({visits:.0f} visits"
                                         f" + {st['n_trees']} leaf reads) per step",
                        peak_source=peak_src, microbench=vp)
        peaks = _peaks()
        hbm_bytes = n * (cfg.n_features * 4) + (hi - lo if fused else n) * 4
        hbm = dict(achieved=hbm_bytes / (ms / 1000.0) / 1e9, peak=peaks["hbm_gbs"], unit="GB/s",
                   frac=hbm_bytes / (ms / 1000.0) / 1e9 / peaks["hbm_gbs"], bytes_per_step=hbm_bytes,
                   peak_source=peaks["source"])
        line = dict(metric=METRIC, value=n / (ms / 1000.0), unit=UNIT, n_gpus=world, steps=args.steps,
                    warmup=args.warmup, ms_per_step=ms, higher_is_better=True,
                    scaling="weak" if args.weak else "strong",
                    vs_baseline=None, dtype="f32", accum="f64", data="synthetic", impl="ours",
                    config={"workload": f"{cfg.name}: {cfg.n_trees} trees depth<={cfg.max_depth}, "
                                        f"{cfg.n_features} features, {n} samples"
                                        + (f" ({reps} copies of {cfg.n_samples})" if reps > 1 else "")
                                        + ", tree-sharded over "
                                        f"{world} GPU(s) + "
                                        + ("fused NVLink reduce + finalize of fp64 partials "
                                           if fused else "NCCL reduce of fp64 partials ")
                                        + f"(BASELINE configs[{cfg.cid - 1}])",
                            "n": n, "trees_per_shard": st["n_trees"],
                            "parallelism": f"tree-sharded x{world}",
                            "reduce": "fused (NCCL device API, LSA)" if fused else "ncclReduce"},
                    strategy="direct", roofline=roofline, hbm=hbm, cpu_baseline=cpu, parity=parity,
                    e2e=e2e,
                    gpu_launches=(2 if (fused or rank == 0) else 1) * args.steps, clocks=clocks,
                    layout_s=layout_s)
        print(json.dumps(line), flush=True)
    if fused:
        comm.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def _config(cfg, n, stats, world: int = 1, weak: bool = False):
    """n: rows of the whole job (strong) or per GPU (weak)."""
    n_local = n if weak else -(-n // world)
    split = (f"{n} samples per GPU (weak scaling)" if weak else
             f"{n} samples split contiguously over {world} GPU(s)")
    c = {"workload": f"{cfg.name}: {cfg.n_trees} trees depth<={cfg.max_depth}, "
                     f"{cfg.n_features} features, {split} (BASELINE configs[{cfg.cid - 1}])",
         "n_total": n * world if weak else n, "n_per_gpu": n_local, "n_trees": cfg.n_trees,
         "n_features": cfg.n_features, "max_depth": cfg.max_depth,
         "agg": {gen.AGG_SUM: "sum", gen.AGG_AVERAGE: "average", gen.AGG_BINARY: "binary margin + class",
                 gen.AGG_CLASS_SUM: f"{cfg.n_classes}-class sums + argmax",
                 gen.AGG_VOTE: "vote"}.get(cfg.agg, str(cfg.agg)),
         "parallelism": f"sample-sharded x{world} (no collective)",
         "l2": f"256 MiB L2 flush between timed steps (inputs {n_local * cfg.n_features * 4 / 1e6:.0f} MB "
               f"per GPU {'<' if n_local * cfg.n_features * 4 < 126e6 else '>'} L2), outside the events"}
    if stats:
        c.update({k: stats[k] for k in ("nodes", "leaves", "n_slices", "slots_max",
                                        "column_balance_expected", "lockstep_eff_sim",
                                        "expected_visits_per_sample", "sliced_bytes") if k in stats})
    return c


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--strategy", type=int, default=-1)
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline / parity leg")
    ap.add_argument("--mode", default=None, choices=["sample", "tree"],
                    help="sample sharding (default; C1-C4) or tree sharding (default for C5)")
    ap.add_argument("--rows", type=int, default=None, help="override the config's row count")
    ap.add_argument("--weak", action="store_true",
                    help="weak scaling: every GPU gets the config's full row count (sample mode: its "
                         "own rows; tree mode: the rows duplicated once per GPU, P:2450-2456)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help=argparse.SUPPRESS)   # gloo: N>1 code path on one GPU (tests only)
    ap.add_argument("--reduce", default="fused", choices=["fused", "nccl"],
                    help="tree mode: fused NVLink reduce + finalize kernel, or ncclReduce + finalize")
    args = ap.parse_args()
    cfg = gen.CONFIGS[args.config]
    if args.rows:
        from dataclasses import replace
        cfg = replace(cfg, n_samples=args.rows)
    if args.impl == "reference":
        return run_reference(args, cfg)
    if (args.mode or ("tree" if cfg.cid == 5 else "sample")) == "tree":
        return run_tree_sharded(args, cfg)

    import torch
    import torch.distributed as dist
    from paper_conf_eurosys_xiedlll21_b200 import tahoe as T

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:   # test hook: several ranks sharing one GPU (NCCL refuses duplicate GPUs)
            dist.init_process_group("gloo")
    T.load(build_if_missing=(rank == 0 and world == 1))
    args.warmup = max(args.warmup, 3)
    n = cfg.n_samples
    lo, hi = rank_rows(cfg, n, rank, world, args.weak)
    n_local = hi - lo
    n_total = n * world if args.weak else n
    f = gen.make_forest(cfg, leaf_mode="normal")
    X = gen.make_rows(cfg, n_local, row0=lo)
    t0 = time.perf_counter()
    F = T.Forest(f, device=local)
    F.layout(gen.make_calibration(cfg))
    layout_s = time.perf_counter() - t0
    stats = F.stats()
    strategy = args.strategy if args.strategy >= 0 else F.select_strategy(n_local, cfg.n_features)
    Xd = torch.from_numpy(X).to(dev)
    coll_dev = dev if args.dist_backend == "nccl" else torch.device("cpu")
    out = torch.empty((n_local, F.n_out), dtype=torch.float32, device=dev)
    cls = torch.empty(n_local, dtype=torch.int32, device=dev)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True),
           torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    for e in ev:
        for x in e:
            x.record(stream)
    torch.cuda.synchronize()

    def step(e=None):
        if e is None:
            F.predict(Xd, out=out, out_class=cls, force_strategy=strategy)
        else:
            e[0].record(stream)
            F.predict(Xd, out=out, out_class=cls, force_strategy=strategy,
                      ev_main_begin=e[2], ev_main_end=e[3])
            e[1].record(stream)

    for _ in range(args.warmup):
        step()
        flush.zero_()
    sampler = ClockSampler(local)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    wall0 = time.perf_counter()
    for k in range(args.steps):
        step(ev[k])
        flush.zero_()   # L2 flush between timed steps (outside the step events)
    torch.cuda.synchronize()
    wall = time.perf_counter() - wall0
    clocks = sampler.stop()
    if world > 1:
        dist.barrier()
    step_ms = [e[0].elapsed_time(e[1]) for e in ev]
    kern_ms = [e[2].elapsed_time(e[3]) for e in ev]
    tot = torch.tensor([sum(step_ms), sum(kern_ms), statistics.median(step_ms), min(step_ms)],
                       dtype=torch.float64, device=coll_dev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.MAX)
    ms_per_step = float(tot[0]) / args.steps
    kern_avg_ms = float(tot[1]) / args.steps
    value = n_total / (ms_per_step / 1000.0)
    out_h = out.cpu().numpy()
    cls_h = cls.cpu().numpy()

    # ---- end to end through the public API with HOST buffers (pinned), copies inside
    Xh = torch.from_numpy(X).pin_memory()
    oh = torch.empty((n_local, F.n_out), dtype=torch.float32).pin_memory()
    ch = torch.empty(n_local, dtype=torch.int32).pin_memory()
    for _ in range(2):
        F.predict_host(Xh, oh, ch)
    torch.cuda.synchronize()
    e2e_ms = []
    for _ in range(max(3, min(args.steps, 20))):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        F.predict_host(Xh, oh, ch)
        b.record(stream)
        torch.cuda.synchronize()
        e2e_ms.append(a.elapsed_time(b))
    e2e_t = torch.tensor([statistics.mean(e2e_ms)], dtype=torch.float64, device=coll_dev)
    if world > 1:
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
    e2e_value = n_total / (float(e2e_t[0]) / 1000.0)
    e2e_same = bool(np.array_equal(oh.numpy(), out_h) and np.array_equal(ch.numpy(), cls_h))
    del Xh

    if rank != 0:
        if world > 1:
            dist.barrier()
            dist.destroy_process_group()
        return 0

    peaks = _peaks()
    # algorithmic bytes (HBM roofline the metric asks for): sample row read + outputs written
    hbm_bytes = n_local * (cfg.n_features * 4 + F.n_out * 4 + 4)
    hbm_gbs = hbm_bytes / (ms_per_step / 1000.0) / 1e9
    cpu = None
    parity = None
    visits = stats["expected_visits_per_sample"]
    visits_src = "calibration estimate"
    if not args.no_cpu and world == 1:
        import oracle
        rate, rows, secs, vis, idx, ref = oracle_rate(f, X, 12.0, 1_000_000)
        r1, m1 = oracle_single_core(f, X)
        cpu = dict(value=rate, unit=UNIT, cores=host_cores(), kind="oracle",
                   sample=f"{rows} seeded rows of this workload ({secs:.1f} s of oracle work)",
                   single_core=dict(value=r1, unit=UNIT, cores=1, sample=f"first {m1} rows"))
        parity = parity_record(f, out_h[idx], cls_h[idx], ref)
        parity["e2e_outputs_equal_device_outputs"] = e2e_same
        visits, visits_src = vis, f"oracle, mean over the {rows} sampled rows"
    # dominant kernel roofline: the walk is bound by the shared-memory LSU pipe; its
    # unit is a node read (internal visit or leaf read), V_int + T per sample; the peak is the
    # node-read rate of the same walk on ideal data, measured live (tahoe_measure_visit_rate)
    code8 = bool(stats.get("code8"))
    kname = {1: "k_sliced", 2: "k_sliced_codes8" if code8 else "k_sliced_codes",
             3: "k_rows"}.get(strategy, "k_direct")
    reads_per_sample = visits + cfg.n_trees
    achieved = n_local * reads_per_sample / (kern_avg_ms / 1000.0) / 1e9
    # peak: the microbenchmark of the walk this strategy runs (0: u16 coded slices, also the
    # closest for the fp32 slices; 1: wide codes; 2: the direct walk through L1, also for ROWS)
    variant = {2: 1 if code8 else 0, 1: 0}.get(strategy, 2)
    vp = visit_peak(local, variant)
    if vp and "node_reads_per_s" in vp:
        what = {0: "the production coded walk on ideal data: conflict-free, perfect lockstep, 32 "
                   "warps/SM on every SM", 1: "the wide-code walk on ideal data, four chains per lane",
                2: "the direct walk with every node read an L1 hit"}[variant]
        peak, peak_src = vp["node_reads_per_s"] / 1e9, (
            "measured live: tahoe_measure_visit_rate variant %d (%s)" % (variant, what))
    else:
        n_sms = stats["num_sms"]
        peak = 128.0 * n_sms * peaks["sm_max_mhz"] * 1e6 / 12.0 / 1e9
        peak_src = (f"derived: 128 B/clk x {n_sms} SMs x {peaks['sm_max_mhz']:.0f} MHz / 12 B per "
                    f"node read (no microbenchmark for this strategy)")
    traffic = None
    sector_eff = None
    path_sector_eff = None   # every LSU global load of the step (pre-pass + walk), same capture
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):
        try:
            rec = json.load(open(tp)).get(f"C{cfg.cid}", {})
            # only a capture of the kernel this run times (e.g. "k_sliced_codes<0>")
            if rec.get("kernel", "").split("<")[0] == kname and rec.get("n") in (None, n_local):
                traffic = rec.get("dram_bytes_per_launch")
                sector_eff = rec.get("global_ld_sector_efficiency")
                path_sector_eff = rec.get("path_global_ld_sector_efficiency")
        except Exception:
            traffic = None
    launches_per_step = 1 if strategy == T.STRATEGY_DIRECT and F.n_out == 1 else (
        1 + (1 if (strategy != T.STRATEGY_DIRECT and stats["n_slices"] > 1) or F.n_out > 1 else 0))
    if strategy == T.STRATEGY_SLICED_CODED:
        launches_per_step += 1   # the row-coding pre-pass (the flag memset is not a kernel of ours)
    line = dict(
        metric=METRIC, value=value, unit=UNIT, n_gpus=world, steps=args.steps, warmup=args.warmup,
        ms_per_step=ms_per_step, ms_median=float(tot[2]), ms_min=float(tot[3]),
        per_gpu=dict(value=value / world, unit=UNIT, n_per_gpu=n_local),
        higher_is_better=True, scaling="weak" if args.weak else "strong", vs_baseline=None,
        dtype="f32", accum="f64", data="synthetic", impl="ours",
        config=_config(cfg, n, stats, world, args.weak),
        strategy={0: "direct", 1: "sliced", 2: "sliced-coded", 3: "rows"}.get(strategy, str(strategy)),
        roofline=dict(bound="alu", pipe="shared-memory LSU data pipe (DESIGN.md §5 Roofline)",
                      kernel=kname, achieved=achieved, peak=peak, unit="G node reads/s",
                      frac=achieved / peak, traffic=traffic, kernel_ms=kern_avg_ms,
                      global_ld_sector_efficiency=sector_eff,
                      path_global_ld_sector_efficiency=path_sector_eff,
                      units_per_launch=f"{n_local} samples x {reads_per_sample:.0f} node reads "
                                       f"({visits:.0f} internal visits ({visits_src}) + "
                                       f"{cfg.n_trees} leaf reads)",
                      peak_source=peak_src, microbench=vp,
                      bytes_view=dict(achieved_gbs=achieved * 12.0, unit="GB/s",
                                      note="node reads x 12 B (8 B node + 4 B attribute)")),
        hbm=dict(achieved=hbm_gbs, peak=peaks["hbm_gbs"], unit="GB/s",
                 frac=hbm_gbs / peaks["hbm_gbs"], bytes_per_step=hbm_bytes,
                 peak_source=peaks["source"]),
        cpu_baseline=cpu, parity=parity,
        e2e=dict(value=e2e_value, unit=UNIT, h2d_bytes_per_step=n_local * cfg.n_features * 4,
                 d2h_bytes_per_step=n_local * (F.n_out * 4 + 4)),
        gpu_launches=launches_per_step * args.steps,
        clocks=clocks, wall_s=wall, layout_s=layout_s)
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
