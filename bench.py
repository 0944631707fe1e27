#!/usr/bin/env python
"""Benchmark of the hot path: batched decision-tree-ensemble prediction (Tahoe, EuroSys '21).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config 2]
    python -m torch.distributed.run --nnodes=1 --nproc-per-node N --master-addr 127.0.0.1 \
        --master-port P bench.py --gpus N ...

Workload (BASELINE.json configs[1], the config the metric is quoted on and that fits one GPU):
C2, a Higgs-shaped binary forest of 500 random post-pruned trees (depth <= 8, 28 attributes) over
1M synthetic samples per GPU.  A step = one tahoe_predict of the whole batch (all §8(a) rows:
traversal, combine, finalize).  N > 1: every rank predicts its own 1M rows (sample sharding, weak
scaling, no data-path collective).  Rank 0 prints one JSON line.

--impl reference: the CPU oracle (oracle/, the "reference arm" of this tier) timed on the box's
host cores on a bounded sample of the same workload per step.
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


def build_workload(cfg, rank: int, n: int):
    f = gen.make_forest(cfg, leaf_mode="normal")
    X = gen.make_rows(cfg, n, row0=rank * n)
    return f, X


def oracle_rate(f, X, target_s: float, max_rows: int):
    """Oracle (as it stands) on a bounded sample of X: returns (rows/s, rows, seconds, visits)."""
    import oracle
    probe = min(2000, X.shape[0])
    t = time.perf_counter()
    oracle.predict(f, X[:probe])
    dt = max(time.perf_counter() - t, 1e-6)
    rows = int(min(max_rows, X.shape[0], max(probe, probe / dt * target_s)))
    idx = gen.subsample(4242, X.shape[0], rows)
    t = time.perf_counter()
    r = oracle.predict(f, X, rows=idx)
    dt = time.perf_counter() - t
    return rows / dt, rows, dt, float(r["visits"].mean())


def run_reference(args, cfg):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    n = cfg.n_samples
    f, X = build_workload(cfg, 0, min(n, 200_000))
    cores = oracle.n_threads()
    rate0, _, _, _ = oracle_rate(f, X, 1.0, 20000)
    rows = int(min(X.shape[0], max(1000, rate0 * 4.0)))   # ~4 s of oracle work per step
    idx = gen.subsample(99, X.shape[0], rows)
    for _ in range(args.warmup):
        oracle.predict(f, X, rows=idx[: max(1, rows // 8)])
    times = []
    for _ in range(args.steps):
        t = time.perf_counter()
        oracle.predict(f, X, rows=idx)
        times.append(time.perf_counter() - t)
    ms = 1000.0 * statistics.mean(times)
    value = rows / (ms / 1000.0)
    sample = f"{rows} seeded rows per step of the {cfg.name} workload (of {n} per GPU)"
    line = dict(metric=METRIC, value=value, unit=UNIT, n_gpus=args.gpus, steps=args.steps,
                warmup=args.warmup, ms_per_step=ms, higher_is_better=True, scaling="weak",
                vs_baseline=None, dtype="f32", data="synthetic", impl="reference",
                config=_config(cfg, n, None),
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
    full = T.Forest(f, device=-1).layout(gen.make_calibration(cfg))
    S = full.shard(rank, world, device=local)
    layout_s = time.perf_counter() - t0
    Xh = gen.make_rows(cfg, cfg.n_samples)
    Xd = torch.from_numpy(Xh).to(dev).repeat(reps, 1)
    stream = torch.cuda.current_stream()
    fused = args.reduce == "fused"
    if fused:
        os.environ.setdefault("NCCL_DEBUG", "WARN")   # keep stdout to the one JSON line
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
        visits = st["expected_visits_per_sample"]   # this rank's shard, calibration estimate
        if not args.no_cpu and world == 1:
            import oracle
            rate, rows, secs, vis = oracle_rate(f, Xh, 12.0, 200_000)
            cpu = dict(value=rate, unit=UNIT, cores=oracle.n_threads(), kind="oracle",
                       sample=f"{rows} seeded rows of this workload, full {cfg.n_trees}-tree forest "
                              f"({secs:.1f} s of oracle work)")
            visits = vis
        # roofline of the traversal (k_direct_tlp over the L2-sized chunks of the shard's image):
        # algorithmic bytes per sample = node visits x (8 B node + 4 B attribute) + leaves x 8 B,
        # against the L1 / shared-memory data pipe the node and attribute loads go through
        # (128 B/clk/SM, the same unit and peak as the sliced kernels' roofline); the time is the
        # whole step (traversal launches + the reduce/finalize kernel, < 1 % of it)
        peaks = _peaks()
        n_sms = st["num_sms"]
        pipe_peak = 128.0 * n_sms * peaks["sm_max_mhz"] * 1e6 / 1e9
        bytes_per_sample = visits * 12.0 + st["n_trees"] * 8.0
        achieved = n * bytes_per_sample / (ms / 1000.0) / 1e9
        roofline = dict(bound="alu", pipe="L1/shared-memory LSU data pipe, 128 B/clk/SM (DESIGN.md Roofline)",
                        kernel="k_direct_tlp", achieved=achieved, peak=pipe_peak, unit="GB/s",
                        frac=achieved / pipe_peak, traffic=None, kernel_ms=ms,
                        units_per_launch=f"{n} samples x {bytes_per_sample:.0f} B ({visits:.0f} visits x 12 B"
                                         f" + {st['n_trees']} leaves x 8 B) per step",
                        peak_source=f"derived: 128 B/clk x {n_sms} SMs x {peaks['sm_max_mhz']:.0f} MHz")
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
                    strategy="direct", roofline=roofline, hbm=hbm, cpu_baseline=cpu, e2e=e2e,
                    gpu_launches=(2 if (fused or rank == 0) else 1) * args.steps, clocks=clocks,
                    layout_s=layout_s)
        print(json.dumps(line), flush=True)
    if fused:
        comm.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def _config(cfg, n, stats):
    c = {"workload": f"{cfg.name}: {cfg.n_trees} trees depth<={cfg.max_depth}, "
                     f"{cfg.n_features} features, {n} samples per GPU (BASELINE configs[{cfg.cid - 1}])",
         "n_per_gpu": n, "n_trees": cfg.n_trees, "n_features": cfg.n_features,
         "max_depth": cfg.max_depth,
         "agg": {gen.AGG_SUM: "sum", gen.AGG_AVERAGE: "average", gen.AGG_BINARY: "binary margin + class",
                 gen.AGG_CLASS_SUM: f"{cfg.n_classes}-class sums + argmax",
                 gen.AGG_VOTE: "vote"}.get(cfg.agg, str(cfg.agg)),
         "parallelism": "sample-sharded (no collective)",
         "l2": f"256 MiB L2 flush between timed steps (inputs {n * cfg.n_features * 4 / 1e6:.0f} MB "
               f"{'<' if n * cfg.n_features * 4 < 126e6 else '>'} L2), outside the events"}
    if stats:
        c.update({k: stats[k] for k in ("nodes", "leaves", "n_slices", "slots_max", "lockstep_eff",
                                        "expected_visits_per_sample", "sliced_bytes") if k in stats})
    return c


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--strategy", type=int, default=-1)
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--mode", default=None, choices=["sample", "tree"],
                    help="sample sharding (default; C1-C4) or tree sharding (default for C5)")
    ap.add_argument("--rows", type=int, default=None, help="override the config's row count")
    ap.add_argument("--weak", action="store_true",
                    help="tree mode: duplicate the rows once per GPU (weak scaling, P:2450-2456)")
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
    f, X = build_workload(cfg, rank, n)
    t0 = time.perf_counter()
    F = T.Forest(f, device=local)
    F.layout(gen.make_calibration(cfg))
    layout_s = time.perf_counter() - t0
    stats = F.stats()
    strategy = args.strategy if args.strategy >= 0 else F.select_strategy(n, cfg.n_features)
    Xd = torch.from_numpy(X).to(dev)
    coll_dev = dev if args.dist_backend == "nccl" else torch.device("cpu")
    out = torch.empty((n, F.n_out), dtype=torch.float32, device=dev)
    cls = torch.empty(n, dtype=torch.int32, device=dev)
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
    tot = torch.tensor([sum(step_ms), sum(kern_ms)], dtype=torch.float64, device=coll_dev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.MAX)
    ms_per_step = float(tot[0]) / args.steps
    kern_avg_ms = float(tot[1]) / args.steps
    value = world * n / (ms_per_step / 1000.0)

    # ---- end to end through the public API with HOST buffers (pinned), copies inside
    Xh = torch.from_numpy(X).pin_memory()
    oh = torch.empty((n, F.n_out), dtype=torch.float32).pin_memory()
    ch = torch.empty(n, dtype=torch.int32).pin_memory()
    for _ in range(2):
        F.predict_host(Xh, oh, ch)
    torch.cuda.synchronize()
    e2e_ms = []
    for _ in range(max(3, min(args.steps, 10))):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        F.predict_host(Xh, oh, ch)
        b.record(stream)
        torch.cuda.synchronize()
        e2e_ms.append(a.elapsed_time(b))
    e2e_t = torch.tensor([statistics.mean(e2e_ms)], dtype=torch.float64, device=coll_dev)
    if world > 1:
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
    e2e_value = world * n / (float(e2e_t[0]) / 1000.0)

    if rank != 0:
        if world > 1:
            dist.barrier()
            dist.destroy_process_group()
        return 0

    peaks = _peaks()
    # algorithmic bytes (HBM roofline the metric asks for): sample row read + outputs written
    hbm_bytes = n * (cfg.n_features * 4 + F.n_out * 4 + 4)
    hbm_gbs = hbm_bytes / (ms_per_step / 1000.0) / 1e9
    # dominant kernel roofline: shared-memory LSU pipe: per node visit
    # 8 B node + 4 B attribute, per leaf 8 B; peak 128 B/clk/SM x SMs x max SM clock
    cpu = None
    visits = stats["expected_visits_per_sample"]
    if not args.no_cpu and world == 1:
        rate, rows, secs, vis = oracle_rate(f, X, 12.0, 1_000_000)
        import oracle
        cpu = dict(value=rate, unit=UNIT, cores=oracle.n_threads(), kind="oracle",
                   sample=f"{rows} seeded rows of this workload ({secs:.1f} s of oracle work)")
        visits = vis
    smem_bytes_per_sample = visits * 12.0 + cfg.n_trees * 8.0
    n_sms = stats["num_sms"]
    smem_peak = 128.0 * n_sms * peaks["sm_max_mhz"] * 1e6 / 1e9
    achieved = n * smem_bytes_per_sample / (kern_avg_ms / 1000.0) / 1e9
    kname = {1: "k_sliced", 2: "k_sliced_codes8" if stats.get("code8") else "k_sliced_codes"}.get(strategy, "k_direct")
    traffic = None
    sector_eff = None
    path_sector_eff = None   # every LSU global load of the step (pre-pass + walk), same capture
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):
        try:
            rec = json.load(open(tp)).get(f"C{cfg.cid}", {})
            # only a capture of the kernel this run times (e.g. "k_sliced_codes<0>")
            if rec.get("kernel", "").split("<")[0] == kname:
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
        ms_per_step=ms_per_step, higher_is_better=True, scaling="weak", vs_baseline=None,
        dtype="f32", accum="f64", data="synthetic", impl="ours",
        config=_config(cfg, n, stats),
        strategy={0: "direct", 1: "sliced", 2: "sliced-coded"}.get(strategy, str(strategy)),
        roofline=dict(bound="alu", pipe="shared-memory LSU, 128 B/clk/SM (DESIGN.md Roofline)",
                      kernel=kname,
                      achieved=achieved, peak=smem_peak, unit="GB/s", frac=achieved / smem_peak,
                      traffic=traffic, kernel_ms=kern_avg_ms,
                      global_ld_sector_efficiency=sector_eff,
                      path_global_ld_sector_efficiency=path_sector_eff,
                      units_per_launch=f"{n} samples x {smem_bytes_per_sample:.0f} B "
                                       f"({visits:.0f} visits x 12 B + {cfg.n_trees} leaves x 8 B)",
                      peak_source=f"derived: 128 B/clk x {n_sms} SMs x {peaks['sm_max_mhz']:.0f} MHz"),
        hbm=dict(achieved=hbm_gbs, peak=peaks["hbm_gbs"], unit="GB/s",
                 frac=hbm_gbs / peaks["hbm_gbs"], bytes_per_step=hbm_bytes,
                 peak_source=peaks["source"]),
        cpu_baseline=cpu,
        e2e=dict(value=e2e_value, unit=UNIT, h2d_bytes_per_step=n * cfg.n_features * 4,
                 d2h_bytes_per_step=n * (F.n_out * 4 + 4)),
        gpu_launches=launches_per_step * args.steps,
        clocks=clocks, wall_s=wall, layout_s=layout_s)
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
