"""Multi-GPU plumbing over torch.distributed; one process per GPU.

Two ways the path shards:

* sample sharding — the paper's scaling runs: "We evenly partition each inference dataset into
  N_G parts ... Each GPU gets one partition" and there is "almost no communication
  between GPUs".  Rows [lo, hi) of rank r are contiguous; the forest is replicated;
  no collective touches the data path.
* tree sharding — for forests too large for one GPU's staging (BASELINE C5): trees are split into
  world shards balanced by expected visits (tahoe_forest_shard), every rank computes raw fp64
  per-sample partial sums of its trees over the SAME rows (tahoe_predict_partial), the partials are
  summed with one reduce (NCCL over NVLink on GPUs, gloo in CPU tests), and the destination rank
  finalizes with the full forest's aggregation (tahoe_finalize).  fp64 partials keep the result
  within the oracle tolerance whatever the reduction order; VOTE partials are exact counts.

The collective helpers take the partial producer as an argument so the same reduce logic runs in
the GPU product path and in the CPU (gloo) tests.
"""
from __future__ import annotations

from typing import Callable

import torch
import torch.distributed as dist


def shard_rows(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous row range [lo, hi) of `rank` (sizes differ by at most one)."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError("bad rank/world")
    return (n * rank) // world, (n * (rank + 1)) // world


def predict_sample_sharded(forest, X_local: torch.Tensor, **kw) -> torch.Tensor:
    """Each rank predicts its own rows; no collective."""
    return forest.predict(X_local, **kw)


def reduce_partials(partial: torch.Tensor, dst: int = 0, group=None) -> torch.Tensor:
    """Sum the per-rank fp64 partial sums onto `dst` (in place; one ncclReduce / gloo reduce)."""
    if partial.dtype != torch.float64:
        raise TypeError("partials are fp64")
    dist.reduce(partial, dst=dst, op=dist.ReduceOp.SUM, group=group)
    return partial


def predict_tree_sharded(full_forest, shard_forest, X: torch.Tensor, dst: int = 0, group=None,
                         partial_fn: Callable | None = None, finalize_fn: Callable | None = None):
    """Tree-sharded prediction of all rows of X (replicated on every rank).

    Returns (out, partial) on `dst` and (None, partial) elsewhere.  partial_fn(X) -> fp64 [n, n_out]
    defaults to shard_forest.predict_partial; finalize_fn(partial) defaults to
    full_forest.finalize."""
    partial_fn = partial_fn or shard_forest.predict_partial
    finalize_fn = finalize_fn or full_forest.finalize
    partial = partial_fn(X)
    reduce_partials(partial, dst=dst, group=group)
    if dist.get_rank(group) == dst:
        return finalize_fn(partial), partial
    return None, partial


def max_over_ranks(value: float, device=None, group=None) -> float:
    """Max of a per-rank timing (device-timed numbers, never wall clock)."""
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
