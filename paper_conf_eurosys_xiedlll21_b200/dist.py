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

  With a tahoe Comm (init_comm) the reduce is fused instead: predict_tree_sharded_fused writes the
  partials into an NCCL symmetric window and one kernel per rank sums the peers' partials over
  NVLink in rank order and finalises its rows (tahoe_predict_reduce).

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


def _global_rank(group, group_rank: int) -> int:
    """Global rank of rank `group_rank` of `group` (None = the default group: the same number)."""
    return group_rank if group is None else dist.get_global_rank(group, group_rank)


def reduce_partials(partial: torch.Tensor, dst: int = 0, group=None) -> torch.Tensor:
    """Sum the per-rank fp64 partial sums onto `dst`, a rank WITHIN `group` (in place; one
    ncclReduce / gloo reduce)."""
    if partial.dtype != torch.float64:
        raise TypeError("partials are fp64")
    dist.reduce(partial, dst=_global_rank(group, dst), op=dist.ReduceOp.SUM, group=group)
    return partial


def predict_tree_sharded(full_forest, shard_forest, X: torch.Tensor, dst: int = 0, group=None,
                         partial_fn: Callable | None = None, finalize_fn: Callable | None = None):
    """Tree-sharded prediction of all rows of X (replicated on every rank); `dst` is a rank within
    `group`.

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


def broadcast_comm_id(make_id: Callable[[], bytes], src: int = 0, group=None) -> bytes:
    """Rank `src` of `group` draws the 128-byte communicator id, every rank returns the same
    bytes."""
    box = [make_id() if dist.get_rank(group) == src else None]
    dist.broadcast_object_list(box, src=_global_rank(group, src), group=group)
    uid = box[0]
    if not isinstance(uid, (bytes, bytearray)) or len(uid) != 128:
        raise RuntimeError("bad communicator id")
    return bytes(uid)


def shared_layout(forest, X_calib, src: int = 0, group=None, **layout_kw):
    """Lay `forest` out on rank `src` of `group` only and apply the same layout on every other rank
    (tahoe_forest_layout_export / _import over torch.distributed): the calibration walk, similarity
    detection and balancing run once instead of once per rank (C5: ~14 s per rank)."""
    if not dist.is_available() or not dist.is_initialized():
        return forest.layout(X_calib, **layout_kw)
    me = dist.get_rank(group)
    box = [forest.layout(X_calib, **layout_kw).layout_state() if me == src else None]
    dist.broadcast_object_list(box, src=_global_rank(group, src), group=group)
    if me != src:
        forest.apply_layout_state(box[0])
    return forest


def init_comm(device: int, group=None):
    """tahoe Comm over the ranks of `group` (one process per GPU, all in one NVLink domain); a
    single process without torch.distributed gets a world-1 communicator."""
    from . import tahoe as T
    if not dist.is_available() or not dist.is_initialized():
        return T.Comm(T.tahoe_comm_unique_id(), 1, 0, device)
    uid = broadcast_comm_id(T.tahoe_comm_unique_id, group=group)
    return T.Comm(uid, dist.get_world_size(group), dist.get_rank(group), device)


def reduce_rows(n: int, world: int, rank: int, scatter: bool = True) -> tuple[int, int]:
    """Rows a rank finalises in the fused reduce (== tahoe_reduce_rows; scatter=False: all)."""
    return shard_rows(n, rank, world) if scatter else (0, n)


def predict_tree_sharded_fused(shard_forest, comm, X: torch.Tensor, scatter: bool = True,
                               out=None, out_class=None, stream=None):
    """Tree-sharded prediction with the fused cross-GPU reduce: returns this rank's rows
    [lo, hi) of the final output (scatter) or all rows (scatter=False)."""
    from . import tahoe as T
    mode = T.REDUCE_SCATTER if scatter else T.REDUCE_ALL
    return shard_forest.predict_reduce(comm, X, mode=mode, out=out, out_class=out_class,
                                       stream=stream)


def max_over_ranks(value: float, device=None, group=None) -> float:
    """Max of a per-rank timing (device-timed numbers, never wall clock)."""
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
