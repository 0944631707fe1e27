"""World-size-2 gloo tests of the multi-GPU host logic on CPU.

* sample sharding: the ranks' row ranges partition [0, n) (no collective on the data path);
* tree sharding: the shards of tahoe_forest_shard (host-only handles here) partition the trees,
  and summing per-shard fp64 partials with the product's reduce_partials over gloo reproduces the
  full forest's raw sums;
* fused reduce (f4) host logic: the 128-byte communicator id drawn on rank 0 (ncclGetUniqueId via
  tahoe_comm_unique_id) reaches every rank unchanged, tahoe_reduce_rows partitions the rows like
  dist.shard_rows, and the rank-order sum of the gathered partials over a rank's rows (what
  k_reduce_lsa computes over NVLink) equals the full forest's raw sums.  The per-shard partial producer in this CPU test is the oracle restricted
  to the shard's trees (test infrastructure); on GPUs it is tahoe_predict_partial (see
  tests/test_gpu_parity.py::test_parity_c5_subsample_direct_and_shards).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _subforest(f, trees):
    """User-level arrays of the listed trees (node ids kept global; unreachable nodes ignored)."""
    return dict(f, root=f["root"][trees], tree_class=f["tree_class"][trees])


def _worker(rank, world, port, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import gen
    import oracle
    from paper_conf_eurosys_xiedlll21_b200 import dist as D
    from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # sample sharding: row ranges
        n = 1001
        lo, hi = D.shard_rows(n, rank, world)
        rng = torch.tensor([lo, hi], dtype=torch.int64)
        allr = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allr, rng)
        cover = np.zeros(n, np.int64)
        for r in allr:
            cover[int(r[0]):int(r[1])] += 1
        assert (cover == 1).all()

        # tree sharding: 3-class forest, host-only handles
        f = gen.make_forest(3, n_trees=56)
        X = gen.make_rows(3, 300)
        full = T.tahoe_forest_build(f, f["n_features"], f["n_classes"], f["agg"], 0.25, -1)
        T.tahoe_forest_layout(full, gen.make_calibration(3, 1000))
        sh = T.tahoe_forest_shard(full, rank, world, -1)
        nt = T.tahoe_forest_n_trees(sh)
        mine = T.tahoe_forest_layout_info(sh, len(f["feature"]), nt)["order"]
        trees = torch.zeros(56, dtype=torch.int64)
        trees[torch.from_numpy(mine.astype(np.int64))] = 1
        dist.all_reduce(trees)
        assert (trees == 1).all(), "shards partition the trees"

        def partial_fn(Xn):
            r = oracle.predict(_subforest(f, np.sort(mine)), Xn, agg=oracle.AGG_CLASS_SUM,
                               base_score=0.0)
            return torch.from_numpy(r["raw"].copy())

        def finalize_fn(p):
            return p  # raw check; GPU finalize is covered by the GPU tests

        out, part = D.predict_tree_sharded(None, None, X, dst=0, partial_fn=partial_fn,
                                           finalize_fn=finalize_fn)
        if rank == 0:
            ref = oracle.predict(f, X, agg=oracle.AGG_CLASS_SUM)
            assert np.array_equal(out.numpy(), ref["raw"]), "dyadic partials sum exactly"
        # fused reduce host logic
        uid = D.broadcast_comm_id(T.tahoe_comm_unique_id)
        ids = [None] * world
        dist.all_gather_object(ids, uid)
        assert all(u == ids[0] for u in ids) and len(uid) == T.COMM_ID_BYTES
        for nn in (0, 1, 7, 300):
            lo, hi = T.tahoe_reduce_rows(nn, world, rank, T.REDUCE_SCATTER)
            assert (lo, hi) == D.reduce_rows(nn, world, rank) == D.shard_rows(nn, rank, world)
            assert T.tahoe_reduce_rows(nn, world, rank, T.REDUCE_ALL) == (0, nn)
        parts = [torch.zeros_like(part) for _ in range(world)]
        dist.all_gather(parts, partial_fn(X))
        lo, hi = T.tahoe_reduce_rows(X.shape[0], world, rank, T.REDUCE_SCATTER)
        s = torch.zeros_like(parts[0][lo:hi])
        for p in parts:          # rank order 0..world-1, as the kernel sums
            s += p[lo:hi]
        ref = oracle.predict(f, X, agg=oracle.AGG_CLASS_SUM)
        assert np.array_equal(s.numpy(), ref["raw"][lo:hi])

        # one rank lays the forest out, every rank applies the same layout (dist.shared_layout)
        g = T.Forest(f, device=-1)
        D.shared_layout(g, gen.make_calibration(3, 1000) if rank == 0 else None)
        order = T.tahoe_forest_layout_info(g.handle, len(f["feature"]), g.n_trees)["order"]
        orders = [None] * world
        dist.all_gather_object(orders, order.tolist())
        ref_order = T.tahoe_forest_layout_info(full, len(f["feature"]), 56)["order"]
        assert all(o == ref_order.tolist() for o in orders), "every rank has rank 0's layout"
        m = D.max_over_ranks(float(rank) + 0.5)
        assert m == world - 0.5
        T.tahoe_forest_free(sh)
        T.tahoe_forest_free(full)
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - surfaced through the queue
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_sample_and_tree_sharding():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res


def _worker_subgroup(rank, world, port, q):
    """dst / src arguments are ranks WITHIN the group: with group = global ranks [1, 2], group rank
    0 is global rank 1 (dist.reduce read dst as a global rank)."""
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    from paper_conf_eurosys_xiedlll21_b200 import dist as D
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        grp = dist.new_group([1, 2])
        if rank in (1, 2):
            part = torch.full((4, 1), float(rank), dtype=torch.float64)
            out, p = D.predict_tree_sharded(None, None, None, dst=0, group=grp,
                                            partial_fn=lambda _x: part, finalize_fn=lambda t: t)
            if rank == 1:   # group rank 0 receives the sum and finalises
                assert out is not None and torch.equal(out, torch.full((4, 1), 3.0, dtype=torch.float64))
            else:
                assert out is None
            uid = D.broadcast_comm_id(lambda: bytes([rank]) * 128, src=0, group=grp)
            assert uid == bytes([1]) * 128, "the id comes from group rank 0 (global rank 1)"
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


def test_gloo_world3_subgroup_ranks():
    world = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_subgroup, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok", 2: "ok"}, res
