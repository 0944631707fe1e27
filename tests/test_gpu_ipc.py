"""Two processes, one GPU: the tree-sharded combine at world = 2 across real process boundaries.

Each process owns one tree shard (tahoe_forest_shard), computes its fp64 partial sums
(tahoe_predict_partial) and hands them to the other process through a CUDA IPC handle (torch
multiprocessing shares the allocation; both processes map the same device memory).  Each process
then calls tahoe_reduce_partials with [partial_0, partial_1] in rank order — the fixed-order sum +
finalize kernel the fused reduce uses over NVLink (reading R5) — for its own row block and for all
rows; the outputs must equal the oracle's bit for bit (dyadic leaves).  This exercises the
multi-rank reduction across address spaces, which a single process cannot (ADVICE r1:
k_reduce_lsa's world > 1 path is otherwise never exercised outside NVLink boxes)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _worker(rank, q_out, q_in, q_res, done):
    import os
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    try:
        import gen
        import oracle
        from paper_conf_eurosys_xiedlll21_b200 import tahoe as T
        torch.cuda.set_device(0)
        world = 2
        f = gen.make_forest(3, n_trees=210)
        F = T.Forest(f, device=0).layout(gen.make_calibration(3, 4096))
        n = 20_011
        X = gen.make_rows(3, n)
        X[::17, 3] = np.nan
        Xd = torch.from_numpy(X).cuda()
        S = F.shard(rank, world)
        part = S.predict_partial(Xd)
        torch.cuda.synchronize()
        q_out.put(part)                  # CUDA IPC handle of this rank's partials
        peer = q_in.get(timeout=300)     # the other rank's partials, mapped into this process
        parts = [part, peer] if rank == 0 else [peer, part]
        ref = oracle.predict(f, X, base_score=0.0)
        for mode in (T.REDUCE_SCATTER, T.REDUCE_ALL):
            lo, hi = T.tahoe_reduce_rows(n, world, rank, mode)
            cls = torch.full((hi - lo,), -1, dtype=torch.int32, device="cuda")
            out = F.reduce_partials(parts, rank, mode=mode, out_class=cls)
            torch.cuda.synchronize()
            assert np.array_equal(out.cpu().numpy(), ref["out"][lo:hi]), (rank, mode)
            assert np.array_equal(cls.cpu().numpy(), ref["cls"][lo:hi]), (rank, mode)
        # the sum of the two shards' partials is the full forest's raw sums (exact, dyadic)
        tot = (part + peer).cpu().numpy()
        assert np.array_equal(tot, ref["raw"]), rank
        q_res.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - surfaced through the queue
        import traceback
        q_res.put((rank, repr(e) + traceback.format_exc()[-1500:]))
    done.wait(timeout=300)   # keep this rank's partials alive until the peer is finished


def test_two_process_ipc_reduce_partials():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q01, q10, res = ctx.Queue(), ctx.Queue(), ctx.Queue()
    done = ctx.Event()
    procs = [ctx.Process(target=_worker, args=(0, q01, q10, res, done)),
             ctx.Process(target=_worker, args=(1, q10, q01, res, done))]
    for p in procs:
        p.start()
    try:
        got = dict(res.get(timeout=600) for _ in range(2))
    finally:
        done.set()
        for p in procs:
            p.join(timeout=120)
    assert got == {0: "ok", 1: "ok"}, got
