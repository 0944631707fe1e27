"""Small runs of every kernel variant for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402

dev = torch.device("cuda", 0)
for cid, n, ntrees in ((2, 3001, 64), (3, 2003, 70), (4, 301, 40)):
    f = gen.make_forest(cid, n_trees=ntrees)
    # small direct chunks (reading R4) so the chunked launches are exercised too
    os.environ["TAHOE_DIRECT_CHUNK_KB"] = "16"
    F = T.Forest(f, device=0).layout(gen.make_calibration(cid, 2048))
    os.environ.pop("TAHOE_DIRECT_CHUNK_KB")
    X = gen.make_rows(cid, n)
    X[::17, 1] = np.nan
    Xd = torch.from_numpy(X).to(dev)
    for s, variant in ((0, "0"), (0, "1"), (0, "2"), (1, "0")):
        os.environ["TAHOE_DIRECT_VARIANT"] = variant   # direct: rows global / staged (lockstep, free)
        out = torch.empty((n, F.n_out), device=dev)
        cls = torch.empty(n, dtype=torch.int32, device=dev)
        leaf = torch.empty((n, F.n_trees), dtype=torch.int32, device=dev)
        fp = torch.empty(n, dtype=torch.int64, device=dev)
        F.predict(Xd, out=out, out_class=cls, force_strategy=s)
        F.predict(Xd, out=out, out_class=cls, out_leaf=leaf, out_fingerprint=fp, force_strategy=s)
    os.environ.pop("TAHOE_DIRECT_VARIANT")
    # large-batch direct kernels (staged rows, P threads per row): C2 / C3 only (d <= 256)
    if X.shape[1] <= 256:
        big = torch.from_numpy(gen.make_rows(cid, 33_001)).to(dev)
        for variant in ("5", "3", "2"):
            os.environ["TAHOE_DIRECT_VARIANT"] = variant
            F.predict(big, force_strategy=0)
        os.environ.pop("TAHOE_DIRECT_VARIANT")
        del big
    # rank-coded slices (reading R7 u16 rows, swizzled rows of >= 128 bytes for C3; reading R8
    # wide codes for C4): both row-coding pre-passes, production and LEAF instantiations, a
    # multi-tile batch so the ring wraps, and the minimum ring depth
    if F.stats()["coded_valid"]:
        big = torch.from_numpy(gen.make_rows(cid, 20_011)).to(dev)
        big[::13, 2] = float("nan")
        for banks in ("1", "0"):
            os.environ["TAHOE_CODE_BANKS"] = banks
            for Xs in (Xd, big):
                m = Xs.shape[0]
                out = torch.empty((m, F.n_out), device=dev)
                F.predict(Xs, out=out, force_strategy=2)
                F.predict(Xs, out=out, out_leaf=torch.empty((m, F.n_trees), dtype=torch.int32, device=dev),
                          out_fingerprint=torch.empty(m, dtype=torch.int64, device=dev), force_strategy=2)
        os.environ.pop("TAHOE_CODE_BANKS")
        os.environ["TAHOE_CODES_RING"] = "3"
        F.predict(big, force_strategy=2)
        os.environ.pop("TAHOE_CODES_RING")
        del big
    # ROWS strategy (f1), with and without leaf diagnostics, and its raw partial path
    if F.stats()["rows_ok"]:
        out = torch.empty((n, F.n_out), device=dev)
        F.predict(Xd, out=out, out_class=torch.empty(n, dtype=torch.int32, device=dev), force_strategy=3)
        F.predict(Xd, out=out, out_leaf=torch.empty((n, F.n_trees), dtype=torch.int32, device=dev),
                  out_fingerprint=torch.empty(n, dtype=torch.int64, device=dev), force_strategy=3)
        os.environ["TAHOE_FORCE_STRATEGY"] = "3"
        F.predict_partial(Xd)
        os.environ.pop("TAHOE_FORCE_STRATEGY")
    # end-to-end host call: chunks alternate between two compute streams (3 chunks of 64K rows)
    if cid == 3:
        Xh = torch.from_numpy(gen.make_rows(cid, 150_001)).pin_memory()
        oh = torch.empty((150_001, F.n_out), dtype=torch.float32).pin_memory()
        F.predict_host(Xh, oh)
        torch.cuda.synchronize()
    # misaligned X -> warp-copy staging path
    buf = torch.empty(X.size + 1, device=dev)
    buf[1:] = Xd.reshape(-1)
    F.predict(buf[1:].view(X.shape), force_strategy=1)
    cnt = torch.zeros(len(f["feature"]), dtype=torch.int32, device=dev)
    T.tahoe_count_visits(F.handle, Xd, n, X.shape[1], cnt)
    S = F.shard(0, 2)
    S.predict_partial(Xd)
    # fused cross-GPU reduce: peer-pointer kernel over two shards' partials, and the NCCL LSA
    # kernel through a world-1 communicator
    parts = [F.shard(r, 2).predict_partial(Xd) for r in range(2)]
    for r in range(2):
        for mode in (T.REDUCE_SCATTER, T.REDUCE_ALL):
            lo, hi = T.tahoe_reduce_rows(n, 2, r, mode)
            F.reduce_partials(parts, r, mode=mode, out_class=torch.empty(hi - lo, dtype=torch.int32, device=dev))
    if cid == 2:
        comm = T.Comm(T.tahoe_comm_unique_id(), 1, 0, 0)
        S1 = F.shard(0, 1)
        S1.predict_reduce(comm, Xd)
        torch.cuda.synchronize()
        comm.close()
# instrumented walk (tahoe_profile_walk, f3) on a C2 forest
fp2 = gen.make_forest(2, n_trees=64)
Fp = T.Forest(fp2, device=0).layout(gen.make_calibration(2, 2048))
Xp = torch.from_numpy(gen.make_rows(2, 9001)).to(dev)
T.tahoe_profile_walk(Fp.handle, Xp, 9001, Xp.shape[1], torch.empty((9001, 1), device=dev))
# microbenchmarks (Algorithm 1 line 4): both walk variants and the raw shared-memory load kernel
T.tahoe_measure_visit_rate(0, 0, 16, 2)
T.tahoe_measure_visit_rate(0, 1, 16, 2)   # steps: a multiple of 8
torch.cuda.synchronize()
print("sanitize case done")
