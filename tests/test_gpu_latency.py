"""Low-parallelism path (the paper's batch-100 workload): the ROWS
strategy (one CTA per sample, lane = tree, fixed-order block reduction, finalize in the same
launch), CUDA-graph replay of a captured predict call, and the L2-persisting forest window — each
against the oracle (dyadic leaves: scores, classes, leaf ids and fingerprints bit-exact)."""
import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_eurosys_xiedlll21_b200 import tahoe as T  # noqa: E402
from test_gpu_parity import _check, _gpu_run  # noqa: E402


@pytest.mark.parametrize("cid,ntrees,n", [(1, None, 1000), (2, None, 100), (2, None, 1000),
                                          (3, None, 257), (4, 200, 100), (5, 300, 64)])
def test_rows_strategy_parity(cid, ntrees, n, monkeypatch):
    f = gen.make_forest(cid, n_trees=ntrees)
    F = T.Forest(f, device=0).layout(gen.make_calibration(cid, 4096))
    assert F.stats()["rows_ok"]
    X = gen.make_rows(cid, n)
    X[::7, 0] = np.nan
    ref = oracle.predict(f, X, want_leaf=True)
    _check(_gpu_run(F, X, T.STRATEGY_ROWS), ref, f["agg"], True)
    _check(_gpu_run(F, X, T.STRATEGY_ROWS, want_leaf=False), ref, f["agg"], True, want_leaf=False)
    part = torch.empty((n, F.n_out), dtype=torch.float64, device="cuda")
    monkeypatch.setenv("TAHOE_FORCE_STRATEGY", str(T.STRATEGY_ROWS))   # raw sums, ROWS kernel
    F.predict_partial(torch.from_numpy(X).cuda(), part)
    torch.cuda.synchronize()
    assert np.array_equal(part.cpu().numpy(), ref["raw"]), "dyadic raw sums are exact"


def test_rows_strategy_vote_average_base():
    from test_oracle_pins import random_forest
    rng = np.random.default_rng(3)
    X = rng.normal(size=(333, 5)).astype(np.float32)
    C = 4
    fv = random_forest(rng, 60, 5, 5, n_classes=C, vote=True)
    F = T.Forest(fv, n_features=5, n_classes=C, agg=oracle.AGG_VOTE, device=0)
    ref = oracle.predict(fv, X, agg=oracle.AGG_VOTE, n_classes=C, want_leaf=True)
    _check(_gpu_run(F, X, T.STRATEGY_ROWS), ref, oracle.AGG_VOTE, True)
    f = random_forest(rng, 45, 6, 5)
    for agg, base in ((oracle.AGG_AVERAGE, 0.625), (oracle.AGG_SUM, -2.0), (oracle.AGG_BINARY, 0.25)):
        F = T.Forest(f, n_features=5, n_classes=1, agg=agg, base_score=base, device=0)
        ref = oracle.predict(f, X, agg=agg, base_score=base, want_leaf=True)
        _check(_gpu_run(F, X, T.STRATEGY_ROWS), ref, agg, True)


def test_rows_strategy_refused_when_too_large():
    """4000 trees x 100 attributes still fit; an over-wide row does not (E_UNSUPPORTED)."""
    from test_oracle_pins import random_forest
    rng = np.random.default_rng(4)
    d = 60_000
    f = random_forest(rng, 8, 3, d)
    F = T.Forest(f, n_features=d, n_classes=1, agg=oracle.AGG_SUM, device=0)
    assert not F.stats()["rows_ok"]
    X = torch.zeros((4, d), dtype=torch.float32, device="cuda")
    with pytest.raises(T.TahoeError):
        F.predict(X, force_strategy=T.STRATEGY_ROWS)


@pytest.mark.parametrize("cid,n", [(2, 100), (2, 1000), (3, 100), (2, 20000)])
def test_cuda_graph_replay_parity(cid, n):
    """A predict call captured in a CUDA graph (strategy chosen by the cost model for n) and
    replayed on new contents of the same input buffer gives the oracle's outputs every time."""
    f = gen.make_forest(cid)
    F = T.Forest(f, device=0).layout(gen.make_calibration(cid, 4096))
    Xd = torch.empty((n, f["n_features"]), dtype=torch.float32, device="cuda")
    out = torch.empty((n, F.n_out), dtype=torch.float32, device="cuda")
    cls = torch.empty(n, dtype=torch.int32, device="cuda")
    s = torch.cuda.Stream()
    Xd.copy_(torch.from_numpy(gen.make_rows(cid, n, row0=0)))
    with torch.cuda.stream(s):
        F.predict(Xd, out=out, out_class=cls, stream=s)   # warm-up (allocator, attributes)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        F.predict(Xd, out=out, out_class=cls, stream=s)
    for rep in range(3):
        X = gen.make_rows(cid, n, row0=(rep + 1) * n)
        Xd.copy_(torch.from_numpy(X))
        g.replay()
        torch.cuda.synchronize()
        ref = oracle.predict(f, X)
        assert np.array_equal(out.cpu().numpy(), ref["out"]), rep
        assert np.array_equal(cls.cpu().numpy(), ref["cls"]), rep


def test_l2_persist_window_parity():
    """With the forest image marked as an L2-persisting window on the stream, every strategy's
    outputs are unchanged (bit-exact against the oracle); removing the window restores the stream."""
    from test_gpu_parity import _strats
    f = gen.make_forest(2, n_trees=200)
    F = T.Forest(f, device=0).layout(gen.make_calibration(2, 4096))
    X = gen.make_rows(2, 5000)
    ref = oracle.predict(f, X, want_leaf=True)
    st = torch.cuda.current_stream()
    T.tahoe_forest_l2_persist(F.handle, st, 1.0)
    try:
        for s in _strats(F):
            _check(_gpu_run(F, X, s), ref, f["agg"], True)
    finally:
        T.tahoe_forest_l2_persist(F.handle, st, 0.0)
    _check(_gpu_run(F, X, -1), ref, f["agg"], True)
