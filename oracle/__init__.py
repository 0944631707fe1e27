"""CPU oracle for batched decision-tree-ensemble prediction — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl
reference`` leg may import this package.  It shares no code with the CUDA path
(``paper_conf_eurosys_xiedlll21_b200``) and neither imports the other.

``predict`` wraps ``tahoe_oracle.c`` (plain traversal + fp64 combine);
``layout_oracle`` holds the layout-side helpers used only by layout tests (P:399-406, P:599-643,
P:773-806, Fig. 1 / Fig. 3).  Parity pins live in ``tests/test_oracle_pins.py`` and
``tests/test_layout_pins.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "tahoe_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

AGG_SUM, AGG_AVERAGE, AGG_BINARY, AGG_CLASS_SUM, AGG_VOTE = 0, 1, 2, 3, 4


def build(force: bool = False) -> str:
    """Compile the oracle (gcc -O2, OpenMP driver, IEEE floating point: no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared",
                               "-fno-fast-math", "-ffp-contract=off", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        i32, i64, f32 = ctypes.c_int32, ctypes.c_int64, ctypes.c_float
        lib.oracle_predict.restype = ctypes.c_int
        lib.oracle_predict.argtypes = [i32, P, i32, P, P, P, P, P, P, P, i32, i32, f32, P, i64,
                                       i32, P, P, P, P, P, P, P, i32]
        lib.oracle_node_counts.argtypes = [i32, P, P, P, P, P, P, P, i64, i32, P]
        lib.oracle_n_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _p(a):
    return None if a is None else ctypes.c_void_p(a.ctypes.data)


def n_threads() -> int:
    return int(_load().oracle_n_threads())


def n_outputs(agg: int, n_classes: int) -> int:
    return n_classes if agg in (AGG_CLASS_SUM, AGG_VOTE) else 1


def predict(forest: dict, X: np.ndarray, rows: np.ndarray | None = None, *, agg: int | None = None,
            base_score: float = 0.0, n_classes: int | None = None, want_leaf: bool = False,
            nthreads: int = 0, use_default_left: bool = True) -> dict:
    """Plain traversal of every (sample, tree) pair + fp64 combine.

    ``forest`` holds the user-level arrays (root, feature, threshold, left, right, leaf_value,
    default_left, tree_class).  ``rows`` optionally selects rows of X.  Returns a dict with
    ``out`` (float32, n x n_out), ``raw`` (float64), ``cls`` (int32), ``fp`` (uint64 fingerprint),
    ``visits`` (uint64) and, with want_leaf, ``leaf`` (int32 n x T original node ids)."""
    lib = _load()
    agg = forest.get("agg", AGG_SUM) if agg is None else agg
    C = forest.get("n_classes", 1) if n_classes is None else n_classes
    X = np.ascontiguousarray(X, dtype=np.float32)
    n = X.shape[0] if rows is None else len(rows)
    d = X.shape[1]
    if rows is not None:
        rows = np.ascontiguousarray(rows, dtype=np.int64)
    T = len(forest["root"])
    no = n_outputs(agg, C)
    arr = {k: np.ascontiguousarray(forest[k]) for k in
           ("root", "feature", "threshold", "left", "right", "leaf_value")}
    dl = forest.get("default_left") if use_default_left else None
    dl = None if dl is None else np.ascontiguousarray(dl, dtype=np.uint8)
    tc = forest.get("tree_class")
    tc = None if tc is None else np.ascontiguousarray(tc, dtype=np.int32)
    out = np.empty((n, no), np.float32)
    raw = np.empty((n, no), np.float64)
    cls = np.zeros(n, np.int32)
    fp = np.empty(n, np.uint64)
    visits = np.empty(n, np.uint64)
    leaf = np.empty((n, T), np.int32) if want_leaf else None
    lib.oracle_predict(T, _p(arr["root"]), len(arr["feature"]), _p(arr["feature"]),
                       _p(arr["threshold"]), _p(arr["left"]), _p(arr["right"]),
                       _p(arr["leaf_value"]), _p(dl), _p(tc), C, agg, float(base_score), _p(X),
                       n, d, _p(rows), _p(out), _p(raw), _p(cls), _p(leaf), _p(fp), _p(visits),
                       nthreads)
    res = dict(out=out, raw=raw, cls=cls, fp=fp, visits=visits)
    if want_leaf:
        res["leaf"] = leaf
    return res


def node_counts(forest: dict, X: np.ndarray) -> np.ndarray:
    """count[k] = number of rows of X whose root->leaf path passes node k."""
    lib = _load()
    X = np.ascontiguousarray(X, dtype=np.float32)
    arr = {k: np.ascontiguousarray(forest[k]) for k in
           ("root", "feature", "threshold", "left", "right")}
    dl = forest.get("default_left")
    dl = None if dl is None else np.ascontiguousarray(dl, dtype=np.uint8)
    cnt = np.zeros(len(arr["feature"]), np.uint64)
    lib.oracle_node_counts(len(arr["root"]), _p(arr["root"]), _p(arr["feature"]),
                           _p(arr["threshold"]), _p(arr["left"]), _p(arr["right"]), _p(dl),
                           _p(X), X.shape[0], X.shape[1], _p(cnt))
    return cnt
