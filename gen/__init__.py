"""Seeded synthetic workloads shaped like the paper's datasets (BASELINE.json configs).

Input generation only: this module is shared by the CPU oracle (``oracle/``) and the CUDA path and
contains none of the method's arithmetic.  The heavy lifting is ``gen/tahoe_gen.c`` (counter-based
RNG, so outputs do not depend on thread count or on which rows are requested).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, replace

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "tahoe_gen.c")
_LIB = os.path.join(_HERE, "libtahoegen.so")

# aggregation codes (same numbering as include/tahoe.h's tahoe_agg; plain data, not arithmetic)
AGG_SUM, AGG_AVERAGE, AGG_BINARY, AGG_CLASS_SUM, AGG_VOTE = 0, 1, 2, 3, 4


@dataclass(frozen=True)
class Config:
    """One BASELINE.json config (SURVEY §8(a) table, §8(d) generator parameters)."""
    cid: int
    name: str
    shape: int            # column-distribution family in tahoe_gen.c
    n_features: int
    n_trees: int
    max_depth: int
    n_classes: int        # output groups: 1 for SUM/AVERAGE/BINARY, C for CLASS_SUM/VOTE
    agg: int
    n_samples: int
    p_split: float
    min_leaf: int
    n_cal: int
    prune_p: float
    quantile_thresholds: int
    leaf_k: int           # dyadic leaves k/256 with |k| <= leaf_k

    @property
    def seed_forest(self) -> int:
        return 1000 + self.cid

    @property
    def seed_cal(self) -> int:
        return 2000 + self.cid

    @property
    def seed_test(self) -> int:
        return 3000 + self.cid


CONFIGS = {
    1: Config(1, "C1-tiny-regression", 1, 8, 10, 4, 1, AGG_SUM, 1_000, 0.8, 4, 4096, 0.25, 0, 256),
    2: Config(2, "C2-higgs-binary", 2, 28, 500, 8, 1, AGG_BINARY, 1_000_000, 0.9, 8, 16384, 0.25, 0, 256),
    3: Config(3, "C3-covtype-7class", 3, 54, 1400, 12, 7, AGG_CLASS_SUM, 4_000_000, 0.9, 4, 16384, 0.25, 0, 256),
    4: Config(4, "C4-epsilon-wide", 4, 2000, 1000, 10, 1, AGG_BINARY, 500_000, 0.9, 4, 16384, 0.25, 0, 256),
    5: Config(5, "C5-large-imbalanced", 5, 100, 4000, 20, 1, AGG_SUM, 10_000_000, 0.97, 2, 65536, 0.10, 1, 64),
}


class _Params(ctypes.Structure):
    _fields_ = [
        ("n_trees", ctypes.c_int32), ("max_depth", ctypes.c_int32), ("n_features", ctypes.c_int32),
        ("n_classes", ctypes.c_int32), ("shape", ctypes.c_int32), ("min_leaf", ctypes.c_int32),
        ("quantile_thresholds", ctypes.c_int32), ("leaf_mode", ctypes.c_int32),
        ("leaf_k", ctypes.c_int32), ("_pad", ctypes.c_int32),
        ("p_split", ctypes.c_double), ("prune_p", ctypes.c_double), ("n_cal", ctypes.c_int64),
        ("seed_forest", ctypes.c_uint64), ("seed_cal", ctypes.c_uint64),
    ]


_lib = None


def build(force: bool = False) -> str:
    """Compile tahoe_gen.c (gcc, OpenMP, no fast-math) if the .so is missing or stale."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared",
                               "-fno-fast-math", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        lib.gen_forest_grow.restype = P
        lib.gen_forest_grow.argtypes = [ctypes.POINTER(_Params), ctypes.c_int32]
        lib.gen_forest_n_nodes.restype = ctypes.c_int64
        lib.gen_forest_n_nodes.argtypes = [P]
        lib.gen_forest_export.argtypes = [P] * 9
        lib.gen_forest_free.argtypes = [P]
        lib.gen_rows.argtypes = [ctypes.c_int32, ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64,
                                 ctypes.c_int32, P, ctypes.c_int32]
        lib.gen_rows_idx.argtypes = [ctypes.c_int32, ctypes.c_uint64, P, ctypes.c_int64,
                                     ctypes.c_int32, P, ctypes.c_int32]
        lib.gen_subsample.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64, P]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def make_forest(cfg: Config | int, leaf_mode: str = "dyadic", n_trees: int | None = None,
                nthreads: int = 0, **overrides) -> dict:
    """Grow the config's forest.  Returns the user-level node arrays that tahoe_forest_build and
    the oracle both consume: root, feature (<0 leaf), threshold, left, right, leaf_value,
    default_left, tree_class, plus n_features / n_classes / agg."""
    if isinstance(cfg, int):
        cfg = CONFIGS[cfg]
    if n_trees is not None:
        overrides["n_trees"] = n_trees
    if overrides:
        cfg = replace(cfg, **overrides)
    lib = _load()
    p = _Params(n_trees=cfg.n_trees, max_depth=cfg.max_depth, n_features=cfg.n_features,
                n_classes=cfg.n_classes, shape=cfg.shape, min_leaf=cfg.min_leaf,
                quantile_thresholds=cfg.quantile_thresholds,
                leaf_mode=0 if leaf_mode == "dyadic" else 1, leaf_k=cfg.leaf_k, _pad=0,
                p_split=cfg.p_split, prune_p=cfg.prune_p, n_cal=cfg.n_cal,
                seed_forest=cfg.seed_forest, seed_cal=cfg.seed_cal)
    h = lib.gen_forest_grow(ctypes.byref(p), nthreads)
    try:
        nn = lib.gen_forest_n_nodes(h)
        T = cfg.n_trees
        out = dict(root=np.empty(T, np.int32), feature=np.empty(nn, np.int32),
                   threshold=np.empty(nn, np.float32), left=np.empty(nn, np.int32),
                   right=np.empty(nn, np.int32), leaf_value=np.empty(nn, np.float32),
                   default_left=np.empty(nn, np.uint8), tree_class=np.empty(T, np.int32))
        lib.gen_forest_export(h, *[_ptr(out[k]) for k in
                                   ("root", "feature", "threshold", "left", "right", "leaf_value",
                                    "default_left", "tree_class")])
    finally:
        lib.gen_forest_free(h)
    out.update(n_features=cfg.n_features, n_classes=cfg.n_classes, agg=cfg.agg, config=cfg)
    return out


def make_rows(cfg: Config | int, n: int, row0: int = 0, seed: int | None = None,
              nthreads: int = 0, d: int | None = None) -> np.ndarray:
    """Rows [row0, row0+n) of the config's test matrix (seed 3000+c), float32 row-major (n, d)."""
    if isinstance(cfg, int):
        cfg = CONFIGS[cfg]
    d = cfg.n_features if d is None else d
    seed = cfg.seed_test if seed is None else seed
    X = np.empty((n, d), np.float32)
    if n:
        _load().gen_rows(cfg.shape, seed, row0, n, d, _ptr(X), nthreads)
    return X


def make_rows_idx(cfg: Config | int, idx: np.ndarray, seed: int | None = None,
                  nthreads: int = 0) -> np.ndarray:
    """Rows at explicit indices of the config's test matrix (for seeded subsamples)."""
    if isinstance(cfg, int):
        cfg = CONFIGS[cfg]
    seed = cfg.seed_test if seed is None else seed
    idx = np.ascontiguousarray(idx, dtype=np.int64)
    X = np.empty((len(idx), cfg.n_features), np.float32)
    if len(idx):
        _load().gen_rows_idx(cfg.shape, seed, _ptr(idx), len(idx), cfg.n_features, _ptr(X), nthreads)
    return X


def make_calibration(cfg: Config | int, n: int | None = None) -> np.ndarray:
    """Calibration rows (seed 2000+c) — the same rows the trees were grown on."""
    if isinstance(cfg, int):
        cfg = CONFIGS[cfg]
    return make_rows(cfg, cfg.n_cal if n is None else n, seed=cfg.seed_cal)


def subsample(seed: int, n: int, k: int) -> np.ndarray:
    """Sorted seeded sample of min(k, n) distinct indices in [0, n)."""
    k = min(k, n)
    out = np.empty(k, np.int64)
    if k:
        _load().gen_subsample(seed, n, k, _ptr(out))
    return out
