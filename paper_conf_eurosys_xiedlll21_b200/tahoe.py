"""Thin Python binding of libtahoe.so (include/tahoe.h): argument marshalling only.

Functions carry the C ABI names (``tahoe_forest_build``, ``tahoe_forest_layout``,
``tahoe_predict`` ...).  Every step of prediction runs in the library's sm_100a kernels; PyTorch is
used only for device memory and streams.  There is no CPU fallback: if the shared library is
missing, importing this module raises.

``Forest`` is a small convenience wrapper that owns a handle and accepts torch tensors / numpy
arrays.
"""
from __future__ import annotations

import ctypes
import json
import os

import numpy as np

from . import build as _build

_lib = None

TAHOE_OK, TAHOE_E_INVAL, TAHOE_E_NOMEM, TAHOE_E_CUDA, TAHOE_E_UNSUPPORTED, TAHOE_E_STATE = range(6)
AGG_SUM, AGG_AVERAGE, AGG_BINARY, AGG_CLASS_SUM, AGG_VOTE = range(5)
STRATEGY_AUTO, STRATEGY_DIRECT, STRATEGY_SLICED, STRATEGY_SLICED_CODED, STRATEGY_ROWS = -1, 0, 1, 2, 3
REDUCE_SCATTER, REDUCE_ALL = 0, 1
COMM_ID_BYTES = 128


class TahoeError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"tahoe status {status}: {msg}")
        self.status = status


class LayoutOpts(ctypes.Structure):
    _fields_ = [("t_nodes", ctypes.c_int32), ("l_hash", ctypes.c_int32),
                ("m_chunks", ctypes.c_int32), ("node_reorder", ctypes.c_int32),
                ("tree_group", ctypes.c_int32), ("_reserved", ctypes.c_int32),
                ("seed", ctypes.c_uint64)]


class PredictOpts(ctypes.Structure):
    _fields_ = [("out_class", ctypes.c_void_p), ("out_leaf", ctypes.c_void_p),
                ("out_fingerprint", ctypes.c_void_p), ("force_strategy", ctypes.c_int32),
                ("_reserved", ctypes.c_int32), ("ev_main_begin", ctypes.c_void_p),
                ("ev_main_end", ctypes.c_void_p)]


SYMBOLS = ("tahoe_forest_build", "tahoe_forest_layout", "tahoe_predict", "tahoe_predict_ex",
           "tahoe_predict_host", "tahoe_forest_shard", "tahoe_predict_partial", "tahoe_finalize",
           "tahoe_forest_n_outputs", "tahoe_forest_n_trees", "tahoe_forest_stats",
           "tahoe_select_strategy", "tahoe_predict_cost_us", "tahoe_forest_free", "tahoe_last_error",
           "tahoe_forest_layout_info", "tahoe_tree_tokens", "tahoe_tree_simhash", "tahoe_simhash",
           "tahoe_lsh_order", "tahoe_sha1", "tahoe_forest_export_sliced", "tahoe_count_visits",
           "tahoe_forest_layout_counts", "tahoe_forest_l2_persist", "tahoe_comm_unique_id",
           "tahoe_comm_init", "tahoe_comm_free", "tahoe_reduce_rows", "tahoe_predict_reduce",
           "tahoe_reduce_partials", "tahoe_measure_visit_rate", "tahoe_profile_walk",
           "tahoe_forest_layout_export", "tahoe_forest_layout_import")


def lib_path() -> str:
    return _build.LIB


def load(build_if_missing: bool = True):
    """Load libtahoe.so (building it with nvcc if missing/stale and allowed)."""
    global _lib
    if _lib is not None:
        return _lib
    path = _build.LIB
    if os.environ.get("TAHOE_LIB_AB"):   # same-box A/B experiments: another in-tree build
        path = os.path.join(os.path.dirname(_build.LIB), os.environ["TAHOE_LIB_AB"])
    elif build_if_missing:
        path = _build.build()
    if not os.path.exists(path):
        raise ImportError(f"libtahoe.so not found at {path}: run __graft_entry__.build()")
    L = ctypes.CDLL(path)
    P, i32, i64, f32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_float
    st = ctypes.c_int
    sig = {
        "tahoe_forest_build": (st, [i32, P, i32, P, P, P, P, P, P, P, i32, i32, i32, f32, i32, P]),
        "tahoe_forest_layout": (st, [P, P, i64, i32, P]),
        "tahoe_predict": (st, [P, P, i64, i32, P, P]),
        "tahoe_predict_ex": (st, [P, P, i64, i32, P, P, P]),
        "tahoe_predict_host": (st, [P, P, i64, i32, P, P, P]),
        "tahoe_forest_shard": (st, [P, i32, i32, i32, P]),
        "tahoe_predict_partial": (st, [P, P, i64, i32, P, P]),
        "tahoe_finalize": (st, [P, P, i64, P, P, P]),
        "tahoe_forest_n_outputs": (i32, [P]),
        "tahoe_forest_n_trees": (i32, [P]),
        "tahoe_forest_stats": (st, [P, P, i64]),
        "tahoe_select_strategy": (i32, [P, i64, i32]),
        "tahoe_predict_cost_us": (ctypes.c_double, [P, i32, i64]),
        "tahoe_forest_free": (None, [P]),
        "tahoe_last_error": (ctypes.c_char_p, []),
        "tahoe_forest_layout_info": (st, [P, P, P, P, P]),
        "tahoe_tree_tokens": (st, [P, i32, i32, P, P, i32, P]),
        "tahoe_tree_simhash": (st, [P, i32, i32, i32, P, P]),
        "tahoe_simhash": (st, [P, P, i32, i32, P, P]),
        "tahoe_lsh_order": (st, [P, i32, i32, i32, P, P]),
        "tahoe_sha1": (st, [P, i64, P]),
        "tahoe_forest_export_sliced": (st, [P, P, P, P, P, P]),
        "tahoe_count_visits": (st, [P, P, i64, i32, P, P]),
        "tahoe_forest_l2_persist": (st, [P, P, f32]),
        "tahoe_forest_layout_counts": (st, [P, P, i64, P, i64, i32, P]),
        "tahoe_comm_unique_id": (st, [P]),
        "tahoe_comm_init": (st, [P, i32, i32, i32, P]),
        "tahoe_comm_free": (None, [P]),
        "tahoe_reduce_rows": (st, [i64, i32, i32, i32, P, P]),
        "tahoe_predict_reduce": (st, [P, P, P, i64, i32, i32, P, P, P]),
        "tahoe_reduce_partials": (st, [P, P, i32, i32, i32, i64, P, P, P]),
        "tahoe_measure_visit_rate": (st, [i32, i32, i32, i32, P, P]),
        "tahoe_profile_walk": (st, [P, P, i64, i32, P, P, P]),
        "tahoe_forest_layout_export": (st, [P, P, i64, P]),
        "tahoe_forest_layout_import": (st, [P, P, i64]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    _lib = L
    return L


def _check(status: int):
    if status != TAHOE_OK:
        raise TahoeError(status, load().tahoe_last_error().decode())


def _np_ptr(a):
    return None if a is None else ctypes.c_void_p(a.ctypes.data)


def _dev_ptr(t):
    """Raw pointer of a torch tensor (device or host) or None."""
    if t is None:
        return None
    return ctypes.c_void_p(t.data_ptr())


def _stream_ptr(stream):
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


# ----------------------------------------------------------------------- C ABI names
def tahoe_forest_build(arrays: dict, n_features: int, n_classes: int = 1, agg: int = AGG_SUM,
                       base_score: float = 0.0, device: int = 0) -> ctypes.c_void_p:
    L = load()
    a = {k: np.ascontiguousarray(arrays[k]) for k in
         ("root", "feature", "threshold", "left", "right", "leaf_value")}
    a["root"] = a["root"].astype(np.int32, copy=False)
    for k in ("feature", "left", "right"):
        a[k] = a[k].astype(np.int32, copy=False)
    for k in ("threshold", "leaf_value"):
        a[k] = a[k].astype(np.float32, copy=False)
    dl = arrays.get("default_left")
    dl = None if dl is None else np.ascontiguousarray(dl, dtype=np.uint8)
    tc = arrays.get("tree_class")
    tc = None if tc is None else np.ascontiguousarray(tc, dtype=np.int32)
    h = ctypes.c_void_p()
    _check(L.tahoe_forest_build(len(a["root"]), _np_ptr(a["root"]), len(a["feature"]),
                                _np_ptr(a["feature"]), _np_ptr(a["threshold"]), _np_ptr(a["left"]),
                                _np_ptr(a["right"]), _np_ptr(a["leaf_value"]), _np_ptr(dl),
                                _np_ptr(tc), int(n_features), int(n_classes), int(agg),
                                float(base_score), int(device), ctypes.byref(h)))
    return h


def tahoe_forest_layout(h, X_calib: np.ndarray, opts: LayoutOpts | None = None):
    X = np.ascontiguousarray(X_calib, dtype=np.float32)
    _check(load().tahoe_forest_layout(h, _np_ptr(X), X.shape[0], X.shape[1],
                                      None if opts is None else ctypes.byref(opts)))


def tahoe_forest_layout_export(h) -> bytes:
    n = ctypes.c_int64()
    _check(load().tahoe_forest_layout_export(h, None, 0, ctypes.byref(n)))
    buf = ctypes.create_string_buffer(max(1, n.value))
    _check(load().tahoe_forest_layout_export(h, buf, n.value, ctypes.byref(n)))
    return buf.raw[: n.value]


def tahoe_forest_layout_import(h, blob: bytes):
    buf = ctypes.create_string_buffer(blob, len(blob))
    _check(load().tahoe_forest_layout_import(h, buf, len(blob)))


def tahoe_forest_l2_persist(h, stream=None, hit_ratio: float = 1.0):
    _check(load().tahoe_forest_l2_persist(h, _stream_ptr(stream), float(hit_ratio)))


def tahoe_count_visits(h, X, n: int, d: int, counts, stream=None):
    _check(load().tahoe_count_visits(h, _dev_ptr(X), n, d, _dev_ptr(counts), _stream_ptr(stream)))


def tahoe_forest_layout_counts(h, counts: np.ndarray, n_calib: int, X_sim: np.ndarray | None = None,
                               opts: LayoutOpts | None = None):
    c = np.ascontiguousarray(counts, dtype=np.uint64)
    Xs = None if X_sim is None else np.ascontiguousarray(X_sim, dtype=np.float32)
    _check(load().tahoe_forest_layout_counts(h, _np_ptr(c), n_calib, _np_ptr(Xs),
                                             0 if Xs is None else Xs.shape[0],
                                             0 if Xs is None else Xs.shape[1],
                                             None if opts is None else ctypes.byref(opts)))


def tahoe_predict(h, X, n: int, d: int, out, stream=None):
    _check(load().tahoe_predict(h, _dev_ptr(X), n, d, _dev_ptr(out), _stream_ptr(stream)))


def tahoe_predict_ex(h, X, n: int, d: int, out, out_class=None, out_leaf=None,
                     out_fingerprint=None, force_strategy: int = -1, stream=None,
                     ev_main_begin=None, ev_main_end=None):
    """ev_main_begin / ev_main_end: optional torch.cuda.Event (timing enabled, already recorded
    once) recorded around the main traversal kernel on ``stream``."""
    o = PredictOpts(_dev_ptr(out_class), _dev_ptr(out_leaf), _dev_ptr(out_fingerprint),
                    int(force_strategy), 0,
                    None if ev_main_begin is None else ctypes.c_void_p(ev_main_begin.cuda_event),
                    None if ev_main_end is None else ctypes.c_void_p(ev_main_end.cuda_event))
    _check(load().tahoe_predict_ex(h, _dev_ptr(X), n, d, _dev_ptr(out), ctypes.byref(o),
                                   _stream_ptr(stream)))


def tahoe_predict_host(h, X_host, n: int, d: int, out_host, class_host=None, stream=None):
    _check(load().tahoe_predict_host(h, _dev_ptr(X_host), n, d, _dev_ptr(out_host),
                                     _dev_ptr(class_host), _stream_ptr(stream)))


def tahoe_forest_shard(h, rank: int, world: int, device: int):
    s = ctypes.c_void_p()
    _check(load().tahoe_forest_shard(h, rank, world, device, ctypes.byref(s)))
    return s


def tahoe_predict_partial(shard, X, n: int, d: int, partial, stream=None):
    _check(load().tahoe_predict_partial(shard, _dev_ptr(X), n, d, _dev_ptr(partial),
                                        _stream_ptr(stream)))


def tahoe_finalize(h, partial, n: int, out, out_class=None, stream=None):
    _check(load().tahoe_finalize(h, _dev_ptr(partial), n, _dev_ptr(out), _dev_ptr(out_class),
                                 _stream_ptr(stream)))


def _nccl_hint():
    """Point the library at torch's NCCL (>= 2.28) unless the caller chose one."""
    if os.environ.get("TAHOE_NCCL_LIB"):
        return
    try:
        import nvidia.nccl as m  # type: ignore
        for base in list(getattr(m, "__path__", [])):
            lib = os.path.join(base, "lib", "libnccl.so.2")
            if os.path.exists(lib):
                os.environ["TAHOE_NCCL_LIB"] = lib
                return
    except ImportError:
        pass


def tahoe_comm_unique_id() -> bytes:
    _nccl_hint()
    buf = (ctypes.c_uint8 * COMM_ID_BYTES)()
    _check(load().tahoe_comm_unique_id(buf))
    return bytes(buf)


def tahoe_comm_init(uid: bytes, world: int, rank: int, device: int):
    _nccl_hint()
    if len(uid) != COMM_ID_BYTES:
        raise ValueError("communicator id must be 128 bytes")
    buf = (ctypes.c_uint8 * COMM_ID_BYTES).from_buffer_copy(uid)
    c = ctypes.c_void_p()
    _check(load().tahoe_comm_init(buf, world, rank, device, ctypes.byref(c)))
    return c


def tahoe_comm_free(c):
    if c:
        load().tahoe_comm_free(c)


def tahoe_reduce_rows(n: int, world: int, rank: int, mode: int = REDUCE_SCATTER) -> tuple[int, int]:
    lo, hi = ctypes.c_int64(), ctypes.c_int64()
    _check(load().tahoe_reduce_rows(n, world, rank, mode, ctypes.byref(lo), ctypes.byref(hi)))
    return lo.value, hi.value


def tahoe_predict_reduce(shard, comm, X, n: int, d: int, mode: int, out, out_class=None,
                         stream=None):
    _check(load().tahoe_predict_reduce(shard, comm, _dev_ptr(X), n, d, mode, _dev_ptr(out),
                                       _dev_ptr(out_class), _stream_ptr(stream)))


def tahoe_reduce_partials(full, partials, world: int, rank: int, mode: int, n: int, out,
                          out_class=None, stream=None):
    """partials: sequence of `world` device tensors (or raw pointers) of fp64 [n x n_out]."""
    arr = (ctypes.c_void_p * max(1, world))(
        *[p if isinstance(p, int) else p.data_ptr() for p in partials])
    _check(load().tahoe_reduce_partials(full, arr, world, rank, mode, n, _dev_ptr(out),
                                        _dev_ptr(out_class), _stream_ptr(stream)))


def tahoe_measure_visit_rate(device: int = 0, variant: int = 0, steps: int = 256,
                             reps: int = 400, smem_bw: bool = True) -> tuple[float, float | None]:
    """(node reads per second of the ideal coded walk, shared-memory bytes per SM clock)."""
    r = ctypes.c_double()
    b = ctypes.c_double()
    _check(load().tahoe_measure_visit_rate(device, variant, steps, reps, ctypes.byref(r),
                                           ctypes.byref(b) if smem_bw else None))
    return r.value, (b.value if smem_bw else None)


def tahoe_profile_walk(h, X, n: int, d: int, out, stream=None) -> dict:
    """Instrumented coded walk (per-lane SM-clock spans): load-balance statistics of the launch."""
    st = np.zeros(8, np.float64)
    _check(load().tahoe_profile_walk(h, _dev_ptr(X), n, d, _dev_ptr(out), _np_ptr(st),
                                     _stream_ptr(stream)))
    u, w = max(st[2], 1.0), max(st[5], 1.0)
    return dict(unit_cv=st[0] / u, unit_lockstep=st[1] / u, mean_span_cycles=st[3] / u,
                lane_total_cv=st[4] / w, units=int(st[2]), warps=int(st[5]))


def tahoe_forest_n_outputs(h) -> int:
    return int(load().tahoe_forest_n_outputs(h))


def tahoe_forest_n_trees(h) -> int:
    return int(load().tahoe_forest_n_trees(h))


def tahoe_forest_stats(h) -> dict:
    buf = ctypes.create_string_buffer(65536)
    _check(load().tahoe_forest_stats(h, buf, len(buf)))
    return json.loads(buf.value.decode())


def tahoe_select_strategy(h, n: int, d: int) -> int:
    return int(load().tahoe_select_strategy(h, n, d))


def tahoe_predict_cost_us(h, strategy: int, n: int) -> float:
    return float(load().tahoe_predict_cost_us(h, strategy, n))


def tahoe_forest_free(h):
    if h:
        load().tahoe_forest_free(h)


def tahoe_last_error() -> str:
    return load().tahoe_last_error().decode()


def tahoe_forest_layout_info(h, n_nodes: int, n_trees: int) -> dict:
    cnt = np.zeros(n_nodes, np.uint64)
    hot = np.zeros(n_nodes, np.uint8)
    er = np.zeros(n_trees, np.float64)
    order = np.zeros(n_trees, np.int32)
    _check(load().tahoe_forest_layout_info(h, _np_ptr(cnt), _np_ptr(hot), _np_ptr(er),
                                           _np_ptr(order)))
    return dict(count=cnt, hot_left=hot, exp_reads=er, order=order)


def tahoe_tree_tokens(h, t: int, t_nodes: int):
    n = ctypes.c_int32()
    _check(load().tahoe_tree_tokens(h, t, t_nodes, None, None, 0, ctypes.byref(n)))
    tok = np.zeros((n.value, t_nodes), np.int32)
    w = np.zeros(n.value, np.float64)
    _check(load().tahoe_tree_tokens(h, t, t_nodes, _np_ptr(tok), _np_ptr(w), n.value,
                                    ctypes.byref(n)))
    return tok, w


def tahoe_tree_simhash(h, t: int, t_nodes: int = 4, l_hash: int = 128):
    cs = np.zeros(l_hash, np.float64)
    bits = np.zeros(l_hash, np.uint8)
    _check(load().tahoe_tree_simhash(h, t, t_nodes, l_hash, _np_ptr(cs), _np_ptr(bits)))
    return cs, bits


def tahoe_simhash(strings: np.ndarray, weights: np.ndarray):
    s = np.ascontiguousarray(strings, dtype=np.int8)
    w = np.ascontiguousarray(weights, dtype=np.float64)
    cs = np.zeros(s.shape[1], np.float64)
    bits = np.zeros(s.shape[1], np.uint8)
    _check(load().tahoe_simhash(_np_ptr(s), _np_ptr(w), s.shape[0], s.shape[1], _np_ptr(cs),
                                _np_ptr(bits)))
    return cs, bits


def tahoe_lsh_order(bits: np.ndarray, m_chunks: int):
    b = np.ascontiguousarray(bits, dtype=np.uint8)
    T, L = b.shape
    col = np.zeros((T, T), np.int32)
    order = np.zeros(T, np.int32)
    _check(load().tahoe_lsh_order(_np_ptr(b), T, L, m_chunks, _np_ptr(col), _np_ptr(order)))
    return col, order


def tahoe_sha1(msg: bytes) -> bytes:
    buf = (ctypes.c_uint8 * max(1, len(msg))).from_buffer_copy(msg or b"\0")
    out = (ctypes.c_uint8 * 20)()
    _check(load().tahoe_sha1(buf, len(msg), out))
    return bytes(out)


def tahoe_forest_export_sliced(h) -> dict | None:
    L = load()
    hdr = np.zeros(8, np.int32)
    _check(L.tahoe_forest_export_sliced(h, _np_ptr(hdr), None, None, None, None))
    ns, smax, C = int(hdr[0]), int(hdr[1]), int(hdr[5])
    if ns == 0:
        return None
    info = np.zeros((ns, 4), np.int32)
    col = np.zeros((ns, C), np.int32)
    nodes = np.zeros((ns, smax, C, 2), np.uint32)
    meta = np.zeros((ns, smax, C, 2), np.int32)
    _check(L.tahoe_forest_export_sliced(h, _np_ptr(hdr), _np_ptr(info), _np_ptr(col),
                                        _np_ptr(nodes), _np_ptr(meta)))
    return dict(n_slices=ns, slots_max=smax, feature_bits=int(hdr[2]), n_trees=int(hdr[3]),
                n_classes=int(hdr[4]), cols=C, slot_bytes=int(hdr[6]), slice_info=info,
                col_len=col, nodes=nodes, leaf_meta=meta)


# ----------------------------------------------------------------------- convenience wrapper
def _need(t, name: str, dtype, shape: tuple, device: int | None):
    """Validate a tensor handed to the C ABI: the library reads raw pointers with a row stride of
    shape[1], so a strided view, a wrong dtype, a wrong shape or a tensor on another device would
    give silently wrong results or a fault.  device None: a host tensor; else cuda:<device>."""
    import torch
    if t is None:
        return
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name}: expected a torch.Tensor, got {type(t).__name__}")
    if t.dtype != dtype:
        raise TypeError(f"{name}: dtype {t.dtype}, expected {dtype}")
    if tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name}: shape {tuple(t.shape)}, expected {tuple(shape)}")
    if not t.is_contiguous():
        raise ValueError(f"{name}: must be contiguous (row-major, row stride = shape[1])")
    if device is None:
        if t.is_cuda:
            raise ValueError(f"{name}: expected a host tensor")
    elif not t.is_cuda or t.device.index != device:
        raise ValueError(f"{name}: on {t.device}, expected cuda:{device}")


def _need_X(X, name: str, device: int | None):
    """X: [n, d] float32, d >= the forest's feature count (checked by the library)."""
    import torch
    if not isinstance(X, torch.Tensor) or X.dim() != 2:
        raise ValueError(f"{name}: expected a 2-D torch tensor")
    _need(X, name, torch.float32, tuple(X.shape), device)
    return X.shape


class Forest:
    """Owns a tahoe_forest handle.  ``arrays`` are the user-level node arrays (as produced by
    gen.make_forest)."""

    def __init__(self, arrays: dict, n_features: int | None = None, n_classes: int | None = None,
                 agg: int | None = None, base_score: float = 0.0, device: int = 0):
        self.n_features = int(arrays.get("n_features") if n_features is None else n_features)
        self.n_classes = int(arrays.get("n_classes", 1) if n_classes is None else n_classes)
        self.agg = int(arrays.get("agg", AGG_SUM) if agg is None else agg)
        self.device = device
        self.n_nodes = len(arrays["feature"])
        self.handle = tahoe_forest_build(arrays, self.n_features, self.n_classes, self.agg,
                                         base_score, device)
        self.n_trees = tahoe_forest_n_trees(self.handle)
        self.n_trees_full = self.n_trees
        self.n_out = tahoe_forest_n_outputs(self.handle)

    @classmethod
    def _wrap(cls, handle, like: "Forest", device: int):
        f = cls.__new__(cls)
        f.n_features, f.n_classes, f.agg = like.n_features, like.n_classes, like.agg
        f.device, f.n_nodes, f.handle = device, like.n_nodes, handle
        f.n_trees = tahoe_forest_n_trees(handle)
        f.n_trees_full = like.n_trees_full   # leaf ids of a shard use the full forest's tree ids
        f.n_out = tahoe_forest_n_outputs(handle)
        return f

    def layout(self, X_calib: np.ndarray, **kw):
        opts = None
        if kw:
            opts = LayoutOpts(kw.get("t_nodes", 0), kw.get("l_hash", 0), kw.get("m_chunks", 0),
                              kw.get("node_reorder", 1), kw.get("tree_group", 1), 0,
                              kw.get("seed", 0))
        tahoe_forest_layout(self.handle, X_calib, opts)
        return self

    def layout_state(self) -> bytes:
        """The handle's layout state (tahoe_forest_layout_export) — ship it to other ranks."""
        return tahoe_forest_layout_export(self.handle)

    def apply_layout_state(self, blob: bytes):
        """Apply another handle's layout of the same forest (tahoe_forest_layout_import)."""
        tahoe_forest_layout_import(self.handle, blob)
        return self

    def layout_gpu(self, X_calib_dev, **kw):
        """Layout from visit counts measured on the GPU (tahoe_count_visits) over the device rows
        X_calib_dev; a host copy of up to 1024 of them feeds the lockstep simulation and balancing."""
        import torch
        n, d = X_calib_dev.shape
        cnt = torch.zeros(self.n_nodes, dtype=torch.int32, device=X_calib_dev.device)
        tahoe_count_visits(self.handle, X_calib_dev, n, d, cnt)
        counts = cnt.cpu().numpy().view(np.uint32).astype(np.uint64)
        step = max(1, n // 1024)
        X_sim = X_calib_dev[::step][:1024].cpu().numpy()
        opts = None
        if kw:
            opts = LayoutOpts(kw.get("t_nodes", 0), kw.get("l_hash", 0), kw.get("m_chunks", 0),
                              kw.get("node_reorder", 1), kw.get("tree_group", 1), 0, kw.get("seed", 0))
        tahoe_forest_layout_counts(self.handle, counts, n, X_sim, opts)
        return counts

    def stats(self) -> dict:
        return tahoe_forest_stats(self.handle)

    def select_strategy(self, n: int, d: int) -> int:
        return tahoe_select_strategy(self.handle, n, d)

    def predict_cost_us(self, strategy: int, n: int) -> float:
        return tahoe_predict_cost_us(self.handle, strategy, n)

    def _stream(self, stream):
        import torch
        return torch.cuda.current_stream(self.device) if stream is None else stream

    def predict(self, X, out=None, out_class=None, out_leaf=None, out_fingerprint=None,
                force_strategy: int = -1, stream=None, ev_main_begin=None, ev_main_end=None):
        """X: torch tensor on the forest's device (n x d float32).  Returns ``out``."""
        import torch
        n, d = _need_X(X, "X", self.device)
        if out is None:
            out = torch.empty((n, self.n_out), dtype=torch.float32, device=X.device)
        _need(out, "out", torch.float32, (n, self.n_out), self.device)
        _need(out_class, "out_class", torch.int32, (n,), self.device)
        _need(out_leaf, "out_leaf", torch.int32, (n, self.n_trees_full), self.device)
        _need(out_fingerprint, "out_fingerprint", torch.int64, (n,), self.device)
        stream = self._stream(stream)
        if (out_class is None and out_leaf is None and out_fingerprint is None
                and force_strategy < 0 and ev_main_begin is None):
            tahoe_predict(self.handle, X, n, d, out, stream)
        else:
            tahoe_predict_ex(self.handle, X, n, d, out, out_class, out_leaf, out_fingerprint,
                             force_strategy, stream, ev_main_begin, ev_main_end)
        return out

    def predict_host(self, X_host, out_host, class_host=None, stream=None):
        import torch
        n, d = _need_X(X_host, "X_host", None)
        _need(out_host, "out_host", torch.float32, (n, self.n_out), None)
        _need(class_host, "class_host", torch.int32, (n,), None)
        tahoe_predict_host(self.handle, X_host, n, d, out_host, class_host, self._stream(stream))
        return out_host

    def shard(self, rank: int, world: int, device: int | None = None) -> "Forest":
        dev = self.device if device is None else device
        return Forest._wrap(tahoe_forest_shard(self.handle, rank, world, dev), self, dev)

    def predict_partial(self, X, partial=None, stream=None):
        import torch
        n, d = _need_X(X, "X", self.device)
        if partial is None:
            partial = torch.empty((n, self.n_out), dtype=torch.float64, device=X.device)
        _need(partial, "partial", torch.float64, (n, self.n_out), self.device)
        tahoe_predict_partial(self.handle, X, n, d, partial, self._stream(stream))
        return partial

    def finalize(self, partial, out=None, out_class=None, stream=None):
        import torch
        n = partial.shape[0]
        _need(partial, "partial", torch.float64, (n, self.n_out), self.device)
        if out is None:
            out = torch.empty((n, self.n_out), dtype=torch.float32, device=partial.device)
        _need(out, "out", torch.float32, (n, self.n_out), self.device)
        _need(out_class, "out_class", torch.int32, (n,), self.device)
        tahoe_finalize(self.handle, partial, n, out, out_class, self._stream(stream))
        return out

    def export_sliced(self):
        return tahoe_forest_export_sliced(self.handle)

    def predict_reduce(self, comm: "Comm", X, mode: int = REDUCE_SCATTER, out=None,
                       out_class=None, stream=None):
        """Collective tree-sharded prediction with this shard (tahoe_predict_reduce): returns this
        rank's rows [lo, hi) of the finalised output."""
        import torch
        n, d = _need_X(X, "X", self.device)
        lo, hi = tahoe_reduce_rows(n, comm.world, comm.rank, mode)
        if out is None:
            out = torch.empty((hi - lo, self.n_out), dtype=torch.float32, device=X.device)
        _need(out, "out", torch.float32, (hi - lo, self.n_out), self.device)
        _need(out_class, "out_class", torch.int32, (hi - lo,), self.device)
        tahoe_predict_reduce(self.handle, comm.handle, X, n, d, mode, out, out_class,
                             self._stream(stream))
        return out

    def reduce_partials(self, partials, rank: int, mode: int = REDUCE_SCATTER, out=None,
                        out_class=None, stream=None):
        """Fixed-order sum + finalisation of per-shard partials resident on this device."""
        import torch
        n = partials[0].shape[0]
        for q, p in enumerate(partials):
            if isinstance(p, torch.Tensor):
                _need(p, f"partials[{q}]", torch.float64, (n, self.n_out), self.device)
        lo, hi = tahoe_reduce_rows(n, len(partials), rank, mode)
        if out is None:
            out = torch.empty((hi - lo, self.n_out), dtype=torch.float32, device=partials[0].device)
        _need(out, "out", torch.float32, (hi - lo, self.n_out), self.device)
        _need(out_class, "out_class", torch.int32, (hi - lo,), self.device)
        tahoe_reduce_partials(self.handle, partials, len(partials), rank, mode, n, out, out_class,
                              self._stream(stream))
        return out

    def close(self):
        if getattr(self, "handle", None):
            tahoe_forest_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Comm:
    """Owns a tahoe_comm (NCCL communicator + device communicator with LSA barriers).  Every rank
    constructs it with the same 128-byte id (tahoe_comm_unique_id on one rank, broadcast by the
    caller; dist.init_comm does both over torch.distributed)."""

    def __init__(self, uid: bytes, world: int, rank: int, device: int):
        self.world, self.rank, self.device = int(world), int(rank), int(device)
        self.handle = tahoe_comm_init(uid, self.world, self.rank, self.device)

    def close(self):
        if getattr(self, "handle", None):
            tahoe_comm_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
