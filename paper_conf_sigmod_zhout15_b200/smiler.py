"""Thin ctypes binding of libsmiler.so (include/smiler.h).

Argument marshalling only: every step of the Search Step runs in the library's
CUDA kernels.  Buffers may be numpy arrays (host) or torch tensors (host or
CUDA); their raw pointers are passed straight to the C ABI.  There is no CPU
fallback: if libsmiler.so is missing or has no usable CUDA device the calls
raise.
"""
from __future__ import annotations

import ctypes
import os
from typing import Any, Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libsmiler.so")

SMILER_I16 = 0
SMILER_F32 = 1
STATUS = {0: "OK", -1: "EINVAL", -2: "ERANGE", -3: "ENOMEM", -4: "ECUDA", -5: "ENCCL"}


class SmilerError(RuntimeError):
    def __init__(self, fn: str, code: int, msg: str):
        super().__init__("%s -> %s: %s" % (fn, STATUS.get(code, code), msg))
        self.code = code


class KnnStats(ctypes.Structure):
    _fields_ = [("candidates", ctypes.c_int64), ("tau_verified", ctypes.c_int64),
                ("survivors", ctypes.c_int64), ("finalists", ctypes.c_int64),
                ("dtw_cells", ctypes.c_double), ("bf_cells", ctypes.c_double),
                ("posting_bytes", ctypes.c_int64), ("lb_bytes", ctypes.c_int64),
                ("kernel_launches", ctypes.c_int32), ("mq_chunks", ctypes.c_int32),
                ("ns_prep", ctypes.c_double), ("ns_window_lb", ctypes.c_double),
                ("ns_group_scan", ctypes.c_double), ("ns_tau", ctypes.c_double),
                ("ns_filter", ctypes.c_double), ("ns_verify", ctypes.c_double),
                ("ns_select", ctypes.c_double), ("ns_total", ctypes.c_double),
                ("cascade_pruned", ctypes.c_int64), ("ns_cascade", ctypes.c_double)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class KnnOpts(ctypes.Structure):
    _fields_ = [("no_prune", ctypes.c_int32), ("timing", ctypes.c_int32),
                ("mq_chunk", ctypes.c_int32), ("two_level", ctypes.c_int32),
                ("lb_kind", ctypes.c_int32), ("horizon", ctypes.c_int32),
                ("exact_postings", ctypes.c_int32), ("tau_mult", ctypes.c_int32), ("variant", ctypes.c_int32),
                ("reserved", ctypes.c_int32), ("tau_keep", ctypes.c_int32), ("shared_tau", ctypes.c_void_p)]


# smiler_knn_opts.variant: kernel paths with the same (exact) result, for tests and A/B timing
VARIANTS = {"auto": 0, "row_fused": 1, "scalar_diag": 2, "wave_dtw": 3, "no_cascade": 4, "no_lag": 5, "packed_dtw": 6, "ring_no_tma": 7, "tma_one_tile": 8, "trim_radix": 9, "trim_two_stage": 10}


# smiler_knn_opts.lb_kind (include/smiler.h): the lower bound that filters candidates
SMILER_LB_INDEX, SMILER_LB_INDEX_EQ, SMILER_LB_INDEX_EC, SMILER_LB_DIRECT, SMILER_LB_DIRECT_SHARED = 0, 1, 2, 3, 4
LB_KINDS = {"index": 0, "index_eq": 1, "index_ec": 2, "direct": 3, "direct_shared": 4}


_lib = None


def lib():
    """Load libsmiler.so (raises if it has not been built: no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError("libsmiler.so not built (run python -m paper_conf_sigmod_zhout15_b200.build); "
                              "there is no CPU fallback")
        L = ctypes.CDLL(LIB_PATH)
        P, i32, i64, f32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_float
        L.smiler_index_build.argtypes = [P, i32, i64, P, i32, i32, f32, i32, P, ctypes.POINTER(P)]
        L.smiler_index_build_shard.argtypes = [P, i32, i64, i64, i64, i64, i64, i32, f32, i32, P,
                                               ctypes.POINTER(P)]
        L.smiler_knn.argtypes = [P, P, P, i32, P, i32, i32, P, P, P]
        L.smiler_knn_ex.argtypes = [P, P, P, i32, P, i32, i32, P, P, P, P]
        L.smiler_knn_step.argtypes = [P, P, P, i32, P, i32, i32, P, i32, P, P, P, P]
        L.smiler_stream_create.argtypes = [P, P, P, i32, P, i32, i32, P, P, ctypes.POINTER(P)]
        L.smiler_stream_create_ex.argtypes = [P, P, P, i32, P, i32, i32, P, P, P, ctypes.POINTER(P)]
        L.smiler_stream_step.argtypes = [P, P, P, P, P, P]
        L.smiler_stream_free.argtypes = [P]
        L.smiler_stream_free.restype = None
        L.smiler_merge_topk.argtypes = [P, P, i32, i32, i32, i32, P, P, i32, P]
        L.smiler_index_envelope.argtypes = [P, i32, i32, P, P]
        L.smiler_lower_bounds.argtypes = [P, P, P, i32, P, i32, P, P]
        L.smiler_lower_bounds_ex.argtypes = [P, P, P, i32, P, i32, i32, P]
        L.smiler_predict.argtypes = [P, P, P, i32, P, i32, P, i32, P, i32, i32, P, P, P, P, P]
        L.smiler_dtw.argtypes = [P, i32, P, i32, i32, P, i64, P]
        L.smiler_free.argtypes = [P]
        L.smiler_free.restype = None
        L.smiler_last_error.restype = ctypes.c_char_p
        L.smiler_abi_version.restype = i32
        for f in ("smiler_index_build", "smiler_index_build_shard", "smiler_knn", "smiler_knn_ex", "smiler_knn_step",
                  "smiler_stream_create", "smiler_stream_create_ex", "smiler_stream_step",
                  "smiler_merge_topk", "smiler_index_envelope", "smiler_lower_bounds", "smiler_lower_bounds_ex",
                  "smiler_dtw", "smiler_predict"):
            getattr(L, f).restype = i32
        _lib = L
    return _lib


def _check(fn: str, rc: int):
    if rc != 0:
        raise SmilerError(fn, rc, lib().smiler_last_error().decode())


def _ptr(x: Any) -> Optional[int]:
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        if not x.flags["C_CONTIGUOUS"]:
            raise ValueError("arrays must be C-contiguous")
        return x.ctypes.data
    if hasattr(x, "data_ptr"):
        if not x.is_contiguous():
            raise ValueError("tensors must be contiguous")
        return x.data_ptr()
    raise TypeError(type(x))


def _np_or_tensor_dtype(x) -> str:
    return str(x.dtype).replace("torch.", "")


def _check_buf(name: str, x, dtype: str, shape) -> None:
    """An argument the C side reads or writes as `dtype` with `shape` elements."""
    if x is None:
        raise ValueError("%s is None" % name)
    got = _np_or_tensor_dtype(x)
    if got != dtype:
        raise TypeError("%s must be %s, got %s" % (name, dtype, got))
    if tuple(x.shape) != tuple(shape):
        raise ValueError("%s must have shape %s, got %s" % (name, tuple(shape), tuple(x.shape)))


def _queries_for(index_code: int, queries, lengths):
    """Queries as the index dtype, [n_mq, D] with D = lengths[-1].  numpy float
    arrays are cast to float32 for an F32 index, integer arrays to int16 for an
    I16 index (values are range-checked by the library, R17); tensors must
    already have the index dtype (no implicit device copy)."""
    want = "int16" if index_code == SMILER_I16 else "float32"
    if queries.ndim != 2 or int(queries.shape[1]) != int(lengths[-1]):
        raise ValueError("queries must be [n_mq, D] with D = lengths[-1] = %d, got shape %s"
                         % (int(lengths[-1]), tuple(queries.shape)))
    if isinstance(queries, np.ndarray):
        if queries.dtype != np.dtype(want):
            if want == "float32" and np.issubdtype(queries.dtype, np.floating):
                queries = queries.astype(np.float32)
            elif want == "int16" and np.issubdtype(queries.dtype, np.integer):
                if queries.size and (queries.max() > 32767 or queries.min() < -32768):
                    raise ValueError("I16 queries must satisfy |x| <= 1023")
                queries = queries.astype(np.int16)
            else:
                raise TypeError("queries must be %s for this index, got %s" % (want, queries.dtype))
        return np.ascontiguousarray(queries)
    if _np_or_tensor_dtype(queries) != want:
        raise TypeError("queries must be %s for this index, got %s" % (want, queries.dtype))
    return queries


def _check_knn_args(queries, lengths, k: int, ids, dists) -> None:
    """Shapes and dtypes the C side relies on: queries [n_mq, D] int16/float32,
    ids int64 and dists int32/float32 (matching the queries) of [n_mq, n_len, k]."""
    qd = _np_or_tensor_dtype(queries)
    if qd not in ("int16", "float32"):
        raise TypeError("queries must be int16 or float32 (the index dtype), got %s" % qd)
    if queries.ndim != 2 or int(queries.shape[1]) != int(lengths[-1]):
        raise ValueError("queries must be [n_mq, D] with D = lengths[-1] = %d, got shape %s"
                         % (int(lengths[-1]), tuple(queries.shape)))
    shape = (int(queries.shape[0]), len(lengths), int(k))
    _check_buf("ids", ids, "int64", shape)
    _check_buf("dists", dists, "int32" if qd == "int16" else "float32", shape)


def _query_sensor(qs, n_mq: int):
    if qs is None:
        return None
    if hasattr(qs, "data_ptr"):
        if _np_or_tensor_dtype(qs) != "int32" or tuple(qs.shape) != (n_mq,):
            raise TypeError("query_sensor tensors must be int32 of shape (%d,)" % n_mq)
        return qs
    a = np.ascontiguousarray(qs, np.int32)
    if a.shape != (n_mq,):
        raise ValueError("query_sensor must have %d entries" % n_mq)
    return a


def _dtype_code(x: Any) -> int:
    name = str(x.dtype)
    if "int16" in name:
        return SMILER_I16
    if "float32" in name:
        return SMILER_F32
    raise TypeError("series dtype must be int16 or float32, got %s" % name)


def _stream_ptr(stream) -> Optional[int]:
    if stream is None:
        return None
    return int(getattr(stream, "cuda_stream", stream))


# ---------------------------------------------------------------------------
# The ABI calls, same names as include/smiler.h
# ---------------------------------------------------------------------------
def smiler_index_build(series, sensor_offsets=None, window: int = 16, band: float = 8.0,
                       device: int = 0, stream=None) -> int:
    h = ctypes.c_void_p()
    offs = None
    ns = 1
    if sensor_offsets is not None:
        offs = np.ascontiguousarray(sensor_offsets, dtype=np.int64)
        ns = len(offs) - 1
    n_total = int(series.shape[0]) if hasattr(series, "shape") else len(series)
    _check("smiler_index_build",
           lib().smiler_index_build(_ptr(series), _dtype_code(series), n_total, _ptr(offs), ns, window,
                                    float(band), device, _stream_ptr(stream), ctypes.byref(h)))
    return h.value


def smiler_index_build_shard(slice_, slice_begin: int, n_global: int, t_begin: int, t_end: int,
                             window: int, band: float, device: int = 0, stream=None) -> int:
    h = ctypes.c_void_p()
    _check("smiler_index_build_shard",
           lib().smiler_index_build_shard(_ptr(slice_), _dtype_code(slice_), int(slice_.shape[0]),
                                          slice_begin, n_global, t_begin, t_end, window, float(band),
                                          device, _stream_ptr(stream), ctypes.byref(h)))
    return h.value


def smiler_knn(handle: int, queries, query_sensor, lengths, k: int, ids, dists,
               stats: Optional[KnnStats] = None, opts: Optional[KnnOpts] = None) -> None:
    """Fills ids [n_mq, n_len, k] int64 and dists [n_mq, n_len, k] int32/float32
    (host numpy or device tensors, caller-allocated)."""
    lens = np.ascontiguousarray(lengths, dtype=np.int32)
    _check_knn_args(queries, lens, k, ids, dists)
    n_mq = int(queries.shape[0])
    qs = _query_sensor(query_sensor, n_mq)
    _check("smiler_knn",
           lib().smiler_knn_ex(handle, _ptr(queries), _ptr(qs), n_mq, _ptr(lens), len(lens), k, _ptr(ids),
                               _ptr(dists), ctypes.byref(stats) if stats is not None else None,
                               ctypes.byref(opts) if opts is not None else None))


def smiler_knn_step(handle: int, queries, query_sensor, lengths, k: int, prev_ids, shift: int, ids, dists,
                    stats: Optional[KnnStats] = None, opts: Optional[KnnOpts] = None) -> None:
    """One continuous step: like smiler_knn, with the previous step's ids of the
    same streams seeding each item query's threshold."""
    lens = np.ascontiguousarray(lengths, dtype=np.int32)
    _check_knn_args(queries, lens, k, ids, dists)
    n_mq = int(queries.shape[0])
    _check_buf("prev_ids", prev_ids, "int64", (n_mq, len(lens), int(k)))
    qs = _query_sensor(query_sensor, n_mq)
    _check("smiler_knn_step",
           lib().smiler_knn_step(handle, _ptr(queries), _ptr(qs), n_mq, _ptr(lens), len(lens), k, _ptr(prev_ids),
                                 shift, _ptr(ids), _ptr(dists), ctypes.byref(stats) if stats is not None else None,
                                 ctypes.byref(opts) if opts is not None else None))


def smiler_stream_create(handle: int, queries, query_sensor, lengths, k: int, ids, dists,
                         opts: Optional[KnnOpts] = None) -> int:
    """Create a batch of continuous streams (Remark 1) and run their first search."""
    h = ctypes.c_void_p()
    lens = np.ascontiguousarray(lengths, dtype=np.int32)
    _check_knn_args(queries, lens, k, ids, dists)
    qs = _query_sensor(query_sensor, int(queries.shape[0]))
    _check("smiler_stream_create",
           lib().smiler_stream_create_ex(handle, _ptr(queries), _ptr(qs), int(queries.shape[0]), _ptr(lens),
                                         len(lens), k, _ptr(ids), _ptr(dists),
                                         ctypes.byref(opts) if opts is not None else None, ctypes.byref(h)))
    return h.value


def smiler_stream_step(stream: int, new_points, ids, dists, stats: Optional[KnnStats] = None,
                       opts: Optional[KnnOpts] = None) -> None:
    _check("smiler_stream_step",
           lib().smiler_stream_step(stream, _ptr(new_points), _ptr(ids), _ptr(dists),
                                    ctypes.byref(stats) if stats is not None else None,
                                    ctypes.byref(opts) if opts is not None else None))


def smiler_stream_free(stream: Optional[int]) -> None:
    lib().smiler_stream_free(stream)


def smiler_merge_topk(ids_in, dists_in, G: int, rows: int, k: int, ids_out, dists_out,
                      device: int = 0, stream=None) -> None:
    _check("smiler_merge_topk",
           lib().smiler_merge_topk(_ptr(ids_in), _ptr(dists_in), _dtype_code_dist(dists_in), G, rows, k,
                                   _ptr(ids_out), _ptr(dists_out), device, _stream_ptr(stream)))


def _dtype_code_dist(x) -> int:
    name = str(x.dtype)
    if "int32" in name:
        return SMILER_I16
    if "float32" in name:
        return SMILER_F32
    raise TypeError("dists dtype must be int32 or float32, got %s" % name)


def smiler_index_envelope(handle: int, sensor: int, rho: int, U, L) -> None:
    _check("smiler_index_envelope", lib().smiler_index_envelope(handle, sensor, rho, _ptr(U), _ptr(L)))


def smiler_lower_bounds(handle: int, queries, query_sensor, lengths, postings, lbw) -> None:
    lens = np.ascontiguousarray(lengths, dtype=np.int32)
    qs = None if query_sensor is None else np.ascontiguousarray(query_sensor, np.int32)
    _check("smiler_lower_bounds",
           lib().smiler_lower_bounds(handle, _ptr(queries), _ptr(qs), int(queries.shape[0]), _ptr(lens),
                                     len(lens), _ptr(postings), _ptr(lbw)))


def smiler_lower_bounds_ex(handle: int, queries, query_sensor, lengths, lb_kind: int, lb) -> None:
    lens = np.ascontiguousarray(lengths, dtype=np.int32)
    qs = None if query_sensor is None else np.ascontiguousarray(query_sensor, np.int32)
    _check("smiler_lower_bounds_ex",
           lib().smiler_lower_bounds_ex(handle, _ptr(queries), _ptr(qs), int(queries.shape[0]), _ptr(lens),
                                        len(lens), int(lb_kind), _ptr(lb)))


def smiler_predict(handle: int, queries, query_sensor, lengths, ids, ekv, horizon: int, theta,
                   ar_mean, ar_var, gp_mean, gp_var) -> None:
    """AR (Eq. 12-13) and GP (Eq. 16-18) predictors of every (MQ, item query, k_j in ekv)
    from the kNN ids (see include/smiler.h).  Host (numpy) or device (torch) buffers."""
    lens = np.ascontiguousarray(lengths, dtype=np.int32)
    ek = np.ascontiguousarray(ekv, dtype=np.int32)
    qs = query_sensor if (query_sensor is None or hasattr(query_sensor, "data_ptr")) \
        else np.ascontiguousarray(query_sensor, np.int32)
    _check("smiler_predict",
           lib().smiler_predict(handle, _ptr(queries), _ptr(qs), int(queries.shape[0]), _ptr(lens), len(lens),
                                _ptr(ids), int(ids.shape[-1]), _ptr(ek), len(ek), int(horizon), _ptr(theta),
                                _ptr(ar_mean), _ptr(ar_var), _ptr(gp_mean), _ptr(gp_var)))


def smiler_dtw(handle: int, sensor: int, q, rho: int, ts, dists) -> None:
    tsa = np.ascontiguousarray(ts, dtype=np.int64) if not hasattr(ts, "data_ptr") else ts
    _check("smiler_dtw", lib().smiler_dtw(handle, sensor, _ptr(q), int(q.shape[0]), rho, _ptr(tsa),
                                          int(tsa.shape[0]), _ptr(dists)))


def smiler_free(handle: Optional[int]) -> None:
    lib().smiler_free(handle)


def smiler_abi_version() -> int:
    return int(lib().smiler_abi_version())


# ---------------------------------------------------------------------------
# Convenience wrapper (host numpy in, host numpy out)
# ---------------------------------------------------------------------------
class Stream:
    """A batch of continuous master-query streams over one Index (host numpy I/O)."""

    def __init__(self, index: "Index", queries, lengths: Sequence[int], k: int, query_sensor=None,
                 exact_postings: bool = False):
        self.index, self.lengths, self.k = index, list(lengths), k
        queries = _queries_for(index.dtype, queries, lengths)
        self.n = int(queries.shape[0])
        self.vt = np.int32 if index.dtype == SMILER_I16 else np.float32
        ids = np.empty((self.n, len(lengths), k), np.int64)
        dists = np.empty((self.n, len(lengths), k), self.vt)
        self.handle = smiler_stream_create(index.handle, queries, query_sensor, lengths, k,
                                           ids, dists, KnnOpts(exact_postings=int(exact_postings)))
        self.first = (ids, dists)

    def step(self, new_points, stats: bool = False, timing: bool = False, tau_mult: int = 0, variant=0):
        ids = np.empty((self.n, len(self.lengths), self.k), np.int64)
        dists = np.empty((self.n, len(self.lengths), self.k), self.vt)
        st = KnnStats() if stats else None
        new_points = np.asarray(new_points)
        if new_points.shape != (self.n,):
            raise ValueError("new_points must have one point per stream (%d)" % self.n)
        new_points = np.ascontiguousarray(new_points, self.vt if self.vt is np.float32 else np.int16)
        smiler_stream_step(self.handle, new_points, ids, dists, st,
                           KnnOpts(timing=int(timing), tau_mult=int(tau_mult),
                                   variant=VARIANTS[variant] if isinstance(variant, str) else int(variant)))
        if stats:
            return ids, dists, st.as_dict()
        return ids, dists

    def close(self):
        if self.handle:
            smiler_stream_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


class Index:
    """RAII-style owner of one smiler_index handle."""

    def __init__(self, series, sensor_offsets=None, window: int = 16, band: float = 8.0,
                 device: int = 0, stream=None, _handle: Optional[int] = None):
        self.dtype = _dtype_code(series)
        self.handle = _handle if _handle is not None else smiler_index_build(
            series, sensor_offsets, window, band, device, stream)

    @classmethod
    def shard(cls, slice_, slice_begin, n_global, t_begin, t_end, window, band, device=0, stream=None):
        h = smiler_index_build_shard(slice_, slice_begin, n_global, t_begin, t_end, window, band, device,
                                     stream)
        return cls(slice_, _handle=h)

    def knn(self, queries, lengths: Sequence[int], k: int, query_sensor=None, stats: bool = False,
            no_prune: bool = False, timing: bool = False, mq_chunk: int = 0, two_level: bool = False,
            lb_kind: int = 0, horizon: int = 0, shared_tau=None, tau_mult: int = 0, variant=0,
            tau_keep: int = 0, exact_postings: bool = False):
        """kNN of every item query (smiler_knn_ex).  shared_tau: optional device
        buffer (torch int64 tensor of n_mq * n_len entries, all ones = -1 at start)
        shared by the window-range shards of one search (NEXT-2)."""
        queries = _queries_for(self.dtype, queries, lengths)
        n_mq = queries.shape[0]
        ids = np.empty((n_mq, len(lengths), k), np.int64)
        dists = np.empty((n_mq, len(lengths), k), np.int32 if self.dtype == SMILER_I16 else np.float32)
        st = KnnStats() if stats else None
        op = KnnOpts(no_prune=int(no_prune), timing=int(timing), mq_chunk=mq_chunk, two_level=int(two_level),
                     lb_kind=int(lb_kind), horizon=int(horizon), tau_mult=int(tau_mult),
                     variant=VARIANTS[variant] if isinstance(variant, str) else int(variant),
                     tau_keep=int(tau_keep), exact_postings=int(exact_postings),
                     shared_tau=_ptr(shared_tau) if shared_tau is not None else None)
        smiler_knn(self.handle, queries, query_sensor, lengths, k, ids, dists, st, op)
        if stats:
            return ids, dists, st.as_dict()
        return ids, dists

    def predict(self, queries, lengths: Sequence[int], ids, ekv: Sequence[int], horizon: int, theta,
                query_sensor=None):
        """(ar_mean, ar_var, gp_mean, gp_var), each [n_mq, n_len, len(ekv)] float64."""
        queries = _queries_for(self.dtype, queries, lengths)
        shape = (queries.shape[0], len(lengths), len(ekv))
        outs = [np.empty(shape, np.float64) for _ in range(4)]
        smiler_predict(self.handle, queries, query_sensor, lengths,
                       np.ascontiguousarray(ids, dtype=np.int64), ekv, horizon,
                       np.ascontiguousarray(theta, dtype=np.float64), *outs)
        return tuple(outs)

    def knn_step(self, queries, lengths: Sequence[int], k: int, prev_ids, shift: int = 1, query_sensor=None,
                 stats: bool = False, timing: bool = False, tau_mult: int = 0):
        queries = _queries_for(self.dtype, queries, lengths)
        n_mq = queries.shape[0]
        ids = np.empty((n_mq, len(lengths), k), np.int64)
        dists = np.empty((n_mq, len(lengths), k), np.int32 if self.dtype == SMILER_I16 else np.float32)
        st = KnnStats() if stats else None
        op = KnnOpts(timing=int(timing), tau_mult=int(tau_mult))
        smiler_knn_step(self.handle, queries, query_sensor, lengths, k,
                        np.ascontiguousarray(prev_ids, dtype=np.int64), shift, ids, dists, st, op)
        if stats:
            return ids, dists, st.as_dict()
        return ids, dists

    def envelope(self, sensor: int, rho: int, n: int):
        dt = np.int16 if self.dtype == SMILER_I16 else np.float32
        U = np.empty(n, dt)
        L = np.empty(n, dt)
        smiler_index_envelope(self.handle, sensor, rho, U, L)
        return U, L

    def lower_bounds(self, queries, lengths, n: int, window: int, query_sensor=None, postings: bool = True):
        """postings=True: two-level path (posting lists materialised and returned);
        postings=False: the fused path (returns post=None)."""
        queries = _queries_for(self.dtype, queries, lengths)
        n_mq, D = queries.shape
        vt = np.int32 if self.dtype == SMILER_I16 else np.float32
        post = np.empty((n_mq, 2, D - window + 1, n // window), vt) if postings else None
        lbw = np.empty((n_mq, len(lengths), n), vt)
        smiler_lower_bounds(self.handle, queries, query_sensor, lengths, post, lbw)
        return post, lbw

    def lower_bounds_kind(self, queries, lengths, n: int, lb_kind: int, query_sensor=None):
        """The per-candidate bound smiler_knn_ex filters with under `lb_kind`:
        [n_mq][n_len][n] (entries with t > n - d_i unspecified)."""
        queries = _queries_for(self.dtype, queries, lengths)
        n_mq = queries.shape[0]
        vt = np.int32 if self.dtype == SMILER_I16 else np.float32
        lb = np.empty((n_mq, len(lengths), n), vt)
        smiler_lower_bounds_ex(self.handle, queries, query_sensor, lengths, lb_kind, lb)
        return lb

    def dtw(self, sensor: int, q, rho: int, ts):
        vt = np.int32 if self.dtype == SMILER_I16 else np.float32
        out = np.empty(len(ts), vt)
        q = _queries_for(self.dtype, np.asarray(q).reshape(1, -1), [len(q)])[0]
        smiler_dtw(self.handle, sensor, np.ascontiguousarray(q), rho, ts, out)
        return out

    def close(self):
        if self.handle:
            smiler_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
