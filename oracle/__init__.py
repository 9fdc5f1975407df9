"""oracle -- TEST INFRASTRUCTURE ONLY.

ctypes wrapper around oracle/oracle.c, the plain brute-force CPU reference for
SMiLer's Search Step (Zhou & Tung, SIGMOD'15).  Only tests/,
__graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import this package.  It never imports paper_conf_sigmod_zhout15_b200 (the
product) and the product never imports it.

Every function cites the PAPER.md passage it follows in oracle.c.  Pins: all
functions are pinned by tests/test_oracle_pins.py (hand-worked DTW values,
warping-path enumeration, closed forms, the paper's Examples 4.1/4.2, the
SURVEY Appendix A golden example, and the LB <= DTW theorems).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import time
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp", "-shared", "-fPIC"]

_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c -> oracle/liboracle.so with gcc (no CUDA involved)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        P = ctypes.c_void_p
        i64, i32 = ctypes.c_int64, ctypes.c_int
        L.orc_envelope_i64.argtypes = [P, i64, i64, P, P]
        L.orc_envelope_f64.argtypes = [P, i64, i64, P, P]
        L.orc_dtw_i64.argtypes = [P, P, i32, i32]
        L.orc_dtw_i64.restype = i64
        L.orc_dtw_f64.argtypes = [P, P, i32, i32]
        L.orc_dtw_f64.restype = ctypes.c_double
        L.orc_dtw_f32.argtypes = [P, P, i32, i32]
        L.orc_dtw_f32.restype = ctypes.c_float
        L.orc_knn_i16.argtypes = [P, i64, P, i32, P, P, i32, i32, i64, i64, i32, P, P]
        L.orc_knn_i16.restype = i32
        L.orc_knn_f64.argtypes = [P, i64, P, i32, P, P, i32, i32, i64, i64, i32, P, P]
        L.orc_knn_f32.argtypes = [P, i64, P, i32, P, P, i32, i32, i64, i64, i32, P, P]
        L.orc_dtw_list_i16.argtypes = [P, P, i32, i32, P, i64, P]
        L.orc_dtw_list_f32.argtypes = [P, P, i32, i32, P, i64, P, P]
        L.orc_postings_i64.argtypes = [P, i64, P, P, P, P, P, i32, i32, P, P]
        L.orc_postings_f64.argtypes = [P, i64, P, P, P, P, P, i32, i32, P, P]
        L.orc_lb_i64.argtypes = [P, i64, P, P, P, P, P, i32, i32, i32, P, P, P, P, P, P, P, P, P]
        L.orc_lb_f64.argtypes = [P, i64, P, P, P, P, P, i32, i32, i32, P, P, P, P, P, P]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _is_int(x: np.ndarray) -> bool:
    return np.issubdtype(x.dtype, np.integer)


# --------------------------------------------------------------------------
# Envelope, Eq. 25, clipped (R3)
# --------------------------------------------------------------------------
def envelope(x: np.ndarray, rho: int) -> Tuple[np.ndarray, np.ndarray]:
    n = len(x)
    if _is_int(x):
        xx = np.ascontiguousarray(x, dtype=np.int64)
        U = np.empty(n, np.int64)
        L = np.empty(n, np.int64)
        lib().orc_envelope_i64(_p(xx), n, rho, _p(U), _p(L))
    else:
        xx = np.ascontiguousarray(x, dtype=np.float64)
        U = np.empty(n, np.float64)
        L = np.empty(n, np.float64)
        lib().orc_envelope_f64(_p(xx), n, rho, _p(U), _p(L))
    return U, L


# --------------------------------------------------------------------------
# Banded DTW, Eq. 21-24
# --------------------------------------------------------------------------
def dtw(q, c, rho: int, mode: Optional[str] = None):
    """mode: 'i64' (exact integer), 'f64', or 'f32' (R16 pinned fma)."""
    q = np.asarray(q)
    c = np.asarray(c)
    d = len(q)
    assert len(c) == d
    if mode is None:
        mode = "i64" if (_is_int(q) and _is_int(c)) else "f64"
    if mode == "i64":
        qq = np.ascontiguousarray(q, np.int64)
        cc = np.ascontiguousarray(c, np.int64)
        return int(lib().orc_dtw_i64(_p(qq), _p(cc), d, rho))
    if mode == "f64":
        qq = np.ascontiguousarray(q, np.float64)
        cc = np.ascontiguousarray(c, np.float64)
        return float(lib().orc_dtw_f64(_p(qq), _p(cc), d, rho))
    if mode == "f32":
        qq = np.ascontiguousarray(q, np.float32)
        cc = np.ascontiguousarray(c, np.float32)
        return float(np.float32(lib().orc_dtw_f32(_p(qq), _p(cc), d, rho)))
    raise ValueError(mode)


def dtw_list(series: np.ndarray, q: np.ndarray, rho: int, ts: np.ndarray):
    """DTW of IQ q against C_{t,d} for each t in ts.  i16 -> int64 array;
    f32 -> (float32 pinned, float64) arrays."""
    ts = np.ascontiguousarray(ts, np.int64)
    d = len(q)
    if series.dtype == np.int16:
        out = np.empty(len(ts), np.int64)
        lib().orc_dtw_list_i16(_p(np.ascontiguousarray(series)), _p(np.ascontiguousarray(q, np.int16)),
                               d, rho, _p(ts), len(ts), _p(out))
        return out
    o32 = np.empty(len(ts), np.float32)
    o64 = np.empty(len(ts), np.float64)
    lib().orc_dtw_list_f32(_p(np.ascontiguousarray(series, np.float32)),
                           _p(np.ascontiguousarray(q, np.float32)), d, rho, _p(ts), len(ts),
                           _p(o32), _p(o64))
    return o32, o64


# --------------------------------------------------------------------------
# Suffix kNN Search, Def. 4.1, brute force
# --------------------------------------------------------------------------
def knn_one(series: np.ndarray, mq: np.ndarray, lengths: Sequence[int], rhos: Sequence[int],
            k: int, mode: Optional[str] = None, t_lo: int = 0, t_hi: Optional[int] = None,
            threads: int = 0):
    """kNN of every item query of one master query over one sensor series.
    Returns (ids [n_len, k] int64, dists [n_len, k]).  mode for f32 series:
    'f64' (the definition in double) or 'f32' (R16 pinned)."""
    n = len(series)
    D = len(mq)
    nl = len(lengths)
    t_hi = n if t_hi is None else t_hi
    lens = np.ascontiguousarray(lengths, np.int32)
    rr = np.ascontiguousarray(list(rhos), np.int32)
    ids = np.empty((nl, k), np.int64)
    if series.dtype == np.int16:
        dists = np.empty((nl, k), np.int64)
        over = lib().orc_knn_i16(_p(np.ascontiguousarray(series)), n, _p(np.ascontiguousarray(mq, np.int16)),
                                 D, _p(lens), _p(rr), nl, k, t_lo, t_hi, threads, _p(ids), _p(dists))
        if over:
            raise OverflowError("a DTW distance reached 2^31: int32 certificate (R17) fails")
        return ids, dists
    s = np.ascontiguousarray(series, np.float32)
    q = np.ascontiguousarray(mq, np.float32)
    mode = mode or "f64"
    if mode == "f64":
        dists = np.empty((nl, k), np.float64)
        lib().orc_knn_f64(_p(s), n, _p(q), D, _p(lens), _p(rr), nl, k, t_lo, t_hi, threads, _p(ids), _p(dists))
    else:
        dists = np.empty((nl, k), np.float32)
        lib().orc_knn_f32(_p(s), n, _p(q), D, _p(lens), _p(rr), nl, k, t_lo, t_hi, threads, _p(ids), _p(dists))
    return ids, dists


def knn(wl, mode: Optional[str] = None, mq_subset: Optional[Sequence[int]] = None,
        threads: int = 0):
    """Oracle kNN for a synth.Workload.  Returns ids [n_mq, n_len, k], dists."""
    sel = list(range(wl.n_mq)) if mq_subset is None else list(mq_subset)
    rhos = wl.rhos()
    I, Dd = [], []
    for j in sel:
        s = int(wl.query_sensor[j])
        ids, d = knn_one(wl.sensor_slice(s), wl.queries[j], wl.lengths, rhos, wl.k, mode=mode,
                         threads=threads)
        I.append(ids)
        Dd.append(d)
    return np.stack(I), np.stack(Dd)


# --------------------------------------------------------------------------
# Lower bounds: window-level postings and per-candidate LB_EQ,
# LB_EC, LB_en (Thm 4.1), LB_w (Thm 4.3 / Eq. 5)
# --------------------------------------------------------------------------
def postings(c: np.ndarray, UC, LC, mq, UQ, LQ, w: int):
    n = len(c)
    D = len(mq)
    n_sw, n_dw = D - w + 1, n // w
    if _is_int(c):
        cv = lambda a: np.ascontiguousarray(a, np.int64)
        PE = np.empty((n_sw, n_dw), np.int64)
        PC = np.empty((n_sw, n_dw), np.int64)
        fn = lib().orc_postings_i64
    else:
        cv = lambda a: np.ascontiguousarray(a, np.float64)
        PE = np.empty((n_sw, n_dw), np.float64)
        PC = np.empty((n_sw, n_dw), np.float64)
        fn = lib().orc_postings_f64
    args = [cv(c), cv(UC), cv(LC), cv(mq), cv(UQ), cv(LQ)]
    fn(_p(args[0]), n, _p(args[1]), _p(args[2]), _p(args[3]), _p(args[4]), _p(args[5]), D, w,
       _p(PE), _p(PC))
    return PE, PC


def lower_bounds(c: np.ndarray, UC, LC, mq, UQ, LQ, d: int, w: int) -> Dict[str, np.ndarray]:
    n = len(c)
    D = len(mq)
    nt = max(n - d + 1, 0)
    if _is_int(c):
        cv = lambda a: np.ascontiguousarray(a, np.int64)
        out = {k: np.empty(nt, np.int64) for k in ("eq", "ec", "en", "w", "b", "r", "m", "weq", "wec")}
        args = [cv(c), cv(UC), cv(LC), cv(mq), cv(UQ), cv(LQ)]
        lib().orc_lb_i64(_p(args[0]), n, _p(args[1]), _p(args[2]), _p(args[3]), _p(args[4]),
                         _p(args[5]), D, d, w, _p(out["eq"]), _p(out["ec"]), _p(out["en"]),
                         _p(out["w"]), _p(out["b"]), _p(out["r"]), _p(out["m"]), _p(out["weq"]), _p(out["wec"]))
        return out
    cv = lambda a: np.ascontiguousarray(a, np.float64)
    out = {k: np.empty(nt, np.float64) for k in ("eq", "ec", "en", "w", "weq", "wec")}
    args = [cv(c), cv(UC), cv(LC), cv(mq), cv(UQ), cv(LQ)]
    lib().orc_lb_f64(_p(args[0]), n, _p(args[1]), _p(args[2]), _p(args[3]), _p(args[4]),
                     _p(args[5]), D, d, w, _p(out["eq"]), _p(out["ec"]), _p(out["en"]), _p(out["w"]),
                     _p(out["weq"]), _p(out["wec"]))
    return out


def mq_lower_bounds(series: np.ndarray, mq: np.ndarray, lengths, rhos, w: int):
    """All lower bounds of one MQ's item queries, with the envelopes of R4/R20
    (rho_env = max rho_i, clipped)."""
    rho_env = max(rhos)
    UC, LC = envelope(series, rho_env)
    UQ, LQ = envelope(mq, rho_env)
    res = []
    for d in lengths:
        res.append(lower_bounds(series, UC, LC, mq, UQ, LQ, d, w))
    return res, (UC, LC, UQ, LQ, rho_env)


def dtw_cells(d: int, rho: int) -> int:
    """Band cells of one d x d banded DTW (|i-j| <= rho)."""
    rho = min(rho, d - 1)
    return d * (2 * rho + 1) - rho * (rho + 1)


def time_knn(series, mq, lengths, rhos, k, t_hi, threads):
    """Wall time of the brute-force oracle over candidates t in [0, t_hi)."""
    t0 = time.perf_counter()
    knn_one(series, mq, lengths, rhos, k, t_hi=t_hi, threads=threads)
    return time.perf_counter() - t0
