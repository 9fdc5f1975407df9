"""oracle.predict -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Plain numpy fp64 reference of the two predictors that consume the Suffix kNN
result (Sec. 5.2), written in the paper's order
and notation.  Only tests/, __graft_entry__.smoke() and bench.py's CPU legs may
import it; it shares nothing with the CUDA path.

kNN data (Sec. 3.2; h-step target P:615-619):
    X_{k,d} = {C_{t_a,d} = c[t_a .. t_a+d)}  a = 1..k      (the k nearest segments)
    Y_h     = {y_{a,h} = c[t_a + d - 1 + h]}               (the value h steps after
                                                           each segment's last point)
AR predictor (Eq. 10-13):
    u~0 = sum_a y_{a,h} / k ,   s~0^2 = sum_a (y_{a,h} - u~0)^2 / k
GP predictor (Eq. 14-18; App. B.3 Eq. 27-31):
    c(x_a, x_b) = theta0^2 exp(-1/2 |x_a - x_b|^2 / theta1^2) + delta_ab theta2^2   (Eq. 18)
    C = [c(x_a, x_b)]_{a,b<=k},  c0 = [c(x_a, x0)]_a  (x0 != x_a: no delta term)
    u0 = c0^T C^{-1} Y_h                                                           (Eq. 16)
    s0^2 = c(x0, x0) - c0^T C^{-1} c0,  c(x0, x0) = theta0^2 + theta2^2           (Eq. 17)
    (reading P1 in DESIGN.md: the test input's own delta term is kept, i.e. the
    variance of a noisy observation y0, as in Eq. 27-31 where every y is noisy)
The multi-k ensemble (Eq. 2-3; multi-k by prefix): the
predictor f_{i,j} of item-query length d_i and k_j in EKV uses the first k_j
neighbours of IQ_i.  Hyperparameters Theta are inputs (their online training,
Eq. 19-20, is out of scope).
"""
from __future__ import annotations

from typing import Sequence

import numpy as np


def knn_data(series: np.ndarray, ts: Sequence[int], d: int, h: int):
    """(X [k, d], Y [k]) of the neighbours starting at ts."""
    c = np.asarray(series, np.float64)
    X = np.stack([c[t:t + d] for t in ts]) if len(ts) else np.zeros((0, d))
    Y = np.array([c[t + d - 1 + h] for t in ts], np.float64)
    return X, Y


def ar(Y: np.ndarray):
    """Eq. 12-13: pseudo-mean and pseudo-variance (divided by k)."""
    k = len(Y)
    u = float(np.sum(Y)) / k
    v = float(np.sum((Y - u) ** 2)) / k
    return u, v


def se_cov(xa: np.ndarray, xb: np.ndarray, theta) -> float:
    """Eq. 18 without the delta term: theta0^2 exp(-|xa-xb|^2 / (2 theta1^2))."""
    t0, t1, _ = theta
    r2 = float(np.sum((np.asarray(xa, np.float64) - np.asarray(xb, np.float64)) ** 2))
    return t0 * t0 * np.exp(-0.5 * r2 / (t1 * t1))


def gp(X: np.ndarray, Y: np.ndarray, x0: np.ndarray, theta):
    """Eq. 16-18: predictive mean and variance of y0 given (X, Y)."""
    t0, t1, t2 = theta
    k = len(Y)
    C = np.empty((k, k))
    for a in range(k):
        for b in range(k):
            C[a, b] = se_cov(X[a], X[b], theta) + (t2 * t2 if a == b else 0.0)
    c0 = np.array([se_cov(X[a], x0, theta) for a in range(k)])
    u0 = float(c0 @ np.linalg.solve(C, Y))
    s2 = t0 * t0 + t2 * t2 - float(c0 @ np.linalg.solve(C, c0))
    return u0, s2


def predict(series_of, queries, query_sensor, lengths, ids, ekv, h, theta):
    """Every predictor f_{i,j} of every master query.

    series_of(s) -> the sensor's series; queries [n_mq, D]; ids [n_mq, n_len, k]
    (the kNN, sorted, -1 padded); ekv ascending k_j <= k; theta [n_mq, n_len, n_k, 3].
    Returns ar_mean, ar_var, gp_mean, gp_var, each [n_mq, n_len, n_k] (NaN when a
    predictor lacks k_j valid neighbours with an h-step-ahead value)."""
    n_mq, D = queries.shape
    nl, nk = len(lengths), len(ekv)
    out = [np.full((n_mq, nl, nk), np.nan) for _ in range(4)]
    for m in range(n_mq):
        c = series_of(int(query_sensor[m]))
        for i, d in enumerate(lengths):
            x0 = np.asarray(queries[m][D - d:], np.float64)        # IQ_i
            for j, kj in enumerate(ekv):
                ts = [int(t) for t in ids[m, i, :kj]]
                if any(t < 0 or t + d - 1 + h >= len(c) for t in ts):
                    continue
                X, Y = knn_data(c, ts, d, h)
                out[0][m, i, j], out[1][m, i, j] = ar(Y)
                out[2][m, i, j], out[3][m, i, j] = gp(X, Y, x0, theta[m, i, j])
    return tuple(out)
