"""Pins of oracle/predict.py (the AR and GP predictors of Sec. 5.2) against
values fixed by the paper's formulas and by closed forms -- not by re-typing the
oracle's own code.  CPU only.

Pinned:
  * Eq. 12-13 on a hand example (mean 3, variance 3.5 with the 1/k of Eq. 13);
  * the h-step target y_{a,h} = c[t_a + d - 1 + h] on a ramp;
  * GP with one neighbour: u0 = c0 y / (theta0^2 + theta2^2), closed form;
  * GP with a huge length-scale (C -> theta0^2 11^T + theta2^2 I): the
    Sherman-Morrison closed form of Eq. 16-17;
  * GP with a vanishing length-scale (independent points): u0 = 0 and
    s0^2 = theta0^2 + theta2^2 (prior), or u0 = theta0^2 y_a / (theta0^2 +
    theta2^2) when x0 coincides with one neighbour;
  * the posterior variance lies in [theta2^2, theta0^2 + theta2^2] and never grows
    with more neighbours (conditioning on more data);
  * the multi-k ensemble uses prefixes of the sorted kNN.
"""
import math

import numpy as np
import pytest

from oracle import predict as P


def test_ar_hand_example():
    u, v = P.ar(np.array([1.0, 2.0, 3.0, 6.0]))
    assert u == 3.0
    assert v == pytest.approx((4 + 1 + 0 + 9) / 4)          # Eq. 13 divides by k


def test_knn_data_h_step_target():
    c = np.arange(100, dtype=np.float64) * 10.0               # c[x] = 10 x
    X, Y = P.knn_data(c, [5, 40], d=8, h=3)
    np.testing.assert_array_equal(X[0], 10.0 * np.arange(5, 13))
    np.testing.assert_array_equal(Y, [10.0 * (5 + 8 - 1 + 3), 10.0 * (40 + 8 - 1 + 3)])


def test_gp_single_neighbour_closed_form():
    rng = np.random.default_rng(1)
    x1, x0 = rng.normal(size=12), rng.normal(size=12)
    th = (1.3, 2.1, 0.4)
    r2 = float(np.sum((x1 - x0) ** 2))
    c0 = th[0] ** 2 * math.exp(-r2 / (2 * th[1] ** 2))
    s = th[0] ** 2 + th[2] ** 2
    u, v = P.gp(x1[None, :], np.array([2.5]), x0, th)
    assert u == pytest.approx(c0 * 2.5 / s, rel=1e-12)
    assert v == pytest.approx(s - c0 * c0 / s, rel=1e-12)


def test_gp_constant_kernel_sherman_morrison():
    rng = np.random.default_rng(2)
    k, d = 9, 16
    X, x0, Y = rng.normal(size=(k, d)), rng.normal(size=d), rng.normal(size=k)
    t0, t2 = 0.8, 0.3
    th = (t0, 1e9, t2)                                       # exp(-r2/(2 t1^2)) = 1
    a, b = t0 ** 2, t2 ** 2
    u_cf = a * Y.sum() / (b + k * a)                           # 1^T (b I + a 11^T)^-1 Y
    v_cf = a + b - k * a * a / (b + k * a)
    u, v = P.gp(X, Y, x0, th)
    assert u == pytest.approx(u_cf, rel=1e-9)
    assert v == pytest.approx(v_cf, rel=1e-9)


def test_gp_independent_points():
    rng = np.random.default_rng(3)
    X, Y = rng.normal(size=(5, 8)) * 10, rng.normal(size=5)
    th = (1.1, 1e-3, 0.5)
    u, v = P.gp(X, Y, rng.normal(size=8) * 10, th)
    assert abs(u) < 1e-12 and v == pytest.approx(1.1 ** 2 + 0.5 ** 2)
    u, v = P.gp(X, Y, X[2].copy(), th)                        # x0 equals neighbour 2
    assert u == pytest.approx(1.1 ** 2 * Y[2] / (1.1 ** 2 + 0.5 ** 2), rel=1e-12)


def test_gp_variance_bounds_and_monotone_in_k():
    rng = np.random.default_rng(4)
    X, Y, x0 = rng.normal(size=(32, 16)), rng.normal(size=32), rng.normal(size=16)
    th = (1.0, 3.0, 0.2)
    vs = [P.gp(X[:k], Y[:k], x0, th)[1] for k in (1, 2, 4, 8, 16, 32)]
    for v in vs:
        assert th[2] ** 2 - 1e-12 <= v <= th[0] ** 2 + th[2] ** 2 + 1e-12
    assert all(b <= a + 1e-12 for a, b in zip(vs, vs[1:]))


def test_predict_uses_prefixes_and_marks_missing():
    rng = np.random.default_rng(5)
    c = rng.normal(size=300)
    q = rng.normal(size=(1, 24))
    ids = np.array([[[10, 50, 90, 130, 170, 210], [7, 77, 150, -1, -1, -1]]], np.int64)
    th = np.tile(np.array([1.0, 4.0, 0.3]), (1, 2, 2, 1))
    ar_m, ar_v, gp_m, gp_v = P.predict(lambda s: c, q, [0], [16, 24], ids, [2, 6], 5, th)
    X, Y = P.knn_data(c, [10, 50], 16, 5)
    assert ar_m[0, 0, 0] == pytest.approx(Y.mean())
    assert gp_m[0, 0, 0] == pytest.approx(P.gp(X, Y, q[0, 8:], (1.0, 4.0, 0.3))[0])
    assert np.isnan(gp_m[0, 1, 1]) and not np.isnan(gp_m[0, 1, 0])   # only 3 valid neighbours
