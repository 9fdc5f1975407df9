"""Parity of the prediction consumers with the oracle (-m gpu).

* smiler_knn_opts.horizon = h keeps only segments whose h-step-ahead value
  exists (t + d - 1 + h < N): the result must equal the oracle's
  brute-force kNN over the series truncated to its first N - h points (the
  same candidate set by definition).
* smiler_predict: AR (Eq. 12-13) and GP (Eq. 16-18) mean and variance of every
  predictor f_{i,j} against oracle/predict.py (fp64 numpy, np.linalg.solve), on
  the same neighbour ids; fp64 on both sides, different operation order
  (Cholesky vs LAPACK LU): rtol 1e-8.
"""
import numpy as np
import pytest

import synth
from oracle import predict as OP

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pkg():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_zhout15_b200 import build
    build.build()
    import paper_conf_sigmod_zhout15_b200 as p
    return p


def oracle_knn_horizon(orc, wl, h, mode):
    rhos = wl.rhos()
    I, Dd = [], []
    for j in range(wl.n_mq):
        s = int(wl.query_sensor[j])
        c = wl.sensor_slice(s)
        ids, d = orc.knn_one(c[:len(c) - h], wl.queries[j], wl.lengths, rhos, wl.k, mode=mode)
        I.append(ids)
        Dd.append(d)
    return np.stack(I), np.stack(Dd)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
@pytest.mark.parametrize("h", [1, 37])
def test_knn_horizon_equals_truncated_series(pkg, orc, dtype, h):
    wl = synth.make_workload("C5", dtype, n=9001, n_sensors=2, mq_per_sensor=2)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        ids, dists = idx.knn(wl.queries, wl.lengths, wl.k, wl.query_sensor, horizon=h)
    oid, od = oracle_knn_horizon(orc, wl, h, None if dtype == "i16" else "f32")
    np.testing.assert_array_equal(ids, oid)
    np.testing.assert_array_equal(dists.astype(od.dtype), od)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
@pytest.mark.parametrize("cfg,ekv", [("C3", [8, 16, 32, 64]), ("C5", [16, 128])])
def test_predictors_match_oracle(pkg, orc, dtype, cfg, ekv):
    h = 6
    wl = synth.make_workload(cfg, dtype, n=12007, n_sensors=2, mq_per_sensor=2)
    rng = np.random.default_rng(7)
    nl, nk = len(wl.lengths), len(ekv)
    scale = 128.0 if dtype == "i16" else 1.0           # i16 stores round(128 z)
    theta = np.stack([rng.uniform(0.5, 1.5, (wl.n_mq, nl, nk)) * scale,
                      rng.uniform(2.0, 8.0, (wl.n_mq, nl, nk)) * scale,
                      rng.uniform(0.1, 0.4, (wl.n_mq, nl, nk)) * scale], axis=-1)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        ids, _ = idx.knn(wl.queries, wl.lengths, wl.k, wl.query_sensor, horizon=h)
        got = idx.predict(wl.queries, wl.lengths, ids, ekv, h, theta, wl.query_sensor)
    exp = OP.predict(wl.sensor_slice, wl.queries, wl.query_sensor, wl.lengths, ids, ekv, h, theta)
    for g, e, name in zip(got, exp, ("ar_mean", "ar_var", "gp_mean", "gp_var")):
        assert np.isfinite(e).all(), name
        np.testing.assert_allclose(g, e, rtol=1e-8, atol=1e-9 * scale * scale, err_msg=name)


def test_predictor_missing_neighbours_is_nan(pkg):
    wl = synth.make_workload("C1", "f32", n=4096)
    theta = np.tile(np.array([1.0, 4.0, 0.3]), (1, 1, 2, 1))
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        ids, _ = idx.knn(wl.queries, wl.lengths, wl.k, horizon=3)
        ids2 = ids.copy()
        ids2[0, 0, 5] = -1                                   # k_j = 8 predictor loses a neighbour
        am, av, gm, gv = idx.predict(wl.queries, wl.lengths, ids2, [4, 8], 3, theta)
    assert np.isfinite([am[0, 0, 0], gm[0, 0, 0], gv[0, 0, 0]]).all()
    assert np.isnan([am[0, 0, 1], av[0, 0, 1], gm[0, 0, 1], gv[0, 0, 1]]).all()


def test_predict_errors(pkg):
    wl = synth.make_workload("C1", "f32", n=4096)
    theta = np.ones((1, 1, 2, 3))
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        ids, _ = idx.knn(wl.queries, wl.lengths, wl.k)
        for ekv in ([8, 4], [0, 4], [4, 9]):                  # not increasing / < 1 / > k
            with pytest.raises(pkg.SmilerError):
                idx.predict(wl.queries, wl.lengths, ids, ekv, 0, theta)
        with pytest.raises(pkg.SmilerError):
            idx.predict(wl.queries, wl.lengths, ids, [2, 4], -1, theta)
