"""Parity of the CUDA path (through the C ABI) with the oracle (-m gpu).

i16: ids and dists bit-exact.  f32: ids and dists bit-exact against the oracle
run in the kernel's precision (R16 pinned fma; the kNN decision is taken in the
same precision on both sides), and dists within relative 1e-5 of the fp64
oracle (BASELINE.json north_star tolerance) with id sets equal up to ties
within that tolerance.
"""
import os

import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu

THREADS = os.cpu_count() or 8


@pytest.fixture(scope="module")
def pkg():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_zhout15_b200 import build
    build.build()
    import paper_conf_sigmod_zhout15_b200 as p
    return p


def gpu_knn(pkg, wl, **kw):
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        return idx.knn(wl.queries, wl.lengths, wl.k, wl.query_sensor, **kw)


def assert_f64_tolerance(ids, dists, oid, od):
    """dists within rel 1e-5 of fp64; ids equal except ties within that tolerance."""
    fin = np.isfinite(od)
    assert (np.isfinite(dists) == fin).all()
    assert np.allclose(dists[fin], od[fin], rtol=1e-5, atol=0)
    for row in np.ndindex(ids.shape[:-1]):
        a, b = ids[row], oid[row]
        if (a == b).all():
            continue
        # differing positions must be near-ties of the oracle distances
        for j in np.nonzero(a != b)[0]:
            dj = od[row][j]
            close = np.abs(od[row] - dj) <= 1e-5 * max(dj, 1e-30)
            assert close.sum() >= 2 or j == len(a) - 1, (row, j)


def check_workload(pkg, orc, wl, mq_subset=None, **kw):
    ids, dists = gpu_knn(pkg, wl, **kw)
    sel = list(range(wl.n_mq)) if mq_subset is None else list(mq_subset)
    if wl.dtype == "i16":
        oid, od = orc.knn(wl, mq_subset=sel, threads=THREADS)
        np.testing.assert_array_equal(ids[sel], oid)
        np.testing.assert_array_equal(dists[sel].astype(np.int64), od)
    else:
        oid32, od32 = orc.knn(wl, mode="f32", mq_subset=sel, threads=THREADS)
        np.testing.assert_array_equal(ids[sel], oid32)
        np.testing.assert_array_equal(dists[sel], od32)
        oid64, od64 = orc.knn(wl, mode="f64", mq_subset=sel, threads=THREADS)
        assert_f64_tolerance(ids[sel], dists[sel], oid64, od64)
    # rows sorted by (dist, t), no duplicate t
    for row in np.ndindex(ids.shape[:-1]):
        r = [(d, t) for d, t in zip(dists[row].tolist(), ids[row].tolist()) if t >= 0]
        assert r == sorted(r) and len({t for _, t in r}) == len(r)
    return ids, dists


# ---------------------------------------------------------------------------
# a1 envelope, a3 postings, a4 LB_w
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("dtype", ["i16", "f32"])
@pytest.mark.parametrize("rho", [0, 1, 4, 25])
def test_envelope_bit_exact(pkg, orc, dtype, rho):
    wl = synth.make_workload("C3", dtype, n=5003, n_sensors=3)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        for s in range(3):
            x = wl.sensor_slice(s)
            U, L = idx.envelope(s, rho, len(x))
            oU, oL = orc.envelope(x, rho)
            np.testing.assert_array_equal(U.astype(oU.dtype), oU)
            np.testing.assert_array_equal(L.astype(oL.dtype), oL)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
@pytest.mark.parametrize("cfg,n,lengths,window,band", [
    ("C2", 9001, [16, 32, 64, 128], 8, 0.1),
    ("C3", 7013, [32, 64, 96], 16, 8.0),
    ("C5", 4099, [16, 32, 64, 128], 8, 0.2),
    ("C1", 1000, [8, 24], 16, 3.0),          # d < 2w-1: candidates with no full DW (R6)
    ("C1", 777, [5, 13, 40], 5, 2.0),         # odd window, generic-w kernel
])
def test_postings_and_lbw(pkg, orc, dtype, cfg, n, lengths, window, band):
    wl = synth.make_workload(cfg, dtype, n=n, n_sensors=1, mq_per_sensor=3, lengths=lengths,
                             window=window, band=band)
    rhos = wl.rhos()
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        post, lbw = idx.lower_bounds(wl.queries, wl.lengths, n, window)
        _, lbw_fused = idx.lower_bounds(wl.queries, wl.lengths, n, window, postings=False)
    for j in range(wl.n_mq):
        res, (UC, LC, UQ, LQ, rho_env) = orc.mq_lower_bounds(wl.series, wl.queries[j], wl.lengths, rhos,
                                                             window)
        PE, PC = orc.postings(wl.series, UC, LC, wl.queries[j], UQ, LQ, window)
        for i, d in enumerate(wl.lengths):
            exp = res[i]["w"]
            for got in (lbw[j, i, :n - d + 1], lbw_fused[j, i, :n - d + 1]):
                if dtype == "i16":
                    np.testing.assert_array_equal(got.astype(np.int64), exp)
                else:
                    np.testing.assert_allclose(got, exp, rtol=2e-5, atol=1e-6)
        if dtype == "i16":
            np.testing.assert_array_equal(post[j, 0].astype(np.int64), PE)
            np.testing.assert_array_equal(post[j, 1].astype(np.int64), PC)
        else:
            np.testing.assert_allclose(post[j, 0], PE, rtol=2e-5, atol=1e-6)
            np.testing.assert_allclose(post[j, 1], PC, rtol=2e-5, atol=1e-6)


# ---------------------------------------------------------------------------
# a7 banded DTW
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("dtype", ["i16", "f32"])
@pytest.mark.parametrize("d,rho", [(1, 0), (2, 1), (7, 3), (16, 1), (32, 4), (33, 8), (64, 6), (96, 8),
                                   (128, 12), (128, 25), (100, 32), (20, 32), (300, 30), (1024, 5), (45, 2), (37, 7), (130, 16),
                                   # rho > 32: the anti-diagonal wavefront kernel (R23: any band)
                                   (70, 33), (200, 60), (256, 255), (640, 100), (1024, 400)])
def test_dtw_kernel(pkg, orc, dtype, d, rho):
    wl = synth.make_workload("C2", dtype, n=3000, mq_per_sensor=1, lengths=[max(d, 1)], window=1, band=1.0)
    rng = np.random.default_rng(d * 100 + rho)
    ts = rng.integers(0, 3000 - d + 1, size=203)   # several warps and a ragged tail
    q = wl.queries[0]
    with pkg.Index(wl.series, None, 1, 1.0) as idx:
        if dtype == "i16" and d > 256:   # R17: int32 exactness needs d <= 256
            with pytest.raises(pkg.SmilerError) as ei:
                idx.dtw(0, q, rho, ts)
            assert ei.value.code == -1
            return
        got = idx.dtw(0, q, rho, ts)
    r = min(rho, d - 1)
    if dtype == "i16":
        exp = orc.dtw_list(wl.series, q, r, ts)
        np.testing.assert_array_equal(got.astype(np.int64), exp)
    else:
        e32, e64 = orc.dtw_list(wl.series, q, r, ts)
        np.testing.assert_array_equal(got, e32)
        np.testing.assert_allclose(got, e64, rtol=1e-5, atol=0)


# ---------------------------------------------------------------------------
# end-to-end kNN, configs C1..C5 at oracle sizes
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_golden_appendix_a_gpu(pkg, orc, dtype):
    import json
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "appendix_a.json")))
    C = np.array(g["C"], np.int16)
    MQ = np.array([g["MQ"]], np.int16)
    if dtype == "f32":   # P13: dyadic scaling keeps every f32 op exact
        C = (C / 8.0).astype(np.float32)
        MQ = (MQ / 8.0).astype(np.float32)
    with pkg.Index(C, None, g["w"], float(g["rho"])) as idx:
        ids, dists = idx.knn(MQ, g["lengths"], g["k"])
        post, lbw = idx.lower_bounds(MQ, g["lengths"], len(C), g["w"])
    scale = 64.0 if dtype == "f32" else 1.0
    for li, iq in enumerate(g["IQ"]):
        assert ids[0, li].tolist() == iq["knn_ids"]
        assert (dists[0, li] * scale).tolist() == iq["knn_dists"]
        assert (lbw[0, li, :len(iq["t"])] * scale).tolist() == iq["LB_w"]
    assert (post[0, 0] * scale).tolist() == g["P_EQ"]
    assert (post[0, 1] * scale).tolist() == g["P_EC"]


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_c1_full(pkg, orc, dtype):
    wl = synth.make_workload("C1", dtype)
    check_workload(pkg, orc, wl)


@pytest.mark.parametrize("two_level", [False, True])
@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_c2_reduced(pkg, orc, dtype, two_level):
    wl = synth.make_workload("C2", dtype, n=20011, mq_per_sensor=4)
    check_workload(pkg, orc, wl, two_level=two_level)


@pytest.mark.parametrize("two_level", [False, True])
@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_c3_reduced(pkg, orc, dtype, two_level):
    wl = synth.make_workload("C3", dtype, n=15007, n_sensors=6)
    check_workload(pkg, orc, wl, two_level=two_level)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_c4_reduced(pkg, orc, dtype):
    wl = synth.make_workload("C4", dtype, n=60013, mq_per_sensor=2)
    check_workload(pkg, orc, wl)


# a5 tau-set trim (tau_trim_kernel / tau_trim_big_kernel): any kept subset of
# verified candidates gives a valid tau, so the kNN must not change; keep = 1 x k
# is the tightest trim, variant 9 forces the radix-select path, -1 disables it
@pytest.mark.parametrize("variant,tau_keep", [(0, 1), (9, 1), (9, 3), (0, -1), (0, 64)])
@pytest.mark.parametrize("cfg,kw", [("C2", dict(n=20011, mq_per_sensor=4)),
                                    ("C4", dict(n=60013, mq_per_sensor=2))])
def test_tau_trim(pkg, orc, cfg, kw, variant, tau_keep):
    wl = synth.make_workload(cfg, "i16", **kw)
    ids, dists, st = gpu_knn(pkg, wl, stats=True, variant=variant, tau_keep=tau_keep)
    oid, od = orc.knn(wl, threads=THREADS)
    np.testing.assert_array_equal(ids, oid)
    np.testing.assert_array_equal(dists.astype(np.int64), od)


# tile lists longer than one chunk (> 8192 scan units per item query): the
# single bitonic trim (default), the two-stage chunked trim (variant 10) and the
# shared-memory radix trim (variant 9)
@pytest.mark.parametrize("variant,tau_keep", [(0, 0), (10, 1), (10, 4), (9, 2)])
def test_tau_trim_long_lists(pkg, orc, variant, tau_keep):
    wl = synth.make_workload("C2", "i16", n=2_200_003, mq_per_sensor=1, lengths=[16, 32])
    ids, dists = gpu_knn(pkg, wl, variant=variant, tau_keep=tau_keep)
    oid, od = orc.knn(wl, threads=THREADS)
    np.testing.assert_array_equal(ids, oid)
    np.testing.assert_array_equal(dists.astype(np.int64), od)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_c5_reduced(pkg, orc, dtype):
    wl = synth.make_workload("C5", dtype, n=12001, n_sensors=4, mq_per_sensor=2, consecutive=True)
    check_workload(pkg, orc, wl)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_pruned_equals_no_prune(pkg, dtype):
    wl = synth.make_workload("C5", dtype, n=30011, n_sensors=3, mq_per_sensor=3)
    a = gpu_knn(pkg, wl)
    b = gpu_knn(pkg, wl, no_prune=True)
    c = gpu_knn(pkg, wl, two_level=True)
    for x in (b, c):
        np.testing.assert_array_equal(a[0], x[0])
        np.testing.assert_array_equal(a[1], x[1])


# ---------------------------------------------------------------------------
# edge cases
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_edges_padding_and_small_series(pkg, orc, dtype):
    # fewer candidates than k (R12), D == N for the longest item query
    wl = synth.make_workload("C1", dtype, n=40, lengths=[8, 16, 40], k=30, window=4, band=3.0)
    ids, dists = check_workload(pkg, orc, wl)
    assert (ids[0, 2, 1:] == -1).all() and ids[0, 2, 0] == 0


@pytest.mark.parametrize("dtype", ["i16", "f32"])
@pytest.mark.parametrize("band", [0.0, 40.0, 0.5])
def test_edges_band_extremes(pkg, orc, dtype, band):
    wl = synth.make_workload("C1", dtype, n=900, lengths=[6, 16, 31], k=5, window=3, band=band)
    check_workload(pkg, orc, wl)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_edges_k1_single_length(pkg, orc, dtype):
    wl = synth.make_workload("C3", dtype, n=5000, n_sensors=2, lengths=[64], k=1, window=16)
    check_workload(pkg, orc, wl)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_edges_uneven_sensors(pkg, orc, dtype):
    parts = [synth.quantise(synth.sensor_series(9, s, n, 200, 144), dtype) for s, n in
             enumerate((3001, 517, 4099))]
    series = np.concatenate([p[:n] for p, n in zip(parts, (3001, 517, 4099))])
    offs = np.array([0, 3001, 3518, 7617], np.int64)
    qs = np.stack([parts[s][n + 3:n + 3 + 64] for s, n in ((0, 3001), (1, 517), (2, 4099), (1, 517))])
    wl = synth.Workload("uneven", dtype, series, offs, np.ascontiguousarray(qs),
                        np.array([0, 1, 2, 1], np.int32), [16, 40, 64], 9, 8, 5.0)
    check_workload(pkg, orc, wl)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_edges_constant_series_ties(pkg, dtype):
    """All distances tie: the lowest t wins (R11); also drives the >4096-finalist
    radix-select path of a8 in no-prune mode."""
    n = 9000
    series = np.full(n, 5, np.int16) if dtype == "i16" else np.full(n, 0.625, np.float32)
    q = np.full((1, 32), 3, np.int16) if dtype == "i16" else np.full((1, 32), 0.375, np.float32)
    for no_prune in (False, True):
        with pkg.Index(series, None, 8, 2.0) as idx:
            ids, dists = idx.knn(q, [16, 32], 7, no_prune=no_prune)
        for li, d in enumerate((16, 32)):
            assert ids[0, li].tolist() == list(range(7))
            exp = d * 4 if dtype == "i16" else d * 0.0625
            assert (dists[0, li] == exp).all()


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_shards_merge_equals_unsharded(pkg, orc, dtype):
    """C4's window-range sharding: G logical shards with halos,
    merged by smiler_merge_topk, equal the unsharded result and the oracle."""
    wl = synth.make_workload("C4", dtype, n=40009, mq_per_sensor=2)
    full_ids, full_d = check_workload(pkg, orc, wl)
    N, D, w = len(wl.series), wl.D, wl.window
    rho_env = max(wl.rhos())
    for G in (2, 3, 4, 8):
        bounds = [((N * g) // G) // w * w for g in range(G)] + [N]
        outs_i, outs_d = [], []
        for g in range(G):
            t0, t1 = bounds[g], bounds[g + 1]
            s0 = max(0, t0 - rho_env) // w * w
            s1 = min(N, t1 + D - 1 + rho_env)
            sl = np.ascontiguousarray(wl.series[s0:s1])
            with pkg.Index.shard(sl, s0, N, t0, t1, w, wl.band) as idx:
                i_, d_ = idx.knn(wl.queries, wl.lengths, wl.k)
            outs_i.append(i_)
            outs_d.append(d_)
        I = np.ascontiguousarray(np.stack(outs_i))
        Dd = np.ascontiguousarray(np.stack(outs_d))
        rows = wl.n_mq * len(wl.lengths)
        mi = np.empty((rows, wl.k), np.int64)
        md = np.empty((rows, wl.k), Dd.dtype)
        pkg.smiler_merge_topk(I, Dd, G, rows, wl.k, mi, md)
        np.testing.assert_array_equal(mi.reshape(full_ids.shape), full_ids)
        np.testing.assert_array_equal(md.reshape(full_d.shape), full_d)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
@pytest.mark.parametrize("tau_mult", [0, 1])
def test_shards_shared_running_tau(pkg, orc, dtype, tau_mult):
    """NEXT-2: shards of one search share a running threshold (atomicMin of
    global keys): the merged top-k is unchanged, later shards verify no more
    candidates than alone, and shards that hold none of the global top-k may
    return padded lists."""
    import torch
    wl = synth.make_workload("C4", dtype, n=40009, mq_per_sensor=2)
    full_ids, full_d = check_workload(pkg, orc, wl)
    N, D, w = len(wl.series), wl.D, wl.window
    rho_env = max(wl.rhos())
    rows = wl.n_mq * len(wl.lengths)
    for G in (2, 4, 8):
        bounds = [((N * g) // G) // w * w for g in range(G)] + [N]
        shared = torch.full((rows,), -1, dtype=torch.int64, device="cuda")
        outs_i, outs_d, surv_sh, surv_alone = [], [], 0, 0
        for g in range(G):
            t0, t1 = bounds[g], bounds[g + 1]
            s0 = max(0, t0 - rho_env) // w * w
            s1 = min(N, t1 + D - 1 + rho_env)
            sl = np.ascontiguousarray(wl.series[s0:s1])
            with pkg.Index.shard(sl, s0, N, t0, t1, w, wl.band) as idx:
                i_, d_, st = idx.knn(wl.queries, wl.lengths, wl.k, stats=True, shared_tau=shared,
                                     tau_mult=tau_mult)
                _, _, st0 = idx.knn(wl.queries, wl.lengths, wl.k, stats=True, tau_mult=tau_mult)
            surv_sh += st["survivors"]
            surv_alone += st0["survivors"]
            outs_i.append(i_)
            outs_d.append(d_)
        I = np.ascontiguousarray(np.stack(outs_i))
        Dd = np.ascontiguousarray(np.stack(outs_d))
        mi = np.empty((rows, wl.k), np.int64)
        md = np.empty((rows, wl.k), Dd.dtype)
        pkg.smiler_merge_topk(I, Dd, G, rows, wl.k, mi, md)
        np.testing.assert_array_equal(mi.reshape(full_ids.shape), full_ids)
        np.testing.assert_array_equal(md.reshape(full_d.shape), full_d)
        assert surv_sh <= surv_alone, (G, surv_sh, surv_alone)


def test_errors_on_gpu(pkg):
    x = np.zeros(100, np.int16)
    x[5] = 2000
    with pytest.raises(pkg.SmilerError) as ei:
        pkg.Index(x, None, 8, 2.0)
    assert ei.value.code == -2
    y = np.zeros(100, np.int16)
    with pkg.Index(y, None, 8, 2.0) as idx:
        with pytest.raises(pkg.SmilerError) as ei:
            idx.knn(np.zeros((1, 16), np.int16), [32, 16], 3)   # lengths not increasing
        assert ei.value.code == -1
        with pytest.raises(pkg.SmilerError):
            idx.knn(np.zeros((1, 200), np.int16), [200], 3)   # D > N
        ids, d = idx.knn(np.zeros((1, 32), np.int16), [16, 32], 3)   # handle still usable
        assert ids[0, 0].tolist() == [0, 1, 2]


def test_repeated_calls_deterministic(pkg):
    wl = synth.make_workload("C5", "f32", n=20000, n_sensors=2, mq_per_sensor=4)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        a = idx.knn(wl.queries, wl.lengths, wl.k, wl.query_sensor)
        b = idx.knn(wl.queries, wl.lengths, wl.k, wl.query_sensor, mq_chunk=3)
    np.testing.assert_array_equal(a[0], b[0])
    np.testing.assert_array_equal(a[1], b[1])


# ---------------------------------------------------------------------------
# full size (BASELINE configs[1], the bench workload), sampled against the oracle
# ---------------------------------------------------------------------------
@pytest.mark.slow
@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_c2_full_size_sampled(pkg, orc, dtype):
    wl = synth.make_workload("C2", dtype, mq_per_sensor=8)
    rhos = wl.rhos()
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        ids, dists, st = idx.knn(wl.queries, wl.lengths, wl.k, stats=True)
        bi, bd = idx.knn(wl.queries[:2], wl.lengths, wl.k, no_prune=True)
        np.testing.assert_array_equal(ids[:2], bi)     # pruning exact at full size
        np.testing.assert_array_equal(dists[:2], bd)
        rng = np.random.default_rng(5)
        for j in range(wl.n_mq):
            for i, d in enumerate(wl.lengths):
                q = wl.queries[j, wl.D - d:]
                # every returned distance is the oracle's DTW of that candidate
                ex = orc.dtw_list(wl.series, q, rhos[i], ids[j, i])
                if dtype == "f32":
                    ex = ex[0]
                np.testing.assert_array_equal(dists[j, i].astype(ex.dtype), ex)
                # random candidates: GPU DTW == oracle, and none beats the k-th result
                ts = rng.integers(0, len(wl.series) - d + 1, size=64)
                g = idx.dtw(0, q, rhos[i], ts)
                e2 = orc.dtw_list(wl.series, q, rhos[i], ts)
                if dtype == "f32":
                    e2 = e2[0]
                np.testing.assert_array_equal(g.astype(e2.dtype), e2)
                kth = (dists[j, i, -1], ids[j, i, -1])
                for t, v in zip(ts.tolist(), g.tolist()):
                    assert (v, t) >= kth or t in ids[j, i]
    assert st["survivors"] < st["candidates"]


# ---------------------------------------------------------------------------
# continuous steps (Def. 4.1; threshold method 2, P:1452-1458 / R9)
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("dtype", ["i16", "f32"])
@pytest.mark.parametrize("tau_mult", [0, -1, 2])
def test_continuous_steps(pkg, orc, dtype, tau_mult):
    """tau_mult -1: thresholds from the previous neighbours only, so the LB
    kernel filters as it scans (a4+a6 fused); 2: plus a tile tau set."""
    kw = dict(n=12001, n_sensors=3, mq_per_sensor=2)
    wl = synth.make_workload("C5", dtype, step=0, **kw)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        ids, dists = idx.knn(wl.queries, wl.lengths, wl.k, wl.query_sensor)
        for s in range(1, 4):
            ws = synth.make_workload("C5", dtype, step=s, **kw)
            assert (ws.series == wl.series).all()
            ids, dists, st = idx.knn_step(ws.queries, ws.lengths, ws.k, ids, 1, ws.query_sensor, stats=True,
                                          tau_mult=tau_mult)
            # the k previous neighbours are part of every item query's tau list
            assert st["tau_verified"] >= ws.n_mq * len(ws.lengths) * ws.k
            if dtype == "i16":
                oid, od = orc.knn(ws, threads=THREADS)
                np.testing.assert_array_equal(ids, oid)
                np.testing.assert_array_equal(dists.astype(np.int64), od)
            else:
                oid, od = orc.knn(ws, mode="f32", threads=THREADS)
                np.testing.assert_array_equal(ids, oid)
                np.testing.assert_array_equal(dists, od)
        # useless previous neighbours (all padding): tau = +inf, still exact
        bad = np.full_like(ids, -1)
        i2, d2 = idx.knn_step(ws.queries, ws.lengths, ws.k, bad, 1, ws.query_sensor, tau_mult=tau_mult)
        np.testing.assert_array_equal(i2, ids)
        np.testing.assert_array_equal(d2, dists)
        # stale neighbours from far away still give a valid (loose) threshold
        i3, d3 = idx.knn_step(ws.queries, ws.lengths, ws.k, ids, 50, ws.query_sensor, tau_mult=tau_mult)
        np.testing.assert_array_equal(i3, ids)
        np.testing.assert_array_equal(d3, dists)


# ---------------------------------------------------------------------------
# more edges: chunking, limits, extreme values
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_forced_chunks_equal_single_chunk(pkg, dtype):
    wl = synth.make_workload("C5", dtype, n=9001, n_sensors=4, mq_per_sensor=3)
    a = gpu_knn(pkg, wl)
    for chunk in (1, 2, 5):
        b = gpu_knn(pkg, wl, mq_chunk=chunk)
        np.testing.assert_array_equal(a[0], b[0])
        np.testing.assert_array_equal(a[1], b[1])
        c = gpu_knn(pkg, wl, mq_chunk=chunk, two_level=True)
        np.testing.assert_array_equal(a[0], c[0])
        np.testing.assert_array_equal(a[1], c[1])


def test_limits_long_query_many_lengths_large_k(pkg, orc):
    """D = 1024 with 16 item queries, k = 1024 (every ABI limit at once, R23;
    F32: I16 stops at D = 256, R17), and the I16 limit D = 256 itself."""
    lens = [16 * (i + 1) for i in range(15)] + [1024]
    wl = synth.make_workload("C2", "f32", n=2500, mq_per_sensor=1, lengths=lens, k=1024, window=16, band=0.02)
    check_workload(pkg, orc, wl)
    lens = [16 * (i + 1) for i in range(15)] + [256]
    wl = synth.make_workload("C2", "i16", n=2500, mq_per_sensor=1, lengths=lens, k=1024, window=16, band=0.05)
    check_workload(pkg, orc, wl)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_extreme_values(pkg, orc, dtype):
    """Series and queries saturating the i16 range (|x| = 1023): int32 sums near
    their bound (R17); f32 with the same large values."""
    rng = np.random.default_rng(17)
    n, D = 3000, 128
    base = rng.choice([-1023, 1023], size=n + D).astype(np.int16)
    if dtype == "f32":
        base = base.astype(np.float32)
    wl = synth.Workload("extreme", dtype, np.ascontiguousarray(base[:n]), np.array([0, n], np.int64),
                        np.ascontiguousarray(base[n:][None, :]), np.array([0], np.int32), [32, 64, 128], 16, 8, 0.1)
    check_workload(pkg, orc, wl)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_shards_fractional_band(pkg, orc, dtype):
    """Window-range shards with a fractional band (rho_max from the longest IQ)."""
    wl = synth.make_workload("C5", dtype, n=20011, n_sensors=1, mq_per_sensor=2)
    full_ids, full_d = gpu_knn(pkg, wl)
    N, D, w = len(wl.series), wl.D, wl.window
    rho_env = max(wl.rhos())
    G = 3
    bounds = [((N * g) // G) // w * w for g in range(G)] + [N]
    outs_i, outs_d = [], []
    for g in range(G):
        t0, t1 = bounds[g], bounds[g + 1]
        s0 = max(0, t0 - rho_env) // w * w
        s1 = min(N, t1 + D - 1 + rho_env)
        with pkg.Index.shard(np.ascontiguousarray(wl.series[s0:s1]), s0, N, t0, t1, w, wl.band) as idx:
            i_, d_ = idx.knn(wl.queries, wl.lengths, wl.k)
        outs_i.append(i_)
        outs_d.append(d_)
    rows = wl.n_mq * len(wl.lengths)
    mi = np.empty((rows, wl.k), np.int64)
    md = np.empty((rows, wl.k), outs_d[0].dtype)
    pkg.smiler_merge_topk(np.ascontiguousarray(np.stack(outs_i)), np.ascontiguousarray(np.stack(outs_d)), G, rows,
                          wl.k, mi, md)
    np.testing.assert_array_equal(mi.reshape(full_ids.shape), full_ids)
    np.testing.assert_array_equal(md.reshape(full_d.shape), full_d)


def test_shard_halo_too_small_is_einval(pkg):
    wl = synth.make_workload("C4", "i16", n=5000, mq_per_sensor=1)
    with pkg.Index.shard(np.ascontiguousarray(wl.series[1024:3000]), 1024, 5000, 1024, 2000, 16, 8.0) as idx:
        with pytest.raises(pkg.SmilerError) as ei:
            idx.knn(wl.queries, wl.lengths, wl.k)   # needs [1016, 2103): slice starts too late
        assert ei.value.code == -1


def test_device_buffers_and_streams(pkg):
    """Device-resident inputs/outputs on a user stream give the host-path result."""
    import torch
    wl = synth.make_workload("C2", "f32", n=30000, mq_per_sensor=8)
    st = torch.cuda.Stream()
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band, stream=st) as idx:
        hi, hd = idx.knn(wl.queries, wl.lengths, wl.k)
        qd = torch.from_numpy(wl.queries).cuda()
        ids = torch.empty(hi.shape, dtype=torch.int64, device="cuda")
        dd = torch.empty(hd.shape, dtype=torch.float32, device="cuda")
        pkg.smiler_knn(idx.handle, qd, None, wl.lengths, wl.k, ids, dd)
        st.synchronize()
        np.testing.assert_array_equal(ids.cpu().numpy(), hi)
        np.testing.assert_array_equal(dd.cpu().numpy(), hd)


# ---------------------------------------------------------------------------
# continuous streams with the reused window-level index (Remark 1)
# ---------------------------------------------------------------------------
def _stream_case(pkg, orc, dtype, name, steps, exact_postings=False, tau_mult=0, variant=0, **kw):
    wl = synth.make_workload(name, dtype, step=0, **kw)
    D = wl.D
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        with pkg.Stream(idx, wl.queries, wl.lengths, wl.k, wl.query_sensor, exact_postings=exact_postings) as st:
            ids, dists = st.first
            for s in range(steps + 1):
                ws = wl if s == 0 else synth.make_workload(name, dtype, step=s, **kw)
                if s > 0:
                    newp = np.ascontiguousarray(ws.queries[:, D - 1])   # the point appended at step s
                    assert (ws.queries[:, :D - 1] == prev_q[:, 1:]).all()
                    ids, dists, stt = st.step(newp, stats=True, tau_mult=tau_mult, variant=variant)
                    assert stt["posting_bytes"] > 0
                prev_q = ws.queries
                if s % 3 and s != steps:
                    continue   # check every third step against the oracle (and the last)
                if dtype == "i16":
                    oid, od = orc.knn(ws, threads=THREADS)
                    np.testing.assert_array_equal(ids, oid)
                    np.testing.assert_array_equal(dists.astype(np.int64), od)
                else:
                    oid, od = orc.knn(ws, mode="f32", threads=THREADS)
                    np.testing.assert_array_equal(ids, oid)
                    np.testing.assert_array_equal(dists, od)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_stream_steps_without_lagged_tau_set(pkg, orc, dtype):
    """opts.variant 5: stream steps with the tile tau set taken after the scan
    (LB_w array + filter pass) -- the path the lagged tau set replaces."""
    _stream_case(pkg, orc, dtype, "C5", 7, variant=5, n=3001, n_sensors=2, mq_per_sensor=2)


# f32 streams store their postings as fp16 rounded toward zero unless
# exact_postings (a valid, slightly looser bound: the kNN must not change)
@pytest.mark.parametrize("tau_mult", [0, -1, 2])
@pytest.mark.parametrize("dtype,exact", [("i16", False), ("f32", False), ("f32", True)])
def test_stream_steps_c5_shape(pkg, orc, dtype, exact, tau_mult):
    _stream_case(pkg, orc, dtype, "C5", 6, exact_postings=exact, tau_mult=tau_mult, n=12001, n_sensors=3,
                 mq_per_sensor=2)


@pytest.mark.parametrize("tau_mult", [0, -1])
@pytest.mark.parametrize("dtype,exact", [("i16", False), ("f32", False), ("f32", True)])
def test_stream_ring_wraps(pkg, orc, dtype, exact, tau_mult):
    """D = 32, w = 8: 25 sliding windows, so 30 steps wrap the ring cursor."""
    _stream_case(pkg, orc, dtype, "C1", 30, exact_postings=exact, tau_mult=tau_mult, n=3000, lengths=[16, 32],
                 window=8, band=3.0, k=6, mq_per_sensor=3)


def test_stream_fp16_postings_saturate(pkg, orc):
    """Values whose posting sums exceed fp16's range (65504): rounding toward
    zero saturates, the bound stays valid, the kNN stays exact."""
    wl = synth.make_workload("C1", "f32", n=3000, lengths=[16, 32], window=8, band=3.0, k=6, mq_per_sensor=3)
    wl.series = (wl.series * 300.0).astype(np.float32)
    wl.queries = (wl.queries * 300.0).astype(np.float32)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        with pkg.Stream(idx, wl.queries, wl.lengths, wl.k, wl.query_sensor) as st:
            ids, dists = st.first
    oid, od = orc.knn(wl, mode="f32", threads=THREADS)
    np.testing.assert_array_equal(ids, oid)
    np.testing.assert_array_equal(dists, od)


# ---------------------------------------------------------------------------
# full size, in the launch configuration bench.py times (BASELINE configs[2..4])
# ---------------------------------------------------------------------------
@pytest.mark.slow
@pytest.mark.parametrize("cfg,dtype", [("C3", "i16"), ("C3", "f32"), ("C5", "f32")])
def test_streams_full_size_sampled(pkg, orc, cfg, dtype):
    """C3 / C5 at full size through the stream calls the bench times: every
    master query of every sensor in one batch, ticks through the reused ring;
    sampled streams equal the oracle's brute-force kNN bit for bit."""
    wl = synth.make_workload(cfg, dtype, step=0, consecutive=True)
    D = wl.D
    rng = np.random.default_rng(11)
    sample = np.sort(rng.choice(wl.n_mq, size=6, replace=False)).tolist()
    mode = None if dtype == "i16" else "f32"

    def check(ws, ids, dists):
        oid, od = orc.knn(ws, mode=mode, mq_subset=sample, threads=THREADS)
        np.testing.assert_array_equal(ids[sample], oid)
        if dtype == "i16":
            np.testing.assert_array_equal(dists[sample].astype(np.int64), od)
        else:
            np.testing.assert_array_equal(dists[sample], od)

    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        with pkg.Stream(idx, wl.queries, wl.lengths, wl.k, wl.query_sensor) as st:
            ids, dists = st.first
            check(wl, ids, dists)
            ws = wl
            for s in (1, 2):
                ws = synth.make_workload(cfg, dtype, step=s, consecutive=True)
                ids, dists, stt = st.step(np.ascontiguousarray(ws.queries[:, D - 1]), stats=True)
                assert stt["survivors"] < stt["candidates"]
            check(ws, ids, dists)


@pytest.mark.slow
@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_c4_full_size_sampled(pkg, orc, dtype):
    """C4 at full size (1e8 points, 16 master queries, one call as the bench
    times it): pruning equals the GPU's exhaustive search, every returned
    distance is the oracle's DTW of that segment, and no sampled candidate
    beats the k-th result."""
    wl = synth.make_workload("C4", dtype)
    rhos = wl.rhos()
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        ids, dists, st = idx.knn(wl.queries, wl.lengths, wl.k, stats=True)
        bi, bd = idx.knn(wl.queries[:2], wl.lengths, wl.k, no_prune=True)
        np.testing.assert_array_equal(ids[:2], bi)
        np.testing.assert_array_equal(dists[:2], bd)
        rng = np.random.default_rng(7)
        for j in range(0, wl.n_mq, 3):
            for i, d in enumerate(wl.lengths):
                q = wl.queries[j, wl.D - d:]
                ex = orc.dtw_list(wl.series, q, rhos[i], ids[j, i])
                if dtype == "f32":
                    ex = ex[0]
                np.testing.assert_array_equal(dists[j, i].astype(ex.dtype), ex)
                ts = rng.integers(0, len(wl.series) - d + 1, size=256)
                g = idx.dtw(0, q, rhos[i], ts)
                kth = (dists[j, i, -1], ids[j, i, -1])
                for t, v in zip(ts.tolist(), g.tolist()):
                    assert (v, t) >= kth or t in ids[j, i]
    assert st["survivors"] < st["candidates"]


# ---------------------------------------------------------------------------
# ABI hygiene and the storage precision of the bounds (R17, R26)
# ---------------------------------------------------------------------------
def test_opts_reserved_and_unknown_variant_are_einval(pkg):
    wl = synth.make_workload("C1", "i16", n=600)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        n_mq, nl = wl.n_mq, len(wl.lengths)
        ids = np.empty((n_mq, nl, wl.k), np.int64)
        dd = np.empty((n_mq, nl, wl.k), np.int32)
        for kw in (dict(reserved=1), dict(reserved=2), dict(variant=11), dict(variant=-1)):
            with pytest.raises(pkg.SmilerError) as ei:
                pkg.smiler_knn(idx.handle, wl.queries, None, wl.lengths, wl.k, ids, dd, None, pkg.KnnOpts(**kw))
            assert ei.value.code == -1, kw
        for v in (0, 1, 6, 9, 10):   # every accepted variant gives the brute-force result
            a = idx.knn(wl.queries, wl.lengths, wl.k, variant=v)
            np.testing.assert_array_equal(a[0], idx.knn(wl.queries, wl.lengths, wl.k)[0])


def test_i16_limits_d_and_query_range(pkg):
    """R17: I16 needs D <= 256 and |q| <= 1023; host queries are refused before
    any work, device queries are flagged by the query-prep kernel (ERANGE when
    the call synchronises) and the handle stays usable."""
    import torch
    wl = synth.make_workload("C2", "i16", n=3000, mq_per_sensor=2)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        with pytest.raises(pkg.SmilerError) as ei:
            idx.knn(np.zeros((1, 300), np.int16), [16, 300], 4)
        assert ei.value.code == -1 and "R17" in str(ei.value)
        bad = wl.queries.copy()
        bad[1, 7] = 1024
        with pytest.raises(pkg.SmilerError) as ei:
            idx.knn(bad, wl.lengths, wl.k)
        assert ei.value.code == -2
        nl = len(wl.lengths)
        ids = np.empty((2, nl, wl.k), np.int64)
        dd = np.empty((2, nl, wl.k), np.int32)
        with pytest.raises(pkg.SmilerError) as ei:
            pkg.smiler_knn(idx.handle, torch.from_numpy(bad).cuda(), None, wl.lengths, wl.k, ids, dd)
        assert ei.value.code == -2
        good = idx.knn(wl.queries, wl.lengths, wl.k)           # flag cleared, handle usable
        pkg.smiler_knn(idx.handle, torch.from_numpy(wl.queries).cuda(), None, wl.lengths, wl.k, ids, dd)
        np.testing.assert_array_equal(ids, good[0])


def test_wrapper_rejects_mismatched_buffers(pkg):
    wl = synth.make_workload("C1", "f32", n=600)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        a = idx.knn(wl.queries.astype(np.float64), wl.lengths, wl.k)   # cast to the index dtype
        np.testing.assert_array_equal(a[0], idx.knn(wl.queries, wl.lengths, wl.k)[0])
        ids = np.empty((1, 1, wl.k), np.int64)
        dd = np.empty((1, 1, wl.k), np.float32)
        with pytest.raises(TypeError):   # float64 straight into the C ABI
            pkg.smiler_knn(idx.handle, wl.queries.astype(np.float64), None, wl.lengths, wl.k, ids, dd)
        with pytest.raises(ValueError):  # narrower than D
            pkg.smiler_knn(idx.handle, np.ascontiguousarray(wl.queries[:, 1:]), None, wl.lengths, wl.k, ids, dd)
        with pytest.raises(ValueError):  # wrong output shape
            pkg.smiler_knn(idx.handle, wl.queries, None, wl.lengths, wl.k + 1, ids, dd)


def test_i16_pruning_survives_tau_above_fp16_range(pkg, orc):
    """R26: the fp16 LB_w array is scaled per MQ by a power of two, so a tau far
    above 65504 (here i16 series of amplitude ~1000, D = 128) still prunes -- the
    unscaled array would round tau up to +inf and verify every candidate."""
    rng = np.random.default_rng(4242)
    n = 60000
    x = np.clip(np.cumsum(rng.integers(-60, 61, size=n + 200)), -1000, 1000)
    x = np.clip(x + rng.integers(-200, 201, size=x.size), -1023, 1023).astype(np.int16)
    series, tail = x[:n], x[n:]
    q = np.stack([tail[0:128], tail[50:178]])
    with pkg.Index(series, None, 8, 0.1) as idx:
        ids, dists, st = idx.knn(q, [16, 32, 64, 128], 16, stats=True)
        # the same search with the LB_w array in int32 (exact_postings: no fp16 storage)
        ids_x, dists_x, st_x = idx.knn(q, [16, 32, 64, 128], 16, stats=True, exact_postings=True)
    assert int(dists[:, -1, -1].min()) > 65504 * 2          # tau well above the fp16 range
    np.testing.assert_array_equal(ids, ids_x)
    # the fp16 array prunes (almost) as well as the exact one: the unscaled array
    # saturated and kept every candidate once tau passed 65504
    assert st["survivors"] <= st_x["survivors"] * 1.02 + 64, (st, st_x)
    assert st_x["survivors"] < 0.9 * st_x["candidates"], st_x
    for j in range(2):
        oid, od = orc.knn_one(series, q[j], [16, 32, 64, 128], [1, 3, 6, 12], 16, threads=THREADS)
        np.testing.assert_array_equal(ids[j], oid)
        np.testing.assert_array_equal(dists[j].astype(np.int64), od)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_tight_lb_equals_tau_fp16_inexact(pkg, orc, dtype):
    """P12 at a bound fp16 cannot represent: constant series a, constant query
    b, k = 1.  Every candidate has DTW = d (a - b)^2 (a tie), the aligned ones
    have LB_w = DTW = tau exactly, so t = 0 (aligned, lowest t) is the answer
    only if the filter keeps a bound equal to tau after the fp16 round-down of
    the stored bound and the round-up of the threshold."""
    a, b = (37, -52) if dtype == "i16" else (0.1, -0.73)
    n, w = 4096, 8
    vt = np.int16 if dtype == "i16" else np.float32
    series = np.full(n, a, vt)
    for d in (16, 48, 128):
        q = np.full((1, d), b, vt)
        tau = d * (float(np.float32(a)) - float(np.float32(b))) ** 2
        with pkg.Index(series, None, w, 3.0) as idx:
            ids, dists = idx.knn(q, [d], 1)
        assert ids[0, 0, 0] == 0, (d, ids[0, 0], dists[0, 0])
        oid, od = orc.knn_one(series, q[0], [d], [3], 1, mode=None if dtype == "i16" else "f32")
        assert oid[0, 0] == 0 and np.float64(dists[0, 0, 0]) == np.float64(od[0, 0])
        m_, _ = np.frexp(tau)
        assert m_ * 2.0 ** 11 != np.floor(m_ * 2.0 ** 11)   # needs > 11 significant bits: fp16-inexact at any scale


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_wide_band_knn(pkg, orc, dtype):
    """A 50% band (rho_i = floor(0.5 d_i) up to 128 > 32): the wavefront DTW path
    end to end, against the oracle."""
    wl = synth.make_workload("C2", dtype, n=2500, mq_per_sensor=2, lengths=[64, 256], k=8, window=16, band=0.5)
    assert max(wl.rhos()) == 128
    check_workload(pkg, orc, wl)


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_wavefront_variant_equals_register_band(pkg, orc, dtype):
    """opts.variant 3 runs the wavefront DTW kernel for every rho (A/B): C5-shaped
    bands {3, 6, 12, 25}, bit-exact with the oracle (the same cells, R16)."""
    wl = synth.make_workload("C5", dtype, n=6007, n_sensors=2, mq_per_sensor=2)
    check_workload(pkg, orc, wl, variant=3)


@pytest.mark.parametrize("cfg", ["C2", "C5"])
def test_packed_dtw_variant(pkg, orc, cfg):
    """opts.variant 6 runs the f32 register band with rows in pairs and fp32x2-packed
    cells (the A/B of the default scalar cells): bit-exact with the oracle."""
    wl = synth.make_workload(cfg, "f32", n=6007, n_sensors=2, mq_per_sensor=2)
    check_workload(pkg, orc, wl, variant=6)


@pytest.mark.parametrize("variant", [0, 4])
def test_phase_timing_includes_the_cascade(pkg, orc, variant):
    """opts.timing: the per-phase times add up to ns_total, and the LB_Keogh
    cascade has its own phase (ns_cascade, ABI 4): non-zero in a continuous step
    where it runs and drops survivors, next to nothing with opts.variant 4 (no
    cascade) and in one-shot searches (which skip it); results unchanged."""
    wl = synth.make_workload("C5", "f32", n=6007, n_sensors=2, mq_per_sensor=2)
    phases = ("ns_prep", "ns_window_lb", "ns_group_scan", "ns_tau", "ns_filter", "ns_cascade", "ns_verify",
              "ns_select")

    def check_phases(st, ran):
        assert all(st[p] >= 0 for p in phases)
        assert abs(sum(st[p] for p in phases) - st["ns_total"]) <= 1e-6 * st["ns_total"] + 1.0
        if ran:
            assert st["cascade_pruned"] >= 0 and st["ns_cascade"] > 0
        else:  # two back-to-back events: only their own resolution
            assert st["cascade_pruned"] == 0 and st["ns_cascade"] < 0.05 * st["ns_total"]

    ids, dists, st = gpu_knn(pkg, wl, stats=True, timing=True, variant=variant)
    check_phases(st, False)  # one-shot: no cascade
    check_workload(pkg, orc, wl, variant=variant)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        stream = pkg.Stream(idx, wl.queries, wl.lengths, wl.k, wl.query_sensor)
        for s in range(1, 3):
            ids, dists, st = stream.step(wl.new_points(s), stats=True, timing=True, variant=variant)
        check_phases(st, variant == 0)
        stream.close()
