"""Small runs of every kernel path through the C ABI, for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck):

    compute-sanitizer --tool racecheck python tools/sanitize_run.py

Reduced C1-C5 shapes: the fused packed-f32 and scalar-int LB kernels, the
two-level path, the TMA ring scan with the stream ring wrapping around, the
register-band (scalar and fp32x2-packed) and the wavefront DTW, every tau-trim path, window-range shards
with the shared running threshold, the direct lower bounds and the predictors.
Each result is checked against the oracle so a silent corruption also fails.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import oracle
import synth
import paper_conf_sigmod_zhout15_b200 as pkg


def check(wl, ids, dists, mode=None):
    oid, od = oracle.knn(wl, mode=mode or (None if wl.dtype == "i16" else "f32"))
    assert np.array_equal(ids, oid), wl.name
    assert np.array_equal(dists.astype(od.dtype), od), wl.name


def knn_cases():
    for dtype in ("i16", "f32"):
        wl = synth.make_workload("C1", dtype, n=1500)
        with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
            check(wl, *idx.knn(wl.queries, wl.lengths, wl.k))
        wl = synth.make_workload("C2", dtype, n=3001, mq_per_sensor=2)
        with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
            for kw in (dict(), dict(two_level=True), dict(variant=9, tau_keep=1), dict(variant=10, tau_keep=1),
                       dict(lb_kind=4), dict(variant=3), dict(variant=6)):
                check(wl, *idx.knn(wl.queries, wl.lengths, wl.k, **kw))
        wl = synth.make_workload("C2", dtype, n=1200, mq_per_sensor=1, lengths=[40, 128], k=4, window=16, band=0.5)
        with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:  # rho 64: the wavefront
            check(wl, *idx.knn(wl.queries, wl.lengths, wl.k))
        print("knn", dtype, "ok", flush=True)


def stream_cases():
    for dtype in ("i16", "f32"):
        wl = synth.make_workload("C5", dtype, n=2003, n_sensors=2, mq_per_sensor=2, consecutive=True)
        with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
            with pkg.Stream(idx, wl.queries, wl.lengths, wl.k, wl.query_sensor) as st:
                ids, dists = st.first
                check(wl, ids, dists)
                for s in range(1, wl.D - wl.window + 4):   # past one full turn of the ring
                    ids, dists = st.step(wl.new_points(s))
                ws = synth.Workload(wl.name, wl.dtype, wl.series, wl.offsets, wl.queries_at(s), wl.query_sensor,
                                    wl.lengths, wl.k, wl.window, wl.band, wl.tails, wl.qoff)
                check(ws, ids, dists)
        print("stream", dtype, "ok", flush=True)


def shard_cases():
    import torch
    wl = synth.make_workload("C4", "f32", n=4001, mq_per_sensor=2)
    N, rho = len(wl.series), max(wl.rhos())
    from paper_conf_sigmod_zhout15_b200 import dist as sdist
    shards = sdist.window_shards(N, wl.D, rho, wl.window, 3)
    shared = torch.full((wl.n_mq * len(wl.lengths),), -1, dtype=torch.int64, device="cuda")
    I, Dd = [], []
    for sh in shards:
        sl = np.ascontiguousarray(wl.series[sh.slice_begin:sh.slice_end])
        with pkg.Index.shard(sl, sh.slice_begin, N, sh.t_begin, sh.t_end, wl.window, wl.band) as idx:
            i_, d_ = idx.knn(wl.queries, wl.lengths, wl.k, shared_tau=shared)
        I.append(i_)
        Dd.append(d_)
    rows = wl.n_mq * len(wl.lengths)
    gi = np.ascontiguousarray(np.stack(I).reshape(3, rows, wl.k))
    gd = np.ascontiguousarray(np.stack(Dd).reshape(3, rows, wl.k))
    mi = np.empty((rows, wl.k), np.int64)
    md = np.empty((rows, wl.k), np.float32)
    pkg.smiler_merge_topk(gi, gd, 3, rows, wl.k, mi, md)
    check(wl, mi.reshape(wl.n_mq, len(wl.lengths), wl.k), md.reshape(wl.n_mq, len(wl.lengths), wl.k))
    print("shards ok", flush=True)


def predict_case():
    wl = synth.make_workload("C3", "f32", n=3000, n_sensors=1, mq_per_sensor=2)
    with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
        ids, _ = idx.knn(wl.queries, wl.lengths, wl.k, horizon=3)
        theta = np.tile(np.array([1.0, 2.0, 0.1]), (wl.n_mq, len(wl.lengths), 2, 1))
        out = idx.predict(wl.queries, wl.lengths, ids, [8, 32], 3, theta)
    assert all(np.isfinite(o).all() for o in out)
    print("predict ok", flush=True)


if __name__ == "__main__":
    knn_cases()
    stream_cases()
    shard_cases()
    predict_case()
    print("sanitize_run: all cases ok")
