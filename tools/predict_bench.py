"""Throughput of smiler_predict on one C5 tick.

    python tools/predict_bench.py [--sensors 1024] [--ekv 32,64,128] [--h 1] [--reps 5]

C5 shape (10 streams per sensor, ELV {16,32,64,128}, band 20%, k = 128): one
horizon-aware kNN (smiler_knn_opts.horizon = h), then every predictor f_{i,j}
(AR + GP, Eq. 12-18) of every stream, all buffers device-resident, timed with
CUDA events on the library stream.  Algorithmic fp64 flops per predictor:
Gram 3 d per pair over the (k_j + 1) k_j / 2 pairs (x0 included), Cholesky
k_j^3 / 3, two forward solves 2 k_j^2; reported against the measured DFMA peak
(profiles/alu_peaks.json "dfma", 2 flops each) when present.
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sensors", type=int, default=1024)
    ap.add_argument("--ekv", default="32,64,128")
    ap.add_argument("--h", type=int, default=1)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--dtype", default="f32")
    args = ap.parse_args()
    import torch

    import bench
    import paper_conf_sigmod_zhout15_b200 as pkg
    ekv = [int(x) for x in args.ekv.split(",")]
    dev = torch.device("cuda", 0)
    st = torch.cuda.Stream(device=dev)
    wl = bench.rank_workload("C5", args.dtype, 0, 1, 16)
    if args.sensors < 1024:
        keep = np.asarray(wl.query_sensor) < args.sensors
        wl.queries, wl.query_sensor = wl.queries[keep], np.asarray(wl.query_sensor)[keep]
    idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band, stream=st)
    nl, nk, k = len(wl.lengths), len(ekv), wl.k
    qd = torch.from_numpy(np.ascontiguousarray(wl.queries)).to(dev)
    qs = np.ascontiguousarray(wl.query_sensor, np.int32)
    ids = torch.empty((wl.n_mq, nl, k), dtype=torch.int64, device=dev)
    dd = torch.empty((wl.n_mq, nl, k), dtype=torch.float32 if args.dtype == "f32" else torch.int32, device=dev)
    op = pkg.KnnOpts(horizon=args.h)
    pkg.smiler_knn(idx.handle, qd, qs, wl.lengths, k, ids, dd, None, op)
    rng = np.random.default_rng(0)
    theta = np.stack([rng.uniform(0.5, 1.5, (wl.n_mq, nl, nk)), rng.uniform(2.0, 8.0, (wl.n_mq, nl, nk)),
                      rng.uniform(0.1, 0.4, (wl.n_mq, nl, nk))], axis=-1)
    th = torch.from_numpy(theta).to(dev)
    outs = [torch.empty((wl.n_mq, nl, nk), dtype=torch.float64, device=dev) for _ in range(4)]
    qs_d = torch.from_numpy(qs).to(dev)
    run = lambda: pkg.smiler_predict(idx.handle, qd, qs_d, wl.lengths, ids, ekv, args.h, th, *outs)
    run()
    torch.cuda.synchronize(dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(args.reps):
        run()
    e1.record(st)
    torch.cuda.synchronize(dev)
    ms = e0.elapsed_time(e1) / args.reps
    n_pred = wl.n_mq * nl * nk
    flops = 0.0
    for d in wl.lengths:
        for kj in ekv:
            flops += 3.0 * d * (kj + 1) * kj / 2 + kj ** 3 / 3.0 + 2.0 * kj * kj
    flops *= wl.n_mq
    peak = None
    ap_ = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "alu_peaks.json")
    if os.path.exists(ap_):
        a = json.load(open(ap_))
        if "dfma_per_s" in a:
            peak = 2.0 * a["dfma_per_s"]
    nan = float(torch.isnan(outs[2]).float().mean().item())
    print(json.dumps({"tool": "predict_bench", "workload": "C5 tick: %d streams, ELV %s, k=%d, EKV %s, h=%d"
                      % (wl.n_mq, wl.lengths, k, ekv, args.h), "dtype": args.dtype, "predictors": n_pred,
                      "ms_per_tick": ms, "predictors_per_s": n_pred / (ms / 1e3),
                      "fp64_gflops": flops / (ms / 1e3) / 1e9,
                      "fp64_peak_gflops": peak / 1e9 if peak else None,
                      "frac": (flops / (ms / 1e3)) / peak if peak else None, "nan_frac": nan}))


if __name__ == "__main__":
    main()
