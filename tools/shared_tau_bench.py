"""NEXT-2 measurement on one GPU: C4 (1e8 points, 16 MQs) split into G window-range
shards (R24) searched one after another, each with or without the shared running
threshold (smiler_knn_opts.shared_tau).  Reports survivors, DTW cells and time per
shard, and checks the merged top-k of both runs are identical.

    python tools/shared_tau_bench.py [--G 8] [--n 100000000]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--G", type=int, default=8)
    ap.add_argument("--n", type=int, default=100_000_000)
    ap.add_argument("--dtype", default="f32")
    args = ap.parse_args()
    import torch

    import synth
    import paper_conf_sigmod_zhout15_b200 as pkg
    from paper_conf_sigmod_zhout15_b200 import dist as sdist
    wl = synth.make_workload("C4", args.dtype, n=args.n, mq_per_sensor=16)
    N, D, w, G = len(wl.series), wl.D, wl.window, args.G
    nl, k = len(wl.lengths), wl.k
    rows = wl.n_mq * nl
    dev = torch.device("cuda", 0)
    qd = torch.from_numpy(wl.queries).to(dev)
    vt = torch.float32 if args.dtype == "f32" else torch.int32
    res = {}
    for mode in ("alone", "shared"):
        shared = torch.full((rows,), -1, dtype=torch.int64, device=dev) if mode == "shared" else None
        ids = torch.empty((G, wl.n_mq, nl, k), dtype=torch.int64, device=dev)
        dd = torch.empty((G, wl.n_mq, nl, k), dtype=vt, device=dev)
        per = []
        for sh in sdist.window_shards(N, D, max(wl.rhos()), w, G):
            sl = np.ascontiguousarray(wl.series[sh.slice_begin:sh.slice_end])
            idx = pkg.Index.shard(sl, sh.slice_begin, N, sh.t_begin, sh.t_end, w, wl.band)
            st = pkg.KnnStats()
            op = pkg.KnnOpts(timing=1, shared_tau=shared.data_ptr() if shared is not None else None)
            pkg.smiler_knn(idx.handle, qd, None, wl.lengths, k, ids[sh.rank], dd[sh.rank], st, op)
            d = st.as_dict()
            per.append({"shard": sh.rank, "survivors": d["survivors"], "dtw_cells": d["dtw_cells"],
                        "ms_tau_verify": (d["ns_tau"] + d["ns_verify"]) / 1e6, "ms_total": d["ns_total"] / 1e6})
            idx.close()
        oi = torch.empty((rows, k), dtype=torch.int64, device=dev)
        od = torch.empty((rows, k), dtype=vt, device=dev)
        pkg.smiler_merge_topk(ids.view(G, rows, k), dd.view(G, rows, k), G, rows, k, oi, od)
        torch.cuda.synchronize(dev)
        res[mode] = (per, oi.cpu().numpy(), od.cpu().numpy())
    same = bool((res["alone"][1] == res["shared"][1]).all() and (res["alone"][2] == res["shared"][2]).all())
    out = {"tool": "shared_tau_bench", "workload": "C4: %d points, 16 MQs, ELV %s, k=%d, %d logical shards on one GPU"
           % (N, wl.lengths, k, G), "merged_identical": same}
    for mode in ("alone", "shared"):
        per = res[mode][0]
        out[mode] = {"survivors": sum(p["survivors"] for p in per), "dtw_cells": sum(p["dtw_cells"] for p in per),
                     "ms_tau_verify": sum(p["ms_tau_verify"] for p in per),
                     "ms_total": sum(p["ms_total"] for p in per),
                     "survivors_per_shard": [p["survivors"] for p in per]}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
