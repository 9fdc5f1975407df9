"""Lower-bound ablations on B200: the synthetic re-run of
Table 3 (verification time and unfiltered candidates per query
per sensor under LB_EQ, LB_EC, LB_en) and Fig. 8 (P:1916-1919, P:2094-2102:
time to compute the lower bound through the index, "SMiLer-Idx", vs directly
per item query, "SMiLer-Dir").

    python tools/ablation.py [CONFIG ...] [--dtype f32] [--reps 5] [--out FILE]

For every config and lb_kind: one-shot smiler_knn_ex over the config's batch
(C3: one MQ per sensor, the paper's protocol; C5: one tick of its streams),
per-phase CUDA events; the kNN result is checked identical across kinds (all
bounds are valid, so filtering is exact).  One JSON line per (config, kind).
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

KINDS = [("index", 0), ("index_eq", 1), ("index_ec", 2), ("direct", 3), ("direct_shared", 4)]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="*", default=["C3", "C2", "C5"])
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    import torch

    import bench
    import paper_conf_sigmod_zhout15_b200 as pkg
    dev = torch.device("cuda", 0)
    stream = torch.cuda.Stream(device=dev)
    lines = []
    for cfg in args.configs:
        wl = bench.rank_workload(cfg, args.dtype, 0, 1, 256 if cfg == "C2" else 16)
        idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band, stream=stream)
        qd = torch.from_numpy(wl.queries).to(dev)
        qs = np.ascontiguousarray(wl.query_sensor)
        nl = len(wl.lengths)
        vt = torch.int32 if args.dtype == "i16" else torch.float32
        ids = torch.empty((wl.n_mq, nl, wl.k), dtype=torch.int64, device=dev)
        dd = torch.empty((wl.n_mq, nl, wl.k), dtype=vt, device=dev)
        ref = None
        for name, kind in KINDS:
            op = pkg.KnnOpts(timing=1, lb_kind=kind)
            st = pkg.KnnStats()
            pkg.smiler_knn(idx.handle, qd, qs, wl.lengths, wl.k, ids, dd, st, op)  # warm-up
            acc = {}
            for _ in range(args.reps):
                pkg.smiler_knn(idx.handle, qd, qs, wl.lengths, wl.k, ids, dd, st, op)
                for k_, v_ in st.as_dict().items():
                    acc[k_] = acc.get(k_, 0) + v_
            torch.cuda.synchronize(dev)
            res = (ids.cpu().numpy().copy(), dd.cpu().numpy().copy())
            if ref is None:
                ref = res
            same = bool((res[0] == ref[0]).all() and (res[1] == ref[1]).all())
            r = args.reps
            ms = {k_[3:]: acc[k_] / r / 1e6 for k_ in acc if k_.startswith("ns_")}
            per_q = acc["survivors"] / r / (wl.n_mq * nl)
            line = {"config": cfg, "dtype": args.dtype, "lb_kind": name, "n_mq": wl.n_mq,
                    "item_queries": wl.lengths, "k": wl.k, "window": wl.window, "band": wl.band,
                    "lb_ms": ms["window_lb"] + ms["group_scan"], "verify_ms": ms["verify"], "tau_ms": ms["tau"],
                    "total_ms": ms["total"], "unfiltered_per_item_query": per_q,
                    "survivor_frac": acc["survivors"] / max(1, acc["candidates"]),
                    "dtw_cells_per_mq": acc["dtw_cells"] / r / wl.n_mq, "mq_per_s": wl.n_mq / (ms["total"] / 1e3),
                    "result_equals_index": same, "phase_ms": ms}
            print(json.dumps(line), flush=True)
            lines.append(line)
        idx.close()
        del qd, ids, dd
        torch.cuda.empty_cache()
    if args.out:
        with open(args.out, "w") as f:
            for ln in lines:
                f.write(json.dumps(ln) + "\n")


if __name__ == "__main__":
    main()
