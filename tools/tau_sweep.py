"""Sweep the tau-set size multiplier on one config.  Usage: python tools/tau_sweep.py C3|C5 [f32|i16]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import bench
import paper_conf_sigmod_zhout15_b200 as pkg

cfg = sys.argv[1]
dtype = sys.argv[2] if len(sys.argv) > 2 else "f32"
wl = bench.rank_workload(cfg, dtype, 0, 1, 256)
dev = torch.device("cuda", 0)
st = torch.cuda.Stream()
idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band, stream=st)
qd = torch.from_numpy(wl.queries).to(dev)
qs = np.ascontiguousarray(wl.query_sensor)
nl = len(wl.lengths)
ids = torch.empty((wl.n_mq, nl, wl.k), dtype=torch.int64, device=dev)
dd = torch.empty((wl.n_mq, nl, wl.k), dtype=torch.int32 if dtype == "i16" else torch.float32, device=dev)
ref = None
cont = len(sys.argv) > 3 and sys.argv[3] == "cont"
prev = None
for mult in ((-1, 2, 4, 8, 16) if cont else (8, 16, 32, 64, 128)):
    op = pkg.KnnOpts(no_prune=0, timing=1, mq_chunk=0, two_level=0)
    op.tau_mult = mult
    s = pkg.KnnStats()
    for it in range(2):
        if cont:
            if prev is None:
                prev = torch.empty_like(ids)
                pkg.smiler_knn(idx.handle, qd, qs, wl.lengths, wl.k, prev, dd)
            pkg.smiler_knn_step(idx.handle, qd, qs, wl.lengths, wl.k, prev, 0, ids, dd, s, op)
        else:
            pkg.smiler_knn(idx.handle, qd, qs, wl.lengths, wl.k, ids, dd, s, op)
    out = (ids.cpu().numpy().copy(), dd.cpu().numpy().copy())
    if ref is None:
        ref = out
    same = (ref[0] == out[0]).all() and (ref[1] == out[1]).all()
    print("mult %4d total %8.2f ms | lb %.2f tau %.2f filter %.2f verify %.2f select %.2f | surv %.4f tau_slots %d | same=%s"
          % (mult, s.ns_total / 1e6, s.ns_window_lb / 1e6, s.ns_tau / 1e6, s.ns_filter / 1e6, s.ns_verify / 1e6,
             s.ns_select / 1e6, s.survivors / s.candidates, s.tau_verified, same))
