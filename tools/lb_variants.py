"""Time the LB variants (diag fused / row fused / two-level) on C2 for one dtype.
Prints per-phase ms per 256-MQ step.  Usage: python tools/lb_variants.py [f32|i16] [mq]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_sigmod_zhout15_b200 as pkg

dtype = sys.argv[1] if len(sys.argv) > 1 else "f32"
nmq = int(sys.argv[2]) if len(sys.argv) > 2 else 256
cfg = os.environ.get("CFG", "C2")
if cfg == "C2":
    wl = synth.make_workload("C2", dtype, mq_per_sensor=nmq)
else:
    import bench
    wl = bench.rank_workload(cfg, dtype, 0, 1, nmq)
dev = torch.device("cuda", 0)
st = torch.cuda.Stream()
idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band, stream=st)
qd = torch.from_numpy(wl.queries).to(dev)
qs = np.ascontiguousarray(wl.query_sensor)
nl = len(wl.lengths)
ids = torch.empty((wl.n_mq, nl, wl.k), dtype=torch.int64, device=dev)
dd = torch.empty((wl.n_mq, nl, wl.k), dtype=torch.int32 if dtype == "i16" else torch.float32, device=dev)
ref = None
variants = [("diag", 0, 0, 0), ("diag_mainonly", 0, 0, 2), ("diag_notau", 0, 0, 3), ("row", 0, 1, 0),
            ("two_level", 1, 0, 0), ("unsplit", 0, 2, 0), ("unsplit_mainonly", 0, 2, 2)]
if len(sys.argv) > 3:
    variants = [v for v in variants if v[0] in sys.argv[3].split(",")]
for name, tl, res, npr in variants:
    op = pkg.KnnOpts(no_prune=1 if npr == 1 else 0, timing=1, mq_chunk=0, two_level=tl)
    op.reserved[0] = res
    op.reserved[1] = {2: 1, 3: 2}.get(npr, 0)
    s = pkg.KnnStats()
    for it in range(1 if npr in (1, 3) else 4):
        pkg.smiler_knn(idx.handle, qd, qs, wl.lengths, wl.k, ids, dd, s, op)
    out = (ids.cpu().numpy().copy(), dd.cpu().numpy().copy())
    if ref is None:
        ref = out
    same = (ref[0] == out[0]).all() and (ref[1] == out[1]).all()
    print("%-10s total %.2f ms | lb %.2f + scan %.2f | tau %.2f filter %.2f verify %.2f select %.2f | same=%s"
          % (name, s.ns_total / 1e6, s.ns_window_lb / 1e6, s.ns_group_scan / 1e6, s.ns_tau / 1e6,
             s.ns_filter / 1e6, s.ns_verify / 1e6, s.ns_select / 1e6, same))
