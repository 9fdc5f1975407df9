"""Small one-shot runs for profiling the fused LB kernel: C2 (w=8, 32 MQs over 2^20)
or C4-shaped (w=16, 16 MQs over 8M points).  usage: prof_lb.py C2|C4 [f32|i16] [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_sigmod_zhout15_b200 as pkg

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
dtype = sys.argv[2] if len(sys.argv) > 2 else "f32"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
if cfg == "C2":
    wl = synth.make_workload("C2", dtype, mq_per_sensor=32)
else:
    wl = synth.make_workload("C4", dtype, n=8 * 1024 * 1024)
dev = torch.device("cuda", 0)
idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band)
qd = torch.from_numpy(wl.queries).to(dev)
nl = len(wl.lengths)
ids = torch.empty((wl.n_mq, nl, wl.k), dtype=torch.int64, device=dev)
dd = torch.empty((wl.n_mq, nl, wl.k), dtype=torch.int32 if dtype == "i16" else torch.float32, device=dev)
st = pkg.KnnStats()
op = pkg.KnnOpts(timing=1, variant=int(os.environ.get("SMILER_AB", "0")))
for _ in range(reps):
    pkg.smiler_knn(idx.handle, qd, np.ascontiguousarray(wl.query_sensor), wl.lengths, wl.k, ids, dd, st, op)
print(cfg, {k: round(v / 1e6, 3) for k, v in st.as_dict().items() if k.startswith("ns_")})
