"""Small C5-shaped run for profiling the DTW kernels (64 sensors x 100k, 10 MQs each)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_sigmod_zhout15_b200 as pkg

dtype = sys.argv[1] if len(sys.argv) > 1 else "f32"
wl = synth.make_workload("C5", dtype, n_sensors=int(sys.argv[2]) if len(sys.argv) > 2 else 64)
dev = torch.device("cuda", 0)
idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band)
qd = torch.from_numpy(wl.queries).to(dev)
nl = len(wl.lengths)
ids = torch.empty((wl.n_mq, nl, wl.k), dtype=torch.int64, device=dev)
dd = torch.empty((wl.n_mq, nl, wl.k), dtype=torch.int32 if dtype == "i16" else torch.float32, device=dev)
st = pkg.KnnStats()
op = pkg.KnnOpts(timing=1)
for _ in range(2):
    pkg.smiler_knn(idx.handle, qd, np.ascontiguousarray(wl.query_sensor), wl.lengths, wl.k, ids, dd, st, op)
print({k: round(v / 1e6, 3) for k, v in st.as_dict().items() if k.startswith("ns_")}, st.survivors / st.candidates,
      st.dtw_cells / ((st.ns_tau + st.ns_verify) * 1e-9) / 1e12, "T cells/s")
