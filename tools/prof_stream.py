"""Continuous-stream run shaped like C3/C5 for ncu (argv: config dtype n_sensors steps)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import synth
import paper_conf_sigmod_zhout15_b200 as pkg

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
dtype = sys.argv[2] if len(sys.argv) > 2 else "f32"
ns = int(sys.argv[3]) if len(sys.argv) > 3 else 256
steps = int(sys.argv[4]) if len(sys.argv) > 4 else 4
wl = synth.make_workload(cfg, dtype, n_sensors=ns, consecutive=True)
nxt = synth.make_workload(cfg, dtype, n_sensors=ns, consecutive=True, step=steps)
idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band)
exact = len(sys.argv) > 5 and sys.argv[5] == "exact"
st = pkg.Stream(idx, wl.queries, wl.lengths, wl.k, wl.query_sensor, exact_postings=exact)
D = wl.D
acc = {}
for s in range(steps):
    # the next point of every stream (a real feed would supply it)
    newp = np.ascontiguousarray(nxt.queries[:, D - steps + s]) if s < steps else None
    _, _, stt = st.step(newp, stats=True, timing=True)
    for k, v in stt.items():
        if k.startswith("ns_"):
            acc[k] = acc.get(k, 0) + v / 1e6 / steps
print(cfg, dtype, ns, {k: round(v, 3) for k, v in acc.items()})
