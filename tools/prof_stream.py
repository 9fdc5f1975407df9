"""Continuous-stream run shaped like C3/C5 for ncu (argv: config dtype n_sensors steps; env SMILER_AB = opts.variant)."""
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
wl = synth.make_workload(cfg, dtype, n_sensors=ns)
idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band)
exact = len(sys.argv) > 5 and sys.argv[5] == "exact"
st = pkg.Stream(idx, wl.queries, wl.lengths, wl.k, wl.query_sensor, exact_postings=exact)
D = wl.D
acc = {}
chunks = 1
for s in range(1, steps + 1):
    # the next point of every stream (a real feed would supply it)
    _, _, stt = st.step(wl.new_points(s), stats=True, timing=True, variant=int(os.environ.get("SMILER_AB", "0")))
    chunks = stt["mq_chunks"]
    for k, v in stt.items():
        if k.startswith("ns_"):
            acc[k] = acc.get(k, 0) + v / 1e6 / steps
print(cfg, dtype, ns, {k: round(v, 3) for k, v in acc.items()})
# master queries per launch of the per-chunk kernels (ncu traffic normalisation)
print("MQ_PER_LAUNCH=%d" % ((wl.n_mq + chunks - 1) // chunks))
