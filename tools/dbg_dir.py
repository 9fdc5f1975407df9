import sys
sys.path.insert(0, ".")
import numpy as np, synth, paper_conf_sigmod_zhout15_b200 as pkg
wl = synth.make_workload("C2", "i16", n=9001, n_sensors=1, mq_per_sensor=3)
with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
    for kind in (0, 4, 3):
        print("kind", kind, flush=True)
        lb = idx.lower_bounds_kind(wl.queries, wl.lengths, 9001, kind)
        print(lb[0, :, :8], flush=True)
