"""Debug: TMA ring scan vs plain ring scan on a small C5-shaped stream batch."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
import paper_conf_sigmod_zhout15_b200 as pkg
from paper_conf_sigmod_zhout15_b200 import smiler as sm

dtype = sys.argv[1] if len(sys.argv) > 1 else "i16"
notma = len(sys.argv) > 2 and sys.argv[2] == "notma"
wl = synth.make_workload("C5", dtype, step=0, n=12001, n_sensors=3, mq_per_sensor=2)
vt = np.int32 if dtype == "i16" else np.float32
with pkg.Index(wl.series, wl.offsets, wl.window, wl.band) as idx:
    n = wl.queries.shape[0]
    ids = np.empty((n, len(wl.lengths), wl.k), np.int64)
    d = np.empty((n, len(wl.lengths), wl.k), vt)
    o = sm.KnnOpts()
    if notma:
        o.reserved[0] = 7
    h = sm.smiler_stream_create(idx.handle, np.ascontiguousarray(wl.queries), wl.query_sensor, wl.lengths, wl.k,
                                ids, d, o)
    import oracle
    oid, od = oracle.knn(wl, mode=(None if dtype == "i16" else "f32"))
    print(dtype, "notma" if notma else "tma", "ids equal:", np.array_equal(ids, oid))
    sm.smiler_stream_free(h)
