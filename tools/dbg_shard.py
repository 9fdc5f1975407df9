import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, synth, paper_conf_sigmod_zhout15_b200 as pkg
from paper_conf_sigmod_zhout15_b200 import dist as sdist
wl = synth.make_workload("C4", "f32", n=2_000_000, mq_per_sensor=4)
N, D, w = len(wl.series), wl.D, wl.window
with pkg.Index(wl.series, wl.offsets, w, wl.band) as idx:
    i0, d0, st = idx.knn(wl.queries, wl.lengths, wl.k, stats=True)
    print("full", st["survivors"], st["tau_verified"], st["candidates"])
    lbf = idx.lower_bounds_kind(wl.queries, wl.lengths, N, 0)
for G in (1, 2):
    for sh in sdist.window_shards(N, D, max(wl.rhos()), w, G):
        sl = np.ascontiguousarray(wl.series[sh.slice_begin:sh.slice_end])
        with pkg.Index.shard(sl, sh.slice_begin, N, sh.t_begin, sh.t_end, w, wl.band) as idx:
            i1, d1, st = idx.knn(wl.queries, wl.lengths, wl.k, stats=True)
            print("G", G, sh, st["survivors"], st["tau_verified"], st["candidates"], "thr?", d1[0, 0, -1], d0[0, 0, -1])
            try:
                lbs = idx.lower_bounds_kind(wl.queries, wl.lengths, len(sl), 0)
                a = sh.t_begin - sh.slice_begin
                print("  lb local[a:a+5]", lbs[0, 0, a:a + 5], "full", lbf[0, 0, sh.t_begin:sh.t_begin + 5])
            except Exception as e:
                print("  lb err", e)
