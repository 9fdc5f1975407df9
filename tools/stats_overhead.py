import os, sys
sys.path.insert(0, "/root/repo")
import numpy as np, torch, synth
import paper_conf_sigmod_zhout15_b200 as pkg
wl = synth.make_workload("C2", "f32", mq_per_sensor=256)
dev = torch.device("cuda", 0); st = torch.cuda.Stream()
idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band, stream=st)
qd = torch.from_numpy(wl.queries).to(dev)
ids = torch.empty((256, 4, 32), dtype=torch.int64, device=dev); dd = torch.empty((256, 4, 32), dtype=torch.float32, device=dev)
S = pkg.KnnStats(); op = pkg.KnnOpts(timing=1)
for _ in range(3): pkg.smiler_knn(idx.handle, qd, None, wl.lengths, 32, ids, dd)
for mode in ("plain", "stats", "plain", "stats"):
    torch.cuda.synchronize(); e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(st); tot = 0.0
    for _ in range(20):
        if mode == "plain": pkg.smiler_knn(idx.handle, qd, None, wl.lengths, 32, ids, dd)
        else:
            pkg.smiler_knn(idx.handle, qd, None, wl.lengths, 32, ids, dd, S, op); tot += S.ns_total
    e1.record(st); torch.cuda.synchronize()
    print(mode, e0.elapsed_time(e1) / 20, "ms/step", (tot / 20 / 1e6) if tot else "")
