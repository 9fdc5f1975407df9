"""Multi-process host logic of the multi-GPU paths on CPU (gloo, world size 2).

The per-rank kNN step is played by the oracle restricted to the rank's owned
candidate range (tests may use the oracle); the plan, the all-gather layout
and the merge semantics are the product's (paper_conf_sigmod_zhout15_b200/dist.py).
"""
import os
import socket

import numpy as np
import pytest

import synth
from paper_conf_sigmod_zhout15_b200 import dist as sdist


def merge_reference_numpy(gi: np.ndarray, gd: np.ndarray, k: int):
    """Plain merge used by the CPU tests to check the gather layout: per row,
    the k smallest (dist, id) of the G lists, padding id -1 last."""
    G, rows, kk = gi.shape
    oi = np.full((rows, k), -1, np.int64)
    od = np.empty((rows, k), gd.dtype)
    pad = np.iinfo(np.int32).max if np.issubdtype(gd.dtype, np.integer) else np.inf
    od[:] = pad
    for r in range(rows):
        cand = [(gd[g, r, j], gi[g, r, j]) for g in range(G) for j in range(kk) if gi[g, r, j] >= 0]
        cand.sort()
        for j, (d, t) in enumerate(cand[:k]):
            oi[r, j] = t
            od[r, j] = d
    return oi, od


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_window_plan_covers_and_has_halos():
    for n, D, rho, w, G in [(100_000_000, 96, 8, 16, 8), (40009, 128, 25, 8, 3), (1000, 32, 4, 16, 4)]:
        sh = sdist.window_shards(n, D, rho, w, G)
        assert sh[0].t_begin == 0 and sh[-1].t_end == n
        for a, b in zip(sh, sh[1:]):
            assert a.t_end == b.t_begin
        for s in sh:
            assert s.t_begin % w == 0 and s.slice_begin % w == 0
            assert s.slice_begin <= max(0, s.t_begin - rho)
            assert s.slice_end >= min(n, s.t_end + D - 1 + rho)


def test_sensor_plan_partitions():
    for ns, G in [(1024, 8), (10, 3), (3, 4)]:
        owned = [sdist.sensor_shard(ns, r, G) for r in range(G)]
        flat = sorted(x for o in owned for x in o)
        assert flat == list(range(ns))


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        wl = synth.make_workload("C4", "i16", n=3011, mq_per_sensor=2)
        rho = max(wl.rhos())
        sh = sdist.window_shards(len(wl.series), wl.D, rho, wl.window, world)[rank]
        # the local step: kNN over the owned candidates only, computed on the
        # rank's halo slice, with ids made global
        sl = wl.series[sh.slice_begin:sh.slice_end]
        ids, dists = [], []
        for j in range(wl.n_mq):
            i_, d_ = oracle.knn_one(sl, wl.queries[j], wl.lengths, wl.rhos(), wl.k,
                                    t_lo=sh.t_begin - sh.slice_begin, t_hi=sh.t_end - sh.slice_begin)
            i_ = np.where(i_ >= 0, i_ + sh.slice_begin, -1)
            ids.append(i_)
            dists.append(np.minimum(d_, np.iinfo(np.int32).max).astype(np.int32))
        ids = torch.from_numpy(np.ascontiguousarray(np.stack(ids).reshape(-1, wl.k)))
        dists = torch.from_numpy(np.ascontiguousarray(np.stack(dists).reshape(-1, wl.k)))
        gi, gd = sdist.all_gather_results(ids, dists)
        mi, md = sdist.merge_gathered(gi, gd, wl.k,
                                      merge=lambda a, b, G, rows, k: merge_reference_numpy(
                                          a.numpy(), b.numpy(), k))
        if rank == 0:
            oi, od = oracle.knn(wl)
            q.put((np.array_equal(mi.reshape(oi.shape), oi),
                   np.array_equal(md.reshape(od.shape).astype(np.int64), od), gi.shape[0]))
    finally:
        dist.destroy_process_group()


def test_window_sharded_gather_merge_gloo():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    ok_ids, ok_d, G = q.get(timeout=10)
    assert G == 2 and ok_ids and ok_d
