"""The multi-GPU product path with real ranks (-m gpu): two processes share the
one GPU of the test box, each owns a window range of one long series (C4
shape, reading R24), runs the library's kNN on its shard, the (ids, dists)
lists are all-gathered through the process group and merged by
smiler_merge_topk (a9).  The merged result must equal the oracle's brute-force
kNN of the whole series bit for bit -- with and without the shared running
threshold (NEXT-2), whose buffer rank 0 allocates and rank 1 maps through CUDA
IPC.  NCCL refuses two ranks on one device, so the group is gloo (host copies
of the result lists); on an 8-GPU box bench.py runs the same code over NCCL.
"""
import os
import socket

import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank(rank, world, port, dtype, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        from paper_conf_sigmod_zhout15_b200 import dist as sdist
        wl = synth.make_workload("C4", dtype, n=200_003, mq_per_sensor=3)
        N = len(wl.series)
        sh = sdist.window_shards(N, wl.D, max(wl.rhos()), wl.window, world)[rank]
        sl = np.ascontiguousarray(wl.series[sh.slice_begin:sh.slice_end])
        search = sdist.WindowShardSearch(sl, sh, N, wl.window, wl.band, device=0)
        qd = torch.from_numpy(wl.queries).cuda()
        rows = wl.n_mq * len(wl.lengths)
        bufs = sdist.shared_tau_buffers(rows, torch.device("cuda", 0))
        out = []
        for step in range(3):   # the shard index is reused across calls
            shared = bufs[step % 2] if step > 0 else None
            if shared is not None and rank == 0:
                sdist.reset_shared_tau(shared)
                torch.cuda.synchronize()
            dist.barrier()
            ids, dd = search.knn(qd, wl.lengths, wl.k, shared_tau=shared)
            torch.cuda.synchronize()
            out.append((ids.cpu().numpy(), dd.cpu().numpy()))
            dist.barrier()
        search.close()
        if rank == 0:
            import oracle
            oid, od = oracle.knn(wl, mode=None if dtype == "i16" else "f32", threads=os.cpu_count() or 8)
            ok = []
            for ids, dd in out:
                ok.append(bool(np.array_equal(ids, oid)) and
                          bool(np.array_equal(dd.astype(od.dtype), od)))
            q.put(ok)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("dtype", ["i16", "f32"])
def test_two_ranks_window_shards_gather_merge(dtype):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_zhout15_b200 import build
    build.build()
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank, args=(r, 2, port, dtype, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=600)
        assert p.exitcode == 0
    ok = q.get(timeout=10)
    assert ok == [True, True, True], ok
