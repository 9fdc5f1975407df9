"""Multi-GPU host logic: one process per GPU,
torch.distributed for the plumbing (NCCL on GPUs, gloo in the CPU tests).

* Sensor sharding (C3/C5): sensors round-robin over ranks; every master query
  runs on the rank that holds its sensor.  No collective on the
  data path.
* Window-range sharding (C4, reading R24): rank g owns candidate starts
  [T_g, T_{g+1}) (T_g a multiple of w) and holds the halo slice
  [floor_w(max(0, T_g - rho_max)), min(N, T_{g+1} + D - 1 + rho_max)); its
  envelopes, disjoint windows and LB_w equal the unsharded ones, every
  candidate is owned by exactly one rank, so the union of the local top-k
  lists contains the global top-k.  One all-gather of the (ids, dists) lists,
  then `smiler_merge_topk` (a9) selects the final k.

This module holds no method arithmetic: planning and collectives only; every
kNN step runs in libsmiler.so.
"""
from __future__ import annotations

import dataclasses
from typing import Callable, List, Optional, Sequence

import numpy as np


def sensor_shard(n_sensors: int, rank: int, world: int) -> List[int]:
    """Sensors owned by `rank` (round-robin)."""
    return list(range(rank, n_sensors, world))


@dataclasses.dataclass(frozen=True)
class WindowShard:
    rank: int
    t_begin: int      # owned candidate starts [t_begin, t_end), global
    t_end: int
    slice_begin: int  # held points [slice_begin, slice_end), global
    slice_end: int


def window_shards(n: int, D: int, rho_max: int, window: int, world: int) -> List[WindowShard]:
    """R24 plan: w-aligned owned ranges covering [0, n) plus halos."""
    bounds = [((n * g) // world) // window * window for g in range(world)] + [n]
    out = []
    for g in range(world):
        t0, t1 = bounds[g], bounds[g + 1]
        s0 = max(0, t0 - rho_max) // window * window
        s1 = min(n, t1 + D - 1 + rho_max)
        out.append(WindowShard(g, t0, t1, s0, s1))
    return out


def all_gather_results(ids, dists, group=None):
    """All-gather per-rank result tensors [rows, k] into [G, rows, k] (torch).
    NCCL gathers the device tensors directly (over NVLink); a gloo group (the
    CPU tests, or several ranks sharing one GPU, which NCCL refuses) gathers
    host copies and returns tensors on the inputs' device."""
    import torch
    import torch.distributed as dist
    G = dist.get_world_size(group)
    rows = int(ids.shape[0])
    dev = ids.device
    if dev.type == "cuda" and dist.get_backend(group) != "nccl":
        ids, dists = ids.cpu(), dists.cpu()
    gi = torch.empty((G * rows,) + tuple(ids.shape[1:]), dtype=ids.dtype, device=ids.device)
    gd = torch.empty((G * rows,) + tuple(dists.shape[1:]), dtype=dists.dtype, device=dists.device)
    dist.all_gather_into_tensor(gi, ids.contiguous(), group=group)
    dist.all_gather_into_tensor(gd, dists.contiguous(), group=group)
    gi, gd = gi.to(dev), gd.to(dev)
    return gi.view((G,) + tuple(ids.shape)), gd.view((G,) + tuple(dists.shape))


def merge_gathered(gi, gd, k: int, merge: Optional[Callable] = None):
    """Final selection over gathered [G, rows, k] lists.  `merge` defaults to
    the library's smiler_merge_topk (a9) on the tensors' device."""
    import torch
    G, rows = int(gi.shape[0]), int(gi.shape[1])
    if merge is not None:
        return merge(gi, gd, G, rows, k)
    from .smiler import smiler_merge_topk
    oi = torch.empty((rows, k), dtype=torch.int64, device=gi.device)
    od = torch.empty((rows, k), dtype=gd.dtype, device=gd.device)
    dev = gi.device.index if gi.device.type == "cuda" else 0
    stream = torch.cuda.current_stream(gi.device) if gi.device.type == "cuda" else None
    smiler_merge_topk(gi, gd, G, rows, k, oi, od, device=dev, stream=stream)
    return oi, od


class WindowShardSearch:
    """One rank's part of the C4 path, kept across calls: the shard index
    (envelopes of its halo slice) is built once; every `knn` call is the local
    Suffix kNN over the owned candidates, one all-gather of the (ids, dists)
    lists and the a9 merge (`smiler_merge_topk`).  With `shared_tau` (NEXT-2)
    the ranks also prune with each other's running thresholds through a
    CUDA-IPC buffer (`shared_tau_buffers`)."""

    def __init__(self, series_slice, shard: WindowShard, n_global: int, window: int, band: float, device: int,
                 stream=None, group=None):
        from .smiler import Index
        self.shard, self.group, self.stream = shard, group, stream
        self.index = Index.shard(series_slice, shard.slice_begin, n_global, shard.t_begin, shard.t_end, window,
                                 band, device=device, stream=stream)

    def knn(self, queries, lengths: Sequence[int], k: int, shared_tau=None):
        """`queries`: CUDA tensor [n_mq, D]; returns (ids, dists) CUDA tensors
        [n_mq, n_len, k], identical on every rank.  shared_tau: a device buffer
        of n_mq * n_len keys, all ones before the first rank uses it."""
        import torch
        from .smiler import KnnOpts, smiler_knn
        n_mq, nl = int(queries.shape[0]), len(lengths)
        ids = torch.empty((n_mq, nl, k), dtype=torch.int64, device=queries.device)
        dists = torch.empty((n_mq, nl, k), dtype=torch.int32 if self.index.dtype == 0 else torch.float32,
                            device=queries.device)
        op = KnnOpts(shared_tau=shared_tau.data_ptr() if shared_tau is not None else None)
        smiler_knn(self.index.handle, queries, None, lengths, k, ids, dists, None, op)
        if self.stream is not None:   # the library runs on `stream`; the collective on torch's
            torch.cuda.current_stream(queries.device).wait_stream(self.stream)
        gi, gd = all_gather_results(ids.view(n_mq * nl, k), dists.view(n_mq * nl, k), self.group)
        oi, od = merge_gathered(gi, gd, k)
        return oi.view(n_mq, nl, k), od.view(n_mq, nl, k)

    def close(self):
        self.index.close()


def window_sharded_knn(series_slice, shard: WindowShard, n_global: int, queries, lengths: Sequence[int],
                       k: int, window: int, band: float, device: int, stream=None, group=None,
                       search: Optional[WindowShardSearch] = None):
    """One rank's step of the C4 path (local kNN on its shard, all-gather,
    merge).  Pass `search` (a WindowShardSearch) to reuse the shard index across
    calls; without it the index is built for this call and freed."""
    if search is not None:
        return search.knn(queries, lengths, k)
    s = WindowShardSearch(series_slice, shard, n_global, window, band, device, stream, group)
    try:
        return s.knn(queries, lengths, k)
    finally:
        s.close()


def shared_tau_buffers(rows: int, device, n: int = 2, group=None):
    """NEXT-2: `n` device buffers of `rows` threshold keys
    (smiler_knn_opts.shared_tau), allocated on rank 0's GPU and mapped into every
    rank through CUDA IPC, so each rank's atomicMin reaches them over NVLink.
    All ones (-1) = no threshold yet.  Use buffer s % n for step s and reset the
    next one (rank 0, `reset_shared_tau`) before the step's collective, so no
    rank can see a previous batch's minima."""
    import torch
    import torch.distributed as dist
    rank = dist.get_rank(group)
    handles = None
    bufs = None
    if rank == 0:
        bufs = [torch.full((rows,), -1, dtype=torch.int64, device=device) for _ in range(n)]
        handles = [b.untyped_storage()._share_cuda_() for b in bufs]
        torch.cuda.synchronize(device)
    obj = [handles]
    dist.broadcast_object_list(obj, src=0, group=group)
    if rank != 0:
        bufs = []
        for h in obj[0]:
            st = torch.UntypedStorage._new_shared_cuda(*h)
            t = torch.empty(0, dtype=torch.int64, device=st.device)
            t.set_(st, 0, (rows,), (1,))
            bufs.append(t)
    return bufs


def reset_shared_tau(buf) -> None:
    """Back to 'no threshold' (all ones); rank 0 only, on its stream."""
    buf.fill_(-1)
