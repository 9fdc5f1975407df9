#!/usr/bin/env python
"""bench.py -- kNN-DTW throughput of the SMiLer Search Step on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--dtype f32|i16]
                    [--impl ours|reference]

A step = one smiler_knn call over one batch of master queries (every row of
SURVEY §8(a): query prep, window-level postings, group-level LB scan, tau,
filter, DTW verification, top-k).  Default workload = BASELINE.json configs[1]
(C2: one sensor of 2^20 points, 256 master queries per step, ELV
{16,32,64,128}, band 10%, k=32, w=8).  Multi-GPU (torchrun): every rank takes
its own batch of master queries over its own copy of the index (independent
units, weak scaling, no data-path collective) -- or, with --config C4, owns a
window range and the per-rank top-k lists are merged by one NCCL all-gather +
smiler_merge_topk.

Rank 0 prints one JSON line (see the keys below).  `--impl reference` times
the oracle (the plain CPU brute force, the only "reference" this paper-only
tier has) on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "kNN-DTW queries/s and DTW cells/s at 1/2/4/8 B200; LB-scan HBM GB/s vs peak"
UNIT = "master_queries/s"


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "sm_max_mhz": 1965.0}, "fallback"


def load_alu_peaks():
    p = os.path.join(ROOT, "profiles", "alu_peaks.json")
    if os.path.exists(p):
        return json.load(open(p))
    return None


# ---------------------------------------------------------------------------
# clocks sampler (nvidia-smi during the timed region)
# ---------------------------------------------------------------------------
class Clocks:
    """SM clock and throttle reasons sampled DURING the timed region: NVML every
    ~5 ms from a thread (short timed regions still get samples), else
    nvidia-smi -lms 100."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    REASONS = (("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
               ("sw_power_cap", 0x4))

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.proc = None
        self.lines = []
        self.t = None
        self.nv = None
        self.samples = []      # NVML: (sm_mhz, max_mhz, reason bits)
        self.stop_flag = False

    def start(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.gpu)
            self.nv = (pynvml, h)
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
            return
        except Exception:
            self.nv = None
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), "--query-gpu=" + self.FIELDS,
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _poll(self):
        nv, h = self.nv
        mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
        while not self.stop_flag:
            try:
                self.samples.append((nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM), mx,
                                     nv.nvmlDeviceGetCurrentClocksEventReasons(h)))
            except Exception:
                pass
            time.sleep(0.005)

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.nv:
            self.stop_flag = True
            self.t.join(timeout=2)
            sm = [x[0] for x in self.samples]
            reasons = {nm for _, _, bits in self.samples for nm, b in self.REASONS if bits & b}
            return {"sm_mhz": statistics.median(sm) if sm else None,
                    "sm_max_mhz": max(x[1] for x in self.samples) if sm else None,
                    "reasons": sorted(reasons), "samples": len(sm), "source": "nvml (5 ms)"}
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm), "source": "nvidia-smi (100 ms)"}


# ---------------------------------------------------------------------------
# workloads
# ---------------------------------------------------------------------------
def rank_workload(cfg: str, dtype: str, rank: int, world: int, mq_per_step: int):
    """The MQ batch of this rank.  Series identical on every rank (same seeds);
    master queries at distinct tail offsets per rank."""
    if cfg == "C2":
        wl = synth.make_workload("C2", dtype, mq_per_sensor=mq_per_step * world)
        sl = slice(rank * mq_per_step, (rank + 1) * mq_per_step)
        wl.queries = np.ascontiguousarray(wl.queries[sl])
        wl.query_sensor = np.ascontiguousarray(wl.query_sensor[sl])
        return wl
    if cfg in ("C3", "C5"):
        # sensors round-robin over ranks; every MQ runs where its sensor lives
        _, ns, N, periods, lens, k, w, band, mqs = synth.CONFIGS[cfg]
        mine = list(range(rank, ns, world))
        parts, qs, qsens, offs, tails, qoff = [], [], [], [0], [], []
        D = lens[-1]
        H = D + 7 * mqs + synth.STEP_MAX + 1   # same history for every continuous step
        for li, s in enumerate(mine):
            z = synth.sensor_series(synth.CONFIGS[cfg][0], s, N, H, periods[s % len(periods)])
            x = synth.quantise(z, dtype)
            parts.append(x[:N])
            offs.append(offs[-1] + N)
            tails.append(x[N:])
            for j in range(mqs):
                qs.append(x[N + 7 * j:N + 7 * j + D])
                qsens.append(li)
                qoff.append(7 * j)
        wl = synth.Workload(cfg, dtype, np.concatenate(parts), np.asarray(offs, np.int64),
                            np.ascontiguousarray(np.stack(qs)), np.asarray(qsens, np.int32), lens, k, w, band)
        wl.tails, wl.qoff = tails, np.asarray(qoff, np.int64)
        return wl
    if cfg == "C4":
        # one long series; every rank holds the same MQ batch and its own window range
        return synth.make_workload("C4", dtype, mq_per_sensor=mq_per_step)
    raise ValueError(cfg)


def cells_per_mq(wl):
    from paper_conf_sigmod_zhout15_b200 import smiler as _s  # noqa: F401
    tot = 0
    rhos = wl.rhos()
    for j in range(wl.n_mq):
        n = wl.offsets[wl.query_sensor[j] + 1] - wl.offsets[wl.query_sensor[j]]
        for d, r in zip(wl.lengths, rhos):
            r = min(r, d - 1)
            tot += (n - d + 1) * (d * (2 * r + 1) - r * (r + 1))
    return tot / wl.n_mq


# ---------------------------------------------------------------------------
# oracle (CPU) baseline
# ---------------------------------------------------------------------------
def oracle_sample(wl, target_s: float):
    """Time the oracle, as it stands, on a bounded sample of the workload: one
    master query, all its item queries, candidates t in [0, T).  Returns
    (master queries/s extrapolated to the full candidate range, cores, sample text)."""
    import oracle
    oracle.build()
    cores = os.cpu_count() or 1
    s = int(wl.query_sensor[0])
    series = wl.sensor_slice(s)
    n = len(series)
    rhos = wl.rhos()
    T = min(n, 2000)
    dt = oracle.time_knn(series, wl.queries[0], wl.lengths, rhos, wl.k, T, cores)
    if dt < target_s / 4 and T < n:
        T = int(min(n, T * max(1.0, target_s / max(dt, 1e-3))))
        dt = oracle.time_knn(series, wl.queries[0], wl.lengths, rhos, wl.k, T, cores)
    frac = T / (n - wl.lengths[0] + 1)
    mqps = frac / dt
    return mqps, cores, dt, ("1 master query (all %d item queries) of %s, candidates t in [0, %d) of %d "
                             "(%.2f%%), %.1f s wall; MQ/s extrapolated linearly to the full candidate range"
                             % (len(wl.lengths), wl.name, T, n, 100 * frac, dt))


def cpu_model() -> str:
    """The host CPU's model name (lscpu / /proc/cpuinfo)."""
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.lower().startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


# ---------------------------------------------------------------------------
CFG_NAMES = {
    "C2": "C2: one sensor, 2^20 points, ELV {16,32,64,128}, band 10%, k=32, w=8, 256 MQs/step/GPU",
    "C3": "C3: 1024 sensors x 100k, ELV {32,64,96}, rho=8, k=64, w=16, 1 MQ stream/sensor (one tick per step), "
          "sharded by sensor",
    "C4": "C4: one series of 1e8 points, ELV {32,64,96}, rho=8, k=32, w=16, 16 MQs/step, window ranges "
          "sharded over GPUs, NCCL all-gather + smiler_merge_topk",
    "C5": "C5: 1024 sensors x 100k, 10 streams/sensor (10,240 MQs/tick), ELV {16,32,64,128}, band 20%, k=128, "
          "w=8, sharded by sensor",
}


class Runner:
    """One configuration's step on this rank.  step() = device-resident inputs
    and outputs; step_e2e() = pinned host inputs -> result on the host."""

    def __init__(self, args, pkg, torch, dist, rank, world, local, dev, stream):
        self.args, self.pkg, self.torch, self.dist = args, pkg, torch, dist
        self.rank, self.world, self.dev, self.stream = rank, world, dev, stream
        cfg = args.config
        wl = rank_workload(cfg, args.dtype, rank, world, args.mq if cfg == "C2" else 16)
        self.wl = wl
        self.n_len, self.k = len(wl.lengths), wl.k
        self.sharded_window = cfg == "C4"
        if self.sharded_window:
            from paper_conf_sigmod_zhout15_b200 import dist as sdist
            self.sdist = sdist
            N = len(wl.series)
            sh = sdist.window_shards(N, wl.D, max(wl.rhos()), wl.window, world)[rank]
            self.shard = sh
            sl = np.ascontiguousarray(wl.series[sh.slice_begin:sh.slice_end])
            self.idx = pkg.Index.shard(sl, sh.slice_begin, N, sh.t_begin, sh.t_end, wl.window, wl.band,
                                       device=local, stream=stream)
            self.index_points = len(sl)
            self.global_mq = wl.n_mq              # every rank serves the same MQs
            # NEXT-2: a running threshold shared by the ranks' shards (opt-in)
            self.tau_bufs = sdist.shared_tau_buffers(wl.n_mq * len(wl.lengths), dev) if args.shared_tau else None
            self.step_no = 0
        else:
            self.idx = pkg.Index(wl.series, wl.offsets, wl.window, wl.band, device=local, stream=stream)
            self.index_points = len(wl.series)
            self.global_mq = None                 # summed over ranks
        self.qd = torch.from_numpy(wl.queries).to(dev)
        self.qs = None if self.sharded_window else np.ascontiguousarray(wl.query_sensor)
        vt = torch.int32 if args.dtype == "i16" else torch.float32
        self.vt = vt
        self.ids = torch.empty((wl.n_mq, self.n_len, self.k), dtype=torch.int64, device=dev)
        self.dd = torch.empty((wl.n_mq, self.n_len, self.k), dtype=vt, device=dev)
        self.op = pkg.KnnOpts(no_prune=0, timing=1, mq_chunk=0, two_level=int(args.two_level))
        self.op.tau_mult = args.tau_mult
        self.op_fast = pkg.KnnOpts(no_prune=0, timing=0, mq_chunk=0, two_level=int(args.two_level))
        self.op_fast.tau_mult = args.tau_mult
        # A/B: kernel-path variant (smiler_knn_opts.variant, same results) and tau-set trim size
        ab = int(os.environ.get("SMILER_AB", "0"))
        self.op.variant = ab
        self.op_fast.variant = ab
        keep = int(os.environ.get("SMILER_TAU_KEEP", "0"))
        self.op.tau_keep = keep
        self.op_fast.tau_keep = keep
        # C5 is a continuous prediction stream: every step is one tick of all
        # streams (each MQ advances one point); after the first tick the previous
        # tick's neighbours seed the thresholds (smiler_knn_step)
        # C3 / C5 are continuous streams: by default every step is one
        # tick through the reused window-level index (Remark 1, smiler_stream_step)
        self.streaming = (not args.no_stream) and cfg in ("C3", "C5")
        self.continuous = (cfg == "C5" and not args.no_continuous) or self.streaming
        self.tick = 0
        if self.continuous:
            D = wl.D
            idx_s = np.asarray(wl.query_sensor)
            tails = np.stack([wl.tails[s_] for s_ in range(len(wl.tails))])
            self.ids2 = torch.empty_like(self.ids)
            self.have_prev = False
            if self.streaming:
                # a tick appends one point per stream: the initial MQs and every later
                # point of each stream's tail, as far as the tail reaches (no wrap:
                # a stream only ever sees its own consecutive points)
                T = tails.shape[1] - int(wl.qoff.max()) - D
                q0 = tails[idx_s[:, None], wl.qoff[:, None] + np.arange(D)[None, :]]
                newp = tails[idx_s[:, None], wl.qoff[:, None] + D - 1 + np.arange(T)[None, :]].T  # [T][n_mq]
                self.q0 = torch.from_numpy(np.ascontiguousarray(q0)).to(dev)
                self.newp_host = torch.from_numpy(np.ascontiguousarray(newp)).pin_memory()
                self.newp = self.newp_host.to(dev)
                self.max_ticks = T - 1
            else:
                T = 2 * args.steps + args.warmup + 12
                cols = wl.qoff[:, None] + np.arange(D)[None, :]
                qt = np.empty((T, wl.n_mq, D), wl.queries.dtype)
                for s_ in range(T):
                    qt[s_] = tails[idx_s[:, None], cols + s_]
                self.qticks_host = torch.from_numpy(qt).pin_memory()
                self.qticks = self.qticks_host.to(dev)

    def mq_per_step(self):
        """Master queries completed per step on this rank (for the value)."""
        if self.sharded_window:
            return self.wl.n_mq / self.world  # each MQ's work is split over the ranks
        return self.wl.n_mq

    def _merge(self, ids, dd):
        rows = self.wl.n_mq * self.n_len
        gi, gd = self.sdist.all_gather_results(ids.view(rows, self.k), dd.view(rows, self.k))
        oi, od = self.sdist.merge_gathered(gi, gd, self.k)
        return oi, od

    def step(self, stats=None, opts=None):
        pkg = self.pkg
        op = opts if opts is not None else (self.op if stats is not None else self.op_fast)
        if self.streaming:
            if not self.have_prev:
                self.stream_h = pkg.smiler_stream_create(self.idx.handle, self.q0, self.qs, self.wl.lengths,
                                                         self.k, self.ids, self.dd)
                self.have_prev = True
                self.tick = 1
            if self.tick > self.max_ticks:
                raise RuntimeError("the streams reached the end of their synthetic tails (%d ticks)" % self.max_ticks)
            pkg.smiler_stream_step(self.stream_h, self.newp[self.tick], self.ids, self.dd, stats, op)
            self.tick += 1
            return
        if self.continuous:
            q = self.qticks[self.tick % self.qticks.shape[0]]
            self.tick += 1
            if self.have_prev:
                pkg.smiler_knn_step(self.idx.handle, q, self.qs, self.wl.lengths, self.k, self.ids, 1,
                                    self.ids2, self.dd, stats, op)
                self.ids, self.ids2 = self.ids2, self.ids
            else:
                pkg.smiler_knn(self.idx.handle, q, self.qs, self.wl.lengths, self.k, self.ids, self.dd,
                               stats, op)
                self.have_prev = True
            return
        self._arm_shared_tau(op)
        pkg.smiler_knn(self.idx.handle, self.qd, self.qs, self.wl.lengths, self.k, self.ids, self.dd, stats, op)
        if self.sharded_window:
            with self.torch.cuda.stream(self.stream):
                self._merge(self.ids, self.dd)

    def _arm_shared_tau(self, op):
        """Step s uses shared buffer s % 2; rank 0 resets the other one first (it is
        next used after this step's all-gather, which orders the reset before it)."""
        if not (self.sharded_window and self.tau_bufs):
            return
        s = self.step_no
        self.step_no += 1
        if self.rank == 0:
            with self.torch.cuda.stream(self.stream):
                self.sdist.reset_shared_tau(self.tau_bufs[(s + 1) % 2])
        op.shared_tau = self.tau_bufs[s % 2].data_ptr()

    def e2e_buffers(self):
        torch = self.torch
        self.qh = torch.from_numpy(self.wl.queries).pin_memory()
        rows = self.wl.n_mq * self.n_len
        self.ih = torch.empty((rows, self.k), dtype=torch.int64).pin_memory()
        self.dh = torch.empty((rows, self.k), dtype=self.vt).pin_memory()
        h2d = self.qh.numel() * self.qh.element_size() + self.n_len * 4 + (0 if self.qs is None else self.qs.nbytes)
        if self.streaming:  # a tick uploads one new point per stream
            h2d = self.wl.n_mq * self.qh.element_size()
        return int(h2d), int(self.ih.numel() * 8 + self.dh.numel() * 4)

    def step_e2e(self):
        pkg, torch = self.pkg, self.torch
        if self.streaming:
            # one tick through the public stream API with pinned host buffers
            if self.tick > self.max_ticks:
                raise RuntimeError("the streams reached the end of their synthetic tails (%d ticks)" % self.max_ticks)
            pkg.smiler_stream_step(self.stream_h, self.newp_host[self.tick], self.ih.view(self.wl.n_mq, self.n_len, self.k),
                                   self.dh.view(self.wl.n_mq, self.n_len, self.k))
            self.tick += 1
            return
        if self.continuous:
            q = self.qticks_host[self.tick % self.qticks_host.shape[0]]
            self.tick += 1
            ih = self.ih.view(self.wl.n_mq, self.n_len, self.k)
            dh = self.dh.view(self.wl.n_mq, self.n_len, self.k)
            if not hasattr(self, "prev_h"):
                self.prev_h = torch.empty_like(ih).pin_memory()
                pkg.smiler_knn(self.idx.handle, q, self.qs, self.wl.lengths, self.k, ih, dh)
            else:
                pkg.smiler_knn_step(self.idx.handle, q, self.qs, self.wl.lengths, self.k, self.prev_h, 1, ih, dh)
            self.prev_h.copy_(ih)
            return
        if not self.sharded_window:
            pkg.smiler_knn(self.idx.handle, self.qh, self.qs, self.wl.lengths, self.k,
                           self.ih.view(self.wl.n_mq, self.n_len, self.k), self.dh.view(self.wl.n_mq, self.n_len,
                                                                                       self.k))
            return
        with torch.cuda.stream(self.stream):
            self.qd.copy_(self.qh, non_blocking=True)
        self._arm_shared_tau(self.op_fast)
        pkg.smiler_knn(self.idx.handle, self.qd, None, self.wl.lengths, self.k, self.ids, self.dd, None,
                       self.op_fast)
        with torch.cuda.stream(self.stream):
            oi, od = self._merge(self.ids, self.dd)
            self.ih.copy_(oi, non_blocking=True)
            self.dh.copy_(od, non_blocking=True)
        self.stream.synchronize()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2", choices=["C2", "C3", "C4", "C5"])
    ap.add_argument("--dtype", default="f32", choices=["f32", "i16"])
    ap.add_argument("--mq", type=int, default=256, help="master queries per step per GPU (C2)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--oracle-seconds", type=float, default=12.0)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-continuous", action="store_true", help="C5: independent ticks (no smiler_knn_step)")
    ap.add_argument("--tau-mult", type=int, default=0, help="tau-set size (x k per item query; -1 = none, 0 = default)")
    ap.add_argument("--no-stream", action="store_true",
                    help="C3/C5: do not use the reused window-level index (smiler_stream_step); C5 then uses "
                         "smiler_knn_step, C3 independent searches")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--shared-tau", action="store_true",
                    help="C4: ranks share a running threshold through CUDA IPC / NVLink atomics (NEXT-2)")
    ap.add_argument("--two-level", action="store_true", help="time the paper's two-level path (a3 -> HBM -> a4)")
    ap.add_argument("--sustain-s", type=float, default=0.0,
                    help="after the timed steps, run back to back for this many seconds and report the sustained "
                         "rate and p50/p99 step latency (the C5 protocol uses 60)")
    ap.add_argument("--prof-steps", type=int, default=10,
                    help="steps of the separate profiled pass (per-phase events, counters)")
    ap.add_argument("--two-level-steps", type=int, default=3,
                    help="extra steps of the two-level path for the LB-scan (a4) HBM figure; 0 = skip")
    args = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    cfg_name = CFG_NAMES[args.config]
    scaling = {"C2": "weak", "C3": "strong", "C4": "strong", "C5": "strong"}[args.config]

    if args.impl == "reference":
        if rank != 0:
            return
        wl = rank_workload(args.config, args.dtype, 0, 1, 4)
        vals = []
        total = 0.0
        cores, sample = 0, ""
        for _ in range(args.steps):
            v, cores, dt, sample = oracle_sample(wl, max(1.0, args.oracle_seconds / max(args.steps, 1)))
            vals.append(v)
            total += dt
        v = statistics.median(vals)
        print(json.dumps({"metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
                          "warmup": args.warmup, "ms_per_step": 1000.0 * total / args.steps,
                          "higher_is_better": True, "scaling": scaling, "vs_baseline": None,
                          "dtype": "int64" if args.dtype == "i16" else "f64", "data": "synthetic",
                          "impl": "reference",
                          "config": {"workload": cfg_name, "parallelism": "host cores (oracle)"},
                          "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "cpu_model": cpu_model(),
                                           "kind": "oracle", "sample": sample},
                          "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}))
        return

    import torch
    import torch.distributed as dist
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    from paper_conf_sigmod_zhout15_b200 import build as _build
    _build.build()
    import paper_conf_sigmod_zhout15_b200 as pkg

    stream = torch.cuda.Stream(device=dev)
    if args.config == "C4" and world == 1:
        # single GPU: the window "shard" is the whole series; the all-gather is a no-op
        pass
    if args.config == "C4" and not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29511")
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    R = Runner(args, pkg, torch, dist, rank, world, local, dev, stream)
    wl, n_len, k = R.wl, R.n_len, R.k

    for _ in range(args.warmup):
        R.step()
    torch.cuda.synchronize(dev)

    # ---- timed region: device-resident inputs/outputs ---------------------------
    # The product call exactly as a user makes it (no stats, no per-phase
    # events, no host synchronisation inside the loop).  One CUDA event pair
    # around the loop gives `value`; one event per step boundary gives the step
    # latencies.  The per-phase split comes from a separate profiled pass below.
    gpu_idx = local
    cvd = os.environ.get("CUDA_VISIBLE_DEVICES")
    if cvd:
        try:
            gpu_idx = int(cvd.split(",")[local])
        except ValueError:
            pass
    clocks = Clocks(gpu_idx)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    clocks.start()
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    evs[0].record(stream)
    for s_ in range(args.steps):
        R.step()
        evs[s_ + 1].record(stream)
    torch.cuda.synchronize(dev)
    ck = clocks.stop()
    if world > 1:
        dist.barrier()
    ms = evs[0].elapsed_time(evs[-1])
    step_ms = [evs[s_].elapsed_time(evs[s_ + 1]) for s_ in range(args.steps)]
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    mq_step = (R.global_mq if R.global_mq is not None else R.mq_per_step() * world)
    mq_total = mq_step * args.steps
    if R.global_mq is None and world > 1:
        tm = torch.tensor([R.mq_per_step()], dtype=torch.float64, device=dev)
        dist.all_reduce(tm, op=dist.ReduceOp.SUM)
        mq_step = float(tm.item())
        mq_total = mq_step * args.steps
    value = mq_total / (ms_max / 1000.0)

    prof_steps_planned = max(1, min(args.steps, args.prof_steps)) + args.steps + 1  # profiled pass + e2e ticks
    # ---- sustained run (C5 protocol: >= 60 s, p50 / p99 step latency)
    sustained = None
    if args.sustain_s > 0:
        ck_s = Clocks(gpu_idx)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        ck_s.start()
        t_wall0 = time.perf_counter()
        lat = []
        n_sus = 0
        dev_ms = 0.0
        while time.perf_counter() - t_wall0 < args.sustain_s and \
                (not R.streaming or R.tick + 32 + 2 * prof_steps_planned <= R.max_ticks):
            batch = [torch.cuda.Event(enable_timing=True) for _ in range(33)]
            batch[0].record(stream)
            for b_ in range(32):
                R.step()
                batch[b_ + 1].record(stream)
            batch[-1].synchronize()
            lat += [batch[b_].elapsed_time(batch[b_ + 1]) for b_ in range(32)]
            dev_ms += batch[0].elapsed_time(batch[-1])
            n_sus += 32
        torch.cuda.synchronize(dev)
        ck2 = ck_s.stop()
        lat.sort()
        tl = torch.tensor([dev_ms], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(tl, op=dist.ReduceOp.MAX)
        sustained = {"seconds": time.perf_counter() - t_wall0, "steps": n_sus,
                     "value": mq_step * n_sus / (float(tl.item()) / 1000.0), "unit": UNIT,
                     "p50_step_ms": lat[len(lat) // 2], "p99_step_ms": lat[min(len(lat) - 1, int(0.99 * len(lat)))],
                     "max_step_ms": lat[-1], "clocks": ck2,
                     "timing": "device time per step (CUDA events between back-to-back steps on the library "
                               "stream), rank-0 distribution; value = MQs / max-over-ranks device time"}

    # ---- profiled pass: per-phase CUDA events and counters (smiler_knn_stats) --
    st = pkg.KnnStats()
    phase = {f: 0.0 for f in ("ns_prep", "ns_window_lb", "ns_group_scan", "ns_tau", "ns_filter", "ns_cascade",
                              "ns_verify", "ns_select", "ns_total")}
    acc = {"survivors": 0, "candidates": 0, "dtw_cells": 0.0, "bf_cells": 0.0, "posting_bytes": 0,
           "lb_bytes": 0, "kernel_launches": 0, "mq_chunks": 0, "tau_verified": 0, "finalists": 0}
    prof_steps = max(1, min(args.steps, args.prof_steps))
    ck_p = Clocks(gpu_idx)
    ck_p.start()
    for _ in range(prof_steps):
        R.step(st)
        for f in phase:
            phase[f] += getattr(st, f)
        for f in acc:
            acc[f] += getattr(st, f)
    torch.cuda.synchronize(dev)
    ck_prof = ck_p.stop()
    launches_per_step = acc["kernel_launches"] / prof_steps + (1 if R.sharded_window else 0)

    # ---- e2e: the same public call with pinned host buffers ------------------
    e2e = None
    if not args.no_e2e:
        h2d, d2h = R.e2e_buffers()
        R.step_e2e()
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        f0 = torch.cuda.Event(enable_timing=True)
        f1 = torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        for _ in range(args.steps):
            R.step_e2e()
        f1.record(stream)
        torch.cuda.synchronize(dev)
        ems = f0.elapsed_time(f1)
        te = torch.tensor([ems], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        ems = float(te.item())
        e2e = {"value": mq_total / (ems / 1000.0), "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h, "ms_per_step": ems / args.steps}

    if rank != 0:
        if dist.is_initialized():
            dist.destroy_process_group()
        return

    # ---- secondary: the paper's two-level path (postings in HBM), for a4's HBM figure
    two = None
    if args.two_level_steps > 0 and not args.two_level and args.config != "C4":
        op2 = pkg.KnnOpts(no_prune=0, timing=1, mq_chunk=0, two_level=1)
        st2 = pkg.KnnStats()
        R.step(st2, op2)
        ph2 = {f: 0.0 for f in phase}
        acc2 = {f: 0 for f in acc}
        for _ in range(args.two_level_steps):
            R.step(st2, op2)
            for f in ph2:
                ph2[f] += getattr(st2, f)
            for f in acc2:
                acc2[f] += getattr(st2, f)
        torch.cuda.synchronize(dev)
        two = (ph2, acc2, args.two_level_steps)

    # ---- rooflines ---------------------------------------------------------------
    peaks, peak_kind = load_peaks()
    alu = load_alu_peaks()
    steps = prof_steps
    sm_mhz = ck.get("sm_mhz") or peaks.get("sm_max_mhz", 1965.0)
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    # ALU rooflines from unit counts: per SM per clock a Blackwell SM
    # issues 4 warp-instructions (128 lane-instructions) and its FP32 (FMA) pipe
    # retires 128 lanes (a packed f32x2 instruction takes two of its cycles).
    #   LB term pair, f32 packed (lb_diag_x2): 6 FP32 lane-ops (4 subtractions in
    #     2 FADD2, 2 FMAs in 1 FFMA2) -> 128 / 6 = 21.33 pairs/clk (5 instructions:
    #     issue bound 25.6); scalar f32 forms (8 instructions): 128 / 8 = 16
    #   DTW cell f32: FADD, FMNMX3, FFMA -> issue bound 128 / 3 = 42.67 cells/clk
    #   i16 (int32) mixes: the alu_bench measurement (profiles/alu_peaks.json)
    if args.dtype == "f32":
        term_pclk = 128.0 / 6.0 if (wl.window in (4, 8, 16) and not R.streaming and not args.two_level) else 16.0
        cell_pclk = 128.0 / 3.0
        alu_src = ("unit counts (128 FP32 lanes / 4 issues per SM per clock; DESIGN.md §6) x median SM clock "
                   "sampled during the timed region")
    else:
        term_pclk = alu["lbterm_i32_per_clk_sm"] if alu else 16.0
        cell_pclk = alu["dtw_cell_i32_per_clk_sm"] if alu else 128.0 / 3.0
        alu_src = "profiles/alu_peaks.json (alu_bench int32 mixes) x median SM clock sampled during the timed region"
    term_peak = term_pclk * sms * sm_mhz * 1e6
    cell_peak = cell_pclk * sms * sm_mhz * 1e6
    n_sw = wl.D - wl.window + 1
    if R.sharded_window:
        pts = [R.index_points] * wl.n_mq
    else:
        pts = [int(wl.offsets[s + 1] - wl.offsets[s]) for s in wl.query_sensor.tolist()]
    # algorithmic work: (SW, DW, j) term pairs = n_sw * n_dw * w per MQ
    win_terms = n_sw * sum(p // wl.window * wl.window for p in pts)
    # bytes per (P_EQ, P_EC) pair as stored: f32 streams keep fp16 entries rounded
    # toward zero (smiler_knn_opts.exact_postings = 0), otherwise 2 x 4 bytes
    pair_bytes = 4 if (R.streaming and args.dtype == "f32" and wl.window in (4, 8, 16, 32)) else 8
    post_bytes_step = pair_bytes * n_sw * sum(p // wl.window for p in pts)
    # LB_w array entry: fp16 rounded down on the product path (one direction of the
    # library's lb_bytes stat, which counts the a4 write and the a6 read), else 4 B
    # (the library's lb_bytes counts the a4 write and the a6 read; 0 when the filter
    # runs inside the scan and no LB_w array exists: lagged stream steps, fused a4+a6)
    lb_bytes_step = acc["lb_bytes"] / 2.0 / steps

    # continuous streams recompute only SW_0 (EQ + EC) and SW_1..SW_rho_max (EQ):
    # (rho_max + 2) / 2 term-pair equivalents per (DW, j) instead of n_sw
    rho_env = max(wl.rhos())
    inc_terms = (min(rho_env + 1, n_sw) + 1) / 2.0 * sum(p // wl.window * wl.window for p in pts)

    def rooflines(ph, ac, nsteps, fused):
        ks = {}
        lbb = ac["lb_bytes"] / 2.0 / nsteps  # the LB_w array written by a4 / read by a6 (0 if fused)
        win_s = ph["ns_window_lb"] / 1e9 / nsteps
        if win_s > 0:
            terms = inc_terms if R.streaming else win_terms
            rate = terms / win_s
            ks["lb_fused" if fused else ("window_lb_a3_incremental" if R.streaming else "window_lb_a3")] = {
                "bound": "alu", "achieved": rate / 1e12, "peak": term_peak / 1e12,
                "unit": "T term-pairs/s", "frac": rate / term_peak, "ms": win_s * 1e3,
                "algorithmic_per_mq": "%d (SW,DW,j) term pairs" % ((inc_terms if R.streaming else win_terms)
                                                                     // wl.n_mq)}
        gs_s = ph["ns_group_scan"] / 1e9 / nsteps
        if not fused and gs_s > 0:
            byts = post_bytes_step + lbb
            gbs = byts / gs_s / 1e9
            ks["group_scan_a4"] = {"bound": "hbm", "achieved": gbs, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                                   "frac": gbs / peaks["hbm_gbs"], "ms": gs_s * 1e3,
                                   "algorithmic_bytes_per_step": byts}
        v_s = (ph["ns_verify"] + ph["ns_tau"]) / 1e9 / nsteps
        if v_s > 0:
            cr = ac["dtw_cells"] / nsteps / v_s
            ks["dtw_verify_a7"] = {"bound": "alu", "achieved": cr / 1e12, "peak": cell_peak / 1e12,
                                   "unit": "T DTW cells/s", "frac": cr / cell_peak, "ms": v_s * 1e3}
            if args.dtype == "f32":
                # the pipes' bound for any instruction mix: FADD + FFMA on the
                # 128-lane FP32 pipe, one FMNMX3 on the 64-lane ALU pipe -> 64 cells/clk/SM
                # (the fp32x2-packed variant issues 2 instructions per cell and could reach it)
                pipe_peak = 64.0 * sms * sm_mhz * 1e6
                ks["dtw_verify_a7"]["peak_pipes"] = pipe_peak / 1e12
                ks["dtw_verify_a7"]["frac_pipes"] = cr / pipe_peak
        f_s = ph["ns_filter"] / 1e9 / nsteps
        if f_s > 0 and lbb > 0:
            gbs = lbb / f_s / 1e9
            ks["filter_a6"] = {"bound": "hbm", "achieved": gbs, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                               "frac": gbs / peaks["hbm_gbs"], "ms": f_s * 1e3}
        return ks

    fused_main = not args.two_level and wl.window in (4, 8, 16) and not R.streaming
    kernels = rooflines(phase, acc, steps, fused_main)
    ph_ms = {k_[3:]: v_ / 1e6 / steps for k_, v_ in phase.items()}
    dom = max(kernels.items(), key=lambda kv: kv[1]["ms"])[0]
    rf = dict(kernels[dom])
    rf["kernel"] = dom
    rf["traffic"] = None
    tfile = os.path.join(ROOT, "profiles", "r02", "prof_c2_traffic_per_mq.json")
    if args.config == "C2" and os.path.exists(tfile):
        tname = {"lb_fused": ("lb_diag_x2_kernel<%d>" % wl.window) if args.dtype == "f32"
                 else ("lb_diag_kernel<short, %d>" % wl.window)}.get(dom)
        tmap = json.load(open(tfile))
        if tname and tname in tmap:
            # DRAM bytes per launch = ncu per-MQ traffic x MQs per launch (one chunk per step)
            rf["traffic"] = tmap[tname] * wl.n_mq
            rf["traffic_source"] = "profiles/r02/prof_c2_traffic_per_mq.json (ncu --set full, %s)" % tname
            rf["algorithmic_bytes_per_launch"] = lb_bytes_step
    rf["peak_source"] = ("MEASURED_PEAKS.json hbm_gbs (%s)" % peak_kind if rf["bound"] == "hbm" else alu_src)
    two_level = None
    if two is not None:
        ph2, acc2, n2 = two
        k2 = rooflines(ph2, acc2, n2, False)
        two_level = {"ms_per_step": ph2["ns_total"] / 1e6 / n2,
                     "value": wl.n_mq / (ph2["ns_total"] / 1e9 / n2),
                     "phase_ms_per_step": {k_[3:]: v_ / 1e6 / n2 for k_, v_ in ph2.items()}, "kernels": k2}
    scan = (two_level or {}).get("kernels", {}).get("group_scan_a4") or kernels.get("group_scan_a4")

    cpu = None
    if world == 1 and not args.no_cpu:
        v, cores, dt, sample = oracle_sample(wl, args.oracle_seconds)
        cpu = {"value": v, "unit": UNIT, "cores": cores, "cpu_model": cpu_model(), "kind": "oracle",
               "sample": sample}

    par = {"C2": "dp%d (independent MQ batches)" % world, "C3": "sensor sharding x%d" % world,
           "C5": "sensor sharding x%d" % world, "C4": "window-range sharding x%d + NCCL all-gather merge" % world}
    out = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
        "scaling": scaling, "vs_baseline": None, "dtype": args.dtype if args.dtype == "f32" else "i16->int32",
        "data": "synthetic",
        "config": {"workload": cfg_name, "master_queries_per_step": mq_total / args.steps,
                   "item_queries": wl.lengths, "k": k, "window": wl.window, "band": wl.band,
                   "indexed_points_rank0": int(R.index_points), "parallelism": par[args.config],
                   "l2": "inputs larger than L2 (LB_w %.0f MB per step; two-level posting lists %.0f MB per MQ)"
                         % (lb_bytes_step / 1e6, post_bytes_step / max(1, wl.n_mq) / 1e6)},
        "item_queries_per_s": value * n_len,
        "dtw_cells_per_s": acc["dtw_cells"] / steps / (ms_max / 1000.0 / args.steps) * world,
        "bf_equiv_cells_per_s": acc["bf_cells"] / steps / (ms_max / 1000.0 / args.steps) * world,
        "survivor_frac": acc["survivors"] / max(1, acc["candidates"]),
        "lb_scan_gbs": scan["achieved"] if scan else None,
        "lb_scan_frac_of_hbm": scan["frac"] if scan else None,
        "lb_path": ("continuous streams: window-level rows reused in an HBM ring (Remark 1) + group scan"
                    if R.streaming else "fused a3+a4 (posting rows on chip)" if fused_main
                    else "two-level (postings in HBM)"),
        "phase_ms_per_step": ph_ms,
        "roofline": rf, "kernels": kernels, "two_level": two_level,
        "gpu_launches": int(round(launches_per_step * args.steps)),
        "phase_timing": ("per-phase CUDA events (smiler_knn_stats) of a separate profiled pass of %d steps right "
                         "after the timed region (the timed loop itself records no phase events and never syncs)"
                         % prof_steps),
        "step_ms": {"p50": sorted(step_ms)[len(step_ms) // 2], "max": max(step_ms)},
        "sustained": sustained,
        "clocks": ck,
        "clocks_profiled_pass": ck_prof,
        "cpu_baseline": cpu,
        "e2e": e2e,
    }
    print(json.dumps(out, default=lambda o: o.item() if hasattr(o, "item") else str(o)))
    if dist.is_initialized():
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
