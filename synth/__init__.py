"""Seeded synthetic sensor workloads shared by the oracle tests and the CUDA path.

This module holds NO arithmetic of the method (no envelope, no lower bound, no
DTW, no selection).  It only draws the inputs: sensor series shaped like the
paper's traffic / sensor datasets and the master queries taken from a held-out
tail, plus the per-config parameters.  Both sides (``oracle/`` and the product
binding) receive the same arrays from here.

Recipe:

  x_t = RW_t + A_d sin(2 pi t / P + phi_s) + A_w sin(2 pi t / (7P) + psi_s) + eps_t

  RW     Gaussian random walk, step sigma = 0.05
  A_d    ~ U(0.5, 1.5),  A_w ~ U(0.1, 0.5),  phi_s, psi_s ~ U(0, 2 pi)
  eps_t  ~ N(0, 0.1^2)
  P      = 144 (10-min sampling, ROAD/MALL-like)
           or 288 (5-min sampling, NET-like)

N + H points are drawn per sensor; [0, N) is indexed, master queries come from
the held-out tail [N, N+H) (the paper's protocol holds out the last points and
queries from them).  Each sensor is z-normalised with the mean and
std of its indexed part, the same affine map applied to the tail.
i16 mode: round(128 z) clipped to [-1023, 1023] (reading R17); f32 mode: float32 z.
Seeds: PCG64(20150531 + 1000 * config + sensor).
"""
from __future__ import annotations

import dataclasses
import math
from typing import List, Optional, Sequence

import numpy as np

I16_SCALE = 128.0
I16_MAX = 1023
SEED_BASE = 20150531
STEP_MAX = 4096  # continuous steps supported by make_workload


def sensor_series(config_id: int, sensor: int, n: int, h: int, period: int) -> np.ndarray:
    """float64 z-normalised series of length n + h for one sensor (see module doc)."""
    rng = np.random.Generator(np.random.PCG64(SEED_BASE + 1000 * config_id + sensor))
    a_d = rng.uniform(0.5, 1.5)
    a_w = rng.uniform(0.1, 0.5)
    phi = rng.uniform(0.0, 2.0 * math.pi)
    psi = rng.uniform(0.0, 2.0 * math.pi)
    total = n + h
    t = np.arange(total, dtype=np.float64)
    rw = np.cumsum(rng.normal(0.0, 0.05, size=total))
    eps = rng.normal(0.0, 0.1, size=total)
    x = (rw + a_d * np.sin(2.0 * math.pi * t / period + phi)
         + a_w * np.sin(2.0 * math.pi * t / (7.0 * period) + psi) + eps)
    mu = x[:n].mean()
    sd = x[:n].std()
    if sd == 0.0:
        sd = 1.0
    return (x - mu) / sd


def quantise(z: np.ndarray, dtype: str) -> np.ndarray:
    if dtype == "i16":
        return np.clip(np.rint(z * I16_SCALE), -I16_MAX, I16_MAX).astype(np.int16)
    if dtype == "f32":
        return z.astype(np.float32)
    raise ValueError(dtype)


@dataclasses.dataclass
class Workload:
    """One batch of Suffix kNN queries (Def. 4.1)."""
    name: str
    dtype: str                     # "i16" | "f32"
    series: np.ndarray             # concatenated indexed parts of all sensors
    offsets: np.ndarray            # int64 [n_sensors + 1]
    queries: np.ndarray            # [n_mq, D] master queries, oldest -> newest
    query_sensor: np.ndarray       # int32 [n_mq]
    lengths: List[int]             # ELV, ascending, last == D
    k: int                         # max(EKV)
    window: int                    # omega
    band: float                    # >= 1: absolute rho; in (0,1): rho_i = floor(band * d_i)
    tails: Optional[List[np.ndarray]] = None  # held-out tail of each sensor (the MQs' source)
    qoff: Optional[np.ndarray] = None         # int64 [n_mq]: tail offset of each MQ's first point

    @property
    def n_sensors(self) -> int:
        return len(self.offsets) - 1

    @property
    def n_mq(self) -> int:
        return int(self.queries.shape[0])

    @property
    def D(self) -> int:
        return int(self.queries.shape[1])

    def sensor_slice(self, s: int) -> np.ndarray:
        return self.series[self.offsets[s]:self.offsets[s + 1]]

    def rhos(self) -> List[int]:
        return band_to_rhos(self.band, self.lengths)

    def queries_at(self, step: int) -> np.ndarray:
        """The master queries after `step` more points of a continuous stream
        (each MQ slides one point per step over its sensor's tail)."""
        D = self.D
        out = np.empty_like(self.queries)
        for j in range(self.n_mq):
            o = int(self.qoff[j]) + step
            out[j] = self.tails[int(self.query_sensor[j])][o:o + D]
        return out

    def new_points(self, step: int) -> np.ndarray:
        """The point each stream appends at continuous step `step` (>= 1)."""
        return np.ascontiguousarray(self.queries_at(step)[:, self.D - 1])


def band_to_rhos(band: float, lengths: Sequence[int]) -> List[int]:
    """Reading R4: band >= 1 is an absolute warping width; band in (0,1) is a
    fraction of each item-query length, rho_i = floor(band * d_i)."""
    if band >= 1.0:
        return [int(band) for _ in lengths]
    return [int(math.floor(band * d)) for d in lengths]


# ---------------------------------------------------------------------------
# The five configs of BASELINE.json.  `scale` shrinks
# series lengths / sensor counts / batch sizes for oracle-sized parity runs.
# ---------------------------------------------------------------------------

CONFIGS = {
    # name: (config_id, n_sensors, N, periods, lengths, k, window, band, n_mq_per_sensor)
    "C1": (1, 1, 4096, (144,), [32], 8, 16, 4.0, 1),
    "C2": (2, 1, 1 << 20, (144,), [16, 32, 64, 128], 32, 8, 0.1, 256),
    "C3": (3, 1024, 100_000, (144, 288), [32, 64, 96], 64, 16, 8.0, 1),
    "C4": (4, 1, 100_000_000, (288,), [32, 64, 96], 32, 16, 8.0, 16),
    "C5": (5, 1024, 100_000, (144, 288), [16, 32, 64, 128], 128, 8, 0.2, 10),
}


def make_workload(name: str, dtype: str = "i16", *, n: Optional[int] = None,
                  n_sensors: Optional[int] = None, mq_per_sensor: Optional[int] = None,
                  k: Optional[int] = None, lengths: Optional[Sequence[int]] = None,
                  window: Optional[int] = None, band: Optional[float] = None,
                  step: int = 0, consecutive: bool = False) -> Workload:
    """Build config `name` (C1..C5), optionally shrunk.

    Master query j of a sensor is tail[off_j : off_j + D].  With
    consecutive=True the offsets are 0,1,2,... (a continuous stream);
    otherwise they are spread over the tail.  `step` shifts every offset (one
    continuous step = one point)."""
    cid, ns, N, periods, lens, kk, w, bd, mqs = CONFIGS[name]
    N = n if n is not None else N
    ns = n_sensors if n_sensors is not None else ns
    mqs = mq_per_sensor if mq_per_sensor is not None else mqs
    kk = k if k is not None else kk
    lens = list(lengths) if lengths is not None else list(lens)
    w = window if window is not None else w
    bd = band if band is not None else bd
    D = lens[-1]
    spread = 1 if consecutive else 7
    # the tail length does not depend on `step`, so every continuous step of a
    # workload sees the same indexed history (noise draws follow the walk's)
    if not 0 <= step < STEP_MAX:
        raise ValueError("step must be in [0, %d)" % STEP_MAX)
    H = D + spread * mqs + STEP_MAX + 1
    parts, queries, qs, tails, qoff = [], [], [], [], []
    offsets = [0]
    for s in range(ns):
        z = sensor_series(cid, s, N, H, periods[s % len(periods)])
        x = quantise(z, dtype)
        parts.append(x[:N])
        offsets.append(offsets[-1] + N)
        tail = x[N:]
        tails.append(tail)
        for j in range(mqs):
            off = spread * j + step
            queries.append(tail[off:off + D])
            qs.append(s)
            qoff.append(off)
    series = np.concatenate(parts)
    return Workload(name=name, dtype=dtype, series=series,
                    offsets=np.asarray(offsets, dtype=np.int64),
                    queries=np.ascontiguousarray(np.stack(queries)),
                    query_sensor=np.asarray(qs, dtype=np.int32),
                    lengths=lens, k=kk, window=w, band=bd, tails=tails,
                    qoff=np.asarray(qoff, dtype=np.int64))


def random_walk_small(seed: int, n: int, dtype: str, lo: int = -40, hi: int = 40) -> np.ndarray:
    """Tiny integer-valued random walks for unit tests (values in [lo, hi])."""
    rng = np.random.Generator(np.random.PCG64(seed))
    x = np.cumsum(rng.integers(-3, 4, size=n))
    x = np.clip(x, lo, hi)
    if dtype == "i16":
        return x.astype(np.int16)
    return (x / 8.0).astype(np.float32)   # dyadic: every f32 op on these is exact (P13)
