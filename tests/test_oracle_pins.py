"""Pins of the oracle against things other than itself (-m "not gpu").

Every oracle function is checked against what the paper or mathematics fixes:
hand-worked values, brute-force enumeration of warping paths, closed forms,
the paper's printed Examples 4.1/4.2, the SURVEY Appendix A golden example,
and the theorems LB_w <= LB_en <= DTW (Thm 4.1, Thm 4.3).
"""
import itertools
import json
import math
import os

import numpy as np
import pytest

import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden", "appendix_a.json")


# --------------------------------------------------------------------------
# Independent DTW by enumerating every warping path (tiny d only).
# A warping path is a contiguous monotone set of cells from (1,1) to (d,d)
# with steps (1,0), (0,1), (1,1) (the three predecessors of
# Eq. 21) staying within the Sakoe-Chiba band |i-j| <= rho.
# --------------------------------------------------------------------------
def dtw_by_paths(q, c, rho):
    d = len(q)
    best = [math.inf]

    def walk(i, j, cost):
        cost += (q[i] - c[j]) ** 2
        if cost >= best[0]:
            return
        if i == d - 1 and j == d - 1:
            best[0] = cost
            return
        for di, dj in ((1, 0), (0, 1), (1, 1)):
            a, b = i + di, j + dj
            if a < d and b < d and abs(a - b) <= rho:
                walk(a, b, cost)

    walk(0, 0, 0)
    return best[0]


HAND = [  # (q, c, rho, DTW) -- SURVEY §8(c) P1, each re-derived by path enumeration below
    ([1, 2, 3], [1, 2, 3], 1, 0),
    ([0, 0, 0], [1, 1, 1], 1, 3),
    ([1, 2, 3, 4], [1, 1, 2, 3], 1, 1),
    ([1, 2, 3, 4], [1, 1, 2, 3], 0, 3),
    ([0, 1, 0, 1], [1, 0, 1, 0], 1, 2),
    ([0, 1, 0, 1], [1, 0, 1, 0], 0, 4),
    ([0, 0, 5, 0, 0], [0, 5, 0, 0, 0], 1, 0),
    ([0, 0, 5, 0, 0], [0, 5, 0, 0, 0], 0, 50),
    ([3, 1, 4, 1, 5], [2, 7, 1, 8, 2], 2, 29),
]


@pytest.mark.parametrize("q,c,rho,val", HAND)
def test_dtw_hand_worked(orc, q, c, rho, val):
    assert dtw_by_paths(q, c, rho) == val            # the worked value itself
    qa, ca = np.array(q, np.int64), np.array(c, np.int64)
    assert orc.dtw(qa, ca, rho) == val
    assert orc.dtw(qa.astype(np.float64), ca.astype(np.float64), rho) == val
    assert orc.dtw(qa.astype(np.float32), ca.astype(np.float32), rho, mode="f32") == val


def test_dtw_equals_path_enumeration(orc):
    rng = np.random.default_rng(7)
    n = 0
    for d in range(1, 7):
        for rho in range(0, d + 1):
            for _ in range(6):
                q = rng.integers(-5, 6, size=d)
                c = rng.integers(-5, 6, size=d)
                assert orc.dtw(q, c, rho) == dtw_by_paths(list(q), list(c), rho), (q, c, rho)
                n += 1
    assert n > 100


def test_dtw_closed_forms_and_invariants(orc):
    rng = np.random.default_rng(11)
    for _ in range(60):
        d = int(rng.integers(1, 40))
        q = rng.integers(-300, 300, size=d)
        c = rng.integers(-300, 300, size=d)
        # rho = 0 reduces to the squared Euclidean distance (Eq. 23 leaves the diagonal)
        assert orc.dtw(q, c, 0) == int(((q - c) ** 2).sum())
        # identity and symmetry (dist symmetric, band symmetric)
        assert orc.dtw(q, q, int(rng.integers(0, d))) == 0
        rho = int(rng.integers(0, d))
        assert orc.dtw(q, c, rho) == orc.dtw(c, q, rho)
        # non-increasing in rho, and rho >= d-1 is unconstrained
        vals = [orc.dtw(q, c, r) for r in range(0, d + 2)]
        assert all(a >= b for a, b in zip(vals, vals[1:]))
        assert vals[d - 1] == vals[d] == vals[d + 1]
        assert min(vals) >= 0


def test_dtw_f32_pinned_vs_f64(orc):
    rng = np.random.default_rng(3)
    for _ in range(40):
        d = int(rng.integers(2, 130))
        rho = int(rng.integers(0, max(1, d // 4) + 1))
        q = rng.normal(size=d).astype(np.float32)
        c = rng.normal(size=d).astype(np.float32)
        a = orc.dtw(q, c, rho, mode="f32")
        b = orc.dtw(q, c, rho, mode="f64")
        assert abs(a - b) <= 1e-5 * max(b, 1e-30)


def test_dyadic_f32_equals_i16_over_64(orc):
    """P13: inputs x/8 with small |x| make every f32 op exact."""
    for seed in range(5):
        xi = synth.random_walk_small(seed, 64, "i16")
        xf = synth.random_walk_small(seed, 64, "f32")
        for d, rho in ((8, 2), (16, 3), (32, 5)):
            q_i, c_i = xi[:d], xi[20:20 + d]
            q_f, c_f = xf[:d], xf[20:20 + d]
            assert orc.dtw(q_f, c_f, rho, mode="f32") * 64 == orc.dtw(q_i, c_i, rho)


# --------------------------------------------------------------------------
# Envelope (Eq. 25) invariants
# --------------------------------------------------------------------------
def test_envelope_invariants(orc):
    rng = np.random.default_rng(5)
    x = rng.integers(-1000, 1000, size=300)
    U0, L0 = orc.envelope(x, 0)
    assert (U0 == x).all() and (L0 == x).all()
    prevU, prevL = U0, L0
    for rho in (1, 2, 5, 17):
        U, L = orc.envelope(x, rho)
        assert (U >= x).all() and (L <= x).all()
        assert (U >= prevU).all() and (L <= prevL).all()     # widening the window
        # each value is attained within the window
        for i in (0, 7, 150, 299):
            lo, hi = max(0, i - rho), min(len(x) - 1, i + rho)
            assert U[i] in x[lo:hi + 1] and L[i] in x[lo:hi + 1]
        prevU, prevL = U, L
    Uc, Lc = orc.envelope(np.full(50, 7), 4)
    assert (Uc == 7).all() and (Lc == 7).all()
    Uf, Lf = orc.envelope(x.astype(np.float32), 3)
    Ui, Li = orc.envelope(x, 3)
    assert (Uf == Ui).all() and (Lf == Li).all()


# --------------------------------------------------------------------------
# Golden example (Fig. 5-shaped)
# --------------------------------------------------------------------------
def test_golden_appendix_a(orc):
    g = json.load(open(GOLD))
    C = np.array(g["C"], np.int64)
    MQ = np.array(g["MQ"], np.int64)
    w, rho, k = g["w"], g["rho"], g["k"]
    UC, LC = orc.envelope(C, rho)
    UQ, LQ = orc.envelope(MQ, rho)
    assert UC.tolist() == g["UC"] and LC.tolist() == g["LC"]
    assert UQ.tolist() == g["UQ"] and LQ.tolist() == g["LQ"]
    PE, PC = orc.postings(C, UC, LC, MQ, UQ, LQ, w)
    assert PE.tolist() == g["P_EQ"] and PC.tolist() == g["P_EC"]
    ids, dists = orc.knn_one(C.astype(np.int16), MQ.astype(np.int16), g["lengths"],
                             [rho] * len(g["lengths"]), k)
    for li, iq in enumerate(g["IQ"]):
        d = iq["d"]
        lb = orc.lower_bounds(C, UC, LC, MQ, UQ, LQ, d, w)
        assert lb["b"].tolist() == iq["b"]
        assert lb["r"].tolist() == iq["r"]
        assert lb["m"].tolist() == iq["m"]
        assert lb["w"].tolist() == iq["LB_w"]
        assert lb["en"].tolist() == iq["LB_en"]
        dt = [orc.dtw(MQ[len(MQ) - d:], C[t:t + d], rho) for t in iq["t"]]
        assert dt == iq["DTW"]
        assert ids[li].tolist() == iq["knn_ids"] and dists[li].tolist() == iq["knn_dists"]
        # R8 tau: verify the k smallest-LB candidates (ties by t), tau = max DTW
        order = sorted(iq["t"], key=lambda t: (iq["LB_w"][t], t))[:k]
        tau = max(iq["DTW"][t] for t in order)
        assert tau == iq["tau_R8"]
        assert sum(1 for t in iq["t"] if iq["LB_w"][t] <= tau) == iq["verified"]


# --------------------------------------------------------------------------
# Index arithmetic: Example 4.1 / 4.2, Lemma 4.1 (Eq. 4), Thm 4.2, Eq. 5
# --------------------------------------------------------------------------
def test_example_4_1_and_4_2(orc):
    w, D = 3, 9
    n_sw = D - w + 1
    csg = {b: [b + j * w for j in range(n_sw) if b + j * w < n_sw] for b in range(w)}
    assert csg == {0: [0, 3, 6], 1: [1, 4], 2: [2, 5]}              # Example 4.1
    d0 = 6   # IQ0
    # CSG_{0,b} = prefix of CSG_b that fits in IQ0: floor((d0-b)/w) windows
    pref = {b: csg[b][:(d0 - b) // w] for b in range(w)}
    assert pref == {0: [0, 3], 1: [1], 2: [2]}                       # Example 4.1
    # Example 4.2: (SW0,DW3)+(SW3,DW2) -> C_{6,6}; +(SW6,DW1) -> C_{3,9}
    C = np.zeros(12, np.int64)
    MQ = np.zeros(9, np.int64)
    lb6 = orc.lower_bounds(C, C, C, MQ, MQ, MQ, 6, w)
    lb9 = orc.lower_bounds(C, C, C, MQ, MQ, MQ, 9, w)
    assert (lb6["b"][6], lb6["r"][6], lb6["m"][6]) == (0, 3, 2)
    assert (lb9["b"][3], lb9["r"][3], lb9["m"][3]) == (0, 3, 3)
    # Eq. 4 gives back the same t
    for d, t, lb in ((6, 6, lb6), (9, 3, lb9)):
        b, r, m = lb["b"][t], lb["r"][t], lb["m"][t]
        assert (r - m + 1) * w - (d - b) % w == t


@pytest.mark.parametrize("n,w,d,uncovered", [(4096, 16, 32, 0), (1000, 16, 16, 923),
                                             (1000, 8, 16, 0), (97, 5, 23, 0)])
def test_eq4_bijection(orc, n, w, d, uncovered):
    """Thm 4.2: each t with >= 1 full DW has exactly one (b, r); Eq. 4 inverts it."""
    z = np.zeros(n, np.int64)
    D = d
    lb = orc.lower_bounds(z, z, z, np.zeros(D, np.int64), np.zeros(D, np.int64),
                          np.zeros(D, np.int64), d, w)
    seen = set()
    unc = 0
    for t in range(n - d + 1):
        b, r, m = int(lb["b"][t]), int(lb["r"][t]), int(lb["m"][t])
        if m < 1:
            unc += 1
            continue
        assert 0 <= b < w and 0 <= r < n // w
        assert m == (d - b) // w                    # |CSG_{i,b}| = floor((d-b)/w)
        assert (r - m + 1) * w - (d - b) % w == t    # Eq. 4
        assert (b, r) not in seen
        seen.add((b, r))
    assert unc == uncovered


def test_lbw_equals_csg_shift_sum(orc):
    """Eq. 5: LB_w(IQ_i, C_t) = max(sum_j P_EQ[b+jw][r-j], sum_j P_EC[...]) -- the
    oracle's LB_w (from point terms, indexed by t) against its postings (by (b,r))."""
    rng = np.random.default_rng(21)
    for trial in range(6):
        w = int(rng.integers(2, 9))
        D = int(rng.integers(2 * w, 6 * w))
        n = int(rng.integers(D + 10, 400))
        rho = int(rng.integers(0, 5))
        c = rng.integers(-200, 200, size=n)
        mq = rng.integers(-200, 200, size=D)
        UC, LC = orc.envelope(c, rho)
        UQ, LQ = orc.envelope(mq, rho)
        PE, PC = orc.postings(c, UC, LC, mq, UQ, LQ, w)
        for d in sorted({D, max(w, D // 2), D - 1}):
            lb = orc.lower_bounds(c, UC, LC, mq, UQ, LQ, d, w)
            for t in range(n - d + 1):
                b, r, m = lb["b"][t], lb["r"][t], lb["m"][t]
                if m < 1:
                    assert lb["w"][t] == 0
                    continue
                se = sum(PE[b + j * w][r - j] for j in range(m))
                sc = sum(PC[b + j * w][r - j] for j in range(m))
                assert lb["w"][t] == max(se, sc)


def test_lb_chain_invariant(orc):
    """Thm 4.1 and Thm 4.3 (and its proof): LB_w <= LB_en <= DTW."""
    rng = np.random.default_rng(99)
    checked = 0
    for trial in range(10):
        w = int(rng.integers(2, 9))
        lengths = sorted(set(int(x) for x in rng.integers(w, 4 * w, size=3)))
        D = lengths[-1]
        n = 300
        rhos = [int(rng.integers(0, 6)) for _ in lengths]
        x = synth.random_walk_small(trial, n + D, "i16", -300, 300).astype(np.int64)
        c, mq = x[:n], x[n:]
        res, (UC, LC, UQ, LQ, rho_env) = orc.mq_lower_bounds(c, mq, lengths, rhos, w)
        for d, rho, lb in zip(lengths, rhos, res):
            for t in range(n - d + 1):
                dt = orc.dtw(mq[D - d:], c[t:t + d], rho)
                assert lb["w"][t] <= lb["en"][t] <= dt
                assert lb["eq"][t] <= dt and lb["ec"][t] <= dt
                checked += 1
    assert checked > 2000


def test_tight_lb_constant_series(orc):
    """P12: c == a, q == b: DTW = LB_EQ = LB_EC = LB_en = d (a-b)^2, LB_w = m w (a-b)^2."""
    a, bq, w, rho = 5, -3, 4, 2
    n, d = 64, 16
    c = np.full(n, a, np.int64)
    mq = np.full(d, bq, np.int64)
    UC, LC = orc.envelope(c, rho)
    UQ, LQ = orc.envelope(mq, rho)
    lb = orc.lower_bounds(c, UC, LC, mq, UQ, LQ, d, w)
    for t in range(n - d + 1):
        full = d * (a - bq) ** 2
        assert orc.dtw(mq, c[t:t + d], rho) == full
        assert lb["eq"][t] == lb["ec"][t] == lb["en"][t] == full
        assert lb["w"][t] == lb["m"][t] * w * (a - bq) ** 2
        if t % w == 0:
            assert lb["w"][t] == full


# --------------------------------------------------------------------------
# kNN = the definition (Def. 4.1), checked against path-enumeration DTW
# --------------------------------------------------------------------------
def test_knn_brute_force_tiny(orc):
    rng = np.random.default_rng(1234)
    for trial in range(4):
        n = 30
        series = rng.integers(-4, 5, size=n).astype(np.int16)   # many ties on purpose
        mq = rng.integers(-4, 5, size=6).astype(np.int16)
        lengths, rhos, k = [3, 5, 6], [1, 2, 1], 7
        ids, dists = orc.knn_one(series, mq, lengths, rhos, k)
        for li, (d, rho) in enumerate(zip(lengths, rhos)):
            iq = [int(v) for v in mq[6 - d:]]
            allk = sorted((dtw_by_paths(iq, [int(v) for v in series[t:t + d]], rho), t)
                          for t in range(n - d + 1))[:k]
            assert ids[li].tolist() == [t for _, t in allk]
            assert dists[li].tolist() == [v for v, _ in allk]


def test_knn_padding(orc):
    series = np.arange(10, dtype=np.int16)
    mq = np.arange(8, dtype=np.int16)
    ids, dists = orc.knn_one(series, mq, [8], [1], 5)
    assert ids[0].tolist()[:3] == [0, 1, 2] and ids[0].tolist()[3:] == [-1, -1]
    assert dists[0].tolist()[3:] == [2 ** 31 - 1] * 2
    idsf, distsf = orc.knn_one(series.astype(np.float32), mq.astype(np.float32), [8], [1], 5)
    assert idsf[0].tolist() == ids[0].tolist() and np.isinf(distsf[0][3:]).all()


def test_knn_prefix_property(orc):
    """Multi-k by prefix: the k1 < k2 result is the prefix."""
    wl = synth.make_workload("C1", "i16", n=600)
    rh = wl.rhos()
    a, da = orc.knn_one(wl.series, wl.queries[0], wl.lengths, rh, 3)
    b, db = orc.knn_one(wl.series, wl.queries[0], wl.lengths, rh, 8)
    assert (a == b[:, :3]).all() and (da == db[:, :3]).all()


def test_knn_f32_modes_agree(orc):
    wl = synth.make_workload("C1", "f32", n=800)
    rh = wl.rhos()
    i32, d32 = orc.knn_one(wl.series, wl.queries[0], wl.lengths, rh, wl.k, mode="f32")
    i64, d64 = orc.knn_one(wl.series, wl.queries[0], wl.lengths, rh, wl.k, mode="f64")
    assert np.allclose(d32, d64, rtol=1e-5, atol=0)
    assert (i32 == i64).all()


def test_int32_certificate_bound():
    """R17: |x| <= 1023 -> every DTW <= 2046^2 (2d-1) < 2^31 for d <= 256."""
    assert 2046 ** 2 * (2 * 256 - 1) < 2 ** 31
    # and every LB sum (<= d terms of at most 2046^2) too
    assert 256 * 2046 ** 2 < 2 ** 31


def test_generator_is_seeded_and_shaped():
    a = synth.make_workload("C2", "i16", n=5000, mq_per_sensor=4)
    b = synth.make_workload("C2", "i16", n=5000, mq_per_sensor=4)
    assert (a.series == b.series).all() and (a.queries == b.queries).all()
    assert a.series.dtype == np.int16 and np.abs(a.series).max() <= 1023
    assert a.queries.shape == (4, 128) and a.rhos() == [1, 3, 6, 12]
    c5 = synth.make_workload("C5", "f32", n=3000, n_sensors=3, mq_per_sensor=2)
    assert c5.rhos() == [3, 6, 12, 25] and c5.n_mq == 6
    z = synth.sensor_series(2, 0, 10000, 100, 144)
    assert abs(z[:10000].mean()) < 1e-9 and abs(z[:10000].std() - 1) < 1e-9


# --------------------------------------------------------------------------
# P13 pins of the oracle's FLOAT paths: inputs x/8 (x small integers) make every
# f32 / f64 operation of the oracle exact, so each float function must equal
# its integer twin divided by 64 exactly -- and the integer twins are pinned
# above (golden example, Eq. 5 shift sums, path enumeration).  A dropped term,
# a wrong sign or index, a transposed operand or a wrong suffix offset in a
# float function breaks the equality.
# --------------------------------------------------------------------------
def _dyadic_cases():
    g = json.load(open(GOLD))
    yield np.array(g["C"], np.int64), np.array(g["MQ"], np.int64), g["w"], g["rho"], [iq["d"] for iq in g["IQ"]]
    rng = np.random.default_rng(1313)
    for seed in range(4):
        w = int(rng.integers(2, 9))
        lengths = sorted(set(int(x) for x in rng.integers(w, 5 * w, size=3)))
        D = lengths[-1]
        n = int(rng.integers(D + 20, 260))
        x = synth.random_walk_small(100 + seed, n + D, "i16", -40, 40).astype(np.int64)
        yield x[:n], x[n:], w, int(rng.integers(0, 6)), lengths


def test_postings_f64_equals_i64_over_64_dyadic(orc):
    """orc_postings_f64 on x/8 inputs == orc_postings_i64 / 64."""
    for c, mq, w, rho, _ in _dyadic_cases():
        UC, LC = orc.envelope(c, rho)
        UQ, LQ = orc.envelope(mq, rho)
        PE, PC = orc.postings(c, UC, LC, mq, UQ, LQ, w)
        f = lambda a: np.asarray(a, np.float64) / 8.0
        FE, FC = orc.postings(f(c), f(UC), f(LC), f(mq), f(UQ), f(LQ), w)
        assert FE.dtype == np.float64
        np.testing.assert_array_equal(FE * 64.0, PE.astype(np.float64))
        np.testing.assert_array_equal(FC * 64.0, PC.astype(np.float64))
        assert PE.any() and PC.any()          # not a vacuous all-zero case


def test_lb_f64_equals_i64_over_64_dyadic(orc):
    """orc_lb_f64 (LB_EQ, LB_EC, LB_en of Thm 4.1; LB_w and its two sums of
    Thm 4.3 / Eq. 5) on x/8 inputs == orc_lb_i64 / 64, for every t and d."""
    for c, mq, w, rho, lengths in _dyadic_cases():
        UC, LC = orc.envelope(c, rho)
        UQ, LQ = orc.envelope(mq, rho)
        f = lambda a: np.asarray(a, np.float64) / 8.0
        for d in lengths:
            li = orc.lower_bounds(c, UC, LC, mq, UQ, LQ, d, w)
            lf = orc.lower_bounds(f(c), f(UC), f(LC), f(mq), f(UQ), f(LQ), d, w)
            for key in ("eq", "ec", "en", "w", "weq", "wec"):
                np.testing.assert_array_equal(lf[key] * 64.0, li[key].astype(np.float64), err_msg=key)
            assert li["w"].any()
            if rho > 0:   # rho = 0: U = L = the series, so both sums are sum (q - c)^2
                assert (li["weq"] != li["wec"]).any()


@pytest.mark.parametrize("mode", ["f32", "f64"])
def test_knn_float_suffix_offsets_dyadic(orc, mode):
    """orc_knn_f32 / orc_knn_f64 with item queries SHORTER than the MQ
    (lengths [3, 5, 6], D = 6: IQ_i = the last d_i points) on x/8
    inputs == orc_knn_i16 / 64 == the kNN of path-enumeration DTWs / 64."""
    for trial in range(4):
        rng = np.random.default_rng(600 + trial)
        n = 40
        xi = rng.integers(-30, 31, size=n + 6)
        series_i, mq_i = xi[:n].astype(np.int16), xi[n:].astype(np.int16)
        series_f, mq_f = (series_i / 8.0).astype(np.float32), (mq_i / 8.0).astype(np.float32)
        lengths, rhos, k = [3, 5, 6], [1, 2, 1], 9
        ids_i, d_i = orc.knn_one(series_i, mq_i, lengths, rhos, k)
        ids_f, d_f = orc.knn_one(series_f, mq_f, lengths, rhos, k, mode=mode)
        np.testing.assert_array_equal(ids_f, ids_i)
        np.testing.assert_array_equal(d_f.astype(np.float64) * 64.0, d_i.astype(np.float64))
        for li, (d, rho) in enumerate(zip(lengths, rhos)):
            iq = [int(v) for v in mq_i[6 - d:]]
            allk = sorted((dtw_by_paths(iq, [int(v) for v in series_i[t:t + d]], rho), t)
                          for t in range(n - d + 1))[:k]
            assert ids_f[li].tolist() == [t for _, t in allk]
            assert (d_f[li].astype(np.float64) * 64.0).tolist() == [float(v) for v, _ in allk]


@pytest.mark.parametrize("mode", ["f32", "f64"])
def test_knn_float_owned_range_dyadic(orc, mode):
    """The t_lo / t_hi candidate window of orc_knn_f32/f64 (window-range shards,
    R24) equals brute force restricted to that window."""
    xi = synth.random_walk_small(77, 300, "i16", -40, 40)
    xf = synth.random_walk_small(77, 300, "f32", -40, 40)
    lengths, rhos, k = [8, 13], [2, 3], 6
    for t_lo, t_hi in ((0, 250), (17, 120), (100, 101)):
        ids_i, d_i = orc.knn_one(xi[:250], xi[250:263], lengths, rhos, k, t_lo=t_lo, t_hi=t_hi)
        ids_f, d_f = orc.knn_one(xf[:250], xf[250:263], lengths, rhos, k, mode=mode, t_lo=t_lo, t_hi=t_hi)
        np.testing.assert_array_equal(ids_f, ids_i)
        fin = ids_i >= 0
        np.testing.assert_array_equal(d_f[fin].astype(np.float64) * 64.0, d_i[fin].astype(np.float64))
        assert np.isinf(d_f[~fin]).all()
        assert ((ids_i[fin] >= t_lo) & (ids_i[fin] < t_hi)).all()
