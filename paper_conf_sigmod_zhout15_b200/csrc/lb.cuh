// lb.cuh -- steps a3/a4 of the Search Step: the SMiLer Index lower bounds.
// Included by kernels.cuh.
//
// Notation (Sec. 4.3): w = omega, n_sw = D - w + 1 sliding windows
// SW_b = MQ[D-w-b .. D-b) (R19), n_dw = floor(N/w) disjoint windows
// DW_r = c[rw .. rw+w).  Posting element (window level):
//   P_EQ[b][r] = sum_j e(c[rw+j]; U(Q), L(Q) at D-w-b+j)
//   P_EC[b][r] = sum_j e(MQ[D-w-b+j]; U(C), L(C) at rw+j)
// Group level (Alg. 1, garbles fixed per R5; Thm 4.3 / Eq. 5):
//   for CSG_b (b < w) and rightmost DW r, the running sums over j of
//   P[b + j w][r - j] give LB_w(IQ_i, C_t) = max(S_EQ, S_EC) as soon as
//   j + 1 = m_i(b) = floor((d_i - b)/w), at t = (r - j) w - (d_i - b) % w (Eq. 4).
// Both the right end e = t + d_i = (r+1) w + b and the tile slot
// (r - Rb) w + b are independent of i, so one CTA buffers the LB_w of a run
// of consecutive r in shared memory and writes each IQ's t range coalesced.
//
// Three kernels:
//   window_lb_kernel  (a3) posting lists -> HBM          [two-level path]
//   group_scan_kernel (a4) HBM posting lists -> LB_w     [two-level path, HBM-bound]
//   lb_fused_kernel   (a3+a4) one CSG row of posting lists at a time lives in
//                     shared memory; nothing but LB_w goes to HBM [one-shot path]
#pragma once
// (included inside namespace smiler by kernels.cuh)

// Build-time A/B switches (tools/build_variants.sh)
#ifndef SMILER_LB_FOLD
#define SMILER_LB_FOLD 1
#endif
#ifndef SMILER_DIAG_UNROLL2
#define SMILER_DIAG_UNROLL2 0
#endif
#ifndef SMILER_DIAG_SPLIT2
#define SMILER_DIAG_SPLIT2 1  // lb_diag w = 16: local chunk sums + one uniform branch instead of slot rotation
#endif
#ifndef SMILER_INC_X2
#define SMILER_INC_X2 1  // f32 continuous-step EQ rows with fp32x2-packed terms (posting_chunk_eq_x2)
#endif
#ifndef SMILER_INC_TILES
#define SMILER_INC_TILES 4  // 128-DW tiles per CTA of the incremental a3 kernel (1: 7.79 ms, 4: 7.00 ms on C5)
#endif
#ifndef SMILER_TMA_SYNC2
#define SMILER_TMA_SYNC2 1  // TMA ring scan: one CTA barrier per two CSG rows
#endif
#ifndef SMILER_DIAG_MINB8
#define SMILER_DIAG_MINB8 6  // lb_diag CTAs per SM for w <= 8 (80 registers, no spills; 5: -0.4%, 4: -3%, 7: -5%)
#endif
#ifndef SMILER_TAU_PACKED
#define SMILER_TAU_PACKED 1  // tau-set keys: LB_w bits with the slot in the low bits
#endif
#ifndef SMILER_EXPERIMENTS
#define SMILER_EXPERIMENTS 0  // 1: timing-only switches (smiler_knn_opts.reserved != 0, results invalid)
#endif
#ifndef SMILER_TMA_EMPTYBAR
#define SMILER_TMA_EMPTYBAR 0  // 1: stages freed by per-warp arrivals, thread 0 waits (measured slower; so
                               // was the last warp to finish a stage refilling it: C5 scan 13.96 -> 17.3 ms)
#endif

// The bound of a candidate from its EQ and EC sums: LB = max(EQ, EC) (Eq. 5,
// Thm 4.1), or one of the two sums alone (the Table 3 ablation).
template <typename V> __device__ __forceinline__ V lbpick(const QParams &P, V eq, V ec) {
    return P.lbsel == 0 ? vmax(eq, ec) : (P.lbsel == 1 ? eq : ec);
}

// CTAs past an MQ's last tile (grids are sized for the longest sensor of the
// chunk) still own tau-list slots: mark them empty (-1) so the tau DTW pass
// never reads a stale t from an earlier call.
__device__ __forceinline__ void tau_clear(const QParams &P, int mq, int units_per_blk, int li0, int li1,
                                          int32_t *tauc, int bx = -1) {
    if (P.E <= 0 || P.k < 0) return;
    const int n = units_per_blk * P.E;
    const int64_t tile = bx >= 0 ? bx : (int)blockIdx.x;
    for (int i = li0; i < li1; i++) {
        int32_t *dst = tauc + (int64_t)(mq * P.n_len + i) * P.LT + tile * n;
        for (int x = threadIdx.x; x < n; x += blockDim.x) dst[x] = -1;
    }
}

// Posting storage.  PV = V keeps the window-level postings exact; PV = __half
// (continuous f32 streams) stores each P_EQ / P_EC rounded toward zero, i.e.
// never above its value (saturating at 65504): a sum of such entries is still
// a lower bound of LB_w, hence of DTW (Thm 4.3), so filtering stays exact while
// the ring -- the bytes the group scan streams every step -- halves.
template <typename PV, typename V> __device__ __forceinline__ void post_st(PV *p, V v, float) { *p = v; }
// fp16 ring: the entry times the stream batch's power-of-two scale (exact),
// rounded toward zero (never above; saturates at 65504, still a lower bound)
template <> __device__ __forceinline__ void post_st<__half, float>(__half *p, float v, float sc) {
    *p = __float2half_rz(v * sc);
}
template <typename V, typename PV> __device__ __forceinline__ V post_cv(PV x) { return x; }
template <> __device__ __forceinline__ float post_cv<float, __half>(__half x) { return __half2float(x); }
// acc += posting entry.  fp16 entries into f32 sums use sm_100's mixed-precision
// add (PTX add.rn.f32.f16, one FHADD): the fp16 -> f32 conversion is exact, so
// the result is bit-identical to converting first and adding in f32.
template <typename V, typename PV> __device__ __forceinline__ void post_acc(V &acc, PV x) { acc += post_cv<V>(x); }
template <> __device__ __forceinline__ void post_acc<float, __half>(float &acc, __half x) {
    float r;
    asm("add.rn.f32.f16 %0, %1, %2;" : "=f"(r) : "h"(__half_as_ushort(x)), "f"(acc));
    acc = r;
}

// emission table: em[j*w + b] = lo | hi << 8, the IQ range [lo, hi) with
// m_i(b) == j + 1 (contiguous in i because d_i increases).
__device__ __forceinline__ void build_emit_table(uint16_t *em, int mmax, int w, const QParams &P) {
    for (int x = threadIdx.x; x < mmax * w; x += blockDim.x) {
        const int j = x / w, b = x % w;
        int lo = 0, hi = 0;
        while (lo < P.n_len && P.len[lo] - b < (j + 1) * w) lo++;
        hi = lo;
        while (hi < P.n_len && P.len[hi] - b < (j + 2) * w) hi++;
        em[x] = (uint16_t)(lo | (hi << 8));
    }
}

// Write a CTA's LB_w tile (slot s <-> e = e0 + s, padded to w+1 per row) to
// lb[mq][i][t] and emit the tau set (E smallest (LB_w, t) per IQ) of the tile.
// The first selection round is folded into the write-out pass.
template <typename V, int W>
__device__ void lb_tile_epilogue(V *tile, int RT, int64_t e0, const MQMeta &m, const QParams &P, V *lb,
                                 int32_t *tauc, int mq, uint64_t *s_red) {
    const int w = W > 0 ? W : P.w;
    const int nl = P.n_len;
    const int stride = RT * (w + 1);
    const int64_t tmin = m.t_lo > 0 ? m.t_lo : 0;
    for (int i = 0; i < nl; i++) {
        const int d = P.len[i];
        const int64_t tend = min(m.t_hi, m.n - m.hz - d + 1);
        V *out = lb + m.seg_off + (int64_t)i * m.n;
        V *row = tile + i * stride;
        uint64_t best = kKeyMax;
        int bs = -1;
        for (int s = threadIdx.x; s < RT * w; s += blockDim.x) {
            const int64_t t = e0 + s - d;
            const int slot = (s / w) * (w + 1) + (s % w);
            if (t >= tmin && t < tend) {
                const V v = row[slot];
                out[t] = v;
                const uint64_t key = ((uint64_t)key_bits(v) << 32) | (uint32_t)t;
                if (key < best) {
                    best = key;
                    bs = slot;
                }
            }
        }
        if (P.E <= 0) continue;
        int32_t *dst = tauc + (int64_t)(mq * nl + i) * P.LT + (int64_t)blockIdx.x * P.E;
        for (int e = 0; e < P.E; e++) {
            if (e > 0) {  // later rounds rescan the thread's slots
                best = kKeyMax;
                bs = -1;
                for (int s = threadIdx.x; s < RT * w; s += blockDim.x) {
                    const int64_t t = e0 + s - d;
                    const int slot = (s / w) * (w + 1) + (s % w);
                    const uint32_t kb = key_bits(row[slot]);
                    if (t >= tmin && t < tend && kb != 0xFFFFFFFFu) {
                        const uint64_t key = ((uint64_t)kb << 32) | (uint32_t)t;
                        if (key < best) {
                            best = key;
                            bs = slot;
                        }
                    }
                }
            }
            const uint64_t win = block_min_u64(best, s_red);
            if (win != kKeyMax && best == win) {  // unique: keys carry t
                uint32_t allones = 0xFFFFFFFFu;   // "taken": not a valid LB >= 0
                row[bs] = *reinterpret_cast<V *>(&allones);
            }
            if (threadIdx.x == 0) {
                dst[e] = win != kKeyMax ? (int32_t)(uint32_t)win : -1;
                if (P.taulb) P.taulb[dst - tauc + e] = (uint32_t)(win >> 32);
            }
            __syncthreads();
        }
    }
}

// Barrier-free epilogue for tiles whose row x is written only by thread x
// (lb_diag_kernel): every thread writes its own W slots (t contiguous) and
// the tau set is chosen per warp (E smallest (LB_w, t) among the warp's slots,
// by warp-shuffle minima).  tauc slot: (mq, i) row, [blockIdx.x * NW + warp] * E + e.
template <typename V, int W>
__device__ void lb_tile_epilogue_warp(V *tile, int RT, int64_t e0, const MQMeta &m, const QParams &P, V *lb,
                                      int32_t *tauc, int mq) {
    const int nl = P.n_len;
    const int stride = RT * (W + 1);
    const int x = threadIdx.x, lane = x & 31, warp = x >> 5, nw = blockDim.x >> 5;
    const int64_t tmin = m.t_lo > 0 ? m.t_lo : 0;
    const int64_t s0 = e0 + (int64_t)x * W;  // e of this thread's slot 0
    for (int i = 0; i < nl; i++) {
        const int d = P.len[i];
        const int64_t tend = min(m.t_hi, m.n - m.hz - d + 1);
        V *out = lb + m.seg_off + (int64_t)i * m.n;
        V *row = tile + i * stride + x * (W + 1);
        uint64_t best = kKeyMax;
        int bs = -1;
#pragma unroll
        for (int b = 0; b < W; b++) {
            const int64_t t = s0 + b - d;
            if (t >= tmin && t < tend) {
                const V v = row[b];
                out[t] = v;
                const uint64_t key = ((uint64_t)key_bits(v) << 32) | (uint32_t)t;
                if (key < best) {
                    best = key;
                    bs = b;
                }
            }
        }
        if (P.E <= 0) continue;
        int32_t *dst = tauc + (int64_t)(mq * nl + i) * P.LT + ((int64_t)blockIdx.x * nw + warp) * P.E;
        for (int e = 0; e < P.E; e++) {
            if (e > 0) {
                best = kKeyMax;
                bs = -1;
#pragma unroll
                for (int b = 0; b < W; b++) {
                    const int64_t t = s0 + b - d;
                    const uint32_t kb = key_bits(row[b]);
                    if (t >= tmin && t < tend && kb != 0xFFFFFFFFu) {
                        const uint64_t key = ((uint64_t)kb << 32) | (uint32_t)t;
                        if (key < best) {
                            best = key;
                            bs = b;
                        }
                    }
                }
            }
            const uint64_t win = warp_min_u64(best);
            if (win != kKeyMax && best == win) {
                uint32_t allones = 0xFFFFFFFFu;
                row[bs] = *reinterpret_cast<V *>(&allones);
            }
            if (lane == 0) {
                dst[e] = win != kKeyMax ? (int32_t)(uint32_t)win : -1;
                if (P.taulb) P.taulb[dst - tauc + e] = (uint32_t)(win >> 32);
            }
        }
    }
}

// Posting elements of one chunk from a preloaded window (see posting_chunk).
template <typename V, int W, int BC, bool CHECK, int WL, typename F>
__device__ __forceinline__ void posting_chunk_w(const V (&c)[W], const V (&U)[W], const V (&L)[W], const V (&wq)[WL],
                                                const V (&wu)[WL], const V (&wl)[WL], int nvalid, F &&store) {
#pragma unroll
    for (int bb = 0; bb < BC; bb++) {
        if (!CHECK || bb < nvalid) {
            V eq = (V)0, ec = (V)0;
#pragma unroll
            for (int j = 0; j < W; j++) {
                const int k = BC - 1 - bb + j;
                lb_term(c[j], wu[k], wl[k], eq);
                lb_term(wq[k], U[j], L[j], ec);
            }
            store(bb, eq, ec);
        }
    }
}

// posting_chunk_w with the terms accumulated straight into the running CSG
// sums (se/sc slot bb): LB_w is the same sum of the same terms (Eq. 5 summed
// over the CSG's postings), one add per posting element shorter.  f32 rounding
// differs only in association; the filter's slack covers any order (R16).
template <typename V, int W, int BC, int WL, int NS>
__device__ __forceinline__ void posting_chunk_w_fold(const V (&c)[W], const V (&U)[W], const V (&L)[W],
                                                     const V (&wq)[WL], const V (&wu)[WL], const V (&wl)[WL],
                                                     V (&se)[NS], V (&sc)[NS]) {
#pragma unroll
    for (int bb = 0; bb < BC; bb++) {
#pragma unroll
        for (int j = 0; j < W; j++) {
            const int k = BC - 1 - bb + j;
            lb_term(c[j], wu[k], wl[k], se[bb]);
            lb_term(wq[k], U[j], L[j], sc[bb]);
        }
    }
}

// One sliding-window chunk of posting elements: SW_{b0+bb} (bb < BC) against
// the thread's DW (c, U, L).  Window registers hold MQ positions
// pb .. pb + W + BC - 2 (pb = D - W - b0 - (BC-1)): q, U(Q), L(Q).
// CHECK: per-bb validity test (only for the last chunk of a CSG row).
template <typename V, int W, int BC, bool CHECK, bool EQONLY = false, typename F>
__device__ __forceinline__ void posting_chunk(const V (&c)[W], const V (&U)[W], const V (&L)[W],
                                              const V *qq, const V *uq, const V *lq, int pb, int nvalid,
                                              F &&store) {
    V wq[W + BC - 1], wu[W + BC - 1], wl[W + BC - 1];
    if (CHECK) {
#pragma unroll
        for (int k = 0; k < W + BC - 1; k++) {
            const int p = max(pb + k, 0);
            wq[k] = qq[p];
            wu[k] = uq[p];
            wl[k] = lq[p];
        }
    } else {  // every position of a full chunk is >= 0: base + immediate offsets
        const V *q0 = qq + pb, *u0 = uq + pb, *l0 = lq + pb;
#pragma unroll
        for (int k = 0; k < W + BC - 1; k++) {
            wq[k] = q0[k];
            wu[k] = u0[k];
            wl[k] = l0[k];
        }
    }
#pragma unroll
    for (int bb = 0; bb < BC; bb++) {
        if (!CHECK || bb < nvalid) {
            V eq = (V)0, ec = (V)0;
#pragma unroll
            for (int j = 0; j < W; j++) {
                const int k = BC - 1 - bb + j;
                lb_term(c[j], wu[k], wl[k], eq);
                if constexpr (!EQONLY) lb_term(wq[k], U[j], L[j], ec);
            }
            store(bb, eq, ec);
        }
    }
}

// ---------------------------------------------------------------------------
// a3: window-level posting lists.  Thread <-> DW r (its w points and envelope
// in registers).  The b loop runs in chunks of BC sliding windows; consecutive
// SWs overlap in w-1 positions, so one chunk needs w+BC-1 MQ positions
// {q, U(Q), L(Q)} loaded once into registers (no shared-memory load per term).
// 8 ALU ops per (b, r, j) term pair.  Output post[mq][b][r] = {P_EQ, P_EC}.
// One disjoint window (w consecutive points of the series or an envelope) into
// registers: 16-byte vector loads when the window is 16-byte aligned (sensors
// start on 64-element boundaries, so every DW of w >= 4 f32 / w >= 8 i16 is).
template <typename S, typename V, int W>
__device__ __forceinline__ void load_dw(const S *p, V (&o)[W]) {
    if constexpr (std::is_same<S, float>::value && W % 4 == 0) {
        if ((reinterpret_cast<uintptr_t>(p) & 15) == 0) {
#pragma unroll
            for (int q = 0; q < W / 4; q++) {
                const float4 v = __ldg(reinterpret_cast<const float4 *>(p) + q);
                o[4 * q] = v.x, o[4 * q + 1] = v.y, o[4 * q + 2] = v.z, o[4 * q + 3] = v.w;
            }
            return;
        }
    } else if constexpr (std::is_same<S, int16_t>::value && W % 8 == 0) {
        if ((reinterpret_cast<uintptr_t>(p) & 15) == 0) {
#pragma unroll
            for (int q = 0; q < W / 8; q++) {
                const int4 v = __ldg(reinterpret_cast<const int4 *>(p) + q);
                const int32_t wv[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                for (int h = 0; h < 4; h++) {
                    o[8 * q + 2 * h] = (V)(int16_t)(wv[h] & 0xFFFF);
                    o[8 * q + 2 * h + 1] = (V)(int16_t)(wv[h] >> 16);
                }
            }
            return;
        }
    }
#pragma unroll
    for (int j = 0; j < W; j++) o[j] = (V)p[j];
}

// ---------------------------------------------------------------------------
template <typename S, int W, typename PV = typename Tr<S>::V>
__global__ void __launch_bounds__(128) window_lb_kernel(const S *series, const S *UC, const S *LC,
                                                       const MQMeta *meta,
                                                       const typename Tr<S>::V4 *qtab, int D,
                                                       int w_rt, PV *post, float pscale) {
    using V = typename Tr<S>::V;
    extern __shared__ __align__(16) unsigned char wl_smem[];
    V *sqq = reinterpret_cast<V *>(wl_smem);
    V *squ = sqq + D;
    V *sql = squ + D;
    const int mq = blockIdx.y;
    const MQMeta m = meta[mq];
    if ((int64_t)blockIdx.x * blockDim.x >= m.n_dw) return;
    for (int p = threadIdx.x; p < D; p += blockDim.x) {
        const typename Tr<S>::V4 e = qtab[(int64_t)mq * D + p];
        sqq[p] = e.x;
        squ[p] = e.y;
        sql[p] = e.z;
    }
    __syncthreads();
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= m.n_dw) return;
    const int64_t ndw = m.n_dw;
    PV *oe = post + m.post_off + r;  // P_EQ plane; P_EC plane `plane` further
    const int64_t pst = m.pstride;
    if constexpr (W > 0) {
        constexpr int BC = W < 8 ? W : 8;
        const int n_sw = D - W + 1;
        const int64_t plane = (int64_t)m.prows * pst;
        const int nmir = m.prows - n_sw;  // mirrored leading rows (TMA ring)
        const int64_t base = m.series_off + r * W;
        V c[W], U[W], L[W];
        load_dw<S, V, W>(series + base, c);
        load_dw<S, V, W>(UC + base, U);
        load_dw<S, V, W>(LC + base, L);
        int b0 = 0;
        auto put = [&](int b, V eq, V ec) {  // ring cursor 0 at a full build: row b
            PV *o = oe + (int64_t)b * pst;
            post_st(o, eq, pscale);
            post_st(o + plane, ec, pscale);
            if (b < nmir) {
                post_st(o + (int64_t)n_sw * pst, eq, pscale);
                post_st(o + (int64_t)n_sw * pst + plane, ec, pscale);
            }
        };
        for (; b0 + BC <= n_sw; b0 += BC)
            posting_chunk<V, W, BC, false>(c, U, L, sqq, squ, sql, D - W - b0 - (BC - 1), BC,
                                           [&](int bb, V eq, V ec) { put(b0 + bb, eq, ec); });
        if (b0 < n_sw)
            posting_chunk<V, W, BC, true>(c, U, L, sqq, squ, sql, D - W - b0 - (BC - 1), n_sw - b0,
                                          [&](int bb, V eq, V ec) { put(b0 + bb, eq, ec); });
    } else {
        const int w = w_rt;
        const int n_sw = D - w + 1;
        const int64_t plane = (int64_t)m.prows * pst;
        const int64_t base = m.series_off + r * w;
        for (int b = 0; b < n_sw; b++) {
            const int p0 = D - w - b;
            V eq = (V)0, ec = (V)0;
            for (int j = 0; j < w; j++) {
                lb_term((V)series[base + j], squ[p0 + j], sql[p0 + j], eq);
                lb_term(sqq[p0 + j], (V)UC[base + j], (V)LC[base + j], ec);
            }
            post_st(oe + (int64_t)b * pst, eq, pscale);
            post_st(oe + (int64_t)b * pst + plane, ec, pscale);
        }
    }
}

// EQ-only chunk of the continuous step, f32, with fp32x2-packed terms: slots
// (bb, bb+1) of one DW point j are MQ positions p and p-1 (consecutive SWs
// overlap shifted by one), so the pair table T[p] = (U_Q[p], U_Q[p-1], L_Q[p],
// L_Q[p-1]) gives both envelope pairs in one 16-byte load and cc[j] = (c_j, c_j):
// A = cc - (U, U'), B = (L, L') - cc (two FADD2, negated operand), m = max3 per
// lane (two FMNMX3), acc = fma(m, m, acc) (one FFMA2): 5 instructions per two
// terms instead of 8, every lane's arithmetic exactly lb_term's (bit-identical).
// Window-position-outer order (one table entry live at a time); each slot still
// receives its terms in increasing j.  CHECK: the last chunk (nvalid < BC
// slots); positions of invalid slots are clamped (never stored).
template <int W, int BC, bool CHECK, typename F>
__device__ __forceinline__ void posting_chunk_eq_x2(const float2 (&cc)[W], const float4 *T, int pb, int nvalid,
                                                    F &&store) {
    static_assert(BC % 2 == 0, "slot pairs");
    float2 acc[BC / 2];
#pragma unroll
    for (int pp = 0; pp < BC / 2; pp++) acc[pp] = make_float2(0.f, 0.f);
#pragma unroll
    for (int k0 = 0; k0 < W + BC - 1; k0++) {
        // pairs (pp, j) with k0 = BC - 1 - 2 pp + j
        bool any = false;
#pragma unroll
        for (int pp = 0; pp < BC / 2; pp++) {
            const int j = k0 - (BC - 1) + 2 * pp;
            any |= (j >= 0 && j < W);
        }
        if (!any) continue;
        const float4 t = T[CHECK ? max(pb + k0, 0) : pb + k0];
#pragma unroll
        for (int pp = 0; pp < BC / 2; pp++) {
            const int j = k0 - (BC - 1) + 2 * pp;
            if (j >= 0 && j < W && (!CHECK || 2 * pp < nvalid)) {
                const float2 a = __fadd2_rn(cc[j], make_float2(-t.x, -t.y));
                const float2 b = __fadd2_rn(make_float2(t.z, t.w), make_float2(-cc[j].x, -cc[j].y));
                const float2 mm = make_float2(fmaxf(fmaxf(a.x, b.x), 0.0f), fmaxf(fmaxf(a.y, b.y), 0.0f));
                acc[pp] = __ffma2_rn(mm, mm, acc[pp]);
            }
        }
    }
#pragma unroll
    for (int pp = 0; pp < BC / 2; pp++) {
        if (!CHECK || 2 * pp < nvalid) store(2 * pp, acc[pp].x);
        if (!CHECK || 2 * pp + 1 < nvalid) store(2 * pp + 1, acc[pp].y);
    }
}

// ---------------------------------------------------------------------------
// Continuous step, static w (Remark 1): rows b in [0, nrows) of the
// ring (physical row (b + cursor) mod n_sw).  SW_0 gets P_EQ and P_EC; SW_1 ..
// SW_{nrows-1} only P_EQ (their MQ envelope changed with the new point; their
// P_EC, same MQ points against the same series envelope, is unchanged), so
// the EC terms are not even computed and the EQ plane takes full 4-byte
// coalesced rows.
// ---------------------------------------------------------------------------
template <typename S, int W, typename PV = typename Tr<S>::V>
__global__ void __launch_bounds__(128) window_lb_inc_kernel(const S *series, const S *UC, const S *LC,
                                                           const MQMeta *meta,
                                                           const typename Tr<S>::V4 *qtab, int D, int nrows,
                                                           int cursor, PV *post, float pscale) {
    using V = typename Tr<S>::V;
    constexpr int BC = W < 8 ? W : 8;
    constexpr bool X2 = std::is_same<V, float>::value && SMILER_INC_X2;
    extern __shared__ __align__(16) unsigned char wi_smem[];
    // X2 (f32): the EQ pair table T[p] = (U_Q[p], U_Q[p-1], L_Q[p], L_Q[p-1]) first
    float4 *sT = reinterpret_cast<float4 *>(wi_smem);
    V *sqq = reinterpret_cast<V *>(wi_smem + (X2 ? (size_t)D * sizeof(float4) : 0));
    V *squ = sqq + D;
    V *sql = squ + D;
    const int mq = blockIdx.y;
    const MQMeta m = meta[mq];
    // SMILER_INC_TILES consecutive 128-DW tiles per CTA: the MQ tables are
    // staged once and the (short) CTAs are fewer
    const int64_t r_first = (int64_t)blockIdx.x * SMILER_INC_TILES * blockDim.x;
    if (r_first >= m.n_dw) return;
    for (int p = threadIdx.x; p < D; p += blockDim.x) {
        const typename Tr<S>::V4 e = qtab[(int64_t)mq * D + p];
        sqq[p] = e.x;
        squ[p] = e.y;
        sql[p] = e.z;
        if constexpr (X2) {
            const typename Tr<S>::V4 e1 = qtab[(int64_t)mq * D + (p > 0 ? p - 1 : 0)];
            sT[p] = make_float4(e.y, e1.y, e.z, e1.z);
        }
    }
    __syncthreads();
    for (int tt = 0; tt < SMILER_INC_TILES; tt++) {
    const int64_t r = r_first + (int64_t)tt * blockDim.x + threadIdx.x;
    if (r >= m.n_dw) return;
    const int64_t ndw = m.n_dw;
    const int n_ring = D - W + 1;
    const int n_sw = min(n_ring, nrows);
    PV *oe = post + m.post_off + r;
    const int64_t base = m.series_off + r * W;
    V c[W], U[W], L[W];
    load_dw<S, V, W>(series + base, c);
    load_dw<S, V, W>(UC + base, U);
    load_dw<S, V, W>(LC + base, L);
    const int64_t pst = m.pstride;
    const int64_t plane = (int64_t)m.prows * pst;
    const int nmir = m.prows - n_ring;  // mirrored leading physical rows (TMA ring)
    // store one entry of logical row b (physical (b + cursor) mod n_sw, and its mirror)
    auto put = [&](int b, int pl, V v) {
        int row = b + cursor;
        row -= row >= n_ring ? n_ring : 0;
        PV *o = oe + (int64_t)pl * plane + (int64_t)row * pst;
        post_st(o, v, pscale);
        if (row < nmir) post_st(o + (int64_t)n_ring * pst, v, pscale);
    };
    // SW_0: both lists
    posting_chunk<V, W, 1, false>(c, U, L, sqq, squ, sql, D - W, 1, [&](int, V eq, V ec) {
        put(0, 0, eq);
        put(0, 1, ec);
    });
    int b0 = 1;
    if constexpr (X2 && BC % 2 == 0) {
        float2 cc[W];
#pragma unroll
        for (int j = 0; j < W; j++) cc[j] = make_float2(c[j], c[j]);
        for (; b0 + BC <= n_sw; b0 += BC)
            posting_chunk_eq_x2<W, BC, false>(cc, sT, D - W - b0 - (BC - 1), BC,
                                              [&](int bb, float eq) { put(b0 + bb, 0, eq); });
        if (b0 < n_sw)
            posting_chunk_eq_x2<W, BC, true>(cc, sT, D - W - b0 - (BC - 1), n_sw - b0,
                                             [&](int bb, float eq) { put(b0 + bb, 0, eq); });
    } else {
        for (; b0 + BC <= n_sw; b0 += BC)
            posting_chunk<V, W, BC, false, true>(c, U, L, sqq, squ, sql, D - W - b0 - (BC - 1), BC,
                                                 [&](int bb, V eq, V) { put(b0 + bb, 0, eq); });
        if (b0 < n_sw)
            posting_chunk<V, W, BC, true, true>(c, U, L, sqq, squ, sql, D - W - b0 - (BC - 1), n_sw - b0,
                                                [&](int bb, V eq, V) { put(b0 + bb, 0, eq); });
    }
    }
}

// ---------------------------------------------------------------------------
// Continuous streams (Remark 1, Fig. 6): after a stream advances by
// one point, the new SW_0 takes the ring slot of the dropped oldest SW, and the
// LB_EQ entries of SW_0 .. SW_rho (whose MQ envelope changed with the new point)
// are recomputed; LB_EC of SW_b for b >= 1 is unchanged (same MQ points, same
// series envelope).  One thread per DW r; rows b in [0, nrows), physical row
// (b + cursor) mod n_sw.  EQ and EC for b = 0, EQ only for b >= 1.
// ---------------------------------------------------------------------------
template <typename S>
__global__ void __launch_bounds__(128) posting_rows_kernel(const S *series, const S *UC, const S *LC,
                                                          const MQMeta *meta, const typename Tr<S>::V4 *qtab,
                                                          int D, int w, int nrows, int cursor,
                                                          typename Tr<S>::V *post) {
    using V = typename Tr<S>::V;
    using V4 = typename Tr<S>::V4;
    const int mq = blockIdx.y;
    const MQMeta m = meta[mq];
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= m.n_dw) return;
    const int n_sw = D - w + 1;
    const int64_t base = m.series_off + r * w;
    const V4 *qt = qtab + (int64_t)mq * D;
    for (int b = 0; b < nrows && b < n_sw; b++) {
        const int p0 = D - w - b;
        V eq = (V)0, ec = (V)0;
        for (int j = 0; j < w; j++) {
            const V4 Q = qt[p0 + j];
            lb_term((V)series[base + j], Q.y, Q.z, eq);
            if (b == 0) lb_term(Q.x, (V)UC[base + j], (V)LC[base + j], ec);
        }
        int row = b + cursor;
        row -= row >= n_sw ? n_sw : 0;
        V *o = post + m.post_off + (int64_t)row * m.n_dw + r;
        *o = eq;
        if (b == 0) o[(int64_t)n_sw * m.n_dw] = ec;
    }
}

// Advance every stream's master query by one point: MQ[0..D-1) = MQ[1..D),
// MQ[D-1] = new point.
template <typename S>
__global__ void __launch_bounds__(256) stream_shift_kernel(S *mq, int D, const S *newpt) {
    __shared__ S s[kMaxD];
    S *q = mq + (int64_t)blockIdx.x * D;
    for (int p = threadIdx.x; p < D; p += blockDim.x) s[p] = q[p];
    __syncthreads();
    for (int p = threadIdx.x; p < D; p += blockDim.x) q[p] = p + 1 < D ? s[p + 1] : newpt[blockIdx.x];
}

// ---------------------------------------------------------------------------
// a4: group-level scan over the posting lists in HBM (HBM-bound).  Thread <->
// rightmost DW r (r = Rb .. Rb+RT-1, Rb = blockIdx.x*RT - 1).  For each CSG_b,
// posting pairs are fetched 8 at a time ahead of the running sums (8 loads of
// 8 B in flight per thread); emission follows the per-CTA table em.
// smem: em [mmax*w] u16 | tile [n_len][RT*(w+1)] V.
// ---------------------------------------------------------------------------
template <typename S, int W>
__global__ void __launch_bounds__(256) group_scan_kernel(const typename Tr<S>::V *post,
                                                        const MQMeta *meta, const QParams P,
                                                        typename Tr<S>::V *lb, int32_t *tauc) {
    using V = typename Tr<S>::V;
    using V2 = typename Tr<S>::V2;
    extern __shared__ __align__(16) unsigned char gs_smem[];
    __shared__ uint64_t s_red[32];
    const int w = W > 0 ? W : P.w;
    const int RT = blockDim.x;
    const int nl = P.n_len;
    const int n_sw = P.D - w + 1;
    const int mmax = P.D / w;
    const int stride = RT * (w + 1);
    uint16_t *em = reinterpret_cast<uint16_t *>(gs_smem);
    V *tile = reinterpret_cast<V *>(gs_smem + ((mmax * w * 2 + 15) & ~15));
    const int mq = blockIdx.y;
    const MQMeta m = meta[mq];
    if ((int)blockIdx.x >= m.nblk) {
        tau_clear(P, mq, 1, 0, P.n_len, tauc);
        return;
    }
    build_emit_table(em, mmax, w, P);
    for (int x = threadIdx.x; x < nl * stride; x += RT) tile[x] = (V)0;
    __syncthreads();
    const int64_t Rb = (int64_t)blockIdx.x * RT - 1;
    const int64_t r = Rb + threadIdx.x;
    if (r >= 0 && r < m.n_dw) {
        const V *pp = post + m.post_off + r;
        const int64_t plane = (int64_t)n_sw * m.n_dw;
        V *trow = tile + threadIdx.x * (w + 1);
        for (int b = 0; b < w && b < n_sw; b++) {
            const int jmax = (n_sw - 1 - b) / w + 1;
            const int jlim = (int)min((int64_t)jmax, r + 1);
            V se = (V)0, sc = (V)0;
            for (int j0 = 0; j0 < jlim; j0 += 8) {
                V2 pv[8];
#pragma unroll
                for (int u = 0; u < 8; u++) {
                    const int j = j0 + u;
                    if (j < jlim) {
                        // continuous streams keep the posting lists in a ring over SWs
                        // (Remark 1): physical row of SW_{b+jw} = (b+jw+cursor) mod n_sw
                        int row = b + j * w + P.ring_cursor;
                        row -= row >= n_sw ? n_sw : 0;
                        const V *q = pp + (int64_t)row * m.n_dw - j;
                        pv[u].x = q[0];
                        pv[u].y = q[plane];
                    }
                }
#pragma unroll
                for (int u = 0; u < 8; u++) {
                    const int j = j0 + u;
                    if (j < jlim) {
                        se += pv[u].x;
                        sc += pv[u].y;
                        const int rng = em[j * w + b];
                        const V lbv = lbpick(P, se, sc);
                        for (int i = rng & 255; i < (rng >> 8); i++) trow[i * stride + b] = lbv;
                    }
                }
            }
        }
    }
    if constexpr (W > 0) {
        // row threadIdx.x of the tile was written by this thread only: barrier-free
        // warp epilogue (the tau units of this kernel are warps)
        lb_tile_epilogue_warp<V, W>(tile, RT, (Rb + 1) * w, m, P, lb, tauc, mq);
    } else {
        __syncthreads();
        lb_tile_epilogue<V, W>(tile, RT, (Rb + 1) * w, m, P, lb, tauc, mq, s_red);
    }
}

// ---------------------------------------------------------------------------
// a3+a4 fused (one-shot batches).  NT threads own NT consecutive DWs r' =
// Rb - HALO + x (HALO = mmax - 1 DWs of left halo); the RT = NT - HALO right
// threads own the tile's rightmost DWs r.  For each CSG row j:
//   phase A: every thread computes P[b + j w][r'] for all b < w into smem Ps
//            (sliding MQ window in registers, as in a3);
//   phase B: tile threads add Ps[b][x - j] = P[b + j w][r - j] to S_b and
//            emit LB_w for the IQs with m_i(b) = j + 1.
// The ALU work equals a3's plus HALO/NT; HBM traffic is only the series
// (read once) and LB_w.  smem: em | sq [D] V4 | Ps [w][NT] V2 | tile.
// ---------------------------------------------------------------------------
constexpr int kFusedThreads = 256;

template <typename S, int W>
__global__ void __launch_bounds__(kFusedThreads, (W <= 8 ? 3 : 1)) lb_fused_kernel(const S *series, const S *UC, const S *LC,
                                                                const MQMeta *meta,
                                                                const typename Tr<S>::V4 *qtab,
                                                                const QParams P, typename Tr<S>::V *lb,
                                                                int32_t *tauc) {
    using V = typename Tr<S>::V;
    using V2 = typename Tr<S>::V2;
    constexpr int NT = kFusedThreads;
    constexpr int BC = W < 8 ? W : 8;
    extern __shared__ __align__(16) unsigned char fz_smem[];
    __shared__ uint64_t s_red[32];
    const int D = P.D;
    const int nl = P.n_len;
    const int n_sw = D - W + 1;
    const int mmax = D / W;
    const int HALO = mmax - 1;
    const int RT = NT - HALO;
    const int stride = RT * (W + 1);
    uint16_t *em = reinterpret_cast<uint16_t *>(fz_smem);
    V2 *Ps = reinterpret_cast<V2 *>(fz_smem + ((mmax * W * 2 + 15) & ~15));  // [2][W][NT]
    V *sqq = reinterpret_cast<V *>(Ps + 2 * W * NT);
    V *squ = sqq + D;
    V *sql = squ + D;
    V *tile = sql + D;
    const int mq = blockIdx.y;
    const MQMeta m = meta[mq];
    if ((int)blockIdx.x >= m.nblk) {
        tau_clear(P, mq, 1, 0, P.n_len, tauc);
        return;
    }
    build_emit_table(em, mmax, W, P);
    for (int p = threadIdx.x; p < D; p += NT) {
        const typename Tr<S>::V4 e = qtab[(int64_t)mq * D + p];
        sqq[p] = e.x;
        squ[p] = e.y;
        sql[p] = e.z;
    }
    for (int x = threadIdx.x; x < nl * stride; x += NT) tile[x] = (V)0;
    const int x = threadIdx.x;
    const int64_t Rb = (int64_t)blockIdx.x * RT - 1;
    const int64_t rp = Rb - HALO + x;  // this thread's DW
    V c[W], U[W], L[W];
    {
        const bool ok = rp >= 0 && rp < m.n_dw;
        const int64_t base = m.series_off + (ok ? rp : 0) * W;
#pragma unroll
        for (int j = 0; j < W; j++) {
            c[j] = ok ? (V)series[base + j] : (V)0;
            U[j] = ok ? (V)UC[base + j] : (V)0;
            L[j] = ok ? (V)LC[base + j] : (V)0;
        }
    }
    V se[W], sc[W];
#pragma unroll
    for (int b = 0; b < W; b++) se[b] = sc[b] = (V)0;
    const bool is_tile = x >= HALO;
    V *trow = tile + (x - HALO) * (W + 1);
    __syncthreads();
    for (int j = 0; j < mmax; j++) {
        V2 *pb_ = Ps + (j & 1) * W * NT;
        const int nrow = min(W, n_sw - j * W);  // valid SWs b + jW in this CSG row (>= 1)
        // phase A: P[b + jW][r'] for b < nrow
#pragma unroll
        for (int b0 = 0; b0 < W; b0 += BC) {
            const int nv = nrow - b0;
            auto store = [&](int bb, V eq, V ec) {
                V2 v;
                v.x = eq;
                v.y = ec;
                pb_[(b0 + bb) * NT + x] = v;
            };
            const int pb = D - W - j * W - b0 - (BC - 1);
            if (nv >= BC)
                posting_chunk<V, W, BC, false>(c, U, L, sqq, squ, sql, pb, BC, store);
            else if (nv > 0)
                posting_chunk<V, W, BC, true>(c, U, L, sqq, squ, sql, pb, nv, store);
        }
        __syncthreads();
        // phase B: running sums along the CSG diagonals + emission
        if (is_tile) {
#pragma unroll
            for (int b = 0; b < W; b++) {
                if (b < nrow) {
                    const V2 pv = pb_[b * NT + x - j];
                    se[b] += pv.x;
                    sc[b] += pv.y;
                    const int rng = em[j * W + b];
                    if ((rng & 255) != (rng >> 8)) {
                        const V lbv = lbpick(P, se[b], sc[b]);
                        for (int i = rng & 255; i < (rng >> 8); i++) trow[i * stride + b] = lbv;
                    }
                }
            }
        }
        // no second barrier: the next row writes the other Ps buffer
    }
    __syncthreads();
    lb_tile_epilogue<V, W>(tile, RT, (Rb + 1) * W, m, P, lb, tauc, mq, s_red);
}

// ---------------------------------------------------------------------------
// a3+a4 fused, diagonal form (one-shot batches, default).  Thread x owns the
// rightmost DW r = Rb + x and walks its CSG diagonals itself: for row j it
// reads DW r - j (points and envelope) from a transposed shared-memory tile of
// the CTA's DWs plus a left halo of mmax-1 DWs, computes P[b + j w][r - j] for
// all b < w with the row's 2w-1 MQ positions in registers, and adds them
// straight into its running sums S_b.  No barrier inside the row loop, no
// halo recomputation, no posting list in memory at all.
// smem: em | sqq, squ, sql [D] | cs, us, ls [w][NT + HALO] | tile.
// ---------------------------------------------------------------------------
constexpr int kDiagThreads = 128;
constexpr int kDiagHaloMax = 128;
constexpr int kDiagCols = kDiagThreads + kDiagHaloMax;  // compile-time tile stride

// Write the W final LB_w values of IQ i held by this thread (slots e = s0 + b,
// t = e - d_i contiguous) and emit its warp's tau candidates.
// LB_w x sc -> fp16 rounded toward -inf: never above the scaled bound.  sc is
// the MQ's power-of-two storage scale (exact product; query_prep_kernel picks it
// so that no bound of the MQ exceeds 65504 after scaling, R26).
__device__ __forceinline__ __half lb_to_half(float v, float sc) { return __float2half_rd(v * sc); }
__device__ __forceinline__ __half lb_to_half(int32_t v, float sc) { return __float2half_rd(__int2float_rd(v) * sc); }
// LB x sc in f32, never above the exact product (the f32 product of a power of two is exact)
__device__ __forceinline__ float lb_scaled_rd(float v, float sc) { return v * sc; }
__device__ __forceinline__ float lb_scaled_rd(int32_t v, float sc) { return __int2float_rd(v) * sc; }

template <typename V, int W, bool FASTMASK = true>
__device__ __forceinline__ void diag_emit(const V (&v)[W], int i, int64_t s0, const MQMeta &m, const QParams &P,
                                          V *lb, int32_t *tauc, int mq, int bx = -1, float lbsc = 0.f) {
    static_assert(W <= 32, "slot mask is 32-bit");
    const int d = P.len[i];
    const int64_t tmin = m.t_lo > 0 ? m.t_lo : 0;
    const int64_t tend = min(m.t_hi, m.n - m.hz - d + 1);
    V *out = lb + m.seg_off + (int64_t)i * m.n;
    const int64_t t0 = s0 - d;
    // valid slots b: tmin <= t0 + b < tend, as one bit mask (two 64-bit
    // compares per emission instead of two per slot)
    constexpr uint32_t kAll = (uint32_t)((1ull << W) - 1ull);
    uint32_t vmask = kAll;  // interior slots (all but the tiles at a range end)
    // (FASTMASK = false: always the general form; lb_diag w = 16 measured faster so)
    if (!FASTMASK || t0 < tmin || t0 + W > tend) {
        const int blo = (int)max((int64_t)0, min((int64_t)W, tmin - t0));
        const int bhi = (int)max((int64_t)0, min((int64_t)W, tend - t0));
        vmask = (uint32_t)(((1ull << bhi) - 1ull) & ~((1ull << blo) - 1ull));
    }
    if (P.fuse) {  // a6 here: keep LB <= thr (ties survive), warp-aggregated append
        const int seg = mq * P.n_len + i;
        const uint32_t th = P.thr[seg];
        auto passes = [&](V x) {
            if constexpr (std::is_same<V, float>::value) return x <= __uint_as_float(th);
            else return x <= (int32_t)th;
        };
        // survivors are rare: one test of the thread's smallest bound decides for most warps
        V vmin = v[0];
#pragma unroll
        for (int b = 1; b < W; b++) vmin = vmin < v[b] ? vmin : v[b];
        if (__any_sync(0xffffffffu, passes(vmin))) {
            uint32_t keep = 0;
#pragma unroll
            for (int b = 0; b < W; b++) keep |= (uint32_t)passes(v[b]) << b;
            keep &= vmask;
            const int lane = threadIdx.x & 31;
            const int cnt = __popc(keep);
            int x = cnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int y = __shfl_up_sync(0xffffffffu, x, o);
                if (lane >= o) x += y;
            }
            const int total = __shfl_sync(0xffffffffu, x, 31);
            int base = 0;
            if (lane == 31 && total) base = atomicAdd(&P.scount[seg], total);
            base = __shfl_sync(0xffffffffu, base, 31);
            int o = base + x - cnt;
            int32_t *dst = P.surv + m.seg_off + (int64_t)i * m.n;
#pragma unroll
            for (int b = 0; b < W; b++)
                if (keep >> b & 1u) dst[o++] = (int32_t)(t0 + b);
        }
        if (P.E <= 0) return;  // a lagged stream step still picks the next step's tile tau set
    } else if (P.lb_half) {  // LB_w array as scaled fp16 rounded down (a valid, slightly looser bound)
        __half *oh = reinterpret_cast<__half *>(lb) + m.seg_off + (int64_t)i * m.n + t0;
        const float sc = lbsc > 0.f ? lbsc : P.lbs[mq];
        if (vmask == kAll && W % 8 == 0 && ((reinterpret_cast<uintptr_t>(oh) & 15) == 0)) {
            // bounds are >= 0, so rounding toward zero is rounding down: one packed
            // conversion (cvt.rz.f16x2.f32) per two bounds
#pragma unroll
            for (int b = 0; b < W; b += 8) {
                uint32_t hw[4];
#pragma unroll
                for (int q = 0; q < 4; q++) {
                    const float lo = lb_scaled_rd(v[b + 2 * q], sc), hi = lb_scaled_rd(v[b + 2 * q + 1], sc);
                    asm("cvt.rz.f16x2.f32 %0, %1, %2;" : "=r"(hw[q]) : "f"(hi), "f"(lo));
                }
                *reinterpret_cast<int4 *>(oh + b) = make_int4((int)hw[0], (int)hw[1], (int)hw[2], (int)hw[3]);
            }
        } else {
#pragma unroll
            for (int b = 0; b < W; b++)
                if (vmask >> b & 1u) oh[b] = lb_to_half(v[b], sc);
        }
    } else if (vmask == kAll && W % 4 == 0 && ((reinterpret_cast<uintptr_t>(out + t0) & 15) == 0)) {
#pragma unroll
        for (int b = 0; b < W; b += 4) {
            typename Tr<int16_t>::V4 pk;  // 4 x 32-bit lanes (int or float bits)
            pk.x = *reinterpret_cast<const int32_t *>(&v[b]);
            pk.y = *reinterpret_cast<const int32_t *>(&v[b + 1]);
            pk.z = *reinterpret_cast<const int32_t *>(&v[b + 2]);
            pk.w = *reinterpret_cast<const int32_t *>(&v[b + 3]);
            *reinterpret_cast<int4 *>(out + t0 + b) = pk;
        }
    } else {
#pragma unroll
        for (int b = 0; b < W; b++)
            if (vmask >> b & 1u) out[t0 + b] = v[b];
    }
    if (P.E <= 0) return;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int unit = (bx >= 0 ? bx : (int)blockIdx.x) * nw + warp;  // tau units are warps of tile bx
    int32_t *dst = tauc + (int64_t)(mq * P.n_len + i) * P.LT + (int64_t)unit * P.E;
#if SMILER_TAU_PACKED
    // The E (near-)smallest LB_w of the warp, one 32-bit key per slot: the
    // LB_w bits (non-negative float or int: unsigned order = value order) with
    // their lowest SB bits replaced by the slot b.  The minimum key names its
    // slot directly (no per-slot hit search), and the stored bound
    // (bits & ~mask) is never above the slot's LB_w.  The tau set only has to
    // hold >= k verified candidates for tau to bound the k-th NN key (R8), so
    // choosing among LB_w equal up to the low SB bits is still valid.
    constexpr int SB = W <= 4 ? 2 : (W <= 8 ? 3 : (W <= 16 ? 4 : 5));
    constexpr uint32_t SM = (1u << SB) - 1u;
    uint32_t kb[W];
#pragma unroll
    for (int b = 0; b < W; b++) kb[b] = (vmask >> b & 1u) ? ((key_bits(v[b]) & ~SM) | (uint32_t)b) : 0xFFFFFFFFu;
    uint32_t best = kb[0];
#pragma unroll
    for (int b = 1; b < W; b++) best = min(best, kb[b]);
    for (int e = 0; e < P.E; e++) {
        const uint32_t win = __reduce_min_sync(0xffffffffu, best);
        const int wl = __ffs(__ballot_sync(0xffffffffu, best == win)) - 1;
        const int tw = __shfl_sync(0xffffffffu, (int)t0, wl) + (int)(win & SM);
        if (lane == wl && e + 1 < P.E) {
            best = 0xFFFFFFFFu;
#pragma unroll
            for (int b = 0; b < W; b++) {
                kb[b] = kb[b] == win ? 0xFFFFFFFFu : kb[b];
                best = min(best, kb[b]);
            }
        }
        if (lane == 0) {
            dst[e] = win != 0xFFFFFFFFu ? tw : -1;
            if (P.taulb) P.taulb[dst - tauc + e] = win != 0xFFFFFFFFu ? (win & ~SM) : win;
        }
    }
}
#else
    // The E smallest (LB_w, t) keys of the warp with 32-bit compares only: t
    // grows with the slot b inside a thread and with the lane across the warp,
    // so among equal LB_w bits the lowest lane, then the lowest b, has the
    // smallest t (the same keys as a 64-bit (LB_w bits << 32 | t) minimum).
    // Per round: the thread minimum (no index tracking), the warp minimum, the
    // lowest lane holding it, and that lane's lowest slot holding it.
    uint32_t kb[W];
#pragma unroll
    for (int b = 0; b < W; b++) kb[b] = (vmask >> b & 1u) ? key_bits(v[b]) : 0xFFFFFFFFu;
    for (int e = 0; e < P.E; e++) {
        uint32_t best = kb[0];
#pragma unroll
        for (int b = 1; b < W; b++) best = min(best, kb[b]);
        const uint32_t win = __reduce_min_sync(0xffffffffu, best);
        const int wl = __ffs(__ballot_sync(0xffffffffu, best == win)) - 1;
        uint32_t hit = 0;
#pragma unroll
        for (int b = 0; b < W; b++) hit |= (uint32_t)(kb[b] == win) << b;
        const int bs = __ffs(hit) - 1;  // valid on lane wl
        const int tw = __shfl_sync(0xffffffffu, (int)(t0 + bs), wl);
        if (lane == wl && e + 1 < P.E) {
#pragma unroll
            for (int b = 0; b < W; b++)
                if (b == bs) kb[b] = 0xFFFFFFFFu;
        }
        if (lane == 0) {
            dst[e] = win != 0xFFFFFFFFu ? tw : -1;
            if (P.taulb) P.taulb[dst - tauc + e] = win;  // the trim reads the bound here, not from LB_w
        }
    }
}
#endif

// ---------------------------------------------------------------------------
// a3+a4 fused, diagonal form (one-shot batches, default).  Thread x owns the
// rightmost DW r = Rb + x and walks its CSG diagonals itself: for row j it
// reads DW r - j (points and envelope) from a transposed shared-memory tile of
// the CTA's DWs plus a left halo of mmax-1 DWs, computes P[b + j w][r - j] for
// all b < w with the row's 2w-1 MQ positions in registers, and adds them
// straight into its running sums S_b.  No barrier inside the row loop, no
// halo recomputation, no posting list in memory at all.
// Emission: m_i(b) = floor((d_i - b)/w) = q_i - [b > r_i] (d_i = q_i w + r_i),
// so IQ i's slots b > r_i are final after row q_i - 2 and b <= r_i after row
// q_i - 1; the thread saves the former and writes all w values of IQ i after
// row q_i - 1 straight from registers (vector stores), choosing the tau set of
// its warp with shuffles.  No LB tile, no epilogue barrier.
// smem: sqq, squ, sql [D] | cs, us, ls [w][kDiagCols].
// ---------------------------------------------------------------------------
// padded column stride (floats) of the DW tile: multiple of 4 for 16-byte
// loads, chosen so the 8 lanes of one LDS.128 phase hit distinct banks
template <int W> struct DiagStride { static constexpr int v = (W == 4) ? 12 : W + 4; };

template <typename S, int W>
__global__ void __launch_bounds__(kDiagThreads, (W <= 8 ? SMILER_DIAG_MINB8 : 3))
    lb_diag_kernel(const S *series, const S *UC, const S *LC, const MQMeta *meta,
                   const typename Tr<S>::V4 *qtab, const QParams P, typename Tr<S>::V *lb,
                   int32_t *tauc) {
    using V = typename Tr<S>::V;
    using V4 = typename Tr<S>::V4;
    constexpr int NT = kDiagThreads;
    constexpr int BC = W < 8 ? W : 8;
    constexpr int DS = DiagStride<W>::v;
    constexpr int WL = ((W + BC - 1) + 3) & ~3;  // window registers, rounded to 16-byte loads
    extern __shared__ __align__(16) unsigned char dg_smem[];
    const int D = P.D;
    const int nl = P.n_len;
    const int n_sw = D - W + 1;
    const int mmax = D / W;
    const int HALO = mmax - 1;
    const int NC = NT + HALO;  // DW columns in the tile
    // MQ arrays shifted so every row's window start is 16-byte aligned
    const int qshift = (4 - ((D - W - BC + 1) % 4 + 4) % 4) % 4;
    const int QL = (D + qshift + WL + 3) & ~3;
    V *sqq = reinterpret_cast<V *>(dg_smem);
    V *squ = sqq + QL;
    V *sql = squ + QL;
    V *cs = sql + QL;  // [kDiagCols][DS]
    V *us = cs + kDiagCols * DS;
    V *ls = us + kDiagCols * DS;
    const int mq = blockIdx.y;
    const MQMeta m = meta[mq];
    if ((int)blockIdx.x >= m.nblk) {
        tau_clear(P, mq, kDiagThreads / 32, 0, P.n_len, tauc);
        return;
    }
    for (int p = threadIdx.x; p < QL; p += NT) {
        const int src = p - qshift;
        V q = (V)0, u = (V)0, l = (V)0;
        if (src >= 0 && src < D) {
            const V4 e = qtab[(int64_t)mq * D + src];
            q = e.x;
            u = e.y;
            l = e.z;
        }
        sqq[p] = q;
        squ[p] = u;
        sql[p] = l;
    }
    const int64_t Rb = (int64_t)blockIdx.x * NT - 1;
    const int64_t R0 = Rb - HALO;  // DW of tile column 0
    // 4 consecutive points per item (16-byte f32 / 8-byte i16 vector loads:
    // sensors start on 64-element boundaries), 16-byte shared-memory stores
    // (DS is a multiple of 4); 4 iterations' loads in flight
    constexpr int W4 = W / 4;
#pragma unroll 4
    for (int idx = threadIdx.x; idx < NC * W4; idx += NT) {
        const int col = idx / W4, q = idx % W4;
        const int64_t rp = R0 + col;
        V4 c = {}, u = {}, l = {};
        if (rp >= 0 && rp < m.n_dw) {
            const int64_t g = m.series_off + rp * W + 4 * q;
            if constexpr (std::is_same<S, float>::value) {
                const float4 a = __ldg(reinterpret_cast<const float4 *>(series + g));
                const float4 b = __ldg(reinterpret_cast<const float4 *>(UC + g));
                const float4 e = __ldg(reinterpret_cast<const float4 *>(LC + g));
                c = make_float4(a.x, a.y, a.z, a.w);
                u = make_float4(b.x, b.y, b.z, b.w);
                l = make_float4(e.x, e.y, e.z, e.w);
            } else {
                auto unpack = [](uint2 v) {
                    return make_int4((int16_t)(v.x & 0xFFFF), (int16_t)((int32_t)v.x >> 16),
                                     (int16_t)(v.y & 0xFFFF), (int16_t)((int32_t)v.y >> 16));
                };
                c = unpack(__ldg(reinterpret_cast<const uint2 *>(series + g)));
                u = unpack(__ldg(reinterpret_cast<const uint2 *>(UC + g)));
                l = unpack(__ldg(reinterpret_cast<const uint2 *>(LC + g)));
            }
        }
        *reinterpret_cast<V4 *>(cs + col * DS + 4 * q) = c;
        *reinterpret_cast<V4 *>(us + col * DS + 4 * q) = u;
        *reinterpret_cast<V4 *>(ls + col * DS + 4 * q) = l;
    }
    __syncthreads();
    const int x = threadIdx.x;
    const int64_t s0 = (Rb + 1 + x) * W;  // e of this thread's slot b = 0
    V se[W], sc[W], saved[W];
#pragma unroll
    for (int b = 0; b < W; b++) se[b] = sc[b] = saved[b] = (V)0;
    uint64_t emit_rows = 0, save_rows = 0;  // rows q_i - 1 / q_i - 2 (block-uniform)
    for (int i = 0; i < nl; i++) {
        const int qi = P.len[i] / W;
        if (qi >= 1) emit_rows |= 1ull << (qi - 1);
        if (qi >= 2) save_rows |= 1ull << (qi - 2);
    }
    // IQs shorter than W have no full DW anywhere (m = 0, R6): LB_w = 0
    for (int i = 0; i < nl && P.len[i] < W; i++) diag_emit<V, W>(saved, i, s0, m, P, lb, tauc, mq);
#if SMILER_DIAG_UNROLL2
#pragma unroll 2
#endif
    // DW r - j of row j: one loop-carried pointer (us / ls at fixed offsets),
    // so the row prologue does not re-derive tid and the tile base each row
    const V *cp = cs + (x + HALO) * DS;
#if SMILER_EXPERIMENTS
    if (P.k < 0) emit_rows = save_rows = 0;  // timing experiment: main loop only (results invalid)
#endif
    for (int j = 0; j < mmax; j++, cp -= DS) {
        V c[W], U[W], L[W];
#pragma unroll
        for (int jj = 0; jj < W; jj += 4) {
            const V4 a = *reinterpret_cast<const V4 *>(cp + jj);
            const V4 u = *reinterpret_cast<const V4 *>(cp + kDiagCols * DS + jj);
            const V4 l = *reinterpret_cast<const V4 *>(cp + 2 * kDiagCols * DS + jj);
            c[jj] = a.x, c[jj + 1] = a.y, c[jj + 2] = a.z, c[jj + 3] = a.w;
            U[jj] = u.x, U[jj + 1] = u.y, U[jj + 2] = u.z, U[jj + 3] = u.w;
            L[jj] = l.x, L[jj + 1] = l.y, L[jj + 2] = l.z, L[jj + 3] = l.w;
        }
        const int nrow = min(W, n_sw - j * W);
        // W / BC chunks of BC sliding windows.  With more than one chunk the
        // chunk loop is NOT unrolled (a fully unrolled w = 16 row is 2048 ALU
        // instructions, 32 KB of code: it thrashes the 32 KB L1.5 I-cache); the
        // chunk always accumulates into slots 0..BC-1 and the slot arrays are
        // rotated by BC afterwards (identity again after W / BC chunks).
        constexpr int NCH = W / BC;
        // two chunks (w = 16): the chunk accumulates into local sums that one
        // uniform branch adds to slots 0..7 or 8..15 (no slot rotation)
        constexpr bool SPLIT2 = SMILER_DIAG_SPLIT2 && NCH == 2;
#pragma unroll 1
        for (int h = 0; h < NCH; h++) {
            const int b0 = h * BC;
            const int nv = nrow - b0;
            V te2[BC], tc2[BC];
            if constexpr (SPLIT2) {
#pragma unroll
                for (int b = 0; b < BC; b++) te2[b] = tc2[b] = (V)0;
            }
            auto acc = [&](int bb, V eq, V ec) {
                if constexpr (SPLIT2) {
                    te2[bb] += eq;
                    tc2[bb] += ec;
                } else {
                    se[bb] += eq;
                    sc[bb] += ec;
                }
            };
            const int pb = D - W - j * W - b0 - (BC - 1);
            if (nv >= BC) {  // full chunk: aligned 16-byte window loads
                V wq[WL], wu[WL], wl[WL];
                const int base = pb + qshift;
#pragma unroll
                for (int k = 0; k < WL; k += 4) {
                    const V4 a = *reinterpret_cast<const V4 *>(sqq + base + k);
                    const V4 u = *reinterpret_cast<const V4 *>(squ + base + k);
                    const V4 l = *reinterpret_cast<const V4 *>(sql + base + k);
                    wq[k] = a.x, wq[k + 1] = a.y, wq[k + 2] = a.z, wq[k + 3] = a.w;
                    wu[k] = u.x, wu[k + 1] = u.y, wu[k + 2] = u.z, wu[k + 3] = u.w;
                    wl[k] = l.x, wl[k + 1] = l.y, wl[k + 2] = l.z, wl[k + 3] = l.w;
                }
                if constexpr (SPLIT2)
                    posting_chunk_w_fold<V, W, BC, WL, BC>(c, U, L, wq, wu, wl, te2, tc2);
                else if constexpr (SMILER_LB_FOLD)
                    posting_chunk_w_fold<V, W, BC, WL, W>(c, U, L, wq, wu, wl, se, sc);
                else
                    posting_chunk_w<V, W, BC, false, WL>(c, U, L, wq, wu, wl, BC, acc);
            } else if (nv > 0) {
                posting_chunk<V, W, BC, true>(c, U, L, sqq + qshift, squ + qshift, sql + qshift, pb, nv, acc);
            }
            if constexpr (SPLIT2) {
                if (h == 0) {
#pragma unroll
                    for (int b = 0; b < BC; b++) se[b] += te2[b], sc[b] += tc2[b];
                } else {
#pragma unroll
                    for (int b = 0; b < BC; b++) se[BC + b] += te2[b], sc[BC + b] += tc2[b];
                }
            } else if (NCH > 1) {  // rotate the slots left by BC
                V te[BC], tc[BC];
#pragma unroll
                for (int b = 0; b < BC; b++) te[b] = se[b], tc[b] = sc[b];
#pragma unroll
                for (int b = 0; b + BC < W; b++) se[b] = se[b + BC], sc[b] = sc[b + BC];
#pragma unroll
                for (int b = 0; b < BC; b++) se[W - BC + b] = te[b], sc[W - BC + b] = tc[b];
            }
        }
        // rows q_i - 1: compose IQ i from the values saved after row q_i - 2
        // (slots b > r_i) and the current sums (b <= r_i), then write it
        if (emit_rows >> j & 1ull) {
            for (int i = 0; i < nl; i++) {
                const int qi = P.len[i] / W, ri = P.len[i] % W;
                if (j == qi - 1) {
                    // saved[] is still all zero at row 0 (the first save follows
                    // row 0's emissions), so q_i = 1 needs no separate case
                    V v[W];
#pragma unroll
                    for (int b = 0; b < W; b++) v[b] = b > ri ? saved[b] : lbpick(P, se[b], sc[b]);
                    diag_emit<V, W, (W <= 8)>(v, i, s0, m, P, lb, tauc, mq);
                }
            }
        }
        // rows q_i - 2: save (after composing, so a row that is q_i - 1 for one
        // IQ and q_i' - 2 for another uses the previous row's saved values)
        if (save_rows >> j & 1ull) {
#pragma unroll
            for (int b = 0; b < W; b++) saved[b] = lbpick(P, se[b], sc[b]);
        }
    }
#if SMILER_EXPERIMENTS
    if (P.k < 0) {  // timing experiment: keep the sums alive
        V acc = (V)0;
#pragma unroll
        for (int b = 0; b < W; b++) acc += se[b] + sc[b];
        if (acc == (V)12345) lb[0] = acc;
    }
#endif
}

// ---------------------------------------------------------------------------
// lb_diag_kernel for f32 with sm_100's packed fp32x2 arithmetic (FADD2 /
// FFMA2).  The EQ and EC terms of one (SW, DW, j) element share each packed
// instruction:
//   A = (c, L_C) - (U_Q, q)     = (c - U_Q, L_C - q)      EQ's v - U, EC's L - v
//   B = (q, L_Q) - (U_C, c)     = (q - U_C, L_Q - c)      EC's v - U, EQ's L - v
//   m = (max(A.x, B.y, 0), max(A.y, B.x, 0))             two FMNMX3
// (the halves of B are crossed so that each FMNMX3 reads one even and one odd
// register of the pairs: no register-bank conflict)
//   (S_EQ, S_EC) = fma(m, m, (S_EQ, S_EC))               one FFMA2
// 5 instructions per term pair instead of 8 (FADD2 negates its second operand
// for free), with exactly the scalar form's roundings and the same per-slot
// summation order, so every LB_w is bit-identical to lb_diag_kernel<float, W>'s.
// The DW tile holds (c, L_C, U_C, c) and the MQ table (U_Q, q, q, L_Q) per point, so
// one LDS.128 yields both operand pairs.  Tile, diagonal walk, emission and
// tau set are lb_diag_kernel's.
// smem: qx [x2_pad + D] float4 | tile [kDiagCols][W + 1] float4 (column stride
// W + 1: the 8 lanes of one LDS.128 phase hit distinct bank quads).
// ---------------------------------------------------------------------------
#ifndef SMILER_DIAG_X2_MINB16
#define SMILER_DIAG_X2_MINB16 3
#endif
#ifndef SMILER_DIAG_X2_MINB8
#define SMILER_DIAG_X2_MINB8 7  // 70 registers, no spills; C2 LB 8.25 ms (6: 8.27, 5: 8.58)
#endif
__device__ __forceinline__ float2 lo2(const float4 &v) { return make_float2(v.x, v.y); }
__device__ __forceinline__ float2 hi2(const float4 &v) { return make_float2(v.z, v.w); }
__device__ __forceinline__ float2 sub2(const float2 &a, const float2 &b) {  // one FADD2 (negated operand)
    return __fadd2_rn(a, make_float2(-b.x, -b.y));
}

// Term pairs of chunk slots bb < BC (valid: bb < nv) against the row's DW
// points Pt[0..W) and the window Q[0..W+BC-1) (element (bb, j) uses
// Q[BC-1-bb+j]).  Window-position-outer order: one Q entry live at a time,
// and every slot still receives its terms in increasing j.
template <int W, int BC, bool CHECK>
__device__ __forceinline__ void x2_chunk(const float4 (&Pt)[W], const float4 *Q, int nv, float2 (&acc)[BC]) {
#pragma unroll
    for (int k = 0; k < W + BC - 1; k++) {
        const float4 q = Q[k];
#pragma unroll
        for (int j = (k - BC + 1 > 0 ? k - BC + 1 : 0); j <= (k < W - 1 ? k : W - 1); j++) {
            const int bb = BC - 1 - k + j;
            if (!CHECK || bb < nv) {
                const float2 a = sub2(lo2(Pt[j]), lo2(q));
                const float2 b = sub2(hi2(q), hi2(Pt[j]));
                const float2 mm = make_float2(fmaxf(fmaxf(a.x, b.y), 0.0f), fmaxf(fmaxf(a.y, b.x), 0.0f));
                acc[bb] = __ffma2_rn(mm, mm, acc[bb]);
            }
        }
    }
}

// qx front padding (entries): windows of the last CSG row's invalid slots start
// up to BC - 1 positions before the MQ; they are never used, only kept in range
template <int W> constexpr int x2_pad() { return 8; }
// qx plus the tile's NT + mmax - 1 columns (sized by the actual halo: more CTAs per SM)
template <int W> size_t x2_smem(int D) {
    return (size_t)(x2_pad<W>() + D + (kDiagThreads + D / W - 1) * (W + 1)) * 16;
}

// The last CSG row with a single valid slot (nv = D mod w + 1 = 1, e.g. D = 128,
// w = 8): slot 0's W term pairs only (the predicated chunk would issue every
// pair's instructions for the one that counts).
template <int W, int BC>
__device__ __forceinline__ void x2_chunk_slot0(const float4 (&Pt)[W], const float4 *Q, float2 (&acc)[BC]) {
#pragma unroll
    for (int j = 0; j < W; j++) {
        const float4 q = Q[BC - 1 + j];
        const float2 a = sub2(lo2(Pt[j]), lo2(q));
        const float2 b = sub2(hi2(q), hi2(Pt[j]));
        const float2 mm = make_float2(fmaxf(fmaxf(a.x, b.y), 0.0f), fmaxf(fmaxf(a.y, b.x), 0.0f));
        acc[0] = __ffma2_rn(mm, mm, acc[0]);
    }
}

template <int W>
__global__ void __launch_bounds__(kDiagThreads, (W <= 8 ? SMILER_DIAG_X2_MINB8 : SMILER_DIAG_X2_MINB16))
    lb_diag_x2_kernel(const float *series, const float *UC, const float *LC, const MQMeta *meta,
                      const float4 *qtab, const QParams P, float *lb, int32_t *tauc) {
    constexpr int NT = kDiagThreads;
    constexpr int BC = W < 8 ? W : 8;
    constexpr int NCH = W / BC;
    constexpr int DS = W + 1;  // float4s per tile column
    constexpr int PAD = x2_pad<W>();
    extern __shared__ __align__(16) unsigned char dx_smem[];
    const int D = P.D;
    const int nl = P.n_len;
    const int n_sw = D - W + 1;
    const int mmax = D / W;
    const int HALO = mmax - 1;
    const int NC = NT + HALO;
    float4 *qx = reinterpret_cast<float4 *>(dx_smem) + PAD;  // qx[p], p in [-PAD, D)
    float4 *tile = qx + D;
    const int mq = blockIdx.y;
    const MQMeta m = meta[mq];
    if ((int)blockIdx.x >= m.nblk) {
        tau_clear(P, mq, kDiagThreads / 32, 0, P.n_len, tauc);
        return;
    }
    for (int p = (int)threadIdx.x - PAD; p < D; p += NT) {
        float4 e = make_float4(0.f, 0.f, 0.f, 0.f);
        if (p >= 0) {
            const float4 t = qtab[(int64_t)mq * D + p];  // (q, U_Q, L_Q, 0)
            e = make_float4(t.y, t.x, t.x, t.z);
        }
        qx[p] = e;
    }
    const int64_t Rb = (int64_t)blockIdx.x * NT - 1;
    const int64_t R0 = Rb - HALO;  // DW of tile column 0
    constexpr int W4 = W / 4;
#pragma unroll 2
    for (int idx = threadIdx.x; idx < NC * W4; idx += NT) {
        const int col = idx / W4, q = idx % W4;
        const int64_t rp = R0 + col;
        float4 c = make_float4(0.f, 0.f, 0.f, 0.f), u = c, l = c;
        if (rp >= 0 && rp < m.n_dw) {
            const int64_t g = m.series_off + rp * W + 4 * q;
            c = __ldg(reinterpret_cast<const float4 *>(series + g));
            u = __ldg(reinterpret_cast<const float4 *>(UC + g));
            l = __ldg(reinterpret_cast<const float4 *>(LC + g));
        }
        float4 *dst = tile + col * DS + 4 * q;
        dst[0] = make_float4(c.x, l.x, u.x, c.x);
        dst[1] = make_float4(c.y, l.y, u.y, c.y);
        dst[2] = make_float4(c.z, l.z, u.z, c.z);
        dst[3] = make_float4(c.w, l.w, u.w, c.w);
    }
    __syncthreads();
    const int x = threadIdx.x;
    const int64_t s0 = (Rb + 1 + x) * W;  // e of this thread's slot b = 0
    float2 acc[W];
    float saved[W];
#pragma unroll
    for (int b = 0; b < W; b++) acc[b] = make_float2(0.f, 0.f), saved[b] = 0.f;
    const float lsc = P.lb_half ? P.lbs[mq] : 0.f;
    // IQs shorter than W have no full DW anywhere (m = 0, R6): LB_w = 0
    int i0 = 0;
    for (; i0 < nl && P.len[i0] < W; i0++) diag_emit<float, W>(saved, i0, s0, m, P, lb, tauc, mq, -1, lsc);
    const float4 *cp = tile + (x + HALO) * DS;  // DW r - j of row j
    // Rows run in segments that end at the emission rows: IQ i (q_i = d_i / w,
    // r_i = d_i % w, ascending in i) needs the sums after row q_i - 2 (saved,
    // slots b > r_i, m_i(b) = q_i - 1) and after row q_i - 1 (slots b <= r_i).
    // LB_w = max(S_EQ, S_EC) (Eq. 5; the EQ / EC ablations run the scalar kernel).
    int j = 0;
    for (int i = i0; i < nl; i++) {
        const int qi = P.len[i] / W, ri = P.len[i] % W;
        for (; j < qi; j++, cp -= DS) {
            if (j == qi - 1) {
#pragma unroll
                for (int b = 0; b < W; b++) saved[b] = fmaxf(acc[b].x, acc[b].y);
            }
            float4 Pt[W];
#pragma unroll
            for (int jj = 0; jj < W; jj++) Pt[jj] = cp[jj];
            const int nrow = min(W, n_sw - j * W);
            if constexpr (NCH == 1) {
                const float4 *Q = qx + (D - W - j * W - (BC - 1));
                if (nrow >= BC) {
                    x2_chunk<W, BC, false>(Pt, Q, nrow, acc);
                } else {
                    // the last CSG row (nrow < BC valid slots, a uniform bound): each
                    // posting element summed on its own, then added (lb_diag_kernel's
                    // association there: bit-identical LB_w)
#pragma unroll
                    for (int bb = 0; bb < BC; bb++) {
                        if (bb < nrow) {
                            float2 t = make_float2(0.f, 0.f);
#pragma unroll
                            for (int jj = 0; jj < W; jj++) {
                                const float4 q = Q[BC - 1 - bb + jj];
                                const float2 a = sub2(lo2(Pt[jj]), lo2(q));
                                const float2 b = sub2(hi2(q), hi2(Pt[jj]));
                                const float2 mm = make_float2(fmaxf(fmaxf(a.x, b.y), 0.0f), fmaxf(fmaxf(a.y, b.x), 0.0f));
                                t = __ffma2_rn(mm, mm, t);
                            }
                            acc[bb] = __fadd2_rn(acc[bb], t);
                        }
                    }
                }
            } else {
                // two chunks (w = 16): local chunk sums added to slots 0..7 or 8..15 by
                // one uniform branch (lb_diag_kernel's SPLIT2 association)
#pragma unroll 1
                for (int h = 0; h < NCH; h++) {
                    const int b0 = h * BC;
                    const int nv = nrow - b0;
                    float2 t2[BC];
#pragma unroll
                    for (int b = 0; b < BC; b++) t2[b] = make_float2(0.f, 0.f);
                    const float4 *Q = qx + (D - W - j * W - b0 - (BC - 1));
                    if (nv >= BC) x2_chunk<W, BC, false>(Pt, Q, nv, t2);
                    else if (nv == 1) x2_chunk_slot0<W, BC>(Pt, Q, t2);
                    else if (nv > 0) x2_chunk<W, BC, true>(Pt, Q, nv, t2);
                    if (h == 0) {
#pragma unroll
                        for (int b = 0; b < BC; b++) acc[b] = __fadd2_rn(acc[b], t2[b]);
                    } else {
#pragma unroll
                        for (int b = 0; b < BC; b++) acc[BC + b] = __fadd2_rn(acc[BC + b], t2[b]);
                    }
                }
            }
        }
        // an IQ with the same q_i as the previous one reuses its saved values
        float v[W];
#pragma unroll
        for (int b = 0; b < W; b++) v[b] = b > ri ? saved[b] : fmaxf(acc[b].x, acc[b].y);
        diag_emit<float, W, (W <= 8)>(v, i, s0, m, P, lb, tauc, mq, -1, lsc);
    }
}

// ---------------------------------------------------------------------------
// a4 for static w (two-level path, continuous-stream ring): thread x owns the
// rightmost DW r = Rb + x and walks CSG row j = 0 .. mmax-1 itself, summing
// P[b + j w][r - j] for all b < w into register sums S_b (the same j order as
// the generic scan, so LB_w is bit-identical).  Emission is lb_diag_kernel's:
// m_i(b) = q_i - [b > r_i], so IQ i's slots b > r_i are final after row
// q_i - 2 (saved) and b <= r_i after row q_i - 1, written straight from
// registers by diag_emit (vector stores, per-warp tau set).  No shared memory,
// no barrier.  Posting addresses are 32-bit offsets from the MQ's posting block
// (host guarantees 2 n_sw n_dw < 2^31: both planes).  Only CTA 0 (DWs r < mmax - 1 lack
// some r - j) and the last CSG row (fewer than w SWs) take predicated loads;
// elsewhere threads past the last DW read DW n_dw - 1 and their slots are
// masked at emission (t >= tend).
// ---------------------------------------------------------------------------
constexpr int kScanThreads = 256;
// measured on C3/C5 streams (profiles/r01/history/group_scan_variants.txt)
#ifndef SMILER_GS_MINB
#define SMILER_GS_MINB(W) ((W) <= 8 ? 4 : (W) <= 16 ? 2 : 1)
#endif

// fp16 ring sums are in units of the ring's storage scale 2^-e: back to the
// bound itself (exact power-of-two product) before emission
template <typename V, typename PV, int W>
__device__ __forceinline__ void ring_unscale(V (&v)[W], const QParams &P) {
    if constexpr (std::is_same<PV, __half>::value) {
#pragma unroll
        for (int b = 0; b < W; b++) v[b] *= P.post_unscale;
    }
}

template <int W, bool CHECK, typename PV>
__device__ __forceinline__ void gs_load_row(PV (&pe)[W], PV (&pc)[W], const PV *pp, uint32_t off, int bw,
                                            uint32_t ndw, uint32_t wrap, int nrow, bool ok) {
#pragma unroll
    for (int b = 0; b < W; b++) {
        // physical rows rr + b >= n_sw wrap to the ring start (bw = n_sw - rr);
        // the P_EC plane sits `wrap` (= n_sw * n_dw) elements after P_EQ
        const uint32_t o = off + (uint32_t)b * ndw - (b >= bw ? wrap : 0u);
        if constexpr (CHECK) {
            pe[b] = pc[b] = (PV)0;
            if (ok && b < nrow) {
                pe[b] = __ldg(pp + o);
                pc[b] = __ldg(pp + o + wrap);
            }
        } else {
            pe[b] = __ldg(pp + o);
            pc[b] = __ldg(pp + o + wrap);
        }
    }
}

template <typename S, int W, typename PV = typename Tr<S>::V>
__global__ void __launch_bounds__(kScanThreads, SMILER_GS_MINB(W)) group_scan_reg_kernel(
    const PV *post, const MQMeta *meta, const QParams P, typename Tr<S>::V *lb, int32_t *tauc) {
    using V = typename Tr<S>::V;
    const int D = P.D;
    const int nl = P.n_len;
    const int n_sw = D - W + 1;
    const int mmax = D / W;
    const int mq = blockIdx.y;
    const MQMeta m = meta[mq];
    if ((int)blockIdx.x >= m.nblk) {
        tau_clear(P, mq, kScanThreads / 32, 0, P.n_len, tauc);
        return;
    }
    const int64_t r = (int64_t)blockIdx.x * kScanThreads - 1 + threadIdx.x;
    const int64_t s0 = (r + 1) * W;  // e of slot b = 0
    const bool valid = r >= 0 && r < m.n_dw;
    const int jall = valid ? (int)min((int64_t)mmax, r + 1) : 0;  // DW r - j must exist
    const bool first = blockIdx.x == 0;
    const uint32_t ndw = (uint32_t)m.n_dw;
    const uint32_t wrap = (uint32_t)n_sw * ndw;
    const int64_t rc = r < 0 ? 0 : (r < m.n_dw ? r : m.n_dw - 1);
    // offsets count from pp - mmax so they stay non-negative across the ring wrap
    const PV *pp = post + m.post_off + rc - mmax;
    // values saved after row q_i - 2 live in shared memory ([b][thread]: no
    // bank conflicts), keeping the registers for sums and loads in flight
    __shared__ V s_saved[W][kScanThreads];
    const int x = threadIdx.x;
    V se[W], sc[W];
#pragma unroll
    for (int b = 0; b < W; b++) se[b] = sc[b] = (V)0;
    uint64_t emit_rows = 0, save_rows = 0;
    for (int i = 0; i < nl; i++) {
        const int qi = P.len[i] / W;
        if (qi >= 1) emit_rows |= 1ull << (qi - 1);
        if (qi >= 2) save_rows |= 1ull << (qi - 2);
    }
    if (nl > 0 && P.len[0] < W) {
        V z[W];
#pragma unroll
        for (int b = 0; b < W; b++) z[b] = (V)0;
        for (int i = 0; i < nl && P.len[i] < W; i++) diag_emit<V, W>(z, i, s0, m, P, lb, tauc, mq);
    }
    // ring row of SW_{j w} (Remark 1): rr = (j w + cursor) mod n_sw,
    // advanced by w per row (mmax >= 2 implies n_sw > w)
    // one row of look-ahead: row j + 1's loads are in flight while row j is summed
    // (the fp16 ring moves half the bytes per load, so it needs the extra depth)
    int rr = P.ring_cursor;
    PV ne[W], nc[W];
    auto load = [&](int jj, int r_) {
        const uint32_t off = (uint32_t)r_ * ndw + (uint32_t)(mmax - jj);
        const int nrow = n_sw - jj * W;
        if (first || nrow < W)
            gs_load_row<W, true, PV>(ne, nc, pp, off, n_sw - r_, ndw, wrap, nrow, jj < jall);
        else
            gs_load_row<W, false, PV>(ne, nc, pp, off, n_sw - r_, ndw, wrap, nrow, true);
    };
    load(0, rr);
    for (int j = 0; j < mmax; j++) {
        PV pe[W], pc[W];
#pragma unroll
        for (int b = 0; b < W; b++) pe[b] = ne[b], pc[b] = nc[b];
        rr += W;
        rr -= rr >= n_sw ? n_sw : 0;
        // look-ahead only where registers allow (w = 8 at 64 registers spills)
        constexpr bool LA = W >= 16;
        if (LA && j + 1 < mmax) load(j + 1, rr);
#pragma unroll
        for (int b = 0; b < W; b++) {
            post_acc<V>(se[b], pe[b]);
            post_acc<V>(sc[b], pc[b]);
        }
        if (!LA && j + 1 < mmax) load(j + 1, rr);
        if (emit_rows >> j & 1ull) {
            for (int i = 0; i < nl; i++) {
                const int qi = P.len[i] / W, ri = P.len[i] % W;
                if (j == qi - 1) {
                    V v[W];
#pragma unroll
                    for (int b = 0; b < W; b++) v[b] = b > ri ? (qi >= 2 ? s_saved[b][x] : (V)0) : lbpick(P, se[b], sc[b]);
                    ring_unscale<V, PV, W>(v, P);
                    diag_emit<V, W>(v, i, s0, m, P, lb, tauc, mq);
                }
            }
        }
        if (save_rows >> j & 1ull) {
#pragma unroll
            for (int b = 0; b < W; b++) s_saved[b][x] = lbpick(P, se[b], sc[b]);
        }
    }
}

// ---------------------------------------------------------------------------
// a4 over the continuous-stream ring, TMA-staged (the HBM-bound "LB scan").
// The ring of every stream is one 2-D tensor: rows = (stream, plane, physical
// SW row) with the first w-1 physical rows mirrored after the last (so the w
// ring rows of one CSG row are contiguous for any cursor), columns = disjoint
// windows (row stride padded to 16 bytes).  For CSG row j the CTA's 256
// rightmost DWs r = Rb .. Rb+255 need columns r - j of the w rows
// (j w + cursor) mod n_sw + b.  A tiled TMA box must start on a 16-byte
// boundary of the innermost dimension (a misaligned start coordinate traps
// with "illegal instruction", measured: tools/tma_probe.cu), so per plane the
// CTA loads a w x 256 box at the aligned column ca = floor((Rb - j) / A) A
// (A = 16 bytes / entry) and, through a second tensor map, a w x A tail box
// at ca + 256; columns < 0 or
// >= n_dw arrive zero-filled.  Both land in a 4-stage shared-memory ring armed
// with mbarriers (persistent CTAs: the ring runs ahead across tiles); thread x
// then reads column x + (Rb - j - ca) of each row
// (from the main box, or the tail for the last few threads) -- conflict-free
// 2- or 4-byte loads, no per-element address arithmetic, whole 512-byte rows
// per request.  Sums, emission and the tau set are group_scan_reg's.
// ---------------------------------------------------------------------------
#ifndef SMILER_TMA_STAGES_W16
#define SMILER_TMA_STAGES_W16 4
#endif
#ifndef SMILER_TMA_MINB_W16
#define SMILER_TMA_MINB_W16 2
#endif
// TMA ring depth (a power of two) and CTAs per SM the register budget must fit
template <int W> constexpr int tma_stages() { return W >= 16 ? SMILER_TMA_STAGES_W16 : 4; }
template <int W> constexpr int tma_minb() { return W >= 16 ? SMILER_TMA_MINB_W16 : SMILER_GS_MINB(W); }
template <typename PV> constexpr int tma_align_elems() { return 16 / (int)sizeof(PV); }
// one stage: per plane a [W][256] main box and a [W][A] tail box, every box at
// a 128-byte aligned shared-memory offset
template <int W, typename PV> constexpr int tma_tail_pitch() {  // elements per tail box incl. padding
    return (int)((W * 16 + 127) / 128 * 128 / sizeof(PV));
}
template <int W, typename PV> constexpr size_t tma_stage_elems() {
    return (size_t)2 * W * kScanThreads + 2 * tma_tail_pitch<W, PV>();
}
template <int W, typename PV> constexpr size_t tma_scan_smem() {
    return (size_t)tma_stages<W>() * tma_stage_elems<W, PV>() * sizeof(PV);
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, int c0, int c1, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::
            "r"(smem_u32(dst)),
        "l"(map), "r"(c0), "r"(c1), "r"(smem_u32(bar))
        : "memory");
}

// One CSG row of the TMA scan for one thread's column: the W P_EQ entries at
// pe[b RS] and the W P_EC entries at pe[PS + b RS]; all 2W loads first, then the
// adds (rows b >= nrow, only in the last CSG row, add zero).
template <typename V, typename PV, int W, int RS, int PS, bool FULL>
__device__ __forceinline__ void tma_row_add(const PV *pe, int nrow, V (&se)[W], V (&sc)[W]) {
    PV ve[W], vc[W];
#pragma unroll
    for (int b = 0; b < W; b++) {
        ve[b] = pe[b * RS];
        vc[b] = pe[PS + b * RS];
    }
#pragma unroll
    for (int b = 0; b < W; b++) {
        if (FULL || b < nrow) {
            post_acc<V>(se[b], ve[b]);
            post_acc<V>(sc[b], vc[b]);
        }
    }
}

template <typename S, int W, typename PV, bool SEL = false>
__global__ void __launch_bounds__(kScanThreads, tma_minb<W>()) group_scan_tma_kernel(
    const __grid_constant__ CUtensorMap tmap, const __grid_constant__ CUtensorMap tmap_tail, const MQMeta *meta,
    const QParams P, typename Tr<S>::V *lb, int32_t *tauc, int nb, int n_mq, int row0, int prows) {
    using V = typename Tr<S>::V;
    constexpr int kTmaStages = tma_stages<W>();
    constexpr int NT = kScanThreads;
    constexpr int A = tma_align_elems<PV>();      // TMA start-column granule (16 bytes)
    constexpr int STAGE = (int)tma_stage_elems<W, PV>();
    constexpr int TP = tma_tail_pitch<W, PV>();
    constexpr uint32_t STAGE_BYTES = 2 * W * (NT + A) * sizeof(PV);  // bytes the four boxes deliver
    extern __shared__ __align__(128) unsigned char tma_smem[];
    // stage st: [plane 0 main W x NT][plane 1 main W x NT][plane 0 tail W x A][plane 1 tail W x A]
    PV *s_ring = reinterpret_cast<PV *>(tma_smem);
    __shared__ __align__(8) uint64_t s_full[kTmaStages];
    __shared__ __align__(8) uint64_t s_empty[kTmaStages];  // SMILER_TMA_EMPTYBAR: one arrival per warp
    __shared__ V s_saved[W][NT];
    const int D = P.D;
    const int nl = P.n_len;
    const int n_sw = D - W + 1;
    const int mmax = D / W;
    const int x = threadIdx.x;
    // Persistent: this CTA scans tiles blockIdx.x, blockIdx.x + gridDim.x, ...
    // (tile = mq * nb + bx); CSG rows are numbered g = k mmax + j over the CTA's
    // k-th tile, and the TMA ring runs ahead across tile boundaries, so the next
    // tile's rows stream in while this one emits.
    const int ntiles = n_mq * nb;
    const int my_tiles = (int)blockIdx.x < ntiles ? (ntiles - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 0;
    const int g_end = my_tiles * mmax;  // rows of this CTA (32-bit: a few thousand)
    // Issue cursor (the thread that refills): rows are issued in increasing g,
    // so (tile, mq, bx, j, physical SW row) advance incrementally -- a division
    // only when a tile starts (the issuing warp is the one every other warp waits
    // for at the next barrier: 240 instructions per issue with divisions per row).
    struct IssueCursor {
        int j, tile, mq, bx, pr;
    } ic;
    ic.j = 0;
    ic.tile = (int)blockIdx.x;
    ic.mq = ic.tile / nb;
    ic.bx = ic.tile - ic.mq * nb;
    ic.pr = P.ring_cursor;  // physical row of SW_0 (< n_sw)
    auto issue = [&](int g) {  // global row g (the next one in order) -> stage g % kTmaStages
        const int j = ic.j, mq = ic.mq, bx = ic.bx, pr = ic.pr;
        if (++ic.j == mmax) {
            ic.j = 0;
            ic.tile += (int)gridDim.x;
            ic.mq = ic.tile / nb;
            ic.bx = ic.tile - ic.mq * nb;
            ic.pr = P.ring_cursor;
        } else {
            ic.pr += W;  // j W < n_sw, cursor < n_sw: one wrap at most
            ic.pr -= ic.pr >= n_sw ? n_sw : 0;
        }
        // tensor row of this stream's P_EQ row 0: the streams' rings are
        // consecutive [2][prows] row blocks (no memory access on the issue path)
        const int row_base = row0 + mq * 2 * prows;
        const int st = g & (kTmaStages - 1);
        mbar_expect_tx(&s_full[st], STAGE_BYTES);
        const int col = bx * NT - 1 - j;
        const int ca = col & ~(A - 1);  // floor to the 16-byte granule (A is a power of two)
        PV *sb = s_ring + (size_t)st * STAGE;
        tma_load_2d(sb, &tmap, ca, row_base + pr, &s_full[st]);
        tma_load_2d(sb + W * NT, &tmap, ca, row_base + prows + pr, &s_full[st]);
        tma_load_2d(sb + 2 * W * NT, &tmap_tail, ca + NT, row_base + pr, &s_full[st]);
        tma_load_2d(sb + 2 * W * NT + TP, &tmap_tail, ca + NT, row_base + prows + pr, &s_full[st]);
    };
    if (x == 0) {
        for (int st = 0; st < kTmaStages; st++) {
            mbar_init(&s_full[st], 1);
            mbar_init(&s_empty[st], NT / 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (x == 0)
        for (int g = 0; g < kTmaStages && g < g_end; g++) issue(g);
    // LB_w = max(S_EQ, S_EC) (Eq. 5) or one sum (Table 3 ablations): max(S_EQ fa, S_EC fb)
    // with fa, fb in {0, 1} (sums are non-negative), times the fp16 ring's
    // unscale factor 2^e (exact), all folded into the two factors
    // SEL = false (P.lbsel == 0, the default): max(S_EQ, S_EC) times the unscale
    // factor once (max(a f, b f) = max(a, b) f for a power of two f > 0, exact),
    // and no multiply at all for float / int32 rings
    const V one = (V)1;
    V fa = P.lbsel == 2 ? (V)0 : one, fb = P.lbsel == 1 ? (V)0 : one;
    if constexpr (std::is_same<PV, __half>::value) {
        fa *= P.post_unscale;
        fb *= P.post_unscale;
    }
    auto pick = [&](V a, V b) -> V {
        if constexpr (SEL) return vmax(a * fa, b * fb);
        else if constexpr (std::is_same<PV, __half>::value) return vmax(a, b) * fa;
        else return vmax(a, b);
    };
    int i0 = 0;  // IQs shorter than W: no full DW (R6), emitted as LB_w = 0 after the rows
    while (i0 < nl && P.len[i0] < W) i0++;
    int g = 0;
    for (int k = 0; k < my_tiles; k++) {
        const int tile = (int)blockIdx.x + k * (int)gridDim.x;
        const int mq = tile / nb, bx = tile - mq * nb;
        // first used at the first emission: the load overlaps the rows
        const MQMeta m = meta[mq];
        const float lsc = P.lb_half ? P.lbs[mq] : 0.f;
        const int64_t Rb = (int64_t)bx * NT - 1;
        const int64_t s0 = (Rb + x + 1) * W;  // e of slot b = 0
        V se[W], sc[W];
#pragma unroll
        for (int b = 0; b < W; b++) se[b] = sc[b] = (V)0;
        // One CSG row: wait for its stage, add this thread's column, release the
        // stage (one CTA barrier per two rows; thread 0 refills both stages).
        auto row = [&](int j) {
            const int st = g & (kTmaStages - 1);
            mbar_wait(&s_full[st], (uint32_t)(g / kTmaStages) & 1u);
            const int nrow = n_sw - j * W;  // SWs of this CSG row (< W only in the last row)
            const int col = (int)(Rb - j);
            const int xo = x + (col & (A - 1));  // this thread's column within the aligned boxes
            const PV *sb = s_ring + (size_t)st * STAGE;
            // main-box columns (all but at most A-1 threads of the last warp) use
            // compile-time row pitches, so the 2W loads take immediate offsets
            if (xo < NT) {
                if (nrow >= W) tma_row_add<V, PV, W, NT, W * NT, true>(sb + xo, nrow, se, sc);
                else tma_row_add<V, PV, W, NT, W * NT, false>(sb + xo, nrow, se, sc);
            } else {
                tma_row_add<V, PV, W, A, TP, false>(sb + 2 * W * NT + (xo - NT), nrow, se, sc);
            }
#if SMILER_TMA_EMPTYBAR
            __syncwarp();
            if ((x & 31) == 0) mbar_arrive(&s_empty[st]);
            if (x == 0 && g + kTmaStages < g_end) {
                mbar_wait(&s_empty[st], (uint32_t)(g / kTmaStages) & 1u);
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                issue(g + kTmaStages);
            }
#else
            if (SMILER_TMA_SYNC2 && kTmaStages >= 4) {
                if ((g & 1) || g + 1 == g_end) {
                    __syncthreads();  // every thread has read the stages of rows g-1, g
                    if (x == 0) {
                        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                        if ((g & 1) && g - 1 + kTmaStages < g_end) issue(g - 1 + kTmaStages);
                        if (g + kTmaStages < g_end) issue(g + kTmaStages);
                    }
                }
            } else {
                __syncthreads();
                if (x == 0 && g + kTmaStages < g_end) {
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                    issue(g + kTmaStages);
                }
            }
#endif
            g++;
        };
        // Rows run in segments ending at the emission rows (lengths ascending):
        // IQ i (q_i = d_i / w, r_i = d_i % w) needs the sums after row q_i - 2
        // (saved in shared memory, slots b > r_i: m_i(b) = q_i - 1) and after row
        // q_i - 1 (slots b <= r_i).  An IQ with the q of the previous one reuses
        // its saved values; q_i = 1 saves the zero sums.
        int j = 0;
        const bool live = bx < m.nblk;  // grids are sized for the longest sensor of the chunk
        for (int i = i0; i < nl; i++) {
            const int qi = P.len[i] / W, ri = P.len[i] % W;
            for (; j < qi; j++) {
                if (j == qi - 1) {
#pragma unroll
                    for (int b = 0; b < W; b++) s_saved[b][x] = pick(se[b], sc[b]);
                }
                row(j);
            }
            if (live) {
                V v[W];
#pragma unroll
                for (int b = 0; b < W; b++) {
                    const V sv = s_saved[b][x];
                    v[b] = b > ri ? sv : pick(se[b], sc[b]);
                }
                diag_emit<V, W>(v, i, s0, m, P, lb, tauc, mq, bx, lsc);
            }
        }
        if (!live) {
            tau_clear(P, mq, NT / 32, 0, P.n_len, tauc, bx);
        } else if (i0 > 0) {
            V z[W];
#pragma unroll
            for (int b = 0; b < W; b++) z[b] = (V)0;
            for (int i = 0; i < i0; i++) diag_emit<V, W>(z, i, s0, m, P, lb, tauc, mq, bx, lsc);
        }
    }
}

// ---------------------------------------------------------------------------
// SMiLer-Dir (ablation, NEXT-4): LB_en(IQ_i, C_t) = max(LB_EQ, LB_EC) over all
// d_i points of the candidate (Thm 4.1; LB_Keogh Eq. 26 with the
// series envelope and the MQ envelope, R4/R20), computed straight from the
// series with no window level -- the "SMiLer-Dir" of Fig. 8 (P:1916-1919,
// P:2094-2097).  Candidates are addressed by their END e = t + d_i: with
// u = 0, 1, ... counted back from the end, the term pair u of every item query
// ending at e is the same (series point e-1-u against MQ position D-1-u, since
// every IQ is a suffix of the MQ), so running sums over u give the
// bound of IQ i as soon as u reaches d_i.  One launch emits the IQs
// [li0, li1): li1 = li0 + 1 is the paper's per-item-query scan
// (SMILER_LB_DIRECT), [0, n_len) shares one pass (SMILER_LB_DIRECT_SHARED).
// Thread x owns the kDirP consecutive ends E0 + x kDirP + p; the CTA stages
// the series (and envelope) range it touches in shared memory with a 4-float
// skew every 32 floats (conflict-free 16-byte loads at an 8-float lane
// stride) and the reversed MQ arrays rq[u] = MQ[D-1-u].  Per chunk of 8 u:
// 16 series values per array and 8 query values per array in registers,
// 8 x 8 term pairs.  Emission reuses diag_emit (slots e = s0 + p, t = e - d_i
// contiguous; tau units are warps).
// ---------------------------------------------------------------------------
constexpr int kDirThreads = 128;
constexpr int kDirP = 8;
constexpr int kDirEnds = kDirThreads * kDirP;  // ends per CTA

__host__ __device__ constexpr int dir_skew(int i) { return i + (i >> 5) * 4; }
// shared memory (elements of V) of lb_direct_kernel for a pass of length dmax
__host__ __device__ inline int dir_tile_len(int dmax) { return kDirEnds + ((dmax + 7) & ~7) + 8; }
__host__ __device__ inline size_t dir_smem_elems(int dmax, int D) {
    return (size_t)3 * dir_skew(dir_tile_len(dmax)) + 3 * (size_t)(((D + 7) & ~7) + 8);
}

template <typename V, bool CHECK>
__device__ __forceinline__ void dir_chunk(const V (&c)[16], const V (&uc)[16], const V (&lc)[16], const V (&q)[8],
                                          const V (&uq)[8], const V (&lq)[8], int ua, int ub, V (&se)[kDirP],
                                          V (&sc)[kDirP]) {
#pragma unroll
    for (int uu = 0; uu < 8; uu++) {
        if (!CHECK || (uu >= ua && uu < ub)) {
#pragma unroll
            for (int p = 0; p < kDirP; p++) {
                const int x = p - uu + 7;  // series point e - 1 - u in the 16-value window
                lb_term(c[x], uq[uu], lq[uu], se[p]);
                lb_term(q[uu], uc[x], lc[x], sc[p]);
            }
        }
    }
}

template <typename S>
__global__ void __launch_bounds__(kDirThreads) lb_direct_kernel(const S *series, const S *UC, const S *LC,
                                                                const MQMeta *meta, const typename Tr<S>::V4 *qtab,
                                                                const QParams P, int li0, int li1,
                                                                typename Tr<S>::V *lb, int32_t *tauc) {
    using V = typename Tr<S>::V;
    using V4 = typename Tr<S>::V4;
    extern __shared__ __align__(16) unsigned char dir_smem[];
    const int D = P.D;
    const int dmax = P.len[li1 - 1];
    const int TL = dir_tile_len(dmax);
    const int DP = TL - kDirEnds;  // tile position of series point E0 is DP
    const int TS = dir_skew(TL);
    const int QL = ((D + 7) & ~7) + 8;
    V *tc = reinterpret_cast<V *>(dir_smem);
    V *tu = tc + TS;
    V *tl = tu + TS;
    V *rq = tl + TS;
    V *ru = rq + QL;
    V *rl = ru + QL;
    const int mq = blockIdx.y;
    const MQMeta m = meta[mq];
    const int64_t E0 = (int64_t)blockIdx.x * kDirEnds;
    if ((int)blockIdx.x >= m.nblk) {  // nblk = n / kDirEnds + 1 (ends 0..n)
        tau_clear(P, mq, kDirThreads / 32, li0, li1, tauc);
        return;
    }
    for (int u = threadIdx.x; u < QL; u += kDirThreads) {
        V a = (V)0, b = (V)0, c = (V)0;
        if (u < D) {
            const V4 e = qtab[(int64_t)mq * D + (D - 1 - u)];
            a = e.x, b = e.y, c = e.z;
        }
        rq[u] = a, ru[u] = b, rl[u] = c;
    }
    const int64_t T0 = E0 - DP;  // series point of tile position 0
#pragma unroll 8
    for (int i = threadIdx.x; i < TL; i += kDirThreads) {
        const int64_t s = T0 + i;
        V a = (V)0, b = (V)0, c = (V)0;
        if (s >= 0 && s < m.n) {
            const int64_t g = m.series_off + s;
            a = (V)series[g], b = (V)UC[g], c = (V)LC[g];
        }
        const int k = dir_skew(i);
        tc[k] = a, tu[k] = b, tl[k] = c;
    }
    __syncthreads();
    const int x = threadIdx.x;
    V se[kDirP], sc[kDirP];
#pragma unroll
    for (int p = 0; p < kDirP; p++) se[p] = sc[p] = (V)0;
    const int64_t s0 = E0 + (int64_t)x * kDirP;  // end e of slot p = 0
    int nexti = li0;
    for (int u0 = 0; u0 < dmax; u0 += 8) {
        // window: tile positions ib .. ib+15 hold series points e0 - 1 - u for the chunk
        const int ib = DP + x * kDirP - u0 - 8;
        V c[16], uc[16], lc[16], q[8], uq[8], lq[8];
#pragma unroll
        for (int g = 0; g < 16; g += 4) {
            const int k = dir_skew(ib + g);
            const V4 a = *reinterpret_cast<const V4 *>(tc + k);
            const V4 b = *reinterpret_cast<const V4 *>(tu + k);
            const V4 d = *reinterpret_cast<const V4 *>(tl + k);
            c[g] = a.x, c[g + 1] = a.y, c[g + 2] = a.z, c[g + 3] = a.w;
            uc[g] = b.x, uc[g + 1] = b.y, uc[g + 2] = b.z, uc[g + 3] = b.w;
            lc[g] = d.x, lc[g + 1] = d.y, lc[g + 2] = d.z, lc[g + 3] = d.w;
        }
#pragma unroll
        for (int g = 0; g < 8; g += 4) {
            const V4 a = *reinterpret_cast<const V4 *>(rq + u0 + g);
            const V4 b = *reinterpret_cast<const V4 *>(ru + u0 + g);
            const V4 d = *reinterpret_cast<const V4 *>(rl + u0 + g);
            q[g] = a.x, q[g + 1] = a.y, q[g + 2] = a.z, q[g + 3] = a.w;
            uq[g] = b.x, uq[g + 1] = b.y, uq[g + 2] = b.z, uq[g + 3] = b.w;
            lq[g] = d.x, lq[g + 1] = d.y, lq[g + 2] = d.z, lq[g + 3] = d.w;
        }
        // split the chunk at item-query lengths (emit when u reaches d_i)
        int ua = 0;
        while (ua < 8) {
            const int dn = nexti < li1 ? P.len[nexti] : 0x7fffffff;
            const int ub = (int)min((int64_t)8, (int64_t)dn - u0);
            if (ua == 0 && ub == 8)
                dir_chunk<V, false>(c, uc, lc, q, uq, lq, 0, 8, se, sc);
            else
                dir_chunk<V, true>(c, uc, lc, q, uq, lq, ua, ub, se, sc);
            if (u0 + ub == dn) {
                V v[kDirP];
#pragma unroll
                for (int p = 0; p < kDirP; p++) v[p] = lbpick(P, se[p], sc[p]);
                diag_emit<V, kDirP>(v, nexti, s0, m, P, lb, tauc, mq);
                nexti++;
            }
            ua = ub;
        }
    }
}
