// dtw.cu -- step a7 (and the DTWs of a5): banded DTW verification.
//
// Recurrence: Eq. 21-24, dist(a,b) = (a-b)^2 (R1).
// The paper's Alg. 2 keeps a compressed 2 x (2rho+2) matrix in
// shared memory per thread.  Here the band lives in REGISTERS: one thread per
// candidate, the 2rho+1 band cells of the current row are a statically indexed
// register array updated in place, rows are the candidate's points c_j and the
// band runs over the item query's points q_i (so q is warp-uniform and c is one
// value per row).  Candidate points are staged 32 rows at a time through
// shared memory as [row][lane] (conflict-free, coalesced loads); the query is
// staged once per task in shared memory and read R rows at a time into
// registers.  Per cell: FADD, FMNMX3, FFMA (f32) or IADD, VIMNMX3, IMAD (int).
// No tensor cores: DTW is a min-plus recurrence, not a contraction.
//
// Band coordinates: row j (1..d) = candidate point c_j, slot u in [0, 2rho]
// = query point i = j + u - rho.  Predecessors of (i, j):
//   (i-1, j)   -> same row, slot u-1      (computed just before)
//   (i-1, j-1) -> previous row, slot u
//   (i, j-1)   -> previous row, slot u+1
// Row 0 is g(0,0) = 0 at slot rho and inf elsewhere (Eq. 22); cells with
// i < 1 or i > d are inf (Eq. 22/23).  For f32 those cells get a query value
// of +inf, which makes every such cell +inf without a mask; for int32 the
// first and last rho rows run a masked variant.
#include <map>
#include <mutex>
#include <type_traits>
#include <utility>

#include "internal.h"

namespace smiler {

#ifndef SMILER_DTW_THREADS
#define SMILER_DTW_THREADS 128  // DTW and cascade CTAs (128: finer register-limited occupancy, +0.1-0.5%; 256 before)
#endif
constexpr int kDtwThreads = SMILER_DTW_THREADS;
constexpr int kDtwWarps = kDtwThreads / 32;
#ifndef SMILER_DTW_KROWS_WIDE
#define SMILER_DTW_KROWS_WIDE 4
#endif
constexpr int kRowsMax = 8;
// rows per register block (interleaved by the scheduler): 4, or the wide-band setting
template <int RHO> constexpr int dtw_krows() { return RHO > 12 ? SMILER_DTW_KROWS_WIDE : 4; }

// Per-warp query staging length (values): d + W + kRowsMax, rounded up to 4.
__host__ __device__ inline int dtw_qstage(int d, int rho) { return (d + 2 * rho + 1 + kRowsMax + 3) & ~3; }

template <typename V> __device__ __forceinline__ V vmin3(V a, V b, V c);
template <> __device__ __forceinline__ float vmin3(float a, float b, float c) {
    return fminf(fminf(a, b), c);
}
template <> __device__ __forceinline__ int32_t vmin3(int32_t a, int32_t b, int32_t c) {
    return min(min(a, b), c);
}
__device__ __forceinline__ float cell(float q, float c, float m) {
    float diff = q - c;
    return fmaf(diff, diff, m);  // R16: pinned
}
__device__ __forceinline__ int32_t cell(int32_t q, int32_t c, int32_t m) {
    int32_t diff = q - c;
    return diff * diff + m;
}
// e(v; U, L) of Eq. 26 accumulated (the same arithmetic as the LB kernels' lb_term)
__device__ __forceinline__ void lb_term(float v, float U, float L, float &acc) {
    const float m = fmaxf(fmaxf(v - U, L - v), 0.0f);
    acc = fmaf(m, m, acc);
}
__device__ __forceinline__ void lb_term(int32_t v, int32_t U, int32_t L, int32_t &acc) {
    const int32_t dd = v - min(max(v, L), U);
    acc += dd * dd;
}
template <typename V> __device__ __forceinline__ uint32_t vbits(V v);
template <> __device__ __forceinline__ uint32_t vbits(float v) { return __float_as_uint(v); }
template <> __device__ __forceinline__ uint32_t vbits(int32_t v) { return (uint32_t)v; }

// One DP row (row index j, 1-based) over the band; qrow[u] = q_{j+u-rho}.
template <typename V, int RHO, bool MASK>
__device__ __forceinline__ void dp_row(V (&band)[2 * RHO + 1], const V *qrow, V cj, int j, int d,
                                       const V INF) {
    constexpr int W = 2 * RHO + 1;
    V left = INF;
#pragma unroll
    for (int u = 0; u < W; u++) {
        V up = (u + 1 < W) ? band[u + 1] : INF;
        V m = vmin3<V>(left, band[u], up);
        V nv = cell(qrow[u], cj, m);
        if (MASK) {
            int i = j + u - RHO;
            nv = (i >= 1 && i <= d) ? nv : INF;
        }
        band[u] = nv;
        left = nv;
    }
}

// Five DP rows j .. j+4 (f32, opts.variant 6) with fp32x2-packed cells: two
// paired-row passes (rows j, j+1 and j+2, j+3) whose step k computes (r, k) and
// (r+1, k-2) -- independent: (r+1, k-2) needs (r+1, k-3), (r, k-2), (r, k-1),
// all from earlier steps -- with one FADD2 and one FFMA2 (per lane exactly q - c
// and fmaf(diff, diff, m), R16: bit-identical to the scalar cell) and one FMNMX3
// each, and one scalar row (j+4), interleaved with a skew of 3
// steps: a pass's step k needs the previous row's slots k and k+1, which
// the stage before writes at its steps k+2 and k+3 (the scalar row's step k:
// k+1 and k+2).  The three stages are independent chains (ILP).  The row carried
// to the next block (j+4) comes from scalar cells: a packed result's halves are
// a register pair, and a long-lived half would pin its pair.  11 instructions
// per 5 cells (2.2) instead of 15 (the unpaired edge cells of each pass run
// scalar).  Measured: the same time as the scalar band (C5 rho = 25: 15% fewer
// instructions, FMA / ALU pipes equally busy, more dispatch and pipe-throttle
// stalls; profiles/r02/ab_dtw_packed.txt), so it is the A/B path, not the default.
// tq[i] = (q_{j+i-rho}, q_{j+i-rho-1}) = (q of (r, k), q of (r+1, k-2)) for
// i = k (pass 1) or k + 2 (pass 2); the scalar row's step u reads
// q_{j+4+u-rho} = tq[u+4].x.  Entries are loaded in groups of
// G, each group AH steps before its first use: ptxas hoists every shared load of
// an unrolled block to its top (the whole table live), so each group's address
// carries a zero computed from a cell value of the step before (a cell is >= 0
// or +inf: its sign bit is 0), which pins the loads in place.  All rows live in
// `band` in place (a slot is overwritten only after its last reader).
#ifndef SMILER_DTW_X2_GROUP
#define SMILER_DTW_X2_GROUP 8  // pair-table entries per load group (even)
#endif
#ifndef SMILER_DTW_X2_AHEAD
#define SMILER_DTW_X2_AHEAD 4  // steps between a group's load and its first use
#endif
constexpr int kX2Rows = 5;
template <int RHO>
__device__ __forceinline__ void dp_rows5(float (&band)[2 * RHO + 1], const float4 *tq, float c0, float c1,
                                         float c2, float c3, float c4, const float INF) {
    constexpr int W = 2 * RHO + 1;
    constexpr int NT = W + 4;  // entries tq[0 .. W + 3]
    constexpr int G = SMILER_DTW_X2_GROUP, AH = SMILER_DTW_X2_AHEAD;
    static_assert(W >= 3, "paired rows need rho >= 1");
    static_assert(G % 2 == 0 && AH >= 1 && AH < G, "load groups");
    float A[W], E[W];  // rows j and j+2
    float2 T[NT + 2];
    const float2 n01 = make_float2(-c0, -c1), n23 = make_float2(-c2, -c3);
    auto load_group = [&](int g0, uint32_t zero) {
        const float4 *p = tq + (g0 >> 1) + zero;
#pragma unroll
        for (int i = 0; i < G; i += 2) {
            if (g0 + i < NT) {
                const float4 v = p[i >> 1];
                T[g0 + i] = make_float2(v.x, v.y);
                T[g0 + i + 1] = make_float2(v.z, v.w);
            }
        }
    };
    // step k of a pass with row r in X, row r+1 written to band, c pair (cA, cB),
    // pair-table offset o (pass 1: 0, pass 2: 2)
    auto step = [&](float (&X)[W], int k, int o, float cA, float cB, const float2 &nc) {
        if (k == 0) {
            X[0] = cell(T[o].x, cA, fminf(band[0], band[1]));
        } else if (k == 1) {
            X[1] = cell(T[o + 1].x, cA, vmin3<float>(X[0], band[1], band[2]));
        } else if (k < W) {
            const float ma = vmin3<float>(X[k - 1], band[k], k + 1 < W ? band[k + 1] : INF);
            const float mb = k >= 3 ? vmin3<float>(band[k - 3], X[k - 2], X[k - 1]) : fminf(X[k - 2], X[k - 1]);
            const float2 dq = __fadd2_rn(T[o + k], nc);
            const float2 r = __ffma2_rn(dq, dq, make_float2(ma, mb));
            X[k] = r.x;
            band[k - 2] = r.y;
        } else if (k == W) {
            band[W - 2] = cell(T[o + W - 1].x, cB, vmin3<float>(band[W - 3], X[W - 2], X[W - 1]));
        } else {
            band[W - 1] = cell(T[o + W].x, cB, fminf(band[W - 2], X[W - 1]));
        }
    };
    // scalar row j+4, step u: left = its slot u-1 (band[u-1], written at step
    // u-1), diag / up = row j+3's slots u, u+1 (band[u], band[u+1])
    float left = INF;
    auto srow = [&](int u) {
        const float nv = cell(T[u + 4].x, c4, vmin3<float>(left, band[u], u + 1 < W ? band[u + 1] : INF));
        band[u] = nv;
        left = nv;
    };
    load_group(0, 0u);
#pragma unroll
    for (int s = 0; s <= W + 7; s++) {
        if (s >= 1 && (s + AH) % G == 0 && s + AH < NT)
            load_group(s + AH, __float_as_uint(A[s - 1 < W ? s - 1 : W - 1]) >> 31);
        if (s <= W + 1) step(A, s, 0, c0, c1, n01);
        if (s >= 3 && s - 3 <= W + 1) step(E, s - 3, 2, c2, c3, n23);
        if (s >= 6 && s - 6 < W) srow(s - 6);
    }
}

#ifndef SMILER_DTW_STAGE_UNROLL
#define SMILER_DTW_STAGE_UNROLL 8  // candidate-row loads in flight per lane before their stores (16: -0.2..0.6%)
#endif
constexpr int kStageUnroll = SMILER_DTW_STAGE_UNROLL;
#ifndef SMILER_DTW_CPASYNC
#define SMILER_DTW_CPASYNC 0  // 1: f32 candidate rows staged with cp.async, double-buffered (measured slower: occupancy)
#endif
// shared-memory row buffers per warp for the candidate staging
#ifndef SMILER_DTW_CPASYNC_MINRHO
#define SMILER_DTW_CPASYNC_MINRHO 1000  // cp.async double buffering only for rho >= this (A/B knob)
#endif
template <typename S, int RHO> constexpr int dtw_cbufs() {
    return (std::is_same<S, float>::value && (SMILER_DTW_CPASYNC || RHO >= SMILER_DTW_CPASYNC_MINRHO)) ? 2 : 1;
}

__device__ __forceinline__ void cp_async4(void *dst, const void *src, bool ok) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"((uint32_t)__cvta_generic_to_shared(dst)),
                 "l"(src), "r"(ok ? 4 : 0)
                 : "memory");
}

#ifndef SMILER_DTW_MINB_WIDE
#define SMILER_DTW_MINB_WIDE 1  // CTAs per SM the compiler must fit for rho > 12 (register cap)
#endif
// X2: f32 rows run in pairs with fp32x2-packed cells (dp_rows2); the query is
// staged as the pair table sqp[e] = (q_{e+1-rho}, q_{e-rho}) (two floats per entry).
#ifndef SMILER_DTW_X2_MINB
#define SMILER_DTW_X2_MINB 1  // CTAs per SM the packed kernels must fit (register cap)
#endif
template <typename S, int RHO, bool X2>
__global__ void __launch_bounds__(kDtwThreads, (X2 ? SMILER_DTW_X2_MINB : RHO > 12 ? SMILER_DTW_MINB_WIDE : 1))
    dtw_kernel(const DtwParams<S> p) {
    using V = typename Tr<S>::V;
    constexpr int W = 2 * RHO + 1;
    constexpr int kRows = dtw_krows<RHO>();
    static_assert(!X2 || (std::is_same<S, float>::value && RHO >= 1 && kRows % 4 == 0), "X2: f32, rho >= 1");
    constexpr int QF = X2 ? 4 : 1;  // floats per staged query entry (X2: two pair tables)
    constexpr bool IS_F = std::is_same<S, float>::value;
    const V INF = Tr<S>::inf();
    extern __shared__ __align__(16) unsigned char dtw_smem[];
    const int lane = threadIdx.x & 31;
    const int wib = threadIdx.x >> 5;
    const int qs = dtw_qstage(p.d, RHO);
    constexpr int NB = dtw_cbufs<S, RHO>();
    constexpr bool ASYNC = NB == 2;
    V *sq = reinterpret_cast<V *>(dtw_smem) + wib * (QF * qs + NB * 32 * 33);
    V (*s_cb)[33] = reinterpret_cast<V (*)[33]>(sq + QF * qs);  // NB buffers of [32][33]
    float2 *sqp = reinterpret_cast<float2 *>(sq);  // X2: the pair table
    const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int nw = (gridDim.x * blockDim.x) >> 5;
    const int total = p.task_off[p.n_mq];
    const int d = p.d;
    int cur_mq = -1;

    for (int task = gw; task < total; task += nw) {
        // segment lookup: largest mq with task_off[mq] <= task
        int lo = 0, hi = p.n_mq;
        while (hi - lo > 1) {
            int mid = (lo + hi) >> 1;
            if (p.task_off[mid] <= task) lo = mid; else hi = mid;
        }
        const int mq = lo;
        const int chunk = task - p.task_off[mq];
        const MQMeta m = p.meta[mq];
        const int seg = mq * p.n_len + p.li;
        int cnt;
        int64_t lbase;
        if (p.mode == 0) {
            cnt = p.LTc;
            lbase = (int64_t)seg * p.LT;
        } else {
            cnt = p.counts[seg];
            lbase = m.seg_off + (int64_t)p.li * m.n;
        }
        const int idx = chunk * 32 + lane;
        const int t = idx < cnt ? p.list[lbase + idx] : -1;

        if (mq != cur_mq) {  // stage IQ_li of this MQ: sq[x] = q_{x-rho+1}
            __syncwarp();
            const V *q = p.qv + (int64_t)mq * p.D + (p.D - d);
            if constexpr (X2) {
                for (int x = lane; x < qs + 1; x += 32) {  // sqp[x] and the shifted copy sqp[qs + x - 1]
                    const int i = x - RHO + 1;
                    const float v1 = (i >= 1 && i <= d) ? q[i - 1] : INF;
                    const float v0 = (i - 1 >= 1 && i - 1 <= d) ? q[i - 2] : INF;
                    if (x < qs) sqp[x] = make_float2(v1, v0);
                    if (x >= 1) sqp[qs + x - 1] = make_float2(v1, v0);
                }
            } else {
                for (int x = lane; x < d + W + kRows; x += 32) {
                    int i = x - RHO + 1;
                    V v = IS_F ? INF : (V)0;
                    if (i >= 1 && i <= d) v = q[i - 1];
                    sq[x] = v;
                }
            }
            cur_mq = mq;
            __syncwarp();
        }

        V band[W];
#pragma unroll
        for (int u = 0; u < W; u++) band[u] = (u == RHO) ? (V)0 : INF;

        const S *cs = p.series + m.series_off;
        // rows j0 .. j0+31 of the warp's 32 candidates -> buf[row][candidate]
        // (f32: asynchronous 4-byte copies, zero-filled outside; one commit group)
        auto stage_async = [&](V (*buf)[33], int j0) {
            const bool in_row = (j0 + lane) < d;
#pragma unroll 4
            for (int l = 0; l < 32; l++) {
                const int tl = __shfl_sync(0xffffffffu, t, l);
                const bool ok = tl >= 0 && in_row;
                cp_async4(&buf[lane][l], ok ? (const void *)(cs + tl + j0 + lane) : (const void *)cs, ok);
            }
            asm volatile("cp.async.commit_group;" ::: "memory");
        };
        if constexpr (ASYNC) stage_async(s_cb, 0);
        for (int j0 = 0, blk = 0; j0 < d; j0 += 32, blk++) {
            V (*s_c)[33] = s_cb + (ASYNC ? (blk & 1) * 32 : 0);
            if constexpr (ASYNC) {
                // the next block streams in while this one is computed
                if (j0 + 32 < d) {
                    stage_async(s_cb + ((blk + 1) & 1) * 32, j0 + 32);
                    asm volatile("cp.async.wait_group 1;" ::: "memory");
                } else {
                    asm volatile("cp.async.wait_group 0;" ::: "memory");
                }
                __syncwarp();
            } else {
                __syncwarp();
                const bool in_row = (j0 + lane) < d;
                // this lane's row of every candidate: cbase[t], one opaque 64-bit base
                // per block (else the address is re-derived in 64 bits per load)
                const S *cbase = cs + (j0 + lane);
                asm("mov.b64 %0, %0;" : "+l"(cbase));
                // kStageUnroll loads in flight before their stores (explicitly
                // batched: the compiler otherwise alternates load / store)
#pragma unroll 1
                for (int l0 = 0; l0 < 32; l0 += kStageUnroll) {
                    S vals[kStageUnroll];
#pragma unroll
                    for (int q = 0; q < kStageUnroll; q++) {
                        const int tl = __shfl_sync(0xffffffffu, t, l0 + q);
                        vals[q] = (tl >= 0 && in_row) ? __ldg(cbase + tl) : (S)0;
                    }
#pragma unroll
                    for (int q = 0; q < kStageUnroll; q++) s_c[lane][l0 + q] = (V)vals[q];
                }
                __syncwarp();
            }
            const int jn = min(32, d - j0);
            int r = 0;
            if constexpr (X2) {
                // blocks of 5 rows from pair-table entry o = j - 1 = j0 + r: the table
                // (even o) or its copy shifted by one entry (odd o), 16-byte aligned
                for (; r + kX2Rows <= jn; r += kX2Rows) {
                    const int o = j0 + r;
                    const float4 *tq = reinterpret_cast<const float4 *>((o & 1) ? sqp + qs + (o - 1) : sqp + o);
                    dp_rows5<RHO>(band, tq, s_c[r][lane], s_c[r + 1][lane], s_c[r + 2][lane], s_c[r + 3][lane],
                                  s_c[r + 4][lane], INF);
                }
                for (; r < jn; r++) {
                    const int j = j0 + r + 1;
                    V qr[W];
#pragma unroll
                    for (int x = 0; x < W; x++) qr[x] = sqp[j - 1 + x].x;
                    dp_row<V, RHO, false>(band, qr, s_c[r][lane], j, d, INF);
                }
            }
            for (; !X2 && r + kRows <= jn; r += kRows) {
                const int j = j0 + r + 1;
                V qr[W + kRows - 1];
#pragma unroll
                for (int x = 0; x < W + kRows - 1; x++) qr[x] = sq[j - 1 + x];
                const bool fast = IS_F || (j - RHO >= 1 && j + kRows - 1 + RHO <= d);
                if (fast) {
#pragma unroll
                    for (int rr = 0; rr < kRows; rr++)
                        dp_row<V, RHO, false>(band, qr + rr, s_c[r + rr][lane], j + rr, d, INF);
                } else {
#pragma unroll
                    for (int rr = 0; rr < kRows; rr++)
                        dp_row<V, RHO, true>(band, qr + rr, s_c[r + rr][lane], j + rr, d, INF);
                }
            }
            for (; !X2 && r < jn; r++) {
                const int j = j0 + r + 1;
                V qr[W];
#pragma unroll
                for (int x = 0; x < W; x++) qr[x] = sq[j - 1 + x];
                dp_row<V, RHO, !IS_F>(band, qr, s_c[r][lane], j, d, INF);
            }
            if constexpr (ASYNC) __syncwarp();  // buffer blk & 1 is refilled two blocks later
        }
        const V dist = band[RHO];
        const uint64_t key = t >= 0 ? (((uint64_t)vbits<V>(dist) << 32) | (uint32_t)t) : kKeyMax;
        if (p.mode == 0) {
            if (idx < cnt) p.keys_out[lbase + idx] = key;
        } else {
            const bool fin = t >= 0 && key <= p.tau_key[seg];
            const unsigned bal = __ballot_sync(0xffffffffu, fin);
            if (bal) {
                int base = 0;
                if (lane == 0) base = atomicAdd(&p.fin_count[seg], __popc(bal));
                base = __shfl_sync(0xffffffffu, base, 0);
                if (fin) p.fin[m.seg_off + (int64_t)p.li * m.n + base + __popc(bal & ((1u << lane) - 1))] = key;
            }
        }
    }
}

// Per-device launch configuration of one dtw_kernel instantiation: the
// shared-memory attribute is a per-device setting and the grid follows the
// device's SM count, so both are kept per device (and guarded: handles on
// different devices / threads are independent).
struct DtwLaunchCfg {
    int occ = 0, sms = 0;
};
template <typename S, int RHO, bool X2>
static DtwLaunchCfg dtw_cfg() {
    using V = typename Tr<S>::V;
    constexpr int NB = dtw_cbufs<S, RHO>();
    constexpr int QF = X2 ? 4 : 1;
    static std::mutex mu;
    static std::map<int, DtwLaunchCfg> per_dev;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lk(mu);
    auto it = per_dev.find(dev);
    if (it != per_dev.end()) return it->second;
    DtwLaunchCfg c;
    cudaFuncSetAttribute(dtw_kernel<S, RHO, X2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)((size_t)kDtwWarps * (QF * dtw_qstage(kMaxD, RHO) + NB * 32 * 33) * sizeof(V)));
    cudaDeviceGetAttribute(&c.sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&c.occ, dtw_kernel<S, RHO, X2>, kDtwThreads,
                                                  (size_t)kDtwWarps * (QF * dtw_qstage(256, RHO) + NB * 32 * 33) * sizeof(V));
    if (c.occ < 1) c.occ = 1;
    if (c.sms < 1) c.sms = 1;
    per_dev[dev] = c;
    return c;
}

template <typename S, int RHO, bool X2>
static void launch_cfg(const DtwParams<S> &p, int grid, cudaStream_t st) {
    using V = typename Tr<S>::V;
    constexpr int NB = dtw_cbufs<S, RHO>();
    constexpr int QF = X2 ? 4 : 1;
    size_t smem = (size_t)kDtwWarps * (QF * dtw_qstage(p.d, RHO) + NB * 32 * 33) * sizeof(V);
    const DtwLaunchCfg c = dtw_cfg<S, RHO, X2>();
    if (grid <= 0) grid = c.sms * c.occ;
    dtw_kernel<S, RHO, X2><<<grid, kDtwThreads, smem, st>>>(p);
}

#ifndef SMILER_DTW_X2_MINRHO
#define SMILER_DTW_X2_MINRHO 4  // f32 bands with rho >= this run the packed row pairs (narrower: the unpaired edge cells dominate)
#endif
template <typename S, int RHO>
static void launch_one(const DtwParams<S> &p, int grid, cudaStream_t st) {
    constexpr bool CAN_X2 = std::is_same<S, float>::value && RHO >= SMILER_DTW_X2_MINRHO && RHO >= 1;
    if constexpr (CAN_X2) {
        if (p.packed) {
            launch_cfg<S, RHO, true>(p, grid, st);
            return;
        }
    }
    launch_cfg<S, RHO, false>(p, grid, st);
}

template <typename S, int... Rs>
static bool dispatch(int rho, const DtwParams<S> &p, int grid, cudaStream_t st,
                     std::integer_sequence<int, Rs...>) {
    bool done = false;
    ((rho == Rs ? (launch_one<S, Rs>(p, grid, st), done = true) : false), ...);
    return done;
}

// ---------------------------------------------------------------------------
// Any rho (the generic path for rho > kMaxRhoFast, and an A/B variant for
// smaller bands): one warp per candidate, anti-diagonal wavefront.  Cells of
// anti-diagonal k = i + j depend only on diagonals k-1 and k-2 (Eq. 21), so
// all of them are computed at once by the warp's lanes.  Indexing the band by
// delta = i - j in [-rho, rho], diagonal k holds the deltas with the parity of
// k, so ONE shared array g[delta] suffices: while diagonal k is computed, the
// slots of the other parity hold diagonal k-1 (the (i-1, j) and (i, j-1)
// predecessors at delta -/+ 1) and its own slots still hold diagonal k-2 (the
// (i-1, j-1) predecessor at delta) -- each cell reads only slots no lane writes
// in this step.  Only valid cells (1 <= i, j <= d, |i - j| <= rho) are
// computed; every read of a never-written slot is the boundary g(0, j) =
// g(i, 0) = inf of Eq. 22, and g[0] starts as g(0, 0) = 0.  The cell is the
// register-band kernel's (f32: fmaf(q - c, q - c, min3), R16), so results are
// bit-identical to it and to the oracle.  The item query and the candidate
// are staged per warp in shared memory.
// ---------------------------------------------------------------------------
constexpr int kWaveWarps = 4;
__host__ __device__ inline int wave_pad(int n) { return (n + 3) & ~3; }
// per-warp shared elements: q [d] | c [d] | g [2 rho + 1]
__host__ __device__ inline size_t wave_smem_elems(int d, int rho) {
    return (size_t)wave_pad(d) * 2 + wave_pad(2 * rho + 1);
}

template <typename S>
__global__ void __launch_bounds__(kWaveWarps * 32) dtw_wave_kernel(const DtwParams<S> p, int rho) {
    using V = typename Tr<S>::V;
    const V INF = Tr<S>::inf();
    extern __shared__ __align__(16) unsigned char wv_smem[];
    const int lane = threadIdx.x & 31;
    const int wib = threadIdx.x >> 5;
    const int d = p.d;
    V *sq = reinterpret_cast<V *>(wv_smem) + (size_t)wib * wave_smem_elems(d, rho);  // q_i at sq[i - 1]
    V *sc = sq + wave_pad(d);                                                        // c_j at sc[j - 1]
    V *g = sc + wave_pad(d);                                                         // g[delta + rho]
    const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int nw = (gridDim.x * blockDim.x) >> 5;
    const int total = p.task_off[p.n_mq];
    int cur_mq = -1;
    for (int task = gw; task < total; task += nw) {
        int lo = 0, hi = p.n_mq;
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (p.task_off[mid] <= task) lo = mid; else hi = mid;
        }
        const int mq = lo;
        const int chunk = task - p.task_off[mq];
        const MQMeta m = p.meta[mq];
        const int seg = mq * p.n_len + p.li;
        int cnt;
        int64_t lbase;
        if (p.mode == 0) {
            cnt = p.LTc;
            lbase = (int64_t)seg * p.LT;
        } else {
            cnt = p.counts[seg];
            lbase = m.seg_off + (int64_t)p.li * m.n;
        }
        const int idx = chunk * 32 + lane;
        const int my_t = idx < cnt ? p.list[lbase + idx] : -1;
        if (mq != cur_mq) {
            __syncwarp();
            const V *q = p.qv + (int64_t)mq * p.D + (p.D - d);
            for (int x = lane; x < d; x += 32) sq[x] = q[x];
            cur_mq = mq;
        }
        const S *cs = p.series + m.series_off;
        V my_dist = INF;
        for (int l = 0; l < 32; l++) {  // the task's candidates, one per pass of the warp
            const int t = __shfl_sync(0xffffffffu, my_t, l);
            if (t < 0) continue;  // warp-uniform
            __syncwarp();
            for (int x = lane; x < d; x += 32) sc[x] = (V)__ldg(cs + t + x);
            for (int x = lane; x < 2 * rho + 1; x += 32) g[x] = x == rho ? (V)0 : INF;
            __syncwarp();
            for (int k = 2; k <= 2 * d; k++) {
                // valid deltas of diagonal k: |delta| <= rho, 1 <= (k + delta) / 2 <= d,
                // 1 <= (k - delta) / 2 <= d, delta = k (mod 2)
                int dlo = max(-rho, max(2 - k, k - 2 * d));
                const int dhi = min(rho, min(2 * d - k, k - 2));
                dlo += (dlo - k) & 1;
                for (int delta = dlo + 2 * lane; delta <= dhi; delta += 64) {
                    const int i = (k + delta) >> 1, j = (k - delta) >> 1;
                    const V up = delta - 1 >= -rho ? g[delta - 1 + rho] : INF;  // (i-1, j)
                    const V lf = delta + 1 <= rho ? g[delta + 1 + rho] : INF;   // (i, j-1)
                    const V dg = g[delta + rho];                                // (i-1, j-1)
                    g[delta + rho] = cell(sq[i - 1], sc[j - 1], vmin3<V>(up, lf, dg));
                }
                __syncwarp();
            }
            const V dist = g[rho];  // (d, d)
            if (lane == l) my_dist = dist;
        }
        const uint64_t key = my_t >= 0 ? (((uint64_t)vbits<V>(my_dist) << 32) | (uint32_t)my_t) : kKeyMax;
        if (p.mode == 0) {
            if (idx < cnt) p.keys_out[lbase + idx] = key;
        } else {
            const bool fin = my_t >= 0 && key <= p.tau_key[seg];
            const unsigned bal = __ballot_sync(0xffffffffu, fin);
            if (bal) {
                int base = 0;
                if (lane == 0) base = atomicAdd(&p.fin_count[seg], __popc(bal));
                base = __shfl_sync(0xffffffffu, base, 0);
                if (fin) p.fin[m.seg_off + (int64_t)p.li * m.n + base + __popc(bal & ((1u << lane) - 1))] = key;
            }
        }
    }
}

template <typename S>
static void launch_wave(int rho, const DtwParams<S> &p, int grid, cudaStream_t st) {
    using V = typename Tr<S>::V;
    static std::mutex mu;
    static std::map<int, int> sms_of;  // device -> SM count
    int dev = 0;
    cudaGetDevice(&dev);
    int sms;
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = sms_of.find(dev);
        if (it == sms_of.end()) {
            int n = 0;
            cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
            cudaFuncSetAttribute(dtw_wave_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)(kWaveWarps * wave_smem_elems(kMaxD, kMaxD) * sizeof(V)));
            it = sms_of.emplace(dev, n > 0 ? n : 1).first;
        }
        sms = it->second;
    }
    const size_t smem = kWaveWarps * wave_smem_elems(p.d, rho) * sizeof(V);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, dtw_wave_kernel<S>, kWaveWarps * 32, smem);
    if (grid <= 0) grid = sms * (occ > 0 ? occ : 1);
    dtw_wave_kernel<S><<<grid, kWaveWarps * 32, smem, st>>>(p, rho);
}

template <typename S> void launch_dtw(int rho, const DtwParams<S> &p, int grid, cudaStream_t st) {
    if (p.wave || rho > kMaxRhoFast) {
        launch_wave<S>(rho, p, grid, st);
        return;
    }
    dispatch<S>(rho, p, grid, st, std::make_integer_sequence<int, kMaxRhoFast + 1>{});
}

// ---------------------------------------------------------------------------
// LB_Keogh cascade (between a6 and a7).  The index bound LB_w (Thm 4.3) uses the
// master query's envelope of width rho_max for every item query (R4, R20) and
// only the candidate's full disjoint windows; LB_EQ(IQ_i, C_t) with IQ_i's own
// envelope of width rho_i over all d_i points (Eq. 26, Keogh's bound for band
// rho_i) is another lower bound of the same DTW, tighter for the short
// item queries.  A survivor whose LB_EQ exceeds the admission threshold cannot be
// among the k nearest (the same argument as the filter), so it is
// dropped before its DTW.  Warp task = 32 survivors (one per lane), candidate
// rows staged through shared memory exactly as the DTW kernel stages them; the
// warp stops early once every lane's partial sum exceeds the threshold.
// ---------------------------------------------------------------------------
#ifndef SMILER_CASC_STAGE_UNROLL
#define SMILER_CASC_STAGE_UNROLL 16  // cascade candidate loads in flight per lane
#endif
constexpr int kCascUnroll = SMILER_CASC_STAGE_UNROLL;
template <typename S>
__global__ void __launch_bounds__(kDtwThreads) cascade_kernel(const CascadeParams<S> p) {
    using V = typename Tr<S>::V;
    using V2 = typename Tr<S>::V2;
    extern __shared__ __align__(16) unsigned char cz_smem[];
    const int lane = threadIdx.x & 31;
    const int wib = threadIdx.x >> 5;
    const int d = p.d;
    V2 *senv = reinterpret_cast<V2 *>(cz_smem) + (size_t)wib * (d + 32 * 33 / 2 + 1);
    V (*s_c)[33] = reinterpret_cast<V (*)[33]>(senv + d);
    const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int nw = (gridDim.x * blockDim.x) >> 5;
    const int total = p.task_off[p.n_mq];
    int cur_mq = -1;
    for (int task = gw; task < total; task += nw) {
        int lo = 0, hi = p.n_mq;
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (p.task_off[mid] <= task) lo = mid; else hi = mid;
        }
        const int mq = lo;
        const int chunk = task - p.task_off[mq];
        const MQMeta m = p.meta[mq];
        const int seg = mq * p.n_len + p.li;
        const int cnt = p.counts[seg];
        const int64_t lbase = m.seg_off + (int64_t)p.li * m.n;
        const int idx = chunk * 32 + lane;
        const int t = idx < cnt ? p.list[lbase + idx] : -1;
        V thr;
        if constexpr (std::is_same<V, float>::value) thr = __uint_as_float(p.thr[seg]);
        else thr = (int32_t)p.thr[seg];
        if (mq != cur_mq) {  // IQ_li's own envelope, positions D - d .. D - 1
            __syncwarp();
            const V2 *e = p.qenv + ((int64_t)mq * p.n_len + p.li) * p.D + (p.D - d);
            for (int x = lane; x < d; x += 32) senv[x] = e[x];
            cur_mq = mq;
        }
        const S *cs = p.series + m.series_off;
        V acc = (V)0;
        for (int j0 = 0; j0 < d; j0 += 32) {
            __syncwarp();
            const bool in_row = (j0 + lane) < d;
            // this lane's row of every candidate: cbase[t] (one 64-bit base per
            // block; per load a shuffle, a predicate and a 32-bit offset)
            const S *cbase = cs + (j0 + lane);
            asm("mov.b64 %0, %0;" : "+l"(cbase));  // opaque: no per-load re-derivation of the 64-bit address
#pragma unroll 1
            for (int l0 = 0; l0 < 32; l0 += kCascUnroll) {
                S vals[kCascUnroll];
#pragma unroll
                for (int q = 0; q < kCascUnroll; q++) {
                    const int tl = __shfl_sync(0xffffffffu, t, l0 + q);
                    vals[q] = (tl >= 0 && in_row) ? __ldg(cbase + tl) : (S)0;
                }
#pragma unroll
                for (int q = 0; q < kCascUnroll; q++) s_c[lane][l0 + q] = (V)vals[q];
            }
            __syncwarp();
            const int jn = min(32, d - j0);
            for (int r = 0; r < jn; r++) {
                const V2 e = senv[j0 + r];  // (U, L) at IQ position j0 + r
                lb_term(s_c[r][lane], e.x, e.y, acc);
            }
            if (__all_sync(0xffffffffu, t < 0 || acc > thr)) break;  // every lane's bound already exceeds it
        }
        const bool keep = t >= 0 && acc <= thr;
        const unsigned bal = __ballot_sync(0xffffffffu, keep);
        if (bal) {
            int base = 0;
            if (lane == 0) base = atomicAdd(&p.out_counts[seg], __popc(bal));
            base = __shfl_sync(0xffffffffu, base, 0);
            if (keep) p.out_list[lbase + base + __popc(bal & ((1u << lane) - 1))] = t;
        }
    }
}

template <typename S> void launch_cascade(const CascadeParams<S> &p, cudaStream_t st) {
    using V = typename Tr<S>::V;
    using V2 = typename Tr<S>::V2;
    static std::mutex mu;
    static std::map<int, int> sms_of;
    int dev = 0;
    cudaGetDevice(&dev);
    int sms;
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = sms_of.find(dev);
        if (it == sms_of.end()) {
            int n = 0;
            cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
            cudaFuncSetAttribute(cascade_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)((size_t)kDtwWarps * (kMaxD * sizeof(V2) + (32 * 33 + 2) * sizeof(V))));
            it = sms_of.emplace(dev, n > 0 ? n : 1).first;
        }
        sms = it->second;
    }
    const size_t smem = (size_t)kDtwWarps * (p.d + 32 * 33 / 2 + 1) * sizeof(V2);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, cascade_kernel<S>, kDtwThreads, smem);
    cascade_kernel<S><<<sms * (occ > 0 ? occ : 1), kDtwThreads, smem, st>>>(p);
}

template void launch_cascade<int16_t>(const CascadeParams<int16_t> &, cudaStream_t);
template void launch_cascade<float>(const CascadeParams<float> &, cudaStream_t);

template void launch_dtw<int16_t>(int, const DtwParams<int16_t> &, int, cudaStream_t);
template void launch_dtw<float>(int, const DtwParams<float> &, int, cudaStream_t);

}  // namespace smiler
