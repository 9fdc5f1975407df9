// kernels.cuh -- steps a1-a6, a8, a9 of the Search Step.
// Included once, by smiler.cu.  DTW (a5/a7) is in dtw.cu.
#pragma once
#include <cuda.h>
#include <cuda_fp16.h>
#include <stdint.h>

#include <type_traits>

#include "internal.h"

namespace smiler {

// ---------------------------------------------------------------------------
// Small device helpers
// ---------------------------------------------------------------------------
template <typename V> __device__ __forceinline__ uint32_t key_bits(V v);
template <> __device__ __forceinline__ uint32_t key_bits(float v) { return __float_as_uint(v); }
template <> __device__ __forceinline__ uint32_t key_bits(int32_t v) { return (uint32_t)v; }

// e(v; U, L) of Eq. 26 accumulated: (v - clamp(v, L, U))^2.
__device__ __forceinline__ void lb_term(float v, float U, float L, float &acc) {
    // (v - clamp(v, L, U))^2 = max(v - U, L - v, 0)^2 (U >= L): bit-identical,
    // one FMNMX3 on the ALU pipe and FADD, FADD, FFMA on the FMA pipe
    const float m = fmaxf(fmaxf(v - U, L - v), 0.0f);
    acc = fmaf(m, m, acc);
}
// clamp form: 2 FMNMX (ALU pipe) + FADD + FFMA (FMA pipe); same value as lb_term
__device__ __forceinline__ void lb_term_clamp(float v, float U, float L, float &acc) {
    const float dd = v - fminf(fmaxf(v, L), U);
    acc = fmaf(dd, dd, acc);
}
__device__ __forceinline__ void lb_term_clamp(int32_t v, int32_t U, int32_t L, int32_t &acc) {
    const int32_t dd = v - min(max(v, L), U);
    acc += dd * dd;
}
__device__ __forceinline__ void lb_term(int32_t v, int32_t U, int32_t L, int32_t &acc) {
    int32_t dd = v - min(max(v, L), U);
    acc += dd * dd;
}
__device__ __forceinline__ float vmax(float a, float b) { return fmaxf(a, b); }
__device__ __forceinline__ int32_t vmax(int32_t a, int32_t b) { return max(a, b); }

__device__ __forceinline__ uint64_t warp_min_u64(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        uint64_t x = __shfl_xor_sync(0xffffffffu, v, o);
        v = x < v ? x : v;
    }
    return v;
}

// Block-wide min of a uint64 (blockDim.x multiple of 32, <= 1024).
__device__ __forceinline__ uint64_t block_min_u64(uint64_t v, uint64_t *s_red) {
    v = warp_min_u64(v);
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    __syncthreads();
    if (lane == 0) s_red[wid] = v;
    __syncthreads();
    if (wid == 0) {
        uint64_t x = lane < nw ? s_red[lane] : kKeyMax;
        x = warp_min_u64(x);
        if (lane == 0) s_red[0] = x;
    }
    __syncthreads();
    return s_red[0];
}

// Exclusive block scan of int (returns exclusive prefix; *total gets the sum).
__device__ __forceinline__ int block_excl_scan(int v, int *s_scan, int *total) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    int x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    __syncthreads();
    if (lane == 31) s_scan[wid] = x;
    __syncthreads();
    if (wid == 0) {
        int w = lane < nw ? s_scan[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int y = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += y;
        }
        if (lane < nw) s_scan[lane] = w;  // inclusive warp totals
    }
    __syncthreads();
    const int before = wid > 0 ? s_scan[wid - 1] : 0;
    *total = s_scan[nw - 1];
    return before + x - v;
}

// Bitonic sort of n (power of two) uint64 keys in shared memory, ascending.
__device__ void bitonic_sort_smem(uint64_t *s, int n) {
    for (int size = 2; size <= n; size <<= 1) {
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            __syncthreads();
            for (int i = threadIdx.x; i < (n >> 1); i += blockDim.x) {
                int lo = 2 * i - (i & (stride - 1));
                int hi = lo + stride;
                bool asc = ((lo & size) == 0);
                uint64_t a = s[lo], b = s[hi];
                if ((a > b) == asc) {
                    s[lo] = b;
                    s[hi] = a;
                }
            }
        }
    }
    __syncthreads();
}

// k-th smallest (1-based) of keys[0..n) (global memory), keys unique except
// kKeyMax padding; returns kKeyMax if fewer than k keys are < kKeyMax.
// MSB radix select, 8 bits per pass, one CTA.  s_hist: 256 ints.
__device__ uint64_t block_radix_kth(const uint64_t *keys, int64_t n, int k, int *s_hist,
                                    uint64_t *s_bcast) {
    uint64_t prefix = 0, mask = 0;
    int krem = k;
    for (int shift = 56; shift >= 0; shift -= 8) {
        for (int i = threadIdx.x; i < 256; i += blockDim.x) s_hist[i] = 0;
        __syncthreads();
        for (int64_t i = threadIdx.x; i < n; i += blockDim.x) {
            uint64_t x = keys[i];
            if (x != kKeyMax && (x & mask) == prefix) atomicAdd(&s_hist[(x >> shift) & 255], 1);
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            int acc = 0, dsel = -1;
            for (int dg = 0; dg < 256; dg++) {
                if (acc + s_hist[dg] >= krem) {
                    dsel = dg;
                    break;
                }
                acc += s_hist[dg];
            }
            if (dsel < 0) {
                s_bcast[0] = kKeyMax;  // fewer than k keys
            } else {
                s_bcast[0] = prefix | ((uint64_t)dsel << shift);
                s_bcast[1] = (uint64_t)(krem - acc);
            }
        }
        __syncthreads();
        if (s_bcast[0] == kKeyMax) return kKeyMax;
        prefix = s_bcast[0];
        krem = (int)s_bcast[1];
        mask |= (uint64_t)255 << shift;
        __syncthreads();
    }
    return prefix;
}

// ---------------------------------------------------------------------------
// a1: envelope E(C) = (U, L), Def. B.1 / Eq. 25, clipped to the
// sensor (R3).  grid (tiles, sensors); each CTA stages tile + 2 rho halo of
// one sensor in shared memory.
// ---------------------------------------------------------------------------
constexpr int kEnvTile = 2048;

template <typename S>
__global__ void __launch_bounds__(256) envelope_kernel(const S *series, const int64_t *soff,
                                                      const int64_t *slen, int rho, S *U, S *L) {
    extern __shared__ __align__(16) unsigned char env_smem[];
    S *tile = reinterpret_cast<S *>(env_smem);
    const int s = blockIdx.y;
    const int64_t n = slen[s];
    const int64_t x0 = (int64_t)blockIdx.x * kEnvTile;
    if (x0 >= n) return;
    const S *c = series + soff[s];
    const int span = kEnvTile + 2 * rho;
    for (int i = threadIdx.x; i < span; i += blockDim.x) {
        int64_t x = x0 - rho + i;
        tile[i] = (x >= 0 && x < n) ? c[x] : (S)0;
    }
    __syncthreads();
    for (int i = threadIdx.x; i < kEnvTile; i += blockDim.x) {
        int64_t x = x0 + i;
        if (x >= n) break;
        int64_t lo = x - rho < 0 ? 0 : x - rho;
        int64_t hi = x + rho > n - 1 ? n - 1 : x + rho;
        S mx = tile[lo - (x0 - rho)], mn = mx;
        for (int64_t y = lo + 1; y <= hi; y++) {
            S v = tile[y - (x0 - rho)];
            mx = v > mx ? v : mx;
            mn = v < mn ? v : mn;
        }
        U[soff[s] + x] = mx;
        L[soff[s] + x] = mn;
    }
}

// ---------------------------------------------------------------------------
// a2: query prep.  One CTA per MQ: MQ values in the arithmetic type (qv) and
// the table {q, U(Q), L(Q), 0} with the MQ envelope of width rho_env clipped
// to the MQ (R3, R4, R20).  Also:
//  * I16: every value must satisfy |q| <= 1023 (R17); a violation sets *qflag
//    (host-mapped) and the value is clamped so no later sum can overflow.
//  * lbs[mq] = the fp16 storage scale of this MQ's bounds (R26): every LB is
//    a sum of at most D terms, each at most (max|q| + max|x|)^2 (both values
//    and both envelopes lie within [-max, max]).
// ---------------------------------------------------------------------------
template <typename S>
__global__ void __launch_bounds__(256) query_prep_kernel(const S *queries, int D, int rho,
                                                        typename Tr<S>::V *qv,
                                                        typename Tr<S>::V4 *qtab, float smax,
                                                        float *lbs, int *qflag, const IQTab tab, int n_len,
                                                        typename Tr<S>::V2 *qenv) {
    using V = typename Tr<S>::V;
    using V4 = typename Tr<S>::V4;
    __shared__ V s[kMaxD];
    __shared__ float s_max[8];
    const int mq = blockIdx.x;
    float amax = 0.0f;
    for (int p = threadIdx.x; p < D; p += blockDim.x) {
        V v = (V)queries[(int64_t)mq * D + p];
        if constexpr (std::is_same<S, int16_t>::value) {
            if (v > 1023 || v < -1023) {
                if (qflag) atomicOr(qflag, 1);
                v = v > 1023 ? 1023 : -1023;
            }
        }
        s[p] = v;
        qv[(int64_t)mq * D + p] = v;
        amax = fmaxf(amax, fabsf((float)v));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) amax = fmaxf(amax, __shfl_xor_sync(0xffffffffu, amax, o));
    if ((threadIdx.x & 31) == 0) s_max[threadIdx.x >> 5] = amax;
    __syncthreads();
    if (lbs && threadIdx.x == 0) {
        float m = 0.0f;
        for (int x = 0; x < (int)(blockDim.x >> 5); x++) m = fmaxf(m, s_max[x]);
        const double a = (double)m + (double)smax;
        lbs[mq] = fp16_fit_scale((double)D * a * a);
    }
    for (int p = threadIdx.x; p < D; p += blockDim.x) {
        int lo = p - rho < 0 ? 0 : p - rho;
        int hi = p + rho > D - 1 ? D - 1 : p + rho;
        V mx = s[lo], mn = s[lo];
        for (int y = lo + 1; y <= hi; y++) {
            mx = s[y] > mx ? s[y] : mx;
            mn = s[y] < mn ? s[y] : mn;
        }
        V4 e;
        e.x = s[p];
        e.y = mx;
        e.z = mn;
        e.w = (V)0;
        qtab[(int64_t)mq * D + p] = e;
    }
    // the cascade's item-query envelopes: IQ_i = MQ[D - d_i, D) with width rho_i,
    // clipped to the item query (Eq. 25 over IQ_i itself, R3)
    if (qenv) {
        for (int i = 0; i < n_len; i++) {
            const int a = D - tab.len[i], r = tab.rho[i];
            typename Tr<S>::V2 *o = qenv + ((int64_t)mq * n_len + i) * D;
            for (int p = a + threadIdx.x; p < D; p += blockDim.x) {
                const int lo = p - r < a ? a : p - r;
                const int hi = p + r > D - 1 ? D - 1 : p + r;
                V mx = s[lo], mn = s[lo];
                for (int y = lo + 1; y <= hi; y++) {
                    mx = s[y] > mx ? s[y] : mx;
                    mn = s[y] < mn ? s[y] : mn;
                }
                typename Tr<S>::V2 e2;
                e2.x = mx;
                e2.y = mn;
                o[p] = e2;
            }
        }
    }
}

#include "lb.cuh"

// ---------------------------------------------------------------------------
// a5 (second half): tau_i = k-th smallest (DTW, t) key of the verified tau set
// (an upper bound on the k-th NN distance: k candidates lie at or below it;
// reading R8).  One CTA per segment (mq, i).  thr = the LB_w admission bound:
// int: dist; f32: dist * (1 + 2^-10) rounded up (R16 rounding slack).
// no candidates enough -> key max / thr = +inf (no pruning).
// ---------------------------------------------------------------------------
// LB admission bound of a threshold key: int: the distance; f32: distance x
// (1 + 2^-10) rounded up (R16 rounding slack); no key -> no pruning.
template <typename V> __device__ __forceinline__ uint32_t thr_from_key(uint64_t key) {
    if (key == kKeyMax) return std::is_same<V, float>::value ? 0x7f800000u : 0x7FFFFFFFu;
    const uint32_t db = (uint32_t)(key >> 32);
    if constexpr (std::is_same<V, float>::value)
        return __float_as_uint(__fmul_ru(__uint_as_float(db), 1.0f + 1.0f / 1024.0f));
    else
        return db;
}

template <typename S>
__global__ void __launch_bounds__(256) tau_select_kernel(const uint64_t *tauk, int LTs, int LT, int k,
                                                        uint64_t *tau_key, uint32_t *thr) {
    // LTs: list stride per segment; LT: entries in use (the verified tau list)
    using V = typename Tr<S>::V;
    __shared__ int s_hist[256];
    __shared__ uint64_t s_b[2];
    __shared__ uint64_t s_keys[kSortCap];
    __shared__ int s_scan[32];
    const int seg = blockIdx.x;
    const uint64_t *src = tauk + (int64_t)seg * LTs;
    uint64_t kth;
    if (LT <= kSortCap) {
        // sort, then the k-th DISTINCT key: the tau list may hold a candidate twice
        // (a tile candidate that is also a shifted previous neighbour), and a
        // duplicate must not count twice (k distinct candidates at or below tau)
        int n2 = 1;
        while (n2 < LT) n2 <<= 1;
        for (int x = threadIdx.x; x < n2; x += blockDim.x) s_keys[x] = x < LT ? src[x] : kKeyMax;
        bitonic_sort_smem(s_keys, n2);
        const int per = (n2 + blockDim.x - 1) / blockDim.x;
        const int x0 = threadIdx.x * per;
        int cnt = 0;
        for (int x = x0; x < min(x0 + per, n2); x++)
            cnt += (s_keys[x] != kKeyMax && (x == 0 || s_keys[x] != s_keys[x - 1]));
        int total;
        int before = block_excl_scan(cnt, s_scan, &total);
        if (threadIdx.x == 0) s_b[0] = kKeyMax;
        __syncthreads();
        if (total >= k) {
            for (int x = x0; x < min(x0 + per, n2); x++) {
                const bool first = s_keys[x] != kKeyMax && (x == 0 || s_keys[x] != s_keys[x - 1]);
                if (first) {
                    if (before == k - 1) s_b[0] = s_keys[x];
                    before++;
                }
            }
        }
        __syncthreads();
        kth = s_b[0];
    } else {
        kth = block_radix_kth(src, LT, k, s_hist, s_b);  // tile candidates only: unique
    }
    if (threadIdx.x == 0) {
        tau_key[seg] = kth;
        thr[seg] = thr_from_key<V>(kth);
    }
}

// ---------------------------------------------------------------------------
// NEXT-2: running threshold shared by the shards of one search (smiler_knn_opts
// .shared_tau).  Each segment's local threshold key becomes global (t + origin),
// is atomically min'ed into the shared entry (system scope: the entry may live
// on a peer GPU), and the minimum read back -- an upper bound of the k-th NN
// key of the whole search, since every shard's key is one -- is converted back
// to this shard's local coordinates: local key <= result  <=>  global key <= g.
// ---------------------------------------------------------------------------
template <typename S>
__global__ void tau_share_kernel(uint64_t *tau_key, uint32_t *thr, unsigned long long *shared, const MQMeta *meta,
                                 int n_len, int nseg) {
    using V = typename Tr<S>::V;
    const int seg = blockIdx.x * blockDim.x + threadIdx.x;
    if (seg >= nseg) return;
    const int64_t origin = meta[seg / n_len].origin;
    const uint64_t k = tau_key[seg];
    uint64_t g;
    if (k != kKeyMax) {
        const uint64_t kg = (k & 0xFFFFFFFF00000000ull) | (uint32_t)((k & 0xFFFFFFFFull) + (uint64_t)origin);
        const uint64_t old = atomicMin_system(shared + seg, (unsigned long long)kg);
        g = old < kg ? old : kg;
    } else {
        g = atomicMin_system(shared + seg, (unsigned long long)kKeyMax);  // read
    }
    uint64_t loc = g;
    if (g != kKeyMax) {
        const uint64_t gt = g & 0xFFFFFFFFull;
        if (gt >= (uint64_t)origin) loc = (g & 0xFFFFFFFF00000000ull) | (gt - (uint64_t)origin);
        else loc = (g & 0xFFFFFFFF00000000ull) - 1;  // same distance, smaller global t: none of ours ties
    }
    if (loc < k) {
        tau_key[seg] = loc;
        thr[seg] = thr_from_key<V>(loc);
    }
}

// ---------------------------------------------------------------------------
// a6: filtering: keep t with LB_w(t) <= thr_i (ties survive).
// Two-phase filter-then-verify keeps warps homogeneous.
// grid (tiles, segments); block-aggregated compaction, one atomic per CTA.
// ---------------------------------------------------------------------------
constexpr int kFiltThreads = 256;
#ifndef SMILER_FILT_ITEMS
#define SMILER_FILT_ITEMS 64  // candidates per thread (multiple of 8, <= 64; 32: C2 filter 0.451 -> 0.462 ms, C4 1.94 -> 2.05 ms)
#endif
constexpr int kFiltItems = SMILER_FILT_ITEMS;
static_assert(kFiltItems % 8 == 0 && kFiltItems <= 64, "filter items per thread");
using FiltFlags = typename std::conditional<(kFiltItems > 32), unsigned long long, uint32_t>::type;

// LH: the LB_w array holds fp16 rounded down (P.lb_half); the comparison is
// then made in float against the threshold rounded up, which keeps a superset
// of the candidates with LB_w <= tau (every survivor is verified exactly).
// fp16 rows are read with 16-byte loads from the aligned address at or below the
// block's first t (a block covers kFiltSpanH candidates, so 1024 vectors of 8
// cover it for any alignment); halves outside the block's range are masked.
constexpr int kFiltSpanH = kFiltThreads * kFiltItems - 8;
template <typename S, bool LH>
__global__ void __launch_bounds__(kFiltThreads) filter_kernel(const typename Tr<S>::V *lb,
                                                             const MQMeta *meta, const QParams P,
                                                             const uint32_t *thr, int32_t *surv,
                                                             int32_t *surv_count) {
    using V = typename Tr<S>::V;
    __shared__ int s_scan[32];
    __shared__ int s_base;
    const int seg = blockIdx.y;
    const int mq = seg / P.n_len, i = seg % P.n_len;
    const MQMeta m = meta[mq];
    const int d = P.len[i];
    const int64_t tb = m.t_lo > 0 ? m.t_lo : 0;
    const int64_t te = min(m.t_hi, m.n - m.hz - d + 1);
    const int span = LH ? kFiltSpanH : kFiltThreads * kFiltItems;
    const int64_t t0 = tb + (int64_t)blockIdx.x * span;
    if (t0 >= te) return;
    const int64_t t1 = min(te, t0 + span);
    const uint32_t th = thr[seg];
    FiltFlags flags = 0;
    int64_t ta = 0;  // LH: t of the first half of the block's aligned window
    if constexpr (LH) {
        float thf;
        if constexpr (std::is_same<V, float>::value)
            thf = __uint_as_float(th);
        else
            thf = __int2float_ru((int32_t)th);
        // stored h = rd(LB x scale): h <= tau x scale (exact power-of-two product,
        // rounded up if it underflows)  <=>  h <= that rounded up to fp16 (h is an
        // fp16 value); the +inf threshold of "no pruning" stays +inf
        const __half2 th2 = __half2half2(__float2half_ru(__fmul_ru(thf, P.lbs[mq])));
        const __half *row = reinterpret_cast<const __half *>(lb) + m.seg_off + (int64_t)i * m.n;
        const uintptr_t a0 = reinterpret_cast<uintptr_t>(row + t0);
        const int4 *vb = reinterpret_cast<const int4 *>(a0 & ~(uintptr_t)15);
        ta = t0 - (int64_t)((a0 & 15) >> 1);
        const int r0 = (int)(t0 - ta), r1 = (int)(t1 - ta);  // block range relative to ta (< 2^31)
        // all vector loads of the thread first (4 x 16 B in flight), then the compares
        constexpr int NV = kFiltItems / 8;
        int4 rawv[NV];
#pragma unroll
        for (int it = 0; it < NV; it++) {
            const int vi = it * kFiltThreads + threadIdx.x;
            const int rv = vi * 8;
            rawv[it] = (rv < r1 && rv + 8 > r0) ? __ldg(vb + vi) : make_int4(0, 0, 0, 0);
        }
#pragma unroll
        for (int it = 0; it < NV; it++) {
            const int vi = it * kFiltThreads + threadIdx.x;
            const int rv = vi * 8;
            if (rv < r1 && rv + 8 > r0) {
                const int lo = max(0, r0 - rv), hi = min(8, r1 - rv);
                const uint32_t vm = ((1u << hi) - 1u) & ~((1u << lo) - 1u);
                const int4 raw = rawv[it];
                const __half2 *h2 = reinterpret_cast<const __half2 *>(&raw);
                uint32_t kb = 0;
#pragma unroll
                for (int q = 0; q < 4; q++) {
                    const uint32_t r = __hle2_mask(h2[q], th2);  // 0xFFFF per lane that holds
                    kb |= ((r & 1u) | ((r >> 15) & 2u)) << (2 * q);
                }
                flags |= (FiltFlags)(kb & vm) << (it * 8);
            }
        }
    } else {
        const V *src = lb + m.seg_off + (int64_t)i * m.n;
#pragma unroll
        for (int it = 0; it < kFiltItems; it++) {
            const int64_t t = t0 + (int64_t)it * kFiltThreads + threadIdx.x;
            if (t < t1) {
                bool keep;
                if constexpr (std::is_same<V, float>::value)
                    keep = src[t] <= __uint_as_float(th);
                else
                    keep = src[t] <= (int32_t)th;
                flags |= (FiltFlags)keep << it;
            }
        }
    }
    int total;
    const int pos = block_excl_scan(kFiltItems > 32 ? __popcll((unsigned long long)flags) : __popc((uint32_t)flags), s_scan, &total);
    if (threadIdx.x == 0) s_base = total ? atomicAdd(&surv_count[seg], total) : 0;
    __syncthreads();
    int o = s_base + pos;
    int32_t *dst = surv + m.seg_off + (int64_t)i * m.n;
#pragma unroll
    for (int it = 0; it < kFiltItems; it++) {
        if (flags >> it & 1) {
            const int64_t t = LH ? ta + (int64_t)((it / 8) * kFiltThreads + threadIdx.x) * 8 + (it % 8)
                                 : t0 + (int64_t)it * kFiltThreads + threadIdx.x;
            dst[o++] = (int32_t)t;
        }
    }
}

// no-prune mode: every owned candidate of every segment is a survivor.
__global__ void all_candidates_kernel(const MQMeta *meta, const QParams P, int32_t *surv,
                                      int32_t *surv_count) {
    const int seg = blockIdx.y;
    const int mq = seg / P.n_len, i = seg % P.n_len;
    const MQMeta m = meta[mq];
    const int d = P.len[i];
    const int64_t tb = m.t_lo > 0 ? m.t_lo : 0;
    const int64_t te = min(m.t_hi, m.n - m.hz - d + 1);
    const int64_t nc = te > tb ? te - tb : 0;
    int32_t *dst = surv + m.seg_off + (int64_t)i * m.n;
    for (int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; x < nc;
         x += (int64_t)gridDim.x * blockDim.x)
        dst[x] = (int32_t)(tb + x);
    if (blockIdx.x == 0 && threadIdx.x == 0) surv_count[seg] = (int32_t)nc;
}

// Warp-task prefix for one item-query index li: task_off[mq] = sum over earlier
// MQs of ceil(count/32).  Single CTA.
__global__ void __launch_bounds__(1024) task_prefix_kernel(const int32_t *counts, int static_count,
                                                          int n_mq, int n_len, int li,
                                                          int32_t *task_off) {
    __shared__ int s_scan[32];
    __shared__ int s_carry;
    if (threadIdx.x == 0) s_carry = 0;
    __syncthreads();
    for (int base = 0; base < n_mq; base += blockDim.x) {
        const int mq = base + threadIdx.x;
        int c = 0;
        if (mq < n_mq) c = static_count >= 0 ? static_count : counts[mq * n_len + li];
        const int tasks = (c + 31) >> 5;
        int total;
        const int ex = block_excl_scan(tasks, s_scan, &total);
        if (mq < n_mq) task_off[mq] = s_carry + ex;
        __syncthreads();
        if (threadIdx.x == 0) s_carry += total;
        __syncthreads();
    }
    if (threadIdx.x == 0) task_off[n_mq] = s_carry;
}

// ---------------------------------------------------------------------------
// a8: selection: the k smallest (DTW, t) keys of each segment,
// sorted ascending; all k are returned (not only the k-th).  One CTA per
// segment.  <= kSortCap finalists: bitonic sort in shared memory; otherwise
// radix-select the k-th key first and sort the k keys at or below it.
// ---------------------------------------------------------------------------
template <typename S>
__global__ void __launch_bounds__(512) topk_kernel(const uint64_t *fin, const int32_t *fin_count,
                                                  const MQMeta *meta, const QParams P,
                                                  int64_t *out_ids, typename Tr<S>::V *out_d) {
    using V = typename Tr<S>::V;
    __shared__ uint64_t s_keys[kSortCap];
    __shared__ int s_hist[256];
    __shared__ uint64_t s_b[2];
    __shared__ int s_cnt;
    const int seg = blockIdx.x;
    const int mq = seg / P.n_len, i = seg % P.n_len;
    const MQMeta m = meta[mq];
    const int k = P.k;
    const int cnt = fin_count[seg];
    const uint64_t *src = fin + m.seg_off + (int64_t)i * m.n;
    int nsort;
    if (cnt <= kSortCap) {
        nsort = 1;
        while (nsort < cnt || nsort < k) nsort <<= 1;
        for (int x = threadIdx.x; x < nsort; x += blockDim.x) s_keys[x] = x < cnt ? src[x] : kKeyMax;
    } else {
        const uint64_t kth = block_radix_kth(src, cnt, k, s_hist, s_b);
        if (threadIdx.x == 0) s_cnt = 0;
        nsort = 1;
        while (nsort < k) nsort <<= 1;
        for (int x = threadIdx.x; x < nsort; x += blockDim.x) s_keys[x] = kKeyMax;
        __syncthreads();
        for (int x = threadIdx.x; x < cnt; x += blockDim.x) {
            uint64_t v = src[x];
            if (v <= kth) {
                int pos = atomicAdd(&s_cnt, 1);
                if (pos < nsort) s_keys[pos] = v;
            }
        }
    }
    bitonic_sort_smem(s_keys, nsort);
    const V INF = Tr<S>::inf();
    for (int j = threadIdx.x; j < k; j += blockDim.x) {
        const uint64_t key = s_keys[j];
        const int64_t o = (int64_t)seg * k + j;
        if (key == kKeyMax) {
            out_ids[o] = -1;
            if constexpr (std::is_same<V, float>::value) out_d[o] = INF;
            else out_d[o] = (V)0x7FFFFFFF;
        } else {
            out_ids[o] = (int64_t)(uint32_t)key + m.origin;
            const uint32_t db = (uint32_t)(key >> 32);
            if constexpr (std::is_same<V, float>::value) out_d[o] = __uint_as_float(db);
            else out_d[o] = (int32_t)db;
        }
    }
}

// ---------------------------------------------------------------------------
// a9: merge of G per-shard top-k lists.  One CTA per row.
// Key = (dist bits << 32) | id (ids < 2^32); padding (id -1) -> key max.
// ---------------------------------------------------------------------------
template <typename V>
__global__ void __launch_bounds__(512) merge_topk_kernel(const int64_t *ids_in, const V *d_in,
                                                        int G, int rows, int k, int64_t *ids_out,
                                                        V *d_out, V pad) {
    __shared__ uint64_t s_keys[kSortCap];
    const int row = blockIdx.x;
    const int n = G * k;
    int nsort = 1;
    while (nsort < n) nsort <<= 1;
    for (int x = threadIdx.x; x < nsort; x += blockDim.x) {
        uint64_t key = kKeyMax;
        if (x < n) {
            const int g = x / k, j = x % k;
            const int64_t o = ((int64_t)g * rows + row) * k + j;
            const int64_t id = ids_in[o];
            if (id >= 0) key = ((uint64_t)key_bits(d_in[o]) << 32) | (uint32_t)id;
        }
        s_keys[x] = key;
    }
    bitonic_sort_smem(s_keys, nsort);
    for (int j = threadIdx.x; j < k; j += blockDim.x) {
        const uint64_t key = s_keys[j];
        const int64_t o = (int64_t)row * k + j;
        if (key == kKeyMax) {
            ids_out[o] = -1;
            d_out[o] = pad;
        } else {
            ids_out[o] = (int64_t)(uint32_t)key;
            const uint32_t db = (uint32_t)(key >> 32);
            d_out[o] = *reinterpret_cast<const V *>(&db);
        }
    }
}

// a5 tau-set trim (reading R8): of the LTt tile candidates of a segment (each
// scan unit's smallest-LB_w candidates), keep the `keep` smallest (LB_w, t) and
// move the previous step's k neighbours (continuous step, at [LTt, LTt + kprev))
// right after them, so the tau DTW pass verifies keep + kprev candidates.  Any
// subset of verified candidates gives a valid tau (the k-th distinct key of k
// verified candidates bounds the k-th NN key); the trim only trades a slightly
// looser tau for fewer DTWs.  One CTA per segment; keys sorted in dynamic
// shared memory (n2 = next power of two >= LTt).
// src: the candidate list of each segment (stride sstride, nsrc entries): the
// tile list itself, or the per-chunk winners of tau_trim_chunk_kernel.
template <typename S>
__global__ void __launch_bounds__(256) tau_trim_kernel(const int32_t *src, int sstride, int nsrc, int32_t *tauc,
                                                      int LT, int LTt, int keep, int kprev,
                                                      const typename Tr<S>::V *lb, const MQMeta *meta,
                                                      int n_len, const uint32_t *slb) {
    // slb: LB_w bits beside src (same layout), or null: gather them from LB_w
    extern __shared__ __align__(16) uint64_t s_tk[];
    const int seg = blockIdx.x;
    const int mq = seg / n_len, i = seg % n_len;
    const MQMeta m = meta[mq];
    int32_t *row = tauc + (int64_t)seg * LT;
    const int32_t *srow = src + (int64_t)seg * sstride;
    const uint32_t *slrow = slb ? slb + (int64_t)seg * sstride : nullptr;
    const typename Tr<S>::V *lbi = lb + m.seg_off + (int64_t)i * m.n;
    int n2 = 1;
    while (n2 < nsrc) n2 <<= 1;
    for (int x = threadIdx.x; x < n2; x += blockDim.x) {
        uint64_t key = kKeyMax;
        if (x < nsrc) {
            const int t = srow[x];
            if (t >= 0) key = ((uint64_t)(slrow ? slrow[x] : key_bits(lbi[t])) << 32) | (uint32_t)t;
        }
        s_tk[x] = key;
    }
    int32_t *s_prev = reinterpret_cast<int32_t *>(s_tk + n2);
    for (int j = threadIdx.x; j < kprev; j += blockDim.x) s_prev[j] = row[LTt + j];
    bitonic_sort_smem(s_tk, n2);  // ends with a barrier
    for (int x = threadIdx.x; x < keep; x += blockDim.x)
        row[x] = s_tk[x] != kKeyMax ? (int32_t)(uint32_t)s_tk[x] : -1;
    for (int j = threadIdx.x; j < kprev; j += blockDim.x) row[keep + j] = s_prev[j];
}

// First level of the trim for very long tile lists (window-range scale): chunk
// c of segment seg (kTrimChunk entries) keeps its `keep` smallest (LB_w, t) in
// out[seg][c keep ..); tau_trim_kernel then trims the chunk winners.
constexpr int kTrimChunk = 8192;
template <typename S>
__global__ void __launch_bounds__(256) tau_trim_chunk_kernel(const int32_t *tauc, int LT, int LTt, int keep,
                                                            const typename Tr<S>::V *lb, const MQMeta *meta,
                                                            int n_len, int32_t *out, int ostride,
                                                            const uint32_t *tlb, uint32_t *olb) {
    extern __shared__ __align__(16) uint64_t s_tk[];
    const int c = blockIdx.x, seg = blockIdx.y;
    const int mq = seg / n_len, i = seg % n_len;
    const MQMeta m = meta[mq];
    const int32_t *row = tauc + (int64_t)seg * LT + (int64_t)c * kTrimChunk;
    const uint32_t *lrow = tlb ? tlb + (int64_t)seg * LT + (int64_t)c * kTrimChunk : nullptr;
    const int n = min(kTrimChunk, LTt - c * kTrimChunk);
    const typename Tr<S>::V *lbi = lb + m.seg_off + (int64_t)i * m.n;
    int n2 = 1;
    while (n2 < n) n2 <<= 1;
    for (int x = threadIdx.x; x < n2; x += blockDim.x) {
        uint64_t key = kKeyMax;
        if (x < n) {
            const int t = row[x];
            if (t >= 0) key = ((uint64_t)(lrow ? lrow[x] : key_bits(lbi[t])) << 32) | (uint32_t)t;
        }
        s_tk[x] = key;
    }
    bitonic_sort_smem(s_tk, n2);
    int32_t *o = out + (int64_t)seg * ostride + (int64_t)c * keep;
    uint32_t *ol = olb ? olb + (int64_t)seg * ostride + (int64_t)c * keep : nullptr;
    for (int x = threadIdx.x; x < keep; x += blockDim.x) {
        const bool ok = x < n2 && s_tk[x] != kKeyMax;
        o[x] = ok ? (int32_t)(uint32_t)s_tk[x] : -1;
        if (ol) ol[x] = ok ? (uint32_t)(s_tk[x] >> 32) : 0xFFFFFFFFu;
    }
}

// tau_trim_kernel for tile lists too long for a 64-bit key sort (window-range
// scale, C4: ~49k per item query): only the 32-bit LB_w bits are kept in shared
// memory with their t (<= kTrimBigCap entries), the keep-th smallest is radix-selected (four
// 8-bit MSB passes over shared memory), and the candidates below it, then those
// equal to it up to `keep`, are compacted to the front in any order (any subset
// of verified candidates gives a valid tau).
template <typename S>
__global__ void __launch_bounds__(256) tau_trim_big_kernel(int32_t *tauc, int LT, int LTt, int keep, int kprev,
                                                          const typename Tr<S>::V *lb, const MQMeta *meta,
                                                          int n_len, const uint32_t *tlb) {
    extern __shared__ __align__(16) uint32_t s_lbk[];  // [LTt] LB bits, then [LTt] t
    __shared__ int s_hist[256];
    __shared__ uint32_t s_sel[2];
    __shared__ int s_cnt;
    int32_t *s_t = reinterpret_cast<int32_t *>(s_lbk + LTt);
    const int seg = blockIdx.x;
    const int mq = seg / n_len, i = seg % n_len;
    const MQMeta m = meta[mq];
    int32_t *row = tauc + (int64_t)seg * LT;
    const typename Tr<S>::V *lbi = lb + m.seg_off + (int64_t)i * m.n;
    const uint32_t *lrow = tlb ? tlb + (int64_t)seg * LT : nullptr;
    for (int x = threadIdx.x; x < LTt; x += blockDim.x) {
        const int t = row[x];
        s_t[x] = t;
        s_lbk[x] = t >= 0 ? (lrow ? lrow[x] : key_bits(lbi[t])) : 0xFFFFFFFFu;
    }
    // keep-th smallest valid value (MSB radix select over shared memory)
    uint32_t prefix = 0, mask = 0;
    int krem = keep;
    bool few = false;
    for (int shift = 24; shift >= 0; shift -= 8) {
        for (int h = threadIdx.x; h < 256; h += blockDim.x) s_hist[h] = 0;
        __syncthreads();
        // LB_w values share their top bits: aggregate equal digits per warp
        // (one shared atomic per distinct digit) instead of one per element
        for (int x0 = threadIdx.x & ~31; x0 < LTt; x0 += blockDim.x) {
            const int x = x0 + (threadIdx.x & 31);
            const uint32_t v = x < LTt ? s_lbk[x] : 0xFFFFFFFFu;
            const bool in = v != 0xFFFFFFFFu && (v & mask) == prefix;
            const int dg = in ? (int)((v >> shift) & 255) : 256;
            const unsigned peers = __match_any_sync(0xffffffffu, dg);
            if (in && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(&s_hist[dg], __popc(peers));
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            int acc = 0, dsel = -1;
            for (int dg = 0; dg < 256; dg++) {
                if (acc + s_hist[dg] >= krem) {
                    dsel = dg;
                    break;
                }
                acc += s_hist[dg];
            }
            s_sel[0] = dsel < 0 ? 0xFFFFFFFFu : (prefix | ((uint32_t)dsel << shift));
            s_sel[1] = (uint32_t)(krem - acc);
        }
        __syncthreads();
        if (s_sel[0] == 0xFFFFFFFFu) {  // fewer than keep valid candidates: keep them all
            few = true;
            break;
        }
        prefix = s_sel[0];
        krem = (int)s_sel[1];
        mask |= 255u << shift;
        __syncthreads();
    }
    const uint32_t thr = few ? 0xFFFFFFFEu : prefix;
    // previous neighbours [LTt, LTt + kprev) -> [keep, keep + kprev): read them first
    int32_t pv[4];  // kprev <= 4 * 256 = kMaxK
#pragma unroll
    for (int r = 0; r < 4; r++) {
        const int j = threadIdx.x + r * 256;
        pv[r] = j < kprev ? row[LTt + j] : -1;
    }
    if (threadIdx.x == 0) s_cnt = 0;
    __syncthreads();
    for (int x = threadIdx.x; x < LTt; x += blockDim.x)
        if (s_lbk[x] < thr) row[atomicAdd(&s_cnt, 1)] = s_t[x];
    __syncthreads();
    for (int x = threadIdx.x; x < LTt; x += blockDim.x) {
        if (s_lbk[x] == thr && s_lbk[x] != 0xFFFFFFFFu) {
            const int o = atomicAdd(&s_cnt, 1);
            if (o < keep) row[o] = s_t[x];
        }
    }
    __syncthreads();
    for (int x = min(s_cnt, keep) + threadIdx.x; x < keep; x += blockDim.x) row[x] = -1;
#pragma unroll
    for (int r = 0; r < 4; r++) {
        const int j = threadIdx.x + r * 256;
        if (j < kprev) row[keep + j] = pv[r];
    }
}

// Continuous step (reading R9): the previous step's k neighbours
// of each stream, shifted by the points the stream advanced, join the tau list
// at [LTt, LTt + k) of their segment (invalid -> -1).
__global__ void prev_tau_kernel(const int64_t *prev, int shift, const MQMeta *meta, const QParams P, int LTt,
                                int32_t *tauc) {
    const int seg = blockIdx.x;
    const int mq = seg / P.n_len, i = seg % P.n_len;
    const MQMeta m = meta[mq];
    const int64_t tb = m.t_lo > 0 ? m.t_lo : 0;
    const int64_t te = min(m.t_hi, m.n - m.hz - P.len[i] + 1);
    for (int j = threadIdx.x; j < P.k; j += blockDim.x) {
        const int64_t id = prev[(int64_t)seg * P.k + j];
        int64_t t = id >= 0 ? id - m.origin + shift : -1;
        if (t < tb || t >= te) t = -1;
        tauc[(int64_t)seg * P.LT + LTt + j] = (int32_t)t;
    }
}

// Lagged tile tau set (stream steps): the previous call's scan-unit candidates
// of each (stream, item query), shifted by the one-point advance, become the
// tile part [0, LTt) of this step's tau list with their (previous) LB_w bits as
// trim keys; a shifted t outside the owned range is dropped (-1).
__global__ void lag_tau_kernel(const int32_t *lag_t, const uint32_t *lag_lb, int LTt, const MQMeta *meta,
                               const QParams P, int32_t *tauc, uint32_t *taulb) {
    const int seg = blockIdx.y;
    const int x = blockIdx.x * blockDim.x + threadIdx.x;
    if (x >= LTt) return;
    const int mq = seg / P.n_len, i = seg % P.n_len;
    const MQMeta m = meta[mq];
    const int64_t tb = m.t_lo > 0 ? m.t_lo : 0;
    const int64_t te = min(m.t_hi, m.n - m.hz - P.len[i] + 1);
    const int32_t t = lag_t[(int64_t)seg * LTt + x];
    const int64_t t1 = t >= 0 ? (int64_t)t + 1 : -1;
    const bool ok = t1 >= tb && t1 < te;
    tauc[(int64_t)seg * P.LT + x] = ok ? (int32_t)t1 : -1;
    taulb[(int64_t)seg * P.LT + x] = ok ? lag_lb[(int64_t)seg * LTt + x] : 0xFFFFFFFFu;
}

// Stats: acc[0] += finalists, acc[1 + i] += candidates DTW-verified for item
// query i (a7), acc[1 + kMaxLen + i] += survivors of a6 the cascade dropped.
// vmask: item queries whose verified list is vcount (the cascade ran), else scount.
__global__ void accum_counts_kernel(const int32_t *vcount, const int32_t *scount, const int32_t *fcount, int nseg,
                                    int n_len, uint32_t vmask, unsigned long long *acc) {
    for (int s = threadIdx.x; s < nseg; s += blockDim.x) {
        const int i = s % n_len;
        const int32_t v = (vmask >> i & 1u) ? vcount[s] : scount[s];
        atomicAdd(&acc[0], (unsigned long long)fcount[s]);
        atomicAdd(&acc[1 + i], (unsigned long long)v);
        atomicAdd(&acc[1 + kMaxLen + i], (unsigned long long)(scount[s] - v));
    }
}

// max |x| over n values (the series bound of the fp16 storage scales, R26);
// *out must start at 0 (non-negative floats order like their bits).
template <typename S>
__global__ void absmax_kernel(const S *x, int64_t n, unsigned *out) {
    float m = 0.0f;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        m = fmaxf(m, fabsf((float)x[i]));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    if ((threadIdx.x & 31) == 0) atomicMax(out, __float_as_uint(m));
}

// int16 range check for the I16 dtype (R17): counts |x| > 1023.
__global__ void range_check_kernel(const int16_t *x, int64_t n, int *bad) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x)
        if (x[i] > 1023 || x[i] < -1023) atomicAdd(bad, 1);
}

// Gather DTW keys of smiler_dtw's candidate list into distances.
template <typename V>
__global__ void keys_to_dists_kernel(const uint64_t *keys, int64_t n, V *out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t db = (uint32_t)(keys[i] >> 32);
        out[i] = *reinterpret_cast<const V *>(&db);
    }
}

}  // namespace smiler
