// internal.h -- device-side data structures shared by the kernels of
// libsmiler.so (not part of the C ABI; see include/smiler.h).
#pragma once
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include "../../include/smiler.h"

namespace smiler {

constexpr int kMaxLen = 16;      // max item queries per master query
constexpr int kMaxD = 1024;      // max master-query length
constexpr int kMaxK = 1024;      // max k
constexpr int kMaxWindow = 64;   // max omega
constexpr int kMaxRhoFast = 32;  // rho handled by the register-band DTW kernels
constexpr int kSortCap = 4096;   // keys sorted in shared memory by one CTA
constexpr int kTrimBigCap = 27648;  // tau-set trim: 32-bit keys + t in shared memory (216 KB)
constexpr int kMaxPredK = 128;   // neighbours per GP predictor (k x k fp64 factor in shared memory)
constexpr uint64_t kKeyMax = ~0ull;

// Value type of the arithmetic for a storage type (R16, R17).
template <typename S> struct Tr;
template <> struct Tr<int16_t> {
    using V = int32_t;
    using V2 = int2;
    using V4 = int4;
    static __device__ __forceinline__ V inf() { return 0x3FFFFFFF; }
};
template <> struct Tr<float> {
    using V = float;
    using V2 = float2;
    using V4 = float4;
    static __device__ __forceinline__ V inf() { return __int_as_float(0x7f800000); }
};

// Per master query (chunk-relative), built on the host.
struct MQMeta {
    int64_t series_off;  // element offset of the sensor's series in the device copy
    int64_t n;           // sensor (slice) length N
    int64_t origin;      // global id of local t = 0
    int64_t t_lo, t_hi;  // owned candidate starts, local coordinates
    int64_t n_dw;        // floor(N / w) disjoint windows
    int64_t post_off;    // element offset of this MQ's P_EQ plane [prows][pstride]; P_EC plane follows
    int64_t pstride;     // posting row stride (elements): n_dw, or n_dw rounded up to 8 (TMA ring)
    int32_t prows;       // posting rows per plane: n_sw, or n_sw + w - 1 (TMA ring: physical rows
                         // 0 .. w-2 mirrored after row n_sw - 1, so any w consecutive ring rows
                         // are contiguous)
    int64_t seg_off;     // offset of this MQ's per-candidate segments; (mq,i) at seg_off + i*n
    int64_t hz;          // prediction horizon h (local): candidates must end by n - hz (C_{t,d} with
                         // c_{t+d-1+h} in the series); 0 = every segment
    int32_t nblk;        // group-scan CTAs for this MQ
    int32_t sensor;
};

// Parameters common to one smiler_knn chunk.
struct QParams {
    int D, w, n_len, k, rho_env, E, LT, n_mq;
    int ring_cursor;  // continuous streams: physical posting row of SW_b is (b + ring_cursor) mod n_sw
    int lbsel;        // which sums make the bound: 0 = max(EQ, EC) (Eq. 5 / Thm 4.1), 1 = EQ, 2 = EC
    int fuse;         // 1: the LB kernel filters (LB <= thr) and appends survivors itself (a4+a6)
    int lb_half;      // 1: the LB_w array holds fp16 of LB_w x lbs[mq] rounded down (R26)
    const float *lbs; // lb_half: per-MQ power-of-two scale (query_prep_kernel: every bound x lbs fits fp16)
    float post_unscale;  // fp16 stream ring: the entries hold P x 2^-e; sums are multiplied by 2^e
    const uint32_t *thr;  // fuse: per-segment admission bound (tau_select_kernel)
    int32_t *surv;        // fuse: survivor t lists (segment layout)
    int32_t *scount;      // fuse: survivors per segment
    uint32_t *taulb;      // LB_w bits of every tile tau candidate (same layout as the tau list), or null
    int len[kMaxLen];
    int rho[kMaxLen];
};

// Work list of one DTW launch (one item-query index `li`, all MQs of a chunk).
template <typename S> struct DtwParams {
    const S *series;
    const MQMeta *meta;
    const typename Tr<S>::V *qv;  // [n_mq][D] master queries in the arithmetic type
    int D, n_len, li, d, n_mq;
    int mode;                     // 0 = tau list -> keys_out; 1 = survivors -> finalists
    const int32_t *list;          // candidate t values
    int LT;                       // tau mode: list stride per segment
    int LTc;                      // tau mode: entries per segment to verify (<= LT)
    const int32_t *counts;        // survivors mode: per-segment counts
    const int32_t *task_off;      // [n_mq + 1] prefix of warp tasks
    uint64_t *keys_out;           // tau mode
    const uint64_t *tau_key;      // survivors mode: per-segment key threshold
    uint64_t *fin;                // survivors mode: finalist keys (segment layout)
    int32_t *fin_count;
    int wave;                     // 1: anti-diagonal wavefront kernel for any rho (else only rho > kMaxRhoFast)
    int packed = 0;               // 1: f32 rows in pairs with fp32x2-packed cells (A/B of the scalar register band)
};

template <typename S> void launch_dtw(int rho, const DtwParams<S> &p, int grid, cudaStream_t st);

// LB_Keogh cascade between the filter (a6) and the DTW verification (a7) of one
// item-query index li: every survivor of the index bound is re-bounded by
// LB_EQ with the item query's own envelope (width rho_i, clipped to the item
// query) over all d_i points, and kept only if that bound is <= the segment's
// admission threshold.
template <typename S> struct CascadeParams {
    const S *series;
    const MQMeta *meta;
    const typename Tr<S>::V2 *qenv;  // [n_mq][n_len][D] (U, L) of IQ_i's own envelope (positions >= D - d_i)
    int D, n_len, li, d, n_mq;
    const int32_t *list;             // survivor t lists (segment layout)
    const int32_t *counts;           // per segment
    const int32_t *task_off;         // [n_mq + 1] prefix of warp tasks (32 survivors each)
    const uint32_t *thr;             // per-segment admission bound (tau_select_kernel)
    int32_t *out_list;               // kept t (segment layout)
    int32_t *out_counts;             // per segment (zeroed by the caller)
};
template <typename S> void launch_cascade(const CascadeParams<S> &p, cudaStream_t st);

// Item-query envelopes of the cascade: IQ_i's own envelope, width rho_i.
struct IQTab {
    int len[kMaxLen];
    int rho[kMaxLen];
};

// Largest power of two 2^e (|e| <= 60) with bound x 2^e <= 65504 (fp16 max):
// the storage scale of bounds that never exceed `bound` (R26).  Scaling by a
// power of two is exact, so rounding the scaled value down to fp16 keeps it a
// lower bound, and no stored bound saturates.
__host__ __device__ inline float fp16_fit_scale(double bound) {
    if (!(bound > 0.0)) return 1.0f;
    int e = 0;
    double b = bound;
    while (b * 2.0 <= 65504.0 && e < 60) { b *= 2.0; e++; }
    while (b > 65504.0 && e > -60) { b *= 0.5; e--; }
    return ldexpf(1.0f, e);
}

// DTW cells of one banded d x d matrix (|i-j| <= rho).
inline int64_t dtw_cells(int d, int rho) {
    if (rho > d - 1) rho = d - 1;
    return (int64_t)d * (2 * rho + 1) - (int64_t)rho * (rho + 1);
}

}  // namespace smiler
