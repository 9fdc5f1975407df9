/*
 * smiler.h -- C ABI of the B200-native Suffix kNN Search under banded DTW
 * (SMiLer Search Step; Zhou & Tung, SIGMOD'15).  Citations "P:<line>" refer
 * to /root/reference/PAPER.md; "R<n>" to the readings listed in DESIGN.md.
 *
 * Conventions for every call:
 *   - Return value is an smiler_status (0 = OK).  No exception, abort or
 *     exit ever crosses the ABI; smiler_last_error() returns a thread-local
 *     message describing the last non-OK status of the calling thread.
 *   - Pointer arguments may be HOST or DEVICE memory (device memory must be
 *     on the handle's device); the library inspects each pointer with
 *     cudaPointerGetAttributes.  The caller owns every input and output
 *     buffer; the library never retains a caller pointer after a call returns.
 *   - The library owns all device state of a handle until smiler_free.
 *   - One handle lives on one device and one CUDA stream.  Calls on one handle
 *     must not run concurrently; separate handles are independent.
 *   - Calls are stream-ordered on the handle's stream.  When any output is a
 *     host buffer (or stats are requested) the call synchronises the stream
 *     before returning; with device outputs and stats == NULL it returns
 *     without a host synchronisation.
 *   - All work runs in this library's CUDA kernels for sm_100a.  There is no
 *     CPU fallback: without a usable CUDA device every call returns
 *     SMILER_ECUDA.
 */
#ifndef SMILER_H
#define SMILER_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SMILER_ABI_VERSION 4  /* 4: smiler_knn_stats.ns_cascade */

#if defined(__GNUC__)
#define SMILER_API __attribute__((visibility("default")))
#else
#define SMILER_API
#endif

typedef struct smiler_index smiler_index; /* opaque, owned by the library */

typedef enum {
    SMILER_I16 = 0, /* int16 values with |x| <= 1023; DTW exact in int32 (R17)  */
    SMILER_F32 = 1  /* float32 values; DTW cell = fmaf(q-c, q-c, min3)  (R16)  */
} smiler_dtype;

typedef enum {
    SMILER_OK = 0,
    SMILER_EINVAL = -1, /* bad argument (message says which)                 */
    SMILER_ERANGE = -2, /* an I16 value outside [-1023, 1023]                */
    SMILER_ENOMEM = -3, /* device allocation failed                          */
    SMILER_ECUDA = -4,  /* CUDA runtime / launch error, or no CUDA device    */
    SMILER_ENCCL = -5   /* reserved for collective errors (merge driver)     */
} smiler_status;

/* Per-call counters and per-phase device times (CUDA events on the handle's
 * stream).  Times are filled only when smiler_knn_opts.timing != 0. */
typedef struct smiler_knn_stats {
    int64_t candidates;   /* sum over (MQ, item query) of candidate starts t      */
    int64_t tau_verified; /* DTWs computed to set the thresholds tau_i (a5)       */
    int64_t survivors;    /* candidates with LB_w <= tau_i that a7 verified by DTW */
    int64_t finalists;    /* verified candidates with key <= tau key (a8 input)   */
    double dtw_cells;     /* banded-DTW cells evaluated (a5 + a7)                 */
    double bf_cells;      /* cells a brute-force scan of every candidate needs    */
    int64_t posting_bytes;/* window-level posting bytes written by a3, read by a4 */
    int64_t lb_bytes;     /* LB_w bytes written by a4 and read by a6              */
    int32_t kernel_launches;
    int32_t mq_chunks;
    double ns_prep, ns_window_lb, ns_group_scan, ns_tau, ns_filter, ns_verify, ns_select;
    double ns_total;
    int64_t cascade_pruned;/* survivors of the index bound (a6) that the LB_Keogh cascade
                              (LB_EQ with IQ_i's own envelope of width rho_i) dropped before
                              a7; `survivors` counts the candidates a7 verified */
    double ns_cascade;    /* time of that cascade (with opts.timing; ns_filter is a6 alone) */
} smiler_knn_stats;

typedef struct smiler_knn_opts {
    int32_t no_prune; /* 1: skip thresholding, verify every candidate (GPU brute force) */
    int32_t timing;   /* 1: record per-phase CUDA events into stats                     */
    int32_t mq_chunk; /* master queries per internal chunk; 0 = automatic               */
    int32_t two_level;/* 1: materialise the window-level posting lists in HBM (a3) and
                         scan them (a4), as the paper's two-level index; 0: automatic
                         (fused a3+a4 with posting rows kept on chip when w is 4/8/16) */
    int32_t lb_kind;  /* which lower bound filters the candidates (SMILER_LB_*); all of
                         them are valid DTW lower bounds, so the kNN result is the same */
    int32_t horizon;  /* h >= 0: only segments C_{t,d} whose h-step-ahead value
                         c_{t+d-1+h} exists are candidates, i.e. t <= N - d - h (the
                         kNN data (X_{k,d}, Y_h) of the predictors);
                         0 = every segment (Def. 4.1).  Shards: N is the full series. */
    int32_t exact_postings; /* smiler_stream_create_ex: 1 keeps the stream's window-level
                         postings in the index arithmetic type; 0 (default) stores them for
                         F32 indices with window 4/8/16/32 as fp16 rounded toward zero --
                         never above the exact value, so every sum of them is still a
                         lower bound of DTW (Thm 4.3) and the kNN is unchanged, while the
                         ring and the bytes the group scan reads per step halve */
    int32_t tau_mult; /* size of the tile tau set (reading R8), in multiples of k per item
                         query: 0 = default (16 one-shot; 2 in continuous steps, which also
                         verify the previous step's k neighbours shifted),
                         > 0 = that many, < 0 = none.  With no tile set in a continuous
                         step the thresholds exist before the scan, and the LB kernel
                         filters as it goes (a4+a6 fused, no LB_w array) */
    int32_t variant;  /* kernel-path selector for tests and A/B timing; every variant computes
                         the same (exact) result: 0 = automatic, 1 = row-form fused LB kernel,
                         2 = scalar (not fp32x2-packed) diagonal LB kernel for F32,
                         3 = the anti-diagonal wavefront DTW kernel for every warping width
                         (by default it runs only for rho > 32, the register band below),
                         4 = no LB_Keogh cascade between the filter and the verification,
                         5 = stream steps without the lagged tile tau set (thresholds after
                         the scan, LB_w array + filter pass),
                         6 = F32 register-band DTW with rows in pairs and fp32x2-packed
                         cells (same cells, bit-identical; measured no faster: A/B only),
                         7 = stream ring scanned without TMA, 8 = one tile per ring-scan CTA,
                         9 = radix-select tau-set trim, 10 = two-stage tau-set trim.  Any other
                         value is EINVAL */
    int32_t reserved; /* must be 0 (EINVAL otherwise) */
    int32_t tau_keep; /* tau-set trim (reading R8): tile candidates kept per item query before
                         the tau DTWs, in multiples of k; 0 = default (4 k one-shot, k / 4 in
                         a continuous step, which also verifies the k shifted previous
                         neighbours), < 0 = verify every tile candidate.  Any choice is a
                         valid tau set; only the threshold's tightness changes */
    uint64_t *shared_tau; /* NULL, or a running threshold shared by calls that split ONE
                         search (window-range shards of the same series and master
                         queries): [n_mq][n_len] keys
                         (float/int dist bits << 32 | global t), device memory of this
                         GPU or of a peer reachable over NVLink, set to all ones before
                         the first call.  Each call atomically lowers entry (m, i) to its
                         own threshold key (a5) and prunes with the minimum it reads
                         back -- every key written is an upper bound of the k-th NN key
                         of the whole search, so the merged top-k is unchanged while later
                         shards verify fewer candidates; a shard's own list may then hold
                         fewer than k entries (padded) */
} smiler_knn_opts;

/* smiler_knn_opts.lb_kind.  The default is the paper's method; the others are
 * the ablations of Table 3 and Fig. 8 (P:1916-1919,
 * P:2094-2102).
 *   SMILER_LB_INDEX     LB_w = max(sum EQ, sum EC) over the full disjoint windows
 *                       of the candidate, through the two-level index (Thm 4.3,
 *                       Eq. 5)
 *   SMILER_LB_INDEX_EQ  the EQ sum of LB_w only ("LB_EQ" row of Table 3)
 *   SMILER_LB_INDEX_EC  the EC sum of LB_w only ("LB_EC" row of Table 3)
 *   SMILER_LB_DIRECT    SMiLer-Dir: LB_en = max(LB_EQ, LB_EC) over all d_i points of
 *                       the candidate (Thm 4.1), computed directly from
 *                       the series for each item query separately
 *   SMILER_LB_DIRECT_SHARED  the same LB_en values for every item query from ONE
 *                       pass: item queries are suffixes of the MQ, so
 *                       the candidates of all item queries that end at the same
 *                       series point share one running sum (cf. Remark 2) */
enum {
    SMILER_LB_INDEX = 0,
    SMILER_LB_INDEX_EQ = 1,
    SMILER_LB_INDEX_EC = 2,
    SMILER_LB_DIRECT = 3,
    SMILER_LB_DIRECT_SHARED = 4
};

/*
 * smiler_index_build -- upload sensor series and build the index (a1).
 *
 * series        n_total values of `dtype`; n_sensors series concatenated.
 *               Each series is the indexed history C of one sensor (P:597-608,
 *               z-normalised by the caller).
 * sensor_offsets n_sensors+1 ascending offsets into `series` (first 0, last
 *               n_total); NULL means one sensor of length n_total.
 * window        omega >= 1, the disjoint/sliding window length.
 * band          Sakoe-Chiba warping width: band >= 1 means an
 *               absolute rho = (int)band for every item query; 0 < band < 1
 *               means rho_i = floor(band * d_i) (R4).  band == 0 means rho = 0.
 *               Envelopes E(C) (Def. B.1, Eq. 25, clipped per
 *               sensor, R3) are built here for an absolute band, lazily on the
 *               first query for a fractional band (width rho_max, R4).
 * device        CUDA device ordinal; cuda_stream a cudaStream_t (NULL = legacy
 *               default stream) used by every call on the handle.
 * out           receives the handle.
 * Errors: EINVAL (n_total < 1, bad offsets, a sensor longer than 2^31 - 1
 *         points (candidate starts are 32-bit), window < 1, band < 0),
 *         ERANGE (I16 value with |x| > 1023), ENOMEM, ECUDA.
 */
SMILER_API int smiler_index_build(const void *series, smiler_dtype dtype, int64_t n_total,
                       const int64_t *sensor_offsets, int32_t n_sensors, int32_t window,
                       float band, int32_t device, void *cuda_stream, smiler_index **out);

/*
 * smiler_index_build_shard -- one sensor, window-range shard for multi-GPU
 * (SURVEY §8(e)).  `slice` holds global points [slice_begin, slice_begin +
 * n_slice) of a series of n_global points; the handle owns candidate starts
 * t in [t_begin, t_end) (global).  slice_begin must be a multiple of window
 * (disjoint windows stay global, so every LB_w equals the unsharded value);
 * the slice must carry a halo: slice_begin <= max(0, t_begin - rho_max) and
 * slice_begin + n_slice >= min(n_global, t_end + D - 1 + rho_max) for every
 * later query (checked by smiler_knn, EINVAL otherwise).  Returned ids are
 * global t.
 */
SMILER_API int smiler_index_build_shard(const void *slice, smiler_dtype dtype, int64_t n_slice,
                             int64_t slice_begin, int64_t n_global, int64_t t_begin,
                             int64_t t_end, int32_t window, float band, int32_t device,
                             void *cuda_stream, smiler_index **out);

/*
 * smiler_knn -- Suffix kNN Search (Def. 4.1) for a batch of master
 * queries, through the two-level index (Sec. 4.3): window-level
 * posting lists (a3), group-level LB_w scan (a4, Thm 4.3 / Eq. 5), per-query
 * threshold tau_i (a5, R8), filtering (a6), banded-DTW verification (a7,
 * Eq. 21-24) and top-k selection (a8).
 *
 * queries       [n_mq][D] master queries, oldest -> newest, same
 *               dtype as the index; D = lengths[n_len-1].  I16 values must
 *               satisfy |x| <= 1023 (R17): host queries are checked before any
 *               work (ERANGE); device queries are checked by the query-prep
 *               kernel, which clamps them for that call and raises a sticky
 *               flag reported as ERANGE by this call when it synchronises
 *               (host outputs or stats) or else by the next call on the handle.
 * query_sensor  [n_mq] sensor searched by each MQ; NULL -> 0.
 * lengths       ELV [n_len], strictly increasing, lengths[0] >= 1, each <= the
 *               sensor's length, lengths[n_len-1] = D <= 1024 (F32) or <= 256
 *               (I16: every DTW and bound then fits int32 exactly, R17),
 *               n_len <= 16.
 *               Item query IQ_i = the last lengths[i] points of the MQ
 *               (P:859-860).
 * k             max(EKV), 1 <= k <= 1024; smaller k are prefixes.
 * ids           [n_mq][n_len][k] int64: start t of C_{t,d_i} (R2) within the
 *               sensor (global t for shards).
 * dists         [n_mq][n_len][k] int32 (I16) or float (F32): DTW with
 *               dist(a,b) = (a-b)^2 (R1).
 *               Rows are sorted by (dist, t) (R11); padding is id -1 with
 *               dist INT32_MAX / +inf (R12).
 * stats         may be NULL.
 * Results are exactly the brute-force kNN (filtering never dismisses a true
 * neighbour: Thm 4.1/4.3 with tau_i >= the k-th distance, R8, R16).
 * Errors: EINVAL (bad argument, non-zero opts->reserved, unknown variant),
 *         ERANGE (I16 query value outside [-1023, 1023]), ENOMEM, ECUDA.
 */
SMILER_API int smiler_knn(smiler_index *idx, const void *queries, const int32_t *query_sensor,
               int32_t n_mq, const int32_t *lengths, int32_t n_len, int32_t k, int64_t *ids,
               void *dists, smiler_knn_stats *stats);

/* smiler_knn with options (opts may be NULL = defaults). */
SMILER_API int smiler_knn_ex(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                  int32_t n_mq, const int32_t *lengths, int32_t n_len, int32_t k, int64_t *ids,
                  void *dists, smiler_knn_stats *stats, const smiler_knn_opts *opts);

/*
 * smiler_knn_step -- one step of the Continuous Suffix kNN Search (Def. 4.1,
 * "from time t to time t+1 ... appending the latest observed point into MQ
 * and delete the oldest point") for a batch of master-query
 * streams.  Same arguments and results as smiler_knn, plus:
 * prev_ids      [n_mq][n_len][k] int64 (host or device): the ids this call's
 *               streams received at their previous step (same lengths, same k).
 * shift         points each stream advanced since then (1 per step, >= 0).
 * The threshold of every item query comes from the paper's second method
 * (reading R9): the previous k neighbours, shifted by `shift`,
 * re-scored against the new item query; tau_i = the largest of their keys.
 * Neighbours that fall outside the series make tau_i = +inf (no pruning).
 * Results are the exact kNN regardless of prev_ids' quality.
 */
SMILER_API int smiler_knn_step(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                               int32_t n_mq, const int32_t *lengths, int32_t n_len, int32_t k,
                               const int64_t *prev_ids, int32_t shift, int64_t *ids, void *dists,
                               smiler_knn_stats *stats, const smiler_knn_opts *opts);

/*
 * Continuous streams with the reused window-level index (Remark 1, P:936-953,
 * Fig. 6).  A stream batch keeps, for every master query, its master query and
 * its window-level posting lists (one per sliding window) in device memory, in
 * a ring over the sliding windows.  Each step appends one point to every
 * master query and drops the oldest; the new SW_0 takes the ring
 * slot of the dropped SW, LB_EQ of SW_0..SW_rho_max (whose query envelope
 * changed) and LB_EC of SW_0 are recomputed, all other posting entries are
 * reused (those of the oldest SWs keep a wider, still valid envelope, R21), the
 * group-level scan reads the ring (HBM-bound), and thresholds come from the
 * previous step's neighbours joined with a small tile set.
 * Results are the exact kNN of the current master queries.
 *
 * smiler_stream_create  queries [n_streams][D] (initial master queries),
 *                       query_sensor/lengths/k as smiler_knn; runs the first
 *                       search and writes its ids/dists ([n][n_len][k], host
 *                       or device).  Memory: 2 planes x (D - w + 1) floor(N/w)
 *                       posting entries per stream, resident (2 bytes each for
 *                       F32 indices with w in {4,8,16,32}, else 4; see
 *                       smiler_knn_opts.exact_postings); ENOMEM if absent.
 *                       The index must outlive the stream.
 * smiler_stream_create_ex  the same with opts (exact_postings; others ignored).
 * smiler_stream_step    new_points [n_streams] (one new point per stream, index
 *                       dtype, host or device); writes the step's results.
 * smiler_stream_free    NULL-safe.
 */
typedef struct smiler_stream smiler_stream;
SMILER_API int smiler_stream_create(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                                    int32_t n_streams, const int32_t *lengths, int32_t n_len, int32_t k,
                                    int64_t *ids, void *dists, smiler_stream **out);
SMILER_API int smiler_stream_create_ex(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                                       int32_t n_streams, const int32_t *lengths, int32_t n_len, int32_t k,
                                       int64_t *ids, void *dists, const smiler_knn_opts *opts,
                                       smiler_stream **out);
SMILER_API int smiler_stream_step(smiler_stream *st, const void *new_points, int64_t *ids, void *dists,
                                  smiler_knn_stats *stats, const smiler_knn_opts *opts);
SMILER_API void smiler_stream_free(smiler_stream *st);

/*
 * smiler_merge_topk -- final selection over G per-shard top-k lists (a9,
 * SURVEY §8(e)); called after an all-gather of the shards' (ids, dists).
 * ids_in [G][rows][k] int64, dists_in [G][rows][k] int32/float (dtype);
 * writes the k smallest by (dist, id) of each row to ids_out/dists_out
 * [rows][k], padding as smiler_knn.  Each candidate must appear in at most
 * one shard (ownership partition), so the merge is exact.  Runs on `device`
 * and `cuda_stream`.
 */
SMILER_API int smiler_merge_topk(const int64_t *ids_in, const void *dists_in, smiler_dtype dtype,
                      int32_t G, int32_t rows, int32_t k, int64_t *ids_out, void *dists_out,
                      int32_t device, void *cuda_stream);

/* ---- Per-step entry points used by the parity tests (same kernels) ------ */

/* Envelope U, L (Eq. 25, clipped, R3) of one sensor with width rho, as built
 * by the a1 kernel.  U, L: [sensor length] of the index dtype. */
SMILER_API int smiler_index_envelope(smiler_index *idx, int32_t sensor, int32_t rho, void *U, void *L);

/* Steps a2-a4 only: for each MQ, the window-level posting lists (P_EQ, P_EC)
 * (may be NULL) as [n_mq][2][D-window+1][n_dw] int32/float, plane 0 = P_EQ,
 * plane 1 = P_EC (the device layout of the two-level path; n_dw = floor(N/w)
 * of the MQ's sensor; all MQs must search sensors of equal length), and LB_w
 * per candidate as [n_mq][n_len][N] int32/float indexed by t (entries with
 * t > N - d_i are unspecified).  Envelope width rho_max as in smiler_knn. */
SMILER_API int smiler_lower_bounds(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                        int32_t n_mq, const int32_t *lengths, int32_t n_len, void *postings,
                        void *lbw);

/* Steps a2-a4 with the lower bound `lb_kind` (SMILER_LB_*): the per-candidate
 * bound that smiler_knn_ex filters with, as [n_mq][n_len][N] int32/float
 * indexed by t (entries with t > N - d_i unspecified).  SMILER_LB_INDEX gives
 * the LB_w of smiler_lower_bounds; SMILER_LB_INDEX_EQ / _EC its two sums
 * (Eq. 5); SMILER_LB_DIRECT / _DIRECT_SHARED give LB_en (Thm 4.1) per
 * candidate, with the series envelope of width rho_max and the MQ envelope
 * (R4, R20).  All MQs must search sensors of equal length.
 * Errors: EINVAL (NULL lb, bad lb_kind, as smiler_knn), ENOMEM, ECUDA. */
SMILER_API int smiler_lower_bounds_ex(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                        int32_t n_mq, const int32_t *lengths, int32_t n_len, int32_t lb_kind,
                        void *lb);

/*
 * smiler_predict -- the predictors that consume the kNN (
 * Sec. 5.2; App. B.3).
 *
 * For master query m (its sensor query_sensor[m], NULL -> 0), item query i
 * (IQ_i = the last lengths[i] points of queries[m]) and k_j = ekv[j],
 * the predictor f_{i,j} uses the kNN data of the first k_j neighbours
 * ids[m][i][0..k_j) (multi-k by prefix):
 *   X = {c[t_a .. t_a+d_i)},  Y_h = {c[t_a + d_i - 1 + horizon]}
 * and returns
 *   ar_mean, ar_var  Eq. 12-13: mean of Y_h and sum (y - mean)^2 / k_j
 *   gp_mean, gp_var  Eq. 16-17 with the covariance of Eq. 18,
 *                    c(x_a, x_b) = th0^2 exp(-|x_a - x_b|^2 / (2 th1^2)) + delta_ab th2^2,
 *                    c(x0, x0) = th0^2 + th2^2 (reading P1)
 * theta: [n_mq][n_len][n_k][3] doubles (th0, th1, th2) per predictor (their
 * online training, Eq. 19-20, is not part of the library).
 * ids: the smiler_knn output [n_mq][n_len][k] (run it with
 * smiler_knn_opts.horizon = horizon so every neighbour has its h-step-ahead
 * value); a predictor whose first k_j ids contain -1 or a t with
 * t + d_i - 1 + horizon >= N, or whose C is not positive definite, gets NaN.
 * Outputs: [n_mq][n_len][n_k] doubles each, row-major.  Every pointer may be
 * host or device memory; the call returns when the outputs are written.
 * Arithmetic: fp64 (Cholesky factor of C in shared memory).
 * Errors: EINVAL (NULL argument, shard index, n_len or lengths as smiler_knn,
 *         ekv not strictly increasing within [1, min(k, 128)], n_k > 64,
 *         horizon < 0, bad sensor), ENOMEM, ECUDA.
 */
SMILER_API int smiler_predict(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                   int32_t n_mq, const int32_t *lengths, int32_t n_len, const int64_t *ids, int32_t k,
                   const int32_t *ekv, int32_t n_k, int32_t horizon, const double *theta,
                   double *ar_mean, double *ar_var, double *gp_mean, double *gp_var);

/* Step a7 only: banded DTW (Eq. 21-24) of item query q[0..d) against
 * C_{t,d} of `sensor` for each t in ts[0..n_t), warping width rho.  dists:
 * [n_t] int32/float.  Every t must satisfy 0 <= t <= N-d. */
SMILER_API int smiler_dtw(smiler_index *idx, int32_t sensor, const void *q, int32_t d, int32_t rho,
               const int64_t *ts, int64_t n_t, void *dists);

/* Release the handle and all its device memory.  NULL-safe. */
SMILER_API void smiler_free(smiler_index *idx);

/* Thread-local message for the last non-OK status ("" if none). */
SMILER_API const char *smiler_last_error(void);

/* SMILER_ABI_VERSION of the loaded library. */
SMILER_API int32_t smiler_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SMILER_H */
