// smiler.cu -- host orchestration and C ABI of libsmiler.so (include/smiler.h).
//
// Per smiler_knn chunk of master queries, on the handle's stream and without
// any host synchronisation inside the pipeline:
//   a2 query_prep -> a3 window_lb -> a4 group_scan (+ tau set)
//   -> a5 DTW(tau set) + tau_select -> a6 filter -> a7 DTW(survivors)
//   -> a8 topk -> copy out
// Data-dependent sizes (survivors, finalists) stay on the device; buffers are
// sized for the worst case (every candidate) and kernels read the counts.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <nvtx3/nvToolsExt.h>
#include <stdarg.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <map>
#include <mutex>
#include <string>
#include <type_traits>
#include <vector>

#include "internal.h"
#include "kernels.cuh"

using namespace smiler;

constexpr int kTauMult = 16;  // tau-set size target, multiples of k (R8 reading)
constexpr int kTauMultCont = 2;  // ... in a continuous step (plus the k previous neighbours)
// Tile tau-set trim (tau_trim_kernel): keep the kTauKeep* x k smallest-LB_w tile
// candidates of the scan units' picks (0 = verify them all).  smiler_knn_opts
// .tau_keep > 0 overrides the multiple, < 0 disables the trim.
#ifndef SMILER_TAU_KEEP_ONESHOT
#define SMILER_TAU_KEEP_ONESHOT 4  // one-shot tile tau set, x k (8: C2 -0.2%, C4 -0.6%)
#endif
#ifndef SMILER_TAU_KEEP_CONT_DIV
#define SMILER_TAU_KEEP_CONT_DIV 4  // continuous steps keep k / 4 tile candidates (beside the k shifted
                                    // neighbours; profiles/r02/ab_tau_keep.txt: k / 4 beat k, k / 2, k / 8)
#endif
constexpr int kTauKeepOneShot = SMILER_TAU_KEEP_ONESHOT;
constexpr int kTauKeepCont = 1;
constexpr int kTrimCap = 16384;   // chunk winners a second bitonic trim may take (two-stage)
constexpr int kTrimSmall = 1024;  // tile lists sorted whole; longer: radix select (tau_trim_big_kernel)
static int tau_keep(const smiler_knn_opts &o, int k, bool cont) {
    int mult = cont ? kTauKeepCont : kTauKeepOneShot;
    if (o.tau_keep > 0) mult = o.tau_keep;
    if (o.tau_keep < 0) mult = 0;
    if (cont && o.tau_keep == 0) return std::max(1, mult * k / SMILER_TAU_KEEP_CONT_DIV);
    return mult * k;
}
constexpr int kTauEMax = 8;   // candidates per tau unit (CTA or warp)

// ---------------------------------------------------------------------------
// errors
// ---------------------------------------------------------------------------
static thread_local std::string g_err;

static int fail(int code, const char *fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_err = buf;
    return code;
}

#define CU(call)                                                                           \
    do {                                                                                   \
        cudaError_t e_ = (call);                                                           \
        if (e_ != cudaSuccess) {                                                           \
            if (e_ == cudaErrorMemoryAllocation)                                           \
                return fail(SMILER_ENOMEM, "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), \
                            __FILE__, __LINE__);                                           \
            return fail(SMILER_ECUDA, "%s: %s (%s:%d)", #call, cudaGetErrorString(e_),     \
                        __FILE__, __LINE__);                                               \
        }                                                                                  \
    } while (0)

#define CHECK_LAUNCH() CU(cudaGetLastError())

#define TRY(x)                      \
    do {                            \
        int r_ = (x);               \
        if (r_ != SMILER_OK) return r_; \
    } while (0)

static bool is_device_ptr(const void *p) {
    if (!p) return false;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// ---------------------------------------------------------------------------
// handle
// ---------------------------------------------------------------------------
struct DevBuf {
    void *p = nullptr;
    size_t cap = 0;
    int ensure(size_t bytes) {
        if (bytes <= cap) return SMILER_OK;
        if (p) cudaFree(p);
        p = nullptr;
        cap = 0;
        size_t want = bytes + bytes / 8 + 256;
        cudaError_t e = cudaMalloc(&p, want);
        if (e != cudaSuccess) {
            cudaGetLastError();
            p = nullptr;
            return fail(SMILER_ENOMEM, "cudaMalloc(%zu): %s", want, cudaGetErrorString(e));
        }
        cap = want;
        return SMILER_OK;
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        cap = 0;
    }
    template <typename T> T *as() const { return reinterpret_cast<T *>(p); }
};

struct SensorInfo {
    int64_t off;     // device element offset (aligned)
    int64_t n;       // length
    int64_t origin;  // global id of local t = 0
    int64_t t_lo, t_hi;
    int64_t n_global;  // shard: the full series length; else n
    int64_t slice_begin;
};

struct smiler_index {
    int device = 0;
    cudaStream_t stream = nullptr;
    smiler_dtype dtype = SMILER_I16;
    int window = 1;
    float band = 0.f;
    bool shard = false;
    std::vector<SensorInfo> sensors;
    int64_t dev_elems = 0;
    void *d_series = nullptr;
    int64_t *d_soff = nullptr, *d_slen = nullptr;
    std::map<int, std::pair<void *, void *>> env;  // rho -> (U, L)
    int num_sms = 148;
    float smax = 0.f;          // max |x| over the indexed series (fp16 storage scales, R26)
    int *qflag_h = nullptr;    // host-mapped sticky flag: an I16 device query outside [-1023, 1023]
    int *qflag_d = nullptr;    // its device alias (written by query_prep_kernel)
    // workspace
    DevBuf queries, qv, qtab, meta, post, lb, surv, fin, tauc, taulb, tauk, taukey, thr, scount, fcount,
        taskoff, out_ids, out_d, tmp, tmp2, pred, lbs, qenv, surv2, scount2;
    std::vector<cudaEvent_t> events;
    size_t budget = (size_t)24 << 30;  // workspace bytes per chunk (set at build)
    // pinned staging ring for per-chunk metadata (async H2D without host sync)
    MQMeta *h_meta[2] = {nullptr, nullptr};
    size_t h_meta_cap[2] = {0, 0};
    cudaEvent_t meta_ev[2] = {nullptr, nullptr};
    int meta_slot = 0;
    // side streams: the per-item-query DTW launches (different rho templates)
    // run concurrently so their grid tails overlap
    cudaStream_t side[kMaxLen] = {};
    cudaEvent_t fork_ev = nullptr;
    cudaEvent_t join_ev[kMaxLen] = {};
};

static inline int64_t m_ndw_of(const SensorInfo &si, int w) { return si.n / w; }

static int side_fork(smiler_index *idx, int n) {
    if (!idx->fork_ev) CU(cudaEventCreateWithFlags(&idx->fork_ev, cudaEventDisableTiming));
    CU(cudaEventRecord(idx->fork_ev, idx->stream));
    for (int i = 0; i < n; i++) {
        if (!idx->side[i]) {
            CU(cudaStreamCreateWithFlags(&idx->side[i], cudaStreamNonBlocking));
            CU(cudaEventCreateWithFlags(&idx->join_ev[i], cudaEventDisableTiming));
        }
        CU(cudaStreamWaitEvent(idx->side[i], idx->fork_ev, 0));
    }
    return SMILER_OK;
}

static int side_join(smiler_index *idx, int n) {
    for (int i = 0; i < n; i++) {
        CU(cudaEventRecord(idx->join_ev[i], idx->side[i]));
        CU(cudaStreamWaitEvent(idx->stream, idx->join_ev[i], 0));
    }
    return SMILER_OK;
}

// Pinned staging slot for n MQMeta; waits until the copy that last used the
// slot has completed.
static int meta_stage(smiler_index *idx, int n, MQMeta **out, int *slot) {
    const int s = idx->meta_slot;
    idx->meta_slot ^= 1;
    if (!idx->meta_ev[s]) CU(cudaEventCreateWithFlags(&idx->meta_ev[s], cudaEventDisableTiming));
    else CU(cudaEventSynchronize(idx->meta_ev[s]));
    if (idx->h_meta_cap[s] < (size_t)n) {
        if (idx->h_meta[s]) cudaFreeHost(idx->h_meta[s]);
        idx->h_meta[s] = nullptr;
        size_t want = (size_t)n + n / 4 + 16;
        CU(cudaMallocHost(&idx->h_meta[s], want * sizeof(MQMeta)));
        idx->h_meta_cap[s] = want;
    }
    *out = idx->h_meta[s];
    *slot = s;
    return SMILER_OK;
}

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) once per kernel and size.
// Opt a kernel in to `bytes` of dynamic shared memory.  Always set (not only
// above 48 KB): the default cap is 48 KB minus the kernel's STATIC shared
// memory, so e.g. 34 KB dynamic + 16 KB static fails to launch without it.
// The attribute is per device, so the record is keyed by (device, kernel) and
// guarded by a mutex (handles on different devices / threads are independent).
static void set_smem(const void *kern, size_t bytes) {
    static std::mutex mu;
    static std::map<std::pair<int, const void *>, size_t> done;
    if (bytes == 0) return;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lk(mu);
    const auto key = std::make_pair(dev, kern);
    auto it = done.find(key);
    if (it != done.end() && it->second >= bytes) return;
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) == cudaSuccess)
        done[key] = bytes;
    else
        cudaGetLastError();  // the launch reports the failure
}

static size_t esize(smiler_dtype t) { return t == SMILER_I16 ? 2 : 4; }

static int set_device(smiler_index *idx) {
    CU(cudaSetDevice(idx->device));
    return SMILER_OK;
}

template <typename T> struct TypeTag { using type = T; };

#ifndef SMILER_CASCADE_ONESHOT
#define SMILER_CASCADE_ONESHOT 0  // 1: the LB_Keogh cascade in one-shot searches too
#endif
#ifndef SMILER_CASCADE_MIN_RHO
#define SMILER_CASCADE_MIN_RHO 0  // the LB_Keogh cascade runs for item queries with rho_i >= this
#endif
// smiler_knn_opts.variant values (include/smiler.h): kernel paths with the same result
constexpr int kVarRowFused = 1, kVarScalarDiag = 2, kVarWaveDtw = 3, kVarNoCascade = 4, kVarNoLag = 5,
              kVarPackedDtw = 6, kVarRingNoTma = 7, kVarTmaOneTile = 8, kVarTrimRadix = 9, kVarTrimTwoStage = 10;
constexpr int kMaxDI16 = 256;  // R17: 2046^2 (2d - 1) < 2^31 for d <= 256

static int check_opts(const smiler_knn_opts &o) {
    const int v = o.variant;
    if (v != 0 && v != kVarRowFused && v != kVarScalarDiag && v != kVarWaveDtw && v != kVarNoCascade && v != kVarNoLag &&
        v != kVarPackedDtw && v != kVarRingNoTma && v != kVarTmaOneTile && v != kVarTrimRadix &&
        v != kVarTrimTwoStage)
        return fail(SMILER_EINVAL, "opts.variant %d is not a known kernel path", v);
#if !SMILER_EXPERIMENTS
    if (o.reserved != 0) return fail(SMILER_EINVAL, "opts.reserved must be 0");
#endif
    return SMILER_OK;
}

// The sticky range flag of I16 device queries (query_prep_kernel sets it
// through the host mapping): reported once, then cleared.
static int take_qflag(smiler_index *idx) {
    volatile int *f = idx->qflag_h;
    if (f && *f) {
        *f = 0;
        return fail(SMILER_ERANGE, "an I16 master query in device memory held a value outside [-1023, 1023] "
                                   "(R17); that call's results are unspecified");
    }
    return SMILER_OK;
}

static int rho_for(float band, int d) {
    if (band >= 1.0f) return (int)band;
    if (band <= 0.0f) return 0;
    return (int)floorf(band * (float)d);
}

// a1: envelope of every sensor with width rho, cached per rho.
static int ensure_envelope(smiler_index *idx, int rho, void **U, void **L) {
    auto it = idx->env.find(rho);
    if (it != idx->env.end()) {
        *U = it->second.first;
        *L = it->second.second;
        return SMILER_OK;
    }
    const size_t bytes = (size_t)idx->dev_elems * esize(idx->dtype);
    void *u = nullptr, *l = nullptr;
    CU(cudaMalloc(&u, bytes));
    cudaError_t e = cudaMalloc(&l, bytes);
    if (e != cudaSuccess) {
        cudaFree(u);
        return fail(SMILER_ENOMEM, "envelope alloc: %s", cudaGetErrorString(e));
    }
    int64_t nmax = 0;
    for (auto &s : idx->sensors) nmax = std::max(nmax, s.n);
    dim3 grid((unsigned)((nmax + kEnvTile - 1) / kEnvTile), (unsigned)idx->sensors.size());
    size_t smem = (size_t)(kEnvTile + 2 * rho) * esize(idx->dtype);
    if (idx->dtype == SMILER_I16) {
        set_smem((const void *)envelope_kernel<int16_t>, smem);
        envelope_kernel<int16_t><<<grid, 256, smem, idx->stream>>>(
            (const int16_t *)idx->d_series, idx->d_soff, idx->d_slen, rho, (int16_t *)u, (int16_t *)l);
    } else {
        set_smem((const void *)envelope_kernel<float>, smem);
        envelope_kernel<float><<<grid, 256, smem, idx->stream>>>(
            (const float *)idx->d_series, idx->d_soff, idx->d_slen, rho, (float *)u, (float *)l);
    }
    CHECK_LAUNCH();
    idx->env[rho] = {u, l};
    *U = u;
    *L = l;
    return SMILER_OK;
}

static int upload_series(smiler_index *idx, const void *series, const int64_t *offs, int ns) {
    const size_t es = esize(idx->dtype);
    const int64_t align = 64;
    int64_t total = 0;
    std::vector<int64_t> dev_off(ns);
    for (int s = 0; s < ns; s++) {
        dev_off[s] = total;
        total += (offs[s + 1] - offs[s] + align - 1) / align * align;
    }
    total += align;
    idx->dev_elems = total;
    CU(cudaMalloc(&idx->d_series, (size_t)total * es));
    CU(cudaMemsetAsync(idx->d_series, 0, (size_t)total * es, idx->stream));
    const bool dev = is_device_ptr(series);
    for (int s = 0; s < ns; s++) {
        const int64_t n = offs[s + 1] - offs[s];
        CU(cudaMemcpyAsync((char *)idx->d_series + dev_off[s] * es,
                           (const char *)series + offs[s] * es, (size_t)n * es,
                           dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, idx->stream));
        idx->sensors[s].off = dev_off[s];
    }
    std::vector<int64_t> so(ns), sl(ns);
    for (int s = 0; s < ns; s++) {
        so[s] = idx->sensors[s].off;
        sl[s] = idx->sensors[s].n;
    }
    CU(cudaMalloc(&idx->d_soff, sizeof(int64_t) * ns));
    CU(cudaMalloc(&idx->d_slen, sizeof(int64_t) * ns));
    CU(cudaMemcpyAsync(idx->d_soff, so.data(), sizeof(int64_t) * ns, cudaMemcpyHostToDevice, idx->stream));
    CU(cudaMemcpyAsync(idx->d_slen, sl.data(), sizeof(int64_t) * ns, cudaMemcpyHostToDevice, idx->stream));
    // I16 range (R17) and max |x| (the series bound of the fp16 storage scales, R26)
    int *chk = nullptr;
    CU(cudaMalloc(&chk, 2 * sizeof(int)));
    CU(cudaMemsetAsync(chk, 0, 2 * sizeof(int), idx->stream));
    if (idx->dtype == SMILER_I16) {
        range_check_kernel<<<idx->num_sms * 4, 256, 0, idx->stream>>>((const int16_t *)idx->d_series, total, chk);
        absmax_kernel<int16_t><<<idx->num_sms * 4, 256, 0, idx->stream>>>((const int16_t *)idx->d_series, total,
                                                                          (unsigned *)chk + 1);
    } else {
        absmax_kernel<float><<<idx->num_sms * 4, 256, 0, idx->stream>>>((const float *)idx->d_series, total,
                                                                        (unsigned *)chk + 1);
    }
    int hb[2] = {0, 0};
    cudaMemcpyAsync(hb, chk, sizeof(hb), cudaMemcpyDeviceToHost, idx->stream);
    cudaError_t e = cudaStreamSynchronize(idx->stream);
    cudaFree(chk);
    if (e != cudaSuccess) return fail(SMILER_ECUDA, "series checks: %s", cudaGetErrorString(e));
    if (hb[0]) return fail(SMILER_ERANGE, "%d I16 values outside [-1023, 1023] (R17)", hb[0]);
    memcpy(&idx->smax, &hb[1], sizeof(float));
    if (!isfinite(idx->smax)) return fail(SMILER_EINVAL, "the series holds a non-finite value");
    return SMILER_OK;
}

static void destroy(smiler_index *idx) {
    if (!idx) return;
    cudaSetDevice(idx->device);
    if (idx->stream) cudaStreamSynchronize(idx->stream);
    if (idx->d_series) cudaFree(idx->d_series);
    if (idx->d_soff) cudaFree(idx->d_soff);
    if (idx->d_slen) cudaFree(idx->d_slen);
    for (auto &kv : idx->env) {
        cudaFree(kv.second.first);
        cudaFree(kv.second.second);
    }
    DevBuf *bufs[] = {&idx->queries, &idx->qv,     &idx->qtab,   &idx->meta,   &idx->post,
                      &idx->lb,      &idx->surv,   &idx->fin,    &idx->tauc,   &idx->taulb,  &idx->tauk,
                      &idx->taukey,  &idx->thr,    &idx->scount, &idx->fcount, &idx->taskoff,
                      &idx->out_ids, &idx->out_d,  &idx->tmp,    &idx->tmp2,   &idx->pred,   &idx->lbs,
                      &idx->qenv,    &idx->surv2,  &idx->scount2};
    for (DevBuf *b : bufs) b->release();
    for (auto ev : idx->events) cudaEventDestroy(ev);
    for (int i = 0; i < kMaxLen; i++) {
        if (idx->side[i]) cudaStreamDestroy(idx->side[i]);
        if (idx->join_ev[i]) cudaEventDestroy(idx->join_ev[i]);
    }
    if (idx->fork_ev) cudaEventDestroy(idx->fork_ev);
    for (int s = 0; s < 2; s++) {
        if (idx->h_meta[s]) cudaFreeHost(idx->h_meta[s]);
        if (idx->meta_ev[s]) cudaEventDestroy(idx->meta_ev[s]);
    }
    if (idx->qflag_h) cudaFreeHost(idx->qflag_h);
    delete idx;
}

static int common_build(smiler_index *idx, int32_t device, void *stream) {
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return fail(SMILER_ECUDA, "no CUDA device available (%s); there is no CPU fallback",
                    cudaGetErrorString(e));
    }
    if (device < 0 || device >= ndev) return fail(SMILER_EINVAL, "device %d out of range [0,%d)", device, ndev);
    idx->device = device;
    idx->stream = (cudaStream_t)stream;
    CU(cudaSetDevice(device));
    CU(cudaDeviceGetAttribute(&idx->num_sms, cudaDevAttrMultiProcessorCount, device));
    size_t fr = 0, tot = 0;
    if (cudaMemGetInfo(&fr, &tot) == cudaSuccess) idx->budget = std::min(idx->budget, fr / 2);
    cudaGetLastError();
    CU(cudaHostAlloc(&idx->qflag_h, sizeof(int), cudaHostAllocMapped));
    *idx->qflag_h = 0;
    CU(cudaHostGetDevicePointer(&idx->qflag_d, idx->qflag_h, 0));
    return SMILER_OK;
}

extern "C" int smiler_index_build(const void *series, smiler_dtype dtype, int64_t n_total,
                                  const int64_t *sensor_offsets, int32_t n_sensors, int32_t window,
                                  float band, int32_t device, void *cuda_stream, smiler_index **out) {
    if (!out) return fail(SMILER_EINVAL, "out is NULL");
    *out = nullptr;
    if (!series) return fail(SMILER_EINVAL, "series is NULL");
    if (dtype != SMILER_I16 && dtype != SMILER_F32) return fail(SMILER_EINVAL, "bad dtype %d", (int)dtype);
    if (n_total < 1) return fail(SMILER_EINVAL, "n_total must be >= 1");
    if (window < 1 || window > kMaxWindow) return fail(SMILER_EINVAL, "window must be in [1, %d]", kMaxWindow);
    if (!(band >= 0.f) || !isfinite(band)) return fail(SMILER_EINVAL, "band must be finite and >= 0");
    std::vector<int64_t> offs;
    if (sensor_offsets) {
        if (n_sensors < 1) return fail(SMILER_EINVAL, "n_sensors must be >= 1");
        std::vector<int64_t> h(n_sensors + 1);
        if (is_device_ptr(sensor_offsets)) {
            if (cudaMemcpy(h.data(), sensor_offsets, sizeof(int64_t) * (n_sensors + 1),
                           cudaMemcpyDeviceToHost) != cudaSuccess)
                return fail(SMILER_ECUDA, "reading sensor_offsets");
        } else {
            memcpy(h.data(), sensor_offsets, sizeof(int64_t) * (n_sensors + 1));
        }
        if (h[0] != 0 || h[n_sensors] != n_total) return fail(SMILER_EINVAL, "sensor_offsets must start at 0 and end at n_total");
        for (int s = 0; s < n_sensors; s++)
            if (h[s + 1] <= h[s]) return fail(SMILER_EINVAL, "sensor %d is empty or offsets not ascending", s);
        offs = h;
    } else {
        n_sensors = 1;
        offs = {0, n_total};
    }
    // candidate starts t are 32-bit in the tau / survivor / finalist lists and keys
    for (int s = 0; s < n_sensors; s++)
        if (offs[s + 1] - offs[s] - 1 > (int64_t)INT32_MAX)
            return fail(SMILER_EINVAL, "sensor %d has more than 2^31 points", s);
    smiler_index *idx = new smiler_index();
    int rc = common_build(idx, device, cuda_stream);
    if (rc) {
        delete idx;
        return rc;
    }
    idx->dtype = dtype;
    idx->window = window;
    idx->band = band;
    idx->sensors.resize(n_sensors);
    for (int s = 0; s < n_sensors; s++) {
        SensorInfo &si = idx->sensors[s];
        si.n = offs[s + 1] - offs[s];
        si.origin = 0;
        si.t_lo = 0;
        si.t_hi = si.n;
        si.n_global = si.n;
        si.slice_begin = 0;
    }
    rc = upload_series(idx, series, offs.data(), n_sensors);
    if (rc == SMILER_OK && band >= 1.0f) {
        void *U, *L;
        rc = ensure_envelope(idx, rho_for(band, 1), &U, &L);
    }
    if (rc == SMILER_OK) {
        cudaError_t e = cudaStreamSynchronize(idx->stream);
        if (e != cudaSuccess) rc = fail(SMILER_ECUDA, "index build: %s", cudaGetErrorString(e));
    }
    if (rc) {
        destroy(idx);
        return rc;
    }
    *out = idx;
    return SMILER_OK;
}

extern "C" int smiler_index_build_shard(const void *slice, smiler_dtype dtype, int64_t n_slice,
                                        int64_t slice_begin, int64_t n_global, int64_t t_begin,
                                        int64_t t_end, int32_t window, float band, int32_t device,
                                        void *cuda_stream, smiler_index **out) {
    if (!out) return fail(SMILER_EINVAL, "out is NULL");
    *out = nullptr;
    if (window < 1 || window > kMaxWindow) return fail(SMILER_EINVAL, "window must be in [1, %d]", kMaxWindow);
    if (n_slice < 1 || slice_begin < 0 || slice_begin + n_slice > n_global)
        return fail(SMILER_EINVAL, "slice [%lld, +%lld) outside the series of %lld points",
                    (long long)slice_begin, (long long)n_slice, (long long)n_global);
    if (slice_begin % window) return fail(SMILER_EINVAL, "slice_begin must be a multiple of window");
    if (t_begin < slice_begin || t_end < t_begin || t_end > slice_begin + n_slice)
        return fail(SMILER_EINVAL, "owned range [%lld, %lld) not inside the slice", (long long)t_begin,
                    (long long)t_end);
    if (n_global - 1 > (int64_t)INT32_MAX) return fail(SMILER_EINVAL, "series longer than 2^31 points");
    int64_t offs[2] = {0, n_slice};
    smiler_index *idx = nullptr;
    int rc = smiler_index_build(slice, dtype, n_slice, offs, 1, window, band, device, cuda_stream, &idx);
    if (rc) return rc;
    idx->shard = true;
    SensorInfo &si = idx->sensors[0];
    si.origin = slice_begin;
    si.t_lo = t_begin - slice_begin;
    si.t_hi = t_end - slice_begin;
    si.n_global = n_global;
    si.slice_begin = slice_begin;
    *out = idx;
    return SMILER_OK;
}

extern "C" void smiler_free(smiler_index *idx) { destroy(idx); }

extern "C" const char *smiler_last_error(void) { return g_err.c_str(); }

extern "C" int32_t smiler_abi_version(void) { return SMILER_ABI_VERSION; }

// ---------------------------------------------------------------------------
// smiler_knn
// ---------------------------------------------------------------------------
struct Plan {
    int D, n_len, k, w, rho_env;
    std::vector<int> len, rho;
    int RT;          // group-scan CTA width (two-level path)
    bool scan_reg;   // a4 by group_scan_reg_kernel (static w, mmax <= 64)
    bool fused;      // a3+a4 fused kernel
    int fused_kind;  // 0 = diagonal form (lb_diag_kernel), 1 = row form (lb_fused_kernel)
    int lb_kind;     // smiler_knn_opts.lb_kind (SMILER_LB_*)
    bool direct;     // SMILER_LB_DIRECT*: lb_direct_kernel, no window level
    int RTf;         // fused: tile DWs per CTA
    bool wave = false;  // opts.variant 3: the wavefront DTW kernel for every rho (A/B)
    bool packed_dtw = false;  // opts.variant 6: f32 register band with fp32x2-packed row pairs (A/B)
    size_t smem_gs, smem_fz;
};

static int validate_query(smiler_index *idx, const int32_t *lengths_h, int n_len, int k, Plan &pl) {
    if (n_len < 1 || n_len > kMaxLen) return fail(SMILER_EINVAL, "n_len must be in [1, %d]", kMaxLen);
    if (k < 1 || k > kMaxK) return fail(SMILER_EINVAL, "k must be in [1, %d]", kMaxK);
    pl.len.assign(lengths_h, lengths_h + n_len);
    for (int i = 0; i < n_len; i++) {
        if (pl.len[i] < 1) return fail(SMILER_EINVAL, "lengths[%d] < 1", i);
        if (i && pl.len[i] <= pl.len[i - 1]) return fail(SMILER_EINVAL, "lengths must be strictly increasing");
    }
    pl.D = pl.len[n_len - 1];
    if (pl.D > kMaxD) return fail(SMILER_EINVAL, "D = %d exceeds %d", pl.D, kMaxD);
    if (idx->dtype == SMILER_I16 && pl.D > kMaxDI16)
        return fail(SMILER_EINVAL, "I16: D = %d exceeds %d (int32 exactness of every DTW and bound, R17)", pl.D,
                    kMaxDI16);
    pl.w = idx->window;
    if (pl.w > pl.D) return fail(SMILER_EINVAL, "window %d longer than D = %d", pl.w, pl.D);
    pl.n_len = n_len;
    pl.k = k;
    pl.rho.resize(n_len);
    pl.rho_env = 0;
    for (int i = 0; i < n_len; i++) {
        int r = rho_for(idx->band, pl.len[i]);
        pl.rho_env = std::max(pl.rho_env, r);  // R4: envelopes use rho_max
        pl.rho[i] = std::min(r, pl.len[i] - 1);  // rho >= d-1 is unconstrained DTW
        // rho > kMaxRhoFast: the anti-diagonal wavefront kernel (any rho)
    }
    const size_t vs = 4;
    const int mmax = pl.D / pl.w;
    const size_t em = ((size_t)mmax * pl.w * 2 + 15) & ~(size_t)15;
    int64_t n_max = 0;
    for (const auto &si : idx->sensors) n_max = std::max<int64_t>(n_max, si.n);
    // register scan: emission bitmasks hold mmax rows; posting offsets are int32
    pl.scan_reg = (pl.w == 4 || pl.w == 8 || pl.w == 16 || pl.w == 32) && mmax <= 64 &&
                  2 * (int64_t)(pl.D - pl.w + 1) * (n_max / pl.w) < ((int64_t)1 << 31);
    if (pl.scan_reg) {
        pl.RT = kScanThreads;
        pl.smem_gs = 0;
    } else {
        pl.RT = 256;
        while (pl.RT > 32 && em + (size_t)n_len * pl.RT * (pl.w + 1) * vs > 160 * 1024) pl.RT >>= 1;
        pl.smem_gs = em + (size_t)n_len * pl.RT * (pl.w + 1) * vs;
    }
    pl.fused = false;
    if (pl.w == 4 || pl.w == 8 || pl.w == 16) {
        const int halo = mmax - 1;
        pl.RTf = kFusedThreads - halo;
        pl.smem_fz = em + (size_t)pl.D * 12 + (size_t)2 * pl.w * kFusedThreads * 8 +
                     (size_t)n_len * pl.RTf * (pl.w + 1) * vs;
        pl.fused = halo <= kFusedThreads / 4 && pl.smem_fz <= 200 * 1024;
        pl.fused_kind = 1;
        const int ds = pl.w == 4 ? 12 : pl.w + 4;
        const size_t smem_dg = (size_t)3 * ((pl.D + 3 + 32 + 3) & ~3) * vs + (size_t)3 * kDiagCols * ds * vs;
        if (halo <= kDiagHaloMax && mmax <= 64 && smem_dg <= 200 * 1024) {
            pl.fused = true;
            pl.fused_kind = 0;
            pl.RTf = kDiagThreads;
            pl.smem_fz = smem_dg;
        }
    }
    return SMILER_OK;
}

template <typename S>
static int run_dtw_list(smiler_index *idx, const Plan &pl, int li, int n_mq, int mode,
                        const int32_t *list, int LT, const int32_t *counts, int32_t *task_off,
                        uint64_t *keys_out, const uint64_t *tau_key, uint64_t *fin,
                        int32_t *fin_count, const MQMeta *d_meta, const typename Tr<S>::V *qv,
                        int D, cudaStream_t st = nullptr, int LTc = -1) {
    if (!st) st = idx->stream;
    if (LTc < 0) LTc = LT;  // tau mode: verify the first LTc entries of each stride-LT list
    task_prefix_kernel<<<1, 1024, 0, st>>>(counts, mode == 0 ? LTc : -1, n_mq, pl.n_len, li, task_off);
    CHECK_LAUNCH();
    DtwParams<S> p;
    p.series = (const S *)idx->d_series;
    p.meta = d_meta;
    p.qv = qv;
    p.D = D;
    p.n_len = pl.n_len;
    p.li = li;
    p.d = pl.len[li];
    p.n_mq = n_mq;
    p.mode = mode;
    p.list = list;
    p.LT = LT;
    p.LTc = LTc;
    p.counts = counts;
    p.task_off = task_off;
    p.keys_out = keys_out;
    p.tau_key = tau_key;
    p.fin = fin;
    p.fin_count = fin_count;
    p.wave = pl.wave ? 1 : 0;
    p.packed = pl.packed_dtw ? 1 : 0;
    launch_dtw<S>(pl.rho[li], p, 0, st);
    CHECK_LAUNCH();
    return SMILER_OK;
}

// NVTX ranges (host timeline; nsys / ncu attribute the kernels launched inside
// them): one range per smiler_knn chunk phase, opened at each phase boundary.
// Without an attached tool the NVTX calls are no-ops.
// kPhaseName[p] names the phase that runs after mark(p) (mark(5): the cascade,
// whose end is mark(8)).
static const char *const kPhaseName[9] = {"smiler a2 query prep", "smiler a3/a4 lower bounds",
                                          "smiler a4 group scan", "smiler a5 tau",
                                          "smiler a6 filter", "smiler a6b cascade",
                                          "smiler a8 select", nullptr, "smiler a7 verify"};
struct PhaseTimer {
    smiler_index *idx;
    bool on;
    std::vector<std::pair<int, int>> marks;  // (phase, event index)
    int next = 0;
    bool nvtx_open = false;
    ~PhaseTimer() {
        if (nvtx_open) nvtxRangePop();
    }
    int mark(int phase) {
        if (nvtx_open) nvtxRangePop();
        nvtx_open = phase < 9 && kPhaseName[phase];
        if (nvtx_open) nvtxRangePushA(kPhaseName[phase]);
        if (!on) return SMILER_OK;
        if (next >= (int)idx->events.size()) {
            cudaEvent_t ev;
            CU(cudaEventCreate(&ev));
            idx->events.push_back(ev);
        }
        CU(cudaEventRecord(idx->events[next], idx->stream));
        marks.push_back({phase, next});
        next++;
        return SMILER_OK;
    }
};

// Continuous-stream context (Remark 1): posting lists live in a per-stream ring.
struct StreamCtx {
    void *ring;                // V [sum over streams of 2 n_sw n_dw]: P_EQ plane, P_EC plane
    const int64_t *ring_off;   // per stream (global index) element offset into ring
    int cursor;                // physical row of SW_0
    int mode;                  // 0: build every row; 1: incremental rows [0, nrows)
    int nrows;
    int64_t *d_prev_out;       // device copy of the results (next step's tau seeds)
    bool post_half;            // ring entries are fp16 rounded toward zero (f32 index, static w)
    bool tma;                  // ring laid out for group_scan_tma_kernel (padded stride, mirrored rows)
    int64_t pstride;           // ring row stride (elements)
    int prows;                 // ring rows per plane
    const CUtensorMap *tmap;   // the ring as one 2-D tensor (tma): w x 256 boxes
    const CUtensorMap *tmap_tail;  // the same tensor, w x (16 bytes) boxes
    float pscale;              // fp16 ring: entries hold P x pscale (a power of two, R26)
    // lagged tile tau set (stream steps): this step's scan-unit candidates are kept
    // per stream and, shifted by one point, form the next step's tile tau set, so
    // the thresholds exist before the next scan and the filter runs inside it
    DevBuf *lag_t, *lag_lb;    // [n_streams][n_len][lag_LTt] t and LB_w bits
    int *lag_LTt;              // entries per (stream, item query) saved by the last call; -1 = none
};

template <typename S>
static int knn_impl(smiler_index *idx, const void *queries, const int32_t *query_sensor_in,
                    int32_t n_mq, const int32_t *lengths_in, int32_t n_len, int32_t k, int64_t *ids,
                    void *dists, smiler_knn_stats *stats, const smiler_knn_opts *opts,
                    bool lb_only, void *post_out, void *lb_out, const int64_t *prev_ids = nullptr,
                    int shift = 0, const StreamCtx *sctx = nullptr) {
    using V = typename Tr<S>::V;
    using V2 = typename Tr<S>::V2;
    using V4 = typename Tr<S>::V4;
    smiler_knn_opts o;
    memset(&o, 0, sizeof(o));
    if (opts) o = *opts;
    TRY(check_opts(o));
    if (!queries) return fail(SMILER_EINVAL, "queries is NULL");
    if (n_mq < 1) return fail(SMILER_EINVAL, "n_mq must be >= 1");
    if (!lengths_in) return fail(SMILER_EINVAL, "lengths is NULL");
    if (!lb_only && (!ids || !dists)) return fail(SMILER_EINVAL, "ids/dists is NULL");
    TRY(set_device(idx));
    std::vector<int32_t> lens_h(n_len > 0 ? n_len : 1);
    if (n_len < 1 || n_len > kMaxLen) return fail(SMILER_EINVAL, "n_len must be in [1, %d]", kMaxLen);
    if (is_device_ptr(lengths_in)) CU(cudaMemcpy(lens_h.data(), lengths_in, 4 * n_len, cudaMemcpyDeviceToHost));
    else memcpy(lens_h.data(), lengths_in, 4 * n_len);
    Plan pl;
    TRY(validate_query(idx, lens_h.data(), n_len, lb_only ? 1 : k, pl));
    if (o.two_level || (lb_only && post_out) || sctx) pl.fused = false;
    if (o.lb_kind < SMILER_LB_INDEX || o.lb_kind > SMILER_LB_DIRECT_SHARED)
        return fail(SMILER_EINVAL, "lb_kind %d is not a SMILER_LB_* value", o.lb_kind);
    pl.lb_kind = o.lb_kind;
    pl.wave = o.variant == kVarWaveDtw;
    pl.packed_dtw = o.variant == kVarPackedDtw;
    if (o.horizon < 0) return fail(SMILER_EINVAL, "horizon must be >= 0");
    pl.direct = o.lb_kind >= SMILER_LB_DIRECT;
    if (pl.direct && (sctx || (lb_only && post_out)))
        return fail(SMILER_EINVAL, "the direct lower bounds have no window level (posting lists / streams)");
    if (pl.direct) pl.fused = false;
    if (pl.fused && o.variant == kVarRowFused && pl.fused_kind == 0) {  // row-form fused kernel (comparison)
        const int mmax = pl.D / pl.w, halo = mmax - 1;
        const size_t em = ((size_t)mmax * pl.w * 2 + 15) & ~(size_t)15;
        pl.fused_kind = 1;
        pl.RTf = kFusedThreads - halo;
        pl.smem_fz = em + (size_t)pl.D * 12 + (size_t)2 * pl.w * kFusedThreads * 8 +
                     (size_t)pl.n_len * pl.RTf * (pl.w + 1) * 4;
        if (halo > kFusedThreads / 4 || pl.smem_fz > 200 * 1024) pl.fused = false;
    }
    const int D = pl.D, w = pl.w, nl = pl.n_len;
    std::vector<int32_t> qsens(n_mq, 0);
    if (query_sensor_in) {
        if (is_device_ptr(query_sensor_in)) CU(cudaMemcpy(qsens.data(), query_sensor_in, 4 * (size_t)n_mq, cudaMemcpyDeviceToHost));
        else memcpy(qsens.data(), query_sensor_in, 4 * (size_t)n_mq);
    }
    for (int j = 0; j < n_mq; j++) {
        if (qsens[j] < 0 || qsens[j] >= (int)idx->sensors.size())
            return fail(SMILER_EINVAL, "query_sensor[%d] = %d out of range", j, qsens[j]);
        const SensorInfo &si = idx->sensors[qsens[j]];
        if (!idx->shard && pl.D > si.n)
            return fail(SMILER_EINVAL, "D = %d longer than sensor %d (%lld points)", pl.D, qsens[j], (long long)si.n);
        if (idx->shard) {
            const int64_t need_lo = std::max<int64_t>(0, si.t_lo + si.slice_begin - pl.rho_env);
            const int64_t need_hi = std::min<int64_t>(si.n_global, si.t_hi + si.slice_begin + pl.D - 1 + pl.rho_env);
            if (si.slice_begin > need_lo || si.slice_begin + si.n < need_hi)
                return fail(SMILER_EINVAL, "shard halo too small: need [%lld, %lld), have [%lld, %lld)",
                            (long long)need_lo, (long long)need_hi, (long long)si.slice_begin,
                            (long long)(si.slice_begin + si.n));
        }
    }
    if (lb_only) {
        for (int j = 1; j < n_mq; j++)
            if (idx->sensors[qsens[j]].n != idx->sensors[qsens[0]].n)
                return fail(SMILER_EINVAL, "smiler_lower_bounds needs sensors of equal length");
    }
    void *dUC, *dLC;
    TRY(ensure_envelope(idx, pl.rho_env, &dUC, &dLC));

    const size_t es = sizeof(S);
    const bool q_dev = is_device_ptr(queries);
    TRY(take_qflag(idx));  // from an earlier call that returned before its kernels ran
    if (std::is_same<S, int16_t>::value && !q_dev) {  // R17 on the host copy
        const int16_t *qq = (const int16_t *)queries;
        for (int64_t x = 0; x < (int64_t)n_mq * D; x++)
            if (qq[x] > 1023 || qq[x] < -1023)
                return fail(SMILER_ERANGE, "queries[%lld] = %d outside [-1023, 1023] (R17)", (long long)x, (int)qq[x]);
    }
    const bool out_dev = lb_only ? (is_device_ptr(lb_out) || (post_out && is_device_ptr(post_out)))
                                 : (is_device_ptr(ids) && is_device_ptr(dists));
    if (!lb_only && (is_device_ptr(ids) != is_device_ptr(dists)))
        return fail(SMILER_EINVAL, "ids and dists must both be host or both be device buffers");

    // ---- per-MQ sizes and chunking -------------------------------------
    const int n_sw = D - w + 1;
    auto mq_bytes = [&](int j) -> size_t {
        const SensorInfo &si = idx->sensors[qsens[j]];
        const size_t ndw = (size_t)(si.n / w);
        return ((pl.fused || pl.direct || sctx) ? 0 : (size_t)n_sw * ndw * 8) + (size_t)nl * si.n * (4 + 4 + 8) +
               4096;
    };
    size_t budget = idx->budget;  // halved on ENOMEM (e.g. a resident stream ring)
    int chunk_max = o.mq_chunk > 0 ? o.mq_chunk : 65535;
    chunk_max = std::min(chunk_max, 65535);

    if (stats) {
        memset(stats, 0, sizeof(*stats));
        TRY(idx->tmp.ensure(8 * (2 * kMaxLen + 1)));
        CU(cudaMemsetAsync(idx->tmp.p, 0, 8 * (2 * kMaxLen + 1), idx->stream));
    }
    PhaseTimer tm{idx, stats != nullptr && o.timing != 0};
    int launches = 0;
    int64_t tau_slots_total = 0;
    double cells_acc = 0, bf_cells = 0;
    int64_t cand_total = 0, surv_total = 0, fin_total = 0, post_bytes = 0, lb_bytes = 0, casc_total = 0;
    int lag_LTt_seen = -2;  // -2: no chunk saved yet; -1: chunks differ (no lagged set next step)
    int n_chunks = 0;

    for (int c0 = 0; c0 < n_mq;) {
        // choose the chunk
        size_t acc = 0;
        int c1 = c0;
        while (c1 < n_mq && c1 - c0 < chunk_max) {
            size_t b = mq_bytes(c1);
            if (c1 > c0 && acc + b > budget) break;
            acc += b;
            c1++;
        }
        const int B = c1 - c0;
        n_chunks++;
        const int64_t cand_before = cand_total;
        const double bf_before = bf_cells;
        // ---- metadata ------------------------------------------------------
        MQMeta *meta;
        int mslot;
        TRY(meta_stage(idx, B, &meta, &mslot));
        int64_t post_tot = 0, seg_tot = 0;
        int nblk_min = INT32_MAX, nblk_max = 0;
        for (int j = 0; j < B; j++) {
            const SensorInfo &si = idx->sensors[qsens[c0 + j]];
            MQMeta &m = meta[j];
            m.series_off = si.off;
            m.n = si.n;
            m.origin = si.origin;
            m.t_lo = si.t_lo;
            m.t_hi = si.t_hi;
            // horizon: t + d + h <= N of the full series; a shard's slice ends at
            // slice_begin + n <= n_global, so locally t + d + hz <= n
            m.hz = std::max<int64_t>(0, (int64_t)o.horizon - (si.n_global - (si.slice_begin + si.n)));
            m.n_dw = si.n / w;
            m.post_off = sctx ? sctx->ring_off[c0 + j] : post_tot;
            m.pstride = (sctx && sctx->tma) ? sctx->pstride : m_ndw_of(si, pl.w);
            m.prows = (sctx && sctx->tma) ? sctx->prows : pl.D - pl.w + 1;
            m.seg_off = seg_tot;
            m.nblk = pl.direct ? (int)(m.n / kDirEnds + 1) : (int)(m.n_dw / (pl.fused ? pl.RTf : pl.RT) + 1);
            m.sensor = qsens[c0 + j];
            if (!pl.direct) post_tot += 2 * (int64_t)n_sw * m.n_dw;  // P_EQ and P_EC planes
            seg_tot += (int64_t)nl * si.n;
            nblk_min = std::min(nblk_min, m.nblk);
            nblk_max = std::max(nblk_max, m.nblk);
            for (int i = 0; i < nl; i++) {
                const int64_t tb = std::max<int64_t>(0, si.t_lo);
                const int64_t te = std::min<int64_t>(si.t_hi, si.n - meta[j].hz - pl.len[i] + 1);
                const int64_t nc = te > tb ? te - tb : 0;
                cand_total += nc;
                bf_cells += (double)nc * (double)dtw_cells(pl.len[i], pl.rho[i]);
            }
        }
        // tau-set units: CTAs (block epilogue) or warps (diagonal kernel's warp epilogue)
        // tau units: warps of the diagonal kernel / of group_scan (w in {4,8,16,32}), else CTAs
        const int units_per_blk = pl.direct                          ? kDirThreads / 32
                                  : (pl.fused && pl.fused_kind == 0) ? kDiagThreads / 32
                                  : (!pl.fused && pl.scan_reg)       ? kScanThreads / 32
                                                                     : 1;
        int E = 0;
        const bool use_prev = prev_ids != nullptr && !lb_only && !o.no_prune;
        // LB_Keogh cascade between a6 and a7 (launch_cascade); variant 4 skips it (A/B)
        // continuous steps only (SMILER_CASCADE_ONESHOT = 0): a one-shot search's tau set
        // (keep x k tile candidates) leaves few survivors per item query and the extra
        // pass does not pay (C2 -0.4%, C4 neutral; C5 / C3 streams +6% / +2%:
        // profiles/r02/ab_cascade_minrho.txt)
        const bool cascade = !lb_only && !o.no_prune && o.variant != kVarNoCascade &&
                             (use_prev || SMILER_CASCADE_ONESHOT);
        // per item query: the cascade costs about one LB term (plus the candidate
        // staging) per row of a survivor, the DTW it may save 2 rho_i + 1 cells per
        // row -- narrow bands skip it (their DTW is barely dearer than the cascade)
        auto casc_iq = [&](int i) { return pl.rho[i] >= SMILER_CASCADE_MIN_RHO; };
        if (!lb_only && !o.no_prune) {
            const int umin = nblk_min * units_per_blk;
            // tau set ~ mult * k tile candidates per IQ (plus k shifted previous
            // neighbours in a continuous step, where a smaller tile set suffices)
            int mult = use_prev ? kTauMultCont : kTauMult;
            if (o.tau_mult > 0) mult = o.tau_mult;
            if (o.tau_mult < 0) mult = 0;
            E = mult > 0 ? std::min(kTauEMax, std::max(1, (mult * pl.k + umin - 1) / umin)) : 0;
            // with previous neighbours the tau list must fit the sorting (dedupe) path
            while (use_prev && E > 0 && nblk_max * units_per_blk * E + pl.k > kSortCap) E--;
        }
        // tau list per segment: the LB kernel's tile candidates [0, LTt), then (continuous
        // step, P:1452-1458 / R9) the previous step's k neighbours shifted by `shift`
        const int LTt = nblk_max * units_per_blk * E;
        const int LT = std::max(1, LTt + (use_prev ? pl.k : 0));
        QParams P;
        memset(&P, 0, sizeof(P));
        P.D = D;
        P.w = w;
        P.n_len = nl;
        P.k = pl.k;
        P.rho_env = pl.rho_env;
        P.E = E;
#if SMILER_EXPERIMENTS
        if (o.reserved == 1) P.k = -1;  // timing experiment (results invalid)
        if (o.reserved == 2) P.E = 0;   // timing experiment: no tau set (no pruning)
#endif
        P.LT = LT;
        P.ring_cursor = sctx ? sctx->cursor : 0;
        P.lbsel = pl.lb_kind == SMILER_LB_INDEX_EQ ? 1 : pl.lb_kind == SMILER_LB_INDEX_EC ? 2 : 0;
        P.n_mq = B;
        for (int i = 0; i < nl; i++) {
            P.len[i] = pl.len[i];
            P.rho[i] = pl.rho[i];
        }
        const int nseg = B * nl;
        auto ensure_all = [&]() -> int {
#define ENS(x)                          \
    do {                                \
        int r_ = (x);                   \
        if (r_ != SMILER_OK) return r_; \
    } while (0)
        ENS(idx->meta.ensure(sizeof(MQMeta) * B));
        ENS(idx->queries.ensure(es * (size_t)B * D));
        ENS(idx->qv.ensure(sizeof(V) * (size_t)B * D));
        ENS(idx->qtab.ensure(sizeof(V4) * (size_t)B * D));
        ENS(idx->lbs.ensure(sizeof(float) * (size_t)B));
        if (!sctx) ENS(idx->post.ensure(sizeof(V) * (size_t)std::max<int64_t>(post_tot, 1)));
        {
            // the filter's 16-byte vector loads also touch the unwritten row tails
            // (t > N - d_i) of the LB_w array (masked, never used): zero the buffer
            // once when it grows so no read is of never-initialised memory
            const void *before = idx->lb.p;
            ENS(idx->lb.ensure(sizeof(V) * (size_t)seg_tot));
            if (idx->lb.p != before) CU(cudaMemsetAsync(idx->lb.p, 0, idx->lb.cap, idx->stream));
        }
        if (cascade) {
            ENS(idx->qenv.ensure(sizeof(V2) * (size_t)B * nl * D));
            ENS(idx->surv2.ensure(4 * (size_t)seg_tot));
            ENS(idx->scount2.ensure(4 * (size_t)nseg));
        }
        if (!lb_only) {
            ENS(idx->surv.ensure(4 * (size_t)seg_tot));
            ENS(idx->fin.ensure(8 * (size_t)seg_tot));
            ENS(idx->tauc.ensure(4 * (size_t)nseg * LT));
            ENS(idx->taulb.ensure(4 * (size_t)nseg * LT));
            ENS(idx->tauk.ensure(8 * (size_t)nseg * LT));
            ENS(idx->taukey.ensure(8 * (size_t)nseg));
            ENS(idx->thr.ensure(4 * (size_t)nseg));
            ENS(idx->scount.ensure(4 * (size_t)nseg));
            ENS(idx->fcount.ensure(4 * (size_t)nseg));
            ENS(idx->taskoff.ensure(4 * (size_t)(B + 1) * nl * 3));
            ENS(idx->out_ids.ensure(8 * (size_t)nseg * pl.k));
            ENS(idx->out_d.ensure(4 * (size_t)nseg * pl.k));
        }
#undef ENS
            return SMILER_OK;
        };
        {
            const int rc_ = ensure_all();
            if (rc_ == SMILER_ENOMEM && B > 1) {  // retry this chunk with half the budget
                budget /= 2;
                n_chunks--;
                cand_total = cand_before;
                bf_cells = bf_before;
                g_err.clear();
                cudaGetLastError();
                continue;
            }
            TRY(rc_);
        }
        if (!lb_only) P.taulb = idx->taulb.as<uint32_t>();  // tile tau candidates' LB_w bits (trim keys)
        V *postbuf = sctx ? reinterpret_cast<V *>(sctx->ring) : idx->post.as<V>();
        MQMeta *d_meta = idx->meta.as<MQMeta>();
        CU(cudaMemcpyAsync(d_meta, meta, sizeof(MQMeta) * B, cudaMemcpyHostToDevice, idx->stream));
        CU(cudaEventRecord(idx->meta_ev[mslot], idx->stream));
        CU(cudaMemcpyAsync(idx->queries.p, (const char *)queries + (size_t)c0 * D * es, es * (size_t)B * D,
                           q_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, idx->stream));
        int32_t *scount = idx->scount.as<int32_t>();
        int32_t *fcount = idx->fcount.as<int32_t>();
        uint64_t *taukey = idx->taukey.as<uint64_t>();
        uint32_t *thr = idx->thr.as<uint32_t>();
        if (!lb_only) {
            CU(cudaMemsetAsync(scount, 0, 4 * (size_t)nseg, idx->stream));
            CU(cudaMemsetAsync(fcount, 0, 4 * (size_t)nseg, idx->stream));
        }
        int32_t *taskoff = idx->taskoff.as<int32_t>();
        auto do_a5 = [&]() -> int {
            // ---- a5: tau ------------------------------------------------------
            if (use_prev) {
                const int64_t *pv = prev_ids + (size_t)c0 * nl * pl.k;
                if (!is_device_ptr(prev_ids)) {
                    TRY(idx->tmp2.ensure(8 * (size_t)nseg * pl.k));
                    CU(cudaMemcpyAsync(idx->tmp2.p, pv, 8 * (size_t)nseg * pl.k, cudaMemcpyHostToDevice, idx->stream));
                    pv = idx->tmp2.as<int64_t>();
                }
                prev_tau_kernel<<<nseg, 128, 0, idx->stream>>>(pv, shift, d_meta, P, LTt, idx->tauc.as<int32_t>());
                CHECK_LAUNCH();
                launches++;
            }
            if (!o.no_prune) {
                // trim the tile tau set to its `keep` smallest-LB_w candidates
                int LTc = LT;
                const int keep = tau_keep(o, pl.k, use_prev);
                const int kpv = use_prev ? pl.k : 0;
                const int nch = (LTt + kTrimChunk - 1) / kTrimChunk;
                const bool two_stage = keep > 0 && nch > 1 && (int64_t)nch * keep <= kTrimCap;
                if (keep > 0 && LTt > keep && (LTt <= kTrimBigCap || two_stage)) {
                    const uint32_t *tlb = idx->taulb.as<uint32_t>();
                    auto trim1 = [&](const int32_t *src, int sstride, int nsrc, const uint32_t *slb) {
                        int n2 = 1;
                        while (n2 < nsrc) n2 <<= 1;
                        const size_t sm = (size_t)8 * n2 + (size_t)4 * kpv;
                        set_smem((const void *)tau_trim_kernel<S>, sm);
                        tau_trim_kernel<S><<<nseg, 256, sm, idx->stream>>>(src, sstride, nsrc, idx->tauc.as<int32_t>(),
                                                                           LT, LTt, keep, kpv, idx->lb.as<V>(),
                                                                           d_meta, nl, slb);
                    };
                    // <= kTrimSmall: one bitonic sort; <= kTrimBigCap: radix select in shared
                    // memory; longer: two-stage (chunk bitonic sorts, then one more trim).
                    // variants 9 / 10 (tests): radix / two-stage for any list length
                    const bool test_alt = o.variant == kVarTrimRadix || o.variant == kVarTrimTwoStage;
                    if (LTt <= kTrimSmall && !test_alt) {
                        trim1(idx->tauc.as<int32_t>(), LT, LTt, tlb);
                    } else if (two_stage && (LTt > kTrimBigCap || o.variant == kVarTrimTwoStage)) {
                        // chunk winners into the survivor buffer (unused until a6), then one more trim
                        // (t in the survivor buffer, their LB_w bits in the finalist buffer:
                        // both unused until a6/a7)
                        const int ostride = nch * keep;
                        TRY(idx->surv.ensure(4 * (size_t)nseg * ostride));
                        TRY(idx->fin.ensure(4 * (size_t)nseg * ostride));
                        const size_t sm = (size_t)8 * kTrimChunk;
                        set_smem((const void *)tau_trim_chunk_kernel<S>, sm);
                        tau_trim_chunk_kernel<S><<<dim3(nch, nseg), 256, sm, idx->stream>>>(
                            idx->tauc.as<int32_t>(), LT, LTt, keep, idx->lb.as<V>(), d_meta, nl,
                            idx->surv.as<int32_t>(), ostride, tlb, reinterpret_cast<uint32_t *>(idx->fin.p));
                        CHECK_LAUNCH();
                        launches++;
                        trim1(idx->surv.as<int32_t>(), ostride, ostride, reinterpret_cast<const uint32_t *>(idx->fin.p));
                    } else {  // 32-bit LB keys, radix select in shared memory
                        const size_t sm = (size_t)8 * LTt;
                        set_smem((const void *)tau_trim_big_kernel<S>, sm);
                        tau_trim_big_kernel<S><<<nseg, 256, sm, idx->stream>>>(
                            idx->tauc.as<int32_t>(), LT, LTt, keep, kpv, idx->lb.as<V>(), d_meta, nl, tlb);
                    }
                    CHECK_LAUNCH();
                    launches++;
                    LTc = keep + kpv;
                }
                TRY(side_fork(idx, nl));
                for (int i = 0; i < nl; i++) {
                    TRY(run_dtw_list<S>(idx, pl, i, B, 0, idx->tauc.as<int32_t>(), LT, nullptr,
                                        taskoff + (size_t)i * (B + 1), idx->tauk.as<uint64_t>(), nullptr,
                                        nullptr, nullptr, d_meta, idx->qv.as<V>(), D, idx->side[i], LTc));
                    launches += 2;
                    tau_slots_total += (int64_t)B * LTc;
                    cells_acc += (double)B * LTc * (double)dtw_cells(pl.len[i], pl.rho[i]);
                }
                TRY(side_join(idx, nl));
                tau_select_kernel<S><<<nseg, 256, 0, idx->stream>>>(idx->tauk.as<uint64_t>(), LT, LTc, pl.k, taukey,
                                                                    thr);
                CHECK_LAUNCH();
                launches++;
                if (o.shared_tau) {  // NEXT-2: running threshold shared across the shards
                    tau_share_kernel<S><<<(nseg + 255) / 256, 256, 0, idx->stream>>>(
                        taukey, thr, reinterpret_cast<unsigned long long *>(o.shared_tau) + (size_t)c0 * nl, d_meta,
                        nl, nseg);
                    CHECK_LAUNCH();
                    launches++;
                }
            } else {
                CU(cudaMemsetAsync(taukey, 0xFF, 8 * (size_t)nseg, idx->stream));
            }
            return SMILER_OK;
        };
        // a4+a6 fused: with thresholds known before the scan (a continuous step
        // seeded only by the previous neighbours, E = 0), the LB kernel compares
        // each LB_w with tau_i as it is produced and appends the survivors; the
        // LB_w array is never written or re-read (P:1437-1448 in one pass).
        const bool diag_emitters = pl.direct || (pl.fused && pl.fused_kind == 0) || (!pl.fused && pl.scan_reg);
        // Stream calls keep this scan's tile tau candidates (lag_save); a stream step
        // whose previous call saved them (same list shape) verifies them, shifted by
        // the one-point advance (the continuation of a good candidate, as R9 shifts
        // the previous neighbours), with the previous neighbours BEFORE its scan:
        // any >= k verified candidates give a valid tau (R8), so the thresholds
        // exist before the scan and the filter runs inside it (lagged fuse).
        const bool lag_save = sctx && !lb_only && !o.no_prune && E > 0 && diag_emitters &&
                              o.variant != kVarNoLag;
        const bool lagged = lag_save && sctx->mode == 1 && use_prev && *sctx->lag_LTt == LTt;
        const bool fuse = (use_prev && E == 0 && !lb_only && !o.no_prune && diag_emitters) || lagged;
        if (lag_save) {
            TRY(sctx->lag_t->ensure(4 * (size_t)n_mq * nl * LTt));
            TRY(sctx->lag_lb->ensure(4 * (size_t)n_mq * nl * LTt));
        }
        // LB_w array as fp16 rounded down for the filter (its only reader besides the
        // tau trim, which takes the bounds from P.taulb): half the bytes written by
        // a4 and read by a6.  lb_only (smiler_lower_bounds) and exact_postings keep V.
        P.lb_half = !lb_only && !o.no_prune && diag_emitters && !o.exact_postings;
        P.lbs = idx->lbs.as<float>();
        P.post_unscale = (sctx && sctx->post_half) ? 1.0f / sctx->pscale : 1.0f;
        TRY(tm.mark(0));
        // ---- a2 ----------------------------------------------------------
        IQTab iqt;
        for (int i = 0; i < nl; i++) {
            iqt.len[i] = pl.len[i];
            iqt.rho[i] = pl.rho[i];
        }
        query_prep_kernel<S><<<B, 256, 0, idx->stream>>>(idx->queries.as<S>(), D, pl.rho_env, idx->qv.as<V>(),
                                                         idx->qtab.as<V4>(), idx->smax, idx->lbs.as<float>(),
                                                         idx->qflag_d, iqt, nl,
                                                         cascade ? idx->qenv.as<V2>() : nullptr);
        CHECK_LAUNCH();
        launches++;
        TRY(tm.mark(1));
        if (fuse) {
            if (lagged) {  // the previous call's tile candidates, shifted by one point
                dim3 g((unsigned)((LTt + 255) / 256), (unsigned)nseg);
                lag_tau_kernel<<<g, 256, 0, idx->stream>>>(sctx->lag_t->as<int32_t>() + (size_t)c0 * nl * LTt,
                                                          sctx->lag_lb->as<uint32_t>() + (size_t)c0 * nl * LTt, LTt,
                                                          d_meta, P, idx->tauc.as<int32_t>(), idx->taulb.as<uint32_t>());
                CHECK_LAUNCH();
                launches++;
            }
            TRY(do_a5());
            TRY(tm.mark(4));
            P.fuse = 1;
            P.thr = thr;
            P.surv = idx->surv.as<int32_t>();
            P.scount = scount;
        }
        if (pl.direct) {
            // ---- SMiLer-Dir (ablation): LB_en per candidate, no window level --
            dim3 grid((unsigned)nblk_max, (unsigned)B);
            auto go = [&](int li0, int li1) -> int {
                const size_t smem = dir_smem_elems(pl.len[li1 - 1], D) * sizeof(V);
                set_smem((const void *)lb_direct_kernel<S>, smem);
                lb_direct_kernel<S><<<grid, kDirThreads, smem, idx->stream>>>(
                    (const S *)idx->d_series, (const S *)dUC, (const S *)dLC, d_meta, idx->qtab.as<V4>(), P, li0,
                    li1, idx->lb.as<V>(), idx->tauc.as<int32_t>());
                CHECK_LAUNCH();
                launches++;
                return SMILER_OK;
            };
            if (pl.lb_kind == SMILER_LB_DIRECT)
                for (int i = 0; i < nl; i++) TRY(go(i, i + 1));  // one scan per item query
            else
                TRY(go(0, nl));
            TRY(tm.mark(2));
        } else if (pl.fused) {
            // ---- a3 + a4 fused ------------------------------------------------
            dim3 grid((unsigned)nblk_max, (unsigned)B);
            const int nthr = pl.fused_kind == 0 ? kDiagThreads : kFusedThreads;
            auto go = [&](auto kern) {
                set_smem((const void *)kern, pl.smem_fz);
                kern<<<grid, nthr, pl.smem_fz, idx->stream>>>(
                    (const S *)idx->d_series, (const S *)dUC, (const S *)dLC, d_meta, idx->qtab.as<V4>(), P,
                    idx->lb.as<V>(), idx->tauc.as<int32_t>());
            };
            if (pl.fused_kind == 0) {
                bool done = false;
                if constexpr (std::is_same<S, float>::value) {
                    // f32: the packed fp32x2 form (same sums); variant 2 = the scalar kernel
                    if (o.variant != kVarScalarDiag && P.lbsel == 0) {
                        auto gx = [&](auto kern, size_t smem) {
                            set_smem((const void *)kern, smem);
                            kern<<<grid, kDiagThreads, smem, idx->stream>>>(
                                (const float *)idx->d_series, (const float *)dUC, (const float *)dLC, d_meta,
                                reinterpret_cast<const float4 *>(idx->qtab.p), P, idx->lb.as<float>(),
                                idx->tauc.as<int32_t>());
                        };
                        switch (w) {
                            case 4: gx(lb_diag_x2_kernel<4>, x2_smem<4>(D)); break;
                            case 8: gx(lb_diag_x2_kernel<8>, x2_smem<8>(D)); break;
                            default: gx(lb_diag_x2_kernel<16>, x2_smem<16>(D)); break;
                        }
                        done = true;
                    }
                }
                if (!done) switch (w) {
                    case 4: go(lb_diag_kernel<S, 4>); break;
                    case 8: go(lb_diag_kernel<S, 8>); break;
                    default: go(lb_diag_kernel<S, 16>); break;
                }
            } else {
                switch (w) {
                    case 4: go(lb_fused_kernel<S, 4>); break;
                    case 8: go(lb_fused_kernel<S, 8>); break;
                    default: go(lb_fused_kernel<S, 16>); break;
                }
            }
            CHECK_LAUNCH();
            launches++;
            TRY(tm.mark(2));
        } else {
            // ---- a3 ----------------------------------------------------------
            int64_t ndw_max = 0;
            for (int j = 0; j < B; j++) ndw_max = std::max(ndw_max, meta[j].n_dw);
            const bool w_static = w == 4 || w == 8 || w == 16 || w == 32;
            if (ndw_max > 0 && sctx && sctx->mode == 1 && !w_static) {
                // continuous step: only SW_0 (EQ + EC) and SW_1..SW_rho (EQ) change
                dim3 grid((unsigned)((ndw_max + 127) / 128), (unsigned)B);
                posting_rows_kernel<S><<<grid, 128, 0, idx->stream>>>(
                    (const S *)idx->d_series, (const S *)dUC, (const S *)dLC, d_meta, idx->qtab.as<V4>(), D, w,
                    sctx->nrows, sctx->cursor, postbuf);
                CHECK_LAUNCH();
                launches++;
            } else if (ndw_max > 0 && sctx && sctx->mode == 1) {
                // continuous step, static w: SW_0 (EQ + EC) and SW_1..SW_rho (EQ only)
                dim3 grid((unsigned)((ndw_max + 128 * SMILER_INC_TILES - 1) / (128 * SMILER_INC_TILES)), (unsigned)B);
                size_t smem = 3 * sizeof(V) * D + (std::is_same<S, float>::value && SMILER_INC_X2 ? 16 * (size_t)D : 0);
                auto go = [&](auto kern, auto *pb) {
                    set_smem((const void *)kern, smem);
                    kern<<<grid, 128, smem, idx->stream>>>((const S *)idx->d_series, (const S *)dUC,
                                                           (const S *)dLC, d_meta, idx->qtab.as<V4>(), D,
                                                           sctx->nrows, sctx->cursor, pb, sctx->pscale);
                };
                if constexpr (std::is_same<S, float>::value) {
                    if (sctx->post_half) {
                        __half *hb = reinterpret_cast<__half *>(sctx->ring);
                        switch (w) {
                            case 4: go(window_lb_inc_kernel<S, 4, __half>, hb); break;
                            case 8: go(window_lb_inc_kernel<S, 8, __half>, hb); break;
                            case 16: go(window_lb_inc_kernel<S, 16, __half>, hb); break;
                            default: go(window_lb_inc_kernel<S, 32, __half>, hb); break;
                        }
                    }
                }
                if (!sctx->post_half) {
                    switch (w) {
                        case 4: go(window_lb_inc_kernel<S, 4>, postbuf); break;
                        case 8: go(window_lb_inc_kernel<S, 8>, postbuf); break;
                        case 16: go(window_lb_inc_kernel<S, 16>, postbuf); break;
                        default: go(window_lb_inc_kernel<S, 32>, postbuf); break;
                    }
                }
                CHECK_LAUNCH();
                launches++;
            } else if (ndw_max > 0) {
                // every row (ring cursor 0 when a stream is created)
                dim3 grid((unsigned)((ndw_max + 127) / 128), (unsigned)B);
                size_t smem = 3 * sizeof(V) * D + (std::is_same<S, float>::value && SMILER_INC_X2 ? 16 * (size_t)D : 0);
                auto go = [&](auto kern, auto *pb) {
                    set_smem((const void *)kern, smem);
                    kern<<<grid, 128, smem, idx->stream>>>((const S *)idx->d_series, (const S *)dUC,
                                                           (const S *)dLC, d_meta, idx->qtab.as<V4>(), D,
                                                           w, pb, sctx ? sctx->pscale : 1.0f);
                };
                bool done_half = false;
                if constexpr (std::is_same<S, float>::value) {
                    if (sctx && sctx->post_half) {
                        __half *hb = reinterpret_cast<__half *>(sctx->ring);
                        done_half = true;
                        switch (w) {
                            case 4: go(window_lb_kernel<S, 4, __half>, hb); break;
                            case 8: go(window_lb_kernel<S, 8, __half>, hb); break;
                            case 16: go(window_lb_kernel<S, 16, __half>, hb); break;
                            default: go(window_lb_kernel<S, 32, __half>, hb); break;
                        }
                    }
                }
                if (!done_half) switch (w) {
                    case 4: go(window_lb_kernel<S, 4>, postbuf); break;
                    case 8: go(window_lb_kernel<S, 8>, postbuf); break;
                    case 16: go(window_lb_kernel<S, 16>, postbuf); break;
                    case 32: go(window_lb_kernel<S, 32>, postbuf); break;
                    default: go(window_lb_kernel<S, 0>, postbuf); break;
                }
                CHECK_LAUNCH();
                launches++;
            }
            post_bytes += post_tot * (int64_t)((sctx && sctx->post_half) ? 2 : sizeof(V));
            TRY(tm.mark(2));
            // ---- a4 ----------------------------------------------------------
            dim3 grid((unsigned)nblk_max, (unsigned)B);
            auto go4 = [&](auto kern, auto *pb) {
                set_smem((const void *)kern, pl.smem_gs);
                kern<<<grid, pl.RT, pl.smem_gs, idx->stream>>>(pb, d_meta, P, idx->lb.as<V>(),
                                                               idx->tauc.as<int32_t>());
            };
            bool done4 = false;
            if (sctx && sctx->tma) {  // TMA-staged ring scan
                done4 = true;
                auto go5 = [&](auto kern, size_t smem) {  // persistent: ~ one wave of CTAs over B x nblk tiles
                    set_smem((const void *)kern, smem);
                    int occ = 0;
                    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kScanThreads, smem);
                    const int64_t tiles = (int64_t)nblk_max * B;
                    // variant 8: one tile per CTA (A/B against the persistent grid)
                    const int g5 = o.variant == kVarTmaOneTile ? (int)tiles
                                   : (int)std::min<int64_t>(tiles, (int64_t)idx->num_sms * std::max(occ, 1));
                    kern<<<g5, kScanThreads, smem, idx->stream>>>(*sctx->tmap, *sctx->tmap_tail, d_meta, P,
                                                                  idx->lb.as<V>(), idx->tauc.as<int32_t>(),
                                                                  nblk_max, B, (int)(sctx->ring_off[c0] / sctx->pstride),
                                                                  sctx->prows);
                };
                // SEL: Table 3's one-sum ablations (P.lbsel != 0) pick S_EQ or S_EC
                auto go5w = [&](auto pv_tag, auto sel_tag) {
                    using PVt = typename decltype(pv_tag)::type;
                    constexpr bool SEL = decltype(sel_tag)::value;
                    switch (w) {
                        case 4: go5(group_scan_tma_kernel<S, 4, PVt, SEL>, tma_scan_smem<4, PVt>()); break;
                        case 8: go5(group_scan_tma_kernel<S, 8, PVt, SEL>, tma_scan_smem<8, PVt>()); break;
                        default: go5(group_scan_tma_kernel<S, 16, PVt, SEL>, tma_scan_smem<16, PVt>()); break;
                    }
                };
                auto go5s = [&](auto pv_tag) {
                    if (P.lbsel != 0) go5w(pv_tag, std::true_type{});
                    else go5w(pv_tag, std::false_type{});
                };
                if constexpr (std::is_same<S, float>::value) {
                    if (sctx->post_half) go5s(TypeTag<__half>{});
                    else go5s(TypeTag<float>{});
                } else {
                    go5s(TypeTag<V>{});
                }
            }
            if constexpr (std::is_same<S, float>::value) {
                if (!done4 && sctx && sctx->post_half) {
                    __half *hb = reinterpret_cast<__half *>(sctx->ring);
                    done4 = true;
                    switch (w) {
                        case 4: go4(group_scan_reg_kernel<S, 4, __half>, hb); break;
                        case 8: go4(group_scan_reg_kernel<S, 8, __half>, hb); break;
                        case 16: go4(group_scan_reg_kernel<S, 16, __half>, hb); break;
                        default: go4(group_scan_reg_kernel<S, 32, __half>, hb); break;
                    }
                }
            }
            if (!done4) switch (pl.scan_reg ? w : 0) {
                case 4: go4(group_scan_reg_kernel<S, 4>, postbuf); break;
                case 8: go4(group_scan_reg_kernel<S, 8>, postbuf); break;
                case 16: go4(group_scan_reg_kernel<S, 16>, postbuf); break;
                case 32: go4(group_scan_reg_kernel<S, 32>, postbuf); break;
                default: go4(group_scan_kernel<S, 0>, postbuf); break;
            }
            CHECK_LAUNCH();
            launches++;
        }
        if (!P.fuse) lb_bytes += 2 * seg_tot * (P.lb_half ? 2 : (int64_t)sizeof(V));  // a4 write + a6 read
        TRY(tm.mark(3));
        if (lb_only) {
            // copy LB_w [n_mq][n_len][N] and postings out
            const size_t lbb = sizeof(V) * (size_t)seg_tot;
            const int64_t lb_off = (int64_t)meta[0].n * nl * c0;
            CU(cudaMemcpyAsync((char *)lb_out + lb_off * sizeof(V), idx->lb.p, lbb,
                               out_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, idx->stream));
            if (post_out) {
                const int64_t po = 2 * (int64_t)n_sw * meta[0].n_dw * c0;
                CU(cudaMemcpyAsync((char *)post_out + po * sizeof(V), idx->post.p, sizeof(V) * (size_t)post_tot,
                                   out_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, idx->stream));
            }
            c0 = c1;
            continue;
        }
        if (lag_save) {  // this scan's tile candidates (before a5's trim reorders them)
            CU(cudaMemcpy2DAsync(sctx->lag_t->as<int32_t>() + (size_t)c0 * nl * LTt, 4 * (size_t)LTt,
                                 idx->tauc.p, 4 * (size_t)LT, 4 * (size_t)LTt, (size_t)nseg, cudaMemcpyDeviceToDevice,
                                 idx->stream));
            CU(cudaMemcpy2DAsync(sctx->lag_lb->as<uint32_t>() + (size_t)c0 * nl * LTt, 4 * (size_t)LTt,
                                 idx->taulb.p, 4 * (size_t)LT, 4 * (size_t)LTt, (size_t)nseg, cudaMemcpyDeviceToDevice,
                                 idx->stream));
            lag_LTt_seen = lag_LTt_seen == -2 ? LTt : (lag_LTt_seen == LTt ? LTt : -1);
        }
        if (!fuse) TRY(do_a5());
        TRY(tm.mark(4));
        // ---- a6 ----------------------------------------------------------
        {
            int64_t nmax = 0;
            for (int j = 0; j < B; j++) nmax = std::max(nmax, meta[j].n);
            if (fuse) {
                // survivors were appended by the LB kernel
            } else if (!o.no_prune) {
                const int span = P.lb_half ? kFiltSpanH : kFiltThreads * kFiltItems;
                dim3 grid((unsigned)((nmax + span - 1) / span), (unsigned)nseg);
                if (P.lb_half)
                    filter_kernel<S, true><<<grid, kFiltThreads, 0, idx->stream>>>(idx->lb.as<V>(), d_meta, P, thr,
                                                                               idx->surv.as<int32_t>(), scount);
                else
                    filter_kernel<S, false><<<grid, kFiltThreads, 0, idx->stream>>>(idx->lb.as<V>(), d_meta, P,
                                                                                thr, idx->surv.as<int32_t>(),
                                                                                scount);
            } else {
                dim3 grid((unsigned)std::min<int64_t>((nmax + 255) / 256, 1024), (unsigned)nseg);
                all_candidates_kernel<<<grid, 256, 0, idx->stream>>>(d_meta, P, idx->surv.as<int32_t>(), scount);
            }
            if (!fuse) {
                CHECK_LAUNCH();
                launches++;
            }
        }
        TRY(tm.mark(5));
        // ---- a6b: LB_Keogh cascade (R27), per item query on its side stream -----
        int32_t *taskoff2 = taskoff + (size_t)nl * (B + 1);
        int32_t *taskoff3 = taskoff + (size_t)2 * nl * (B + 1);
        const int32_t *vlist = idx->surv.as<int32_t>();
        const int32_t *vcnt = scount;
        if (cascade) {
            CU(cudaMemsetAsync(idx->scount2.p, 0, 4 * (size_t)nseg, idx->stream));
            vlist = idx->surv2.as<int32_t>();
            vcnt = idx->scount2.as<int32_t>();
            TRY(side_fork(idx, nl));
            for (int i = 0; i < nl; i++) {
                if (!casc_iq(i)) continue;
                int32_t *to = taskoff3 + (size_t)i * (B + 1);
                task_prefix_kernel<<<1, 1024, 0, idx->side[i]>>>(scount, -1, B, nl, i, to);
                CHECK_LAUNCH();
                CascadeParams<S> cp;
                cp.series = (const S *)idx->d_series;
                cp.meta = d_meta;
                cp.qenv = idx->qenv.as<V2>();
                cp.D = D;
                cp.n_len = nl;
                cp.li = i;
                cp.d = pl.len[i];
                cp.n_mq = B;
                cp.list = idx->surv.as<int32_t>();
                cp.counts = scount;
                cp.task_off = to;
                cp.thr = thr;
                cp.out_list = idx->surv2.as<int32_t>();
                cp.out_counts = idx->scount2.as<int32_t>();
                launch_cascade<S>(cp, idx->side[i]);
                CHECK_LAUNCH();
                launches += 2;
            }
            TRY(side_join(idx, nl));
        }
        TRY(tm.mark(8));  // the cascade (ns_cascade)
        // ---- a7: DTW verification ------------------------------------------
        TRY(side_fork(idx, nl));
        for (int i = 0; i < nl; i++) {
            const bool ci = cascade && casc_iq(i);  // this IQ's survivors: the cascade's or the filter's
            TRY(run_dtw_list<S>(idx, pl, i, B, 1, ci ? vlist : idx->surv.as<int32_t>(), 0, ci ? vcnt : scount,
                                taskoff2 + (size_t)i * (B + 1), nullptr, taukey, idx->fin.as<uint64_t>(), fcount,
                                d_meta, idx->qv.as<V>(), D, idx->side[i]));
            launches += 2;
        }
        TRY(side_join(idx, nl));
        TRY(tm.mark(6));
        // ---- a8 ----------------------------------------------------------
        topk_kernel<S><<<nseg, 512, 0, idx->stream>>>(idx->fin.as<uint64_t>(), fcount, d_meta, P,
                                                      idx->out_ids.as<int64_t>(), idx->out_d.as<V>());
        CHECK_LAUNCH();
        launches++;
        TRY(tm.mark(7));
        const size_t ob = (size_t)nseg * pl.k;
        CU(cudaMemcpyAsync(ids + (size_t)c0 * nl * pl.k, idx->out_ids.p, 8 * ob,
                           out_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, idx->stream));
        CU(cudaMemcpyAsync((char *)dists + (size_t)c0 * nl * pl.k * 4, idx->out_d.p, 4 * ob,
                           out_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, idx->stream));
        if (sctx && sctx->d_prev_out)
            CU(cudaMemcpyAsync(sctx->d_prev_out + (size_t)c0 * nl * pl.k, idx->out_ids.p, 8 * ob,
                               cudaMemcpyDeviceToDevice, idx->stream));
        if (stats) {
            uint32_t vmask = 0;
            for (int i = 0; i < nl; i++) vmask |= (uint32_t)(cascade && casc_iq(i)) << i;
            accum_counts_kernel<<<1, 256, 0, idx->stream>>>(vcnt, scount, fcount, nseg, nl, vmask,
                                                            idx->tmp.as<unsigned long long>());
            CHECK_LAUNCH();
        }
        c0 = c1;
    }
    if (sctx) *sctx->lag_LTt = lag_LTt_seen >= 0 ? lag_LTt_seen : -1;  // the next step may use the saved lists
    unsigned long long acc_h[2 * kMaxLen + 1] = {0};
    if (stats && !lb_only)
        CU(cudaMemcpyAsync(acc_h, idx->tmp.p, 8 * (2 * kMaxLen + 1), cudaMemcpyDeviceToHost, idx->stream));
    if (!out_dev || stats) {
        CU(cudaStreamSynchronize(idx->stream));
        TRY(take_qflag(idx));
    }
    CHECK_LAUNCH();
    if (stats) {
        fin_total = (int64_t)acc_h[0];
        for (int i = 0; i < nl; i++) {
            surv_total += (int64_t)acc_h[1 + i];
            casc_total += (int64_t)acc_h[1 + kMaxLen + i];
            cells_acc += (double)acc_h[1 + i] * (double)dtw_cells(pl.len[i], pl.rho[i]);
        }
        stats->candidates = cand_total;
        stats->tau_verified = tau_slots_total;
        stats->survivors = surv_total;
        stats->cascade_pruned = casc_total;
        stats->finalists = fin_total;
        stats->dtw_cells = cells_acc;
        stats->bf_cells = bf_cells;
        stats->posting_bytes = post_bytes;
        stats->lb_bytes = lb_bytes;
        stats->kernel_launches = launches;
        stats->mq_chunks = n_chunks;
        if (tm.on) {
            double *slots[9] = {nullptr, &stats->ns_prep, &stats->ns_window_lb, &stats->ns_group_scan,
                                &stats->ns_tau, &stats->ns_filter, &stats->ns_verify, &stats->ns_select,
                                &stats->ns_cascade};
            for (size_t x = 1; x < tm.marks.size(); x++) {
                int ph = tm.marks[x].first;
                if (ph == 0) continue;
                float ms = 0;
                CU(cudaEventElapsedTime(&ms, idx->events[tm.marks[x - 1].second], idx->events[tm.marks[x].second]));
                *slots[ph] += ms * 1e6;
                stats->ns_total += ms * 1e6;
            }
        }
    }
    return SMILER_OK;
}

struct NvtxRange {
    explicit NvtxRange(const char *n) { nvtxRangePushA(n); }
    ~NvtxRange() { nvtxRangePop(); }
};

extern "C" int smiler_knn_ex(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                             int32_t n_mq, const int32_t *lengths, int32_t n_len, int32_t k, int64_t *ids,
                             void *dists, smiler_knn_stats *stats, const smiler_knn_opts *opts) {
    NvtxRange nr("smiler_knn");
    if (!idx) return fail(SMILER_EINVAL, "index is NULL");
    if (idx->dtype == SMILER_I16)
        return knn_impl<int16_t>(idx, queries, query_sensor, n_mq, lengths, n_len, k, ids, dists, stats,
                                 opts, false, nullptr, nullptr);
    return knn_impl<float>(idx, queries, query_sensor, n_mq, lengths, n_len, k, ids, dists, stats, opts,
                           false, nullptr, nullptr);
}

extern "C" int smiler_knn(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                          int32_t n_mq, const int32_t *lengths, int32_t n_len, int32_t k, int64_t *ids,
                          void *dists, smiler_knn_stats *stats) {
    return smiler_knn_ex(idx, queries, query_sensor, n_mq, lengths, n_len, k, ids, dists, stats, nullptr);
}

extern "C" int smiler_knn_step(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                               int32_t n_mq, const int32_t *lengths, int32_t n_len, int32_t k,
                               const int64_t *prev_ids, int32_t shift, int64_t *ids, void *dists,
                               smiler_knn_stats *stats, const smiler_knn_opts *opts) {
    if (!idx) return fail(SMILER_EINVAL, "index is NULL");
    if (!prev_ids) return fail(SMILER_EINVAL, "prev_ids is NULL (use smiler_knn for a first step)");
    if (shift < 0) return fail(SMILER_EINVAL, "shift must be >= 0");
    if (idx->dtype == SMILER_I16)
        return knn_impl<int16_t>(idx, queries, query_sensor, n_mq, lengths, n_len, k, ids, dists, stats, opts,
                                 false, nullptr, nullptr, prev_ids, shift);
    return knn_impl<float>(idx, queries, query_sensor, n_mq, lengths, n_len, k, ids, dists, stats, opts, false,
                           nullptr, nullptr, prev_ids, shift);
}

// ---------------------------------------------------------------------------
// Continuous streams (Def. 4.1; Remark 1; tau method 2,
// P:1452-1458)
// ---------------------------------------------------------------------------
struct smiler_stream {
    smiler_index *idx = nullptr;
    int n = 0, D = 0, n_len = 0, k = 0, n_sw = 0, nrows = 0;
    std::vector<int32_t> lens, qsens;
    std::vector<int64_t> ring_off;
    void *d_mq = nullptr;      // [n][D] current master queries (storage type)
    void *d_new = nullptr;     // [n] staging for new points
    void *ring = nullptr;      // posting-list rings
    int64_t *d_prev = nullptr; // [n][n_len][k] last results
    bool post_half = false;    // ring entries fp16 rounded toward zero (see post_st in lb.cuh)
    bool tma = false;          // ring as one TMA tensor (group_scan_tma_kernel)
    int64_t pstride = 0;       // ring row stride (elements)
    int prows = 0;             // ring rows per plane
    CUtensorMap tmap, tmap_tail;
    float pscale = 1.f;        // fp16 ring storage scale (power of two)
    DevBuf lag_t, lag_lb;      // lagged tile tau set (StreamCtx)
    int lag_LTt = -1;
    int cursor = 0;
    int64_t steps = 0;
};

static void stream_release(smiler_stream *st) {
    if (!st) return;
    if (st->idx) cudaSetDevice(st->idx->device);
    if (st->idx && st->idx->stream) cudaStreamSynchronize(st->idx->stream);
    if (st->d_mq) cudaFree(st->d_mq);
    if (st->d_new) cudaFree(st->d_new);
    if (st->ring) cudaFree(st->ring);
    if (st->d_prev) cudaFree(st->d_prev);
    st->lag_t.release();
    st->lag_lb.release();
    delete st;
}

template <typename S>
static int stream_run(smiler_stream *st, int64_t *ids, void *dists, smiler_knn_stats *stats,
                      const smiler_knn_opts *opts, int mode) {
    StreamCtx sc;
    sc.ring = st->ring;
    sc.ring_off = st->ring_off.data();
    sc.cursor = st->cursor;
    sc.mode = mode;
    sc.nrows = st->nrows;
    sc.d_prev_out = st->d_prev;
    sc.post_half = st->post_half;
    sc.tma = st->tma;
    sc.pstride = st->pstride;
    sc.prows = st->prows;
    sc.tmap = &st->tmap;
    sc.tmap_tail = &st->tmap_tail;
    sc.pscale = st->pscale;
    sc.lag_t = &st->lag_t;
    sc.lag_lb = &st->lag_lb;
    sc.lag_LTt = &st->lag_LTt;
    return knn_impl<S>(st->idx, st->d_mq, st->qsens.data(), st->n, st->lens.data(), st->n_len, st->k, ids, dists,
                       stats, opts, false, nullptr, nullptr, mode == 1 ? st->d_prev : nullptr, 1, &sc);
}

extern "C" int smiler_stream_create_ex(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                                       int32_t n_streams, const int32_t *lengths, int32_t n_len, int32_t k,
                                       int64_t *ids, void *dists, const smiler_knn_opts *opts,
                                       smiler_stream **out) {
    if (!out) return fail(SMILER_EINVAL, "out is NULL");
    *out = nullptr;
    if (!idx || !queries || !lengths || !ids || !dists) return fail(SMILER_EINVAL, "NULL argument");
    if (idx->shard) return fail(SMILER_EINVAL, "streams on window-range shards are not supported");
    if (n_streams < 1) return fail(SMILER_EINVAL, "n_streams must be >= 1");
    if (n_len < 1 || n_len > kMaxLen) return fail(SMILER_EINVAL, "n_len must be in [1, %d]", kMaxLen);
    TRY(set_device(idx));
    smiler_stream *st = new smiler_stream();
    st->idx = idx;
    st->n = n_streams;
    st->n_len = n_len;
    st->k = k;
    st->lens.resize(n_len);
    if (is_device_ptr(lengths)) {
        if (cudaMemcpy(st->lens.data(), lengths, 4 * n_len, cudaMemcpyDeviceToHost) != cudaSuccess) {
            stream_release(st);
            return fail(SMILER_ECUDA, "reading lengths");
        }
    } else {
        memcpy(st->lens.data(), lengths, 4 * n_len);
    }
    Plan pl;
    int rc = validate_query(idx, st->lens.data(), n_len, k, pl);
    if (rc) {
        stream_release(st);
        return rc;
    }
    st->D = pl.D;
    st->n_sw = pl.D - pl.w + 1;
    st->nrows = std::min(pl.rho_env + 1, st->n_sw);
    // fp16 ring (rounded toward zero) for f32 indices on the register group scan
    st->post_half = idx->dtype == SMILER_F32 && pl.scan_reg && !(opts && opts->exact_postings);
    st->qsens.assign(n_streams, 0);
    if (query_sensor) {
        if (is_device_ptr(query_sensor)) cudaMemcpy(st->qsens.data(), query_sensor, 4 * (size_t)n_streams, cudaMemcpyDeviceToHost);
        else memcpy(st->qsens.data(), query_sensor, 4 * (size_t)n_streams);
    }
    int64_t tot = 0;
    st->ring_off.resize(n_streams);
    int64_t ndw0 = -1;
    bool same_ndw = true;
    for (int j = 0; j < n_streams; j++) {
        if (st->qsens[j] < 0 || st->qsens[j] >= (int)idx->sensors.size()) {
            stream_release(st);
            return fail(SMILER_EINVAL, "query_sensor[%d] out of range", j);
        }
        const int64_t ndw = idx->sensors[st->qsens[j]].n / pl.w;
        if (ndw0 < 0) ndw0 = ndw;
        same_ndw = same_ndw && ndw == ndw0;
    }
    // TMA ring (group_scan_tma_kernel): every stream's sensor has the same n_dw,
    // row stride padded to 8 entries (16-byte rows), first w-1 rows mirrored
    const int pbytes = st->post_half ? 2 : 4;
    st->tma = pl.scan_reg && (pl.w == 4 || pl.w == 8 || pl.w == 16) && same_ndw && ndw0 >= 1 &&
              !(opts && opts->variant == kVarRingNoTma);  // variant 7: A/B without TMA
    st->pstride = st->tma ? (ndw0 + 7) / 8 * 8 : 0;
    st->prows = st->tma ? st->n_sw + pl.w - 1 : st->n_sw;
    for (int j = 0; j < n_streams; j++) {
        st->ring_off[j] = tot;
        const int64_t ndw = idx->sensors[st->qsens[j]].n / pl.w;
        tot += st->tma ? 2 * (int64_t)st->prows * st->pstride : 2 * (int64_t)st->n_sw * ndw;
    }
    if (st->tma && tot / st->pstride > INT32_MAX) st->tma = false;  // TMA row coordinates are int32
    if (!st->tma) {  // plain layout
        tot = 0;
        st->prows = st->n_sw;
        for (int j = 0; j < n_streams; j++) {
            st->ring_off[j] = tot;
            tot += 2 * (int64_t)st->n_sw * (idx->sensors[st->qsens[j]].n / pl.w);
        }
    }
    const size_t es = esize(idx->dtype);
    if (st->post_half) {
        // fp16 ring scale: entries are sums of w terms, each at most (|q| + max|x|)^2;
        // the initial master queries bound |q|, with 2x headroom for later points
        // (an entry above the range saturates at 65504: still a lower bound)
        std::vector<float> qh((size_t)n_streams * pl.D);
        if (cudaMemcpy(qh.data(), queries, es * qh.size(), cudaMemcpyDefault) != cudaSuccess) {
            stream_release(st);
            return fail(SMILER_ECUDA, "reading the initial queries");
        }
        double qm = 0.0;
        for (float v : qh) qm = std::max(qm, (double)fabsf(v));
        const double a = 2.0 * (qm + (double)idx->smax);
        st->pscale = fp16_fit_scale((double)pl.w * a * a);
    }
    cudaError_t e = cudaMalloc(&st->ring, (size_t)pbytes * (size_t)std::max<int64_t>(tot, 1));
    if (e == cudaSuccess && st->tma) {
        // the mirror rows and the row padding are never read as valid data, but
        // start them at zero so the ring holds no uninitialised bytes
        e = cudaMemsetAsync(st->ring, 0, (size_t)pbytes * (size_t)tot, idx->stream);
        static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
        if (!encode) {
            void *fn = nullptr;
            cudaDriverEntryPointQueryResult q;
            if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) == cudaSuccess &&
                q == cudaDriverEntryPointSuccess)
                encode = (PFN_cuTensorMapEncodeTiled_v12000)fn;
        }
        if (!encode) {
            stream_release(st);
            return fail(SMILER_ECUDA, "cuTensorMapEncodeTiled unavailable");
        }
        const CUtensorMapDataType dt = st->post_half ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16
                                       : idx->dtype == SMILER_F32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                                                                  : CU_TENSOR_MAP_DATA_TYPE_INT32;
        const cuuint64_t gdim[2] = {(cuuint64_t)ndw0, (cuuint64_t)(tot / st->pstride)};
        const cuuint64_t gstride[1] = {(cuuint64_t)st->pstride * pbytes};
        const cuuint32_t box[2] = {(cuuint32_t)kScanThreads, (cuuint32_t)pl.w};
        const cuuint32_t estr[2] = {1, 1};
        // tail boxes: 16 bytes wide (group_scan_tma_kernel loads from 16-byte aligned columns)
        const cuuint32_t box_tail[2] = {(cuuint32_t)(16 / pbytes), (cuuint32_t)pl.w};
        CUresult cr = encode(&st->tmap, dt, 2, st->ring, gdim, gstride, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                             CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (cr == CUDA_SUCCESS)
            cr = encode(&st->tmap_tail, dt, 2, st->ring, gdim, gstride, box_tail, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (cr != CUDA_SUCCESS) {
            stream_release(st);
            return fail(SMILER_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)cr);
        }
    }
    if (e == cudaSuccess) e = cudaMalloc(&st->d_mq, es * (size_t)n_streams * pl.D);
    if (e == cudaSuccess) e = cudaMalloc(&st->d_new, es * (size_t)n_streams);
    if (e == cudaSuccess) e = cudaMalloc(&st->d_prev, 8 * (size_t)n_streams * n_len * k);
    if (e != cudaSuccess) {
        cudaGetLastError();
        stream_release(st);
        return fail(SMILER_ENOMEM, "stream buffers (%lld posting entries): %s", (long long)tot, cudaGetErrorString(e));
    }
    e = cudaMemcpyAsync(st->d_mq, queries, es * (size_t)n_streams * pl.D, cudaMemcpyDefault, idx->stream);
    if (e != cudaSuccess) {
        stream_release(st);
        return fail(SMILER_ECUDA, "copying queries: %s", cudaGetErrorString(e));
    }
    rc = idx->dtype == SMILER_I16 ? stream_run<int16_t>(st, ids, dists, nullptr, nullptr, 0)
                                  : stream_run<float>(st, ids, dists, nullptr, nullptr, 0);
    if (rc) {
        stream_release(st);
        return rc;
    }
    *out = st;
    return SMILER_OK;
}

extern "C" int smiler_stream_create(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                                    int32_t n_streams, const int32_t *lengths, int32_t n_len, int32_t k,
                                    int64_t *ids, void *dists, smiler_stream **out) {
    return smiler_stream_create_ex(idx, queries, query_sensor, n_streams, lengths, n_len, k, ids, dists, nullptr,
                                   out);
}

extern "C" int smiler_stream_step(smiler_stream *st, const void *new_points, int64_t *ids, void *dists,
                                  smiler_knn_stats *stats, const smiler_knn_opts *opts) {
    NvtxRange nr("smiler_stream_step");
    if (!st) return fail(SMILER_EINVAL, "stream is NULL");
    if (!new_points || !ids || !dists) return fail(SMILER_EINVAL, "NULL argument");
    smiler_index *idx = st->idx;
    TRY(set_device(idx));
    const size_t es = esize(idx->dtype);
    CU(cudaMemcpyAsync(st->d_new, new_points, es * (size_t)st->n, cudaMemcpyDefault, idx->stream));
    if (idx->dtype == SMILER_I16) {
        // R17 range of the appended points, checked on the host copy when available
        if (!is_device_ptr(new_points)) {
            const int16_t *np = (const int16_t *)new_points;
            for (int j = 0; j < st->n; j++)
                if (np[j] > 1023 || np[j] < -1023) return fail(SMILER_ERANGE, "new point %d outside [-1023, 1023]", j);
        }
        stream_shift_kernel<int16_t><<<st->n, 256, 0, idx->stream>>>((int16_t *)st->d_mq, st->D,
                                                                     (const int16_t *)st->d_new);
    } else {
        stream_shift_kernel<float><<<st->n, 256, 0, idx->stream>>>((float *)st->d_mq, st->D,
                                                                   (const float *)st->d_new);
    }
    CHECK_LAUNCH();
    // ring: the new SW_0 takes the slot of the dropped oldest SW (Fig. 6)
    st->cursor = (st->cursor + st->n_sw - 1) % st->n_sw;
    st->steps++;
    return idx->dtype == SMILER_I16 ? stream_run<int16_t>(st, ids, dists, stats, opts, 1)
                                    : stream_run<float>(st, ids, dists, stats, opts, 1);
}

extern "C" void smiler_stream_free(smiler_stream *st) { stream_release(st); }

extern "C" int smiler_lower_bounds(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                                   int32_t n_mq, const int32_t *lengths, int32_t n_len, void *postings,
                                   void *lbw) {
    if (!idx) return fail(SMILER_EINVAL, "index is NULL");
    if (!lbw) return fail(SMILER_EINVAL, "lbw is NULL");
    smiler_knn_opts o;
    memset(&o, 0, sizeof(o));
    if (idx->dtype == SMILER_I16)
        return knn_impl<int16_t>(idx, queries, query_sensor, n_mq, lengths, n_len, 1, nullptr, nullptr,
                                 nullptr, &o, true, postings, lbw);
    return knn_impl<float>(idx, queries, query_sensor, n_mq, lengths, n_len, 1, nullptr, nullptr, nullptr,
                           &o, true, postings, lbw);
}

extern "C" int smiler_lower_bounds_ex(smiler_index *idx, const void *queries, const int32_t *query_sensor,
                                      int32_t n_mq, const int32_t *lengths, int32_t n_len, int32_t lb_kind,
                                      void *lb) {
    if (!idx) return fail(SMILER_EINVAL, "index is NULL");
    if (!lb) return fail(SMILER_EINVAL, "lb is NULL");
    smiler_knn_opts o;
    memset(&o, 0, sizeof(o));
    o.lb_kind = lb_kind;
    if (idx->dtype == SMILER_I16)
        return knn_impl<int16_t>(idx, queries, query_sensor, n_mq, lengths, n_len, 1, nullptr, nullptr,
                                 nullptr, &o, true, nullptr, lb);
    return knn_impl<float>(idx, queries, query_sensor, n_mq, lengths, n_len, 1, nullptr, nullptr, nullptr, &o,
                           true, nullptr, lb);
}

// ---------------------------------------------------------------------------
// smiler_predict (NEXT-3): AR and GP predictors on the kNN data (Sec. 5.2)
// ---------------------------------------------------------------------------
namespace smiler {
template <typename S>
int launch_predict(const void *series, const int64_t *soff_n, int n_sensors, const int32_t *qsens,
                   const void *queries, int D, const int32_t *lens, int n_len, const int64_t *ids, int k,
                   const int32_t *ekv, int n_k, int kmax, int h, const double *theta, int n_pred, double *ar_mean,
                   double *ar_var, double *gp_mean, double *gp_var, cudaStream_t st);
}

extern "C" int smiler_predict(smiler_index *idx, const void *queries, const int32_t *query_sensor, int32_t n_mq,
                              const int32_t *lengths, int32_t n_len, const int64_t *ids, int32_t k,
                              const int32_t *ekv, int32_t n_k, int32_t horizon, const double *theta,
                              double *ar_mean, double *ar_var, double *gp_mean, double *gp_var) {
    if (!idx) return fail(SMILER_EINVAL, "index is NULL");
    if (!queries || !lengths || !ids || !ekv || !theta || !ar_mean || !ar_var || !gp_mean || !gp_var)
        return fail(SMILER_EINVAL, "NULL argument");
    if (idx->shard) return fail(SMILER_EINVAL, "smiler_predict needs a whole-series index (not a shard)");
    if (n_mq < 1 || n_len < 1 || n_len > kMaxLen || k < 1 || n_k < 1 || n_k > 64 || horizon < 0)
        return fail(SMILER_EINVAL, "need n_mq >= 1, 1 <= n_len <= %d, k >= 1, 1 <= n_k <= 64, horizon >= 0",
                    kMaxLen);
    TRY(set_device(idx));
    std::vector<int32_t> lens(n_len), ek(n_k), qs(n_mq, 0);
    CU(cudaMemcpy(lens.data(), lengths, 4 * (size_t)n_len, cudaMemcpyDefault));
    CU(cudaMemcpy(ek.data(), ekv, 4 * (size_t)n_k, cudaMemcpyDefault));
    if (query_sensor) CU(cudaMemcpy(qs.data(), query_sensor, 4 * (size_t)n_mq, cudaMemcpyDefault));
    for (int i = 0; i < n_len; i++)
        if (lens[i] < 1 || (i && lens[i] <= lens[i - 1])) return fail(SMILER_EINVAL, "lengths must increase");
    const int D = lens[n_len - 1];
    if (D > kMaxD) return fail(SMILER_EINVAL, "D = %d exceeds %d", D, kMaxD);
    for (int j = 0; j < n_k; j++)
        if (ek[j] < 1 || ek[j] > k || ek[j] > kMaxPredK || (j && ek[j] <= ek[j - 1]))
            return fail(SMILER_EINVAL, "ekv must increase within [1, min(k, %d)]", kMaxPredK);
    for (int m = 0; m < n_mq; m++)
        if (qs[m] < 0 || qs[m] >= (int)idx->sensors.size())
            return fail(SMILER_EINVAL, "query_sensor[%d] out of range", m);
    const int kmax = ek[n_k - 1];
    const int64_t n_pred = (int64_t)n_mq * n_len * n_k;
    if (n_pred > INT32_MAX) return fail(SMILER_EINVAL, "too many predictors");
    const size_t es = esize(idx->dtype);
    // device workspace: sensors | qsens | lens | ekv | queries | ids | theta | 4 outputs
    const size_t ns = idx->sensors.size();
    size_t off = 0;
    auto take = [&](size_t b) { size_t o = off; off += (b + 255) & ~(size_t)255; return o; };
    const size_t o_sens = take(16 * ns), o_qs = take(4 * (size_t)n_mq), o_len = take(4 * (size_t)n_len),
                 o_ek = take(4 * (size_t)n_k), o_q = take(es * (size_t)n_mq * D),
                 o_ids = take(8 * (size_t)n_mq * n_len * k), o_th = take(24 * (size_t)n_pred),
                 o_out = take(32 * (size_t)n_pred);
    TRY(idx->pred.ensure(off));
    char *b = idx->pred.as<char>();
    std::vector<int64_t> sn(2 * ns);
    for (size_t x = 0; x < ns; x++) {
        sn[2 * x] = idx->sensors[x].off;
        sn[2 * x + 1] = idx->sensors[x].n;
    }
    cudaStream_t st = idx->stream;
    CU(cudaMemcpyAsync(b + o_sens, sn.data(), 16 * ns, cudaMemcpyHostToDevice, st));
    CU(cudaMemcpyAsync(b + o_qs, qs.data(), 4 * (size_t)n_mq, cudaMemcpyHostToDevice, st));
    CU(cudaMemcpyAsync(b + o_len, lens.data(), 4 * (size_t)n_len, cudaMemcpyHostToDevice, st));
    CU(cudaMemcpyAsync(b + o_ek, ek.data(), 4 * (size_t)n_k, cudaMemcpyHostToDevice, st));
    CU(cudaMemcpyAsync(b + o_q, queries, es * (size_t)n_mq * D, cudaMemcpyDefault, st));
    CU(cudaMemcpyAsync(b + o_ids, ids, 8 * (size_t)n_mq * n_len * k, cudaMemcpyDefault, st));
    CU(cudaMemcpyAsync(b + o_th, theta, 24 * (size_t)n_pred, cudaMemcpyDefault, st));
    double *outs = reinterpret_cast<double *>(b + o_out);
    int rc = idx->dtype == SMILER_I16
                 ? smiler::launch_predict<int16_t>(idx->d_series, (const int64_t *)(b + o_sens), (int)ns,
                                           (const int32_t *)(b + o_qs), b + o_q, D, (const int32_t *)(b + o_len),
                                           n_len, (const int64_t *)(b + o_ids), k, (const int32_t *)(b + o_ek), n_k,
                                           kmax, horizon, (const double *)(b + o_th), (int)n_pred, outs,
                                           outs + n_pred, outs + 2 * n_pred, outs + 3 * n_pred, st)
                 : smiler::launch_predict<float>(idx->d_series, (const int64_t *)(b + o_sens), (int)ns,
                                         (const int32_t *)(b + o_qs), b + o_q, D, (const int32_t *)(b + o_len),
                                         n_len, (const int64_t *)(b + o_ids), k, (const int32_t *)(b + o_ek), n_k,
                                         kmax, horizon, (const double *)(b + o_th), (int)n_pred, outs,
                                         outs + n_pred, outs + 2 * n_pred, outs + 3 * n_pred, st);
    if (rc != cudaSuccess) return fail(SMILER_ECUDA, "predict_kernel: %s", cudaGetErrorString((cudaError_t)rc));
    double *dst[4] = {ar_mean, ar_var, gp_mean, gp_var};
    for (int x = 0; x < 4; x++)
        CU(cudaMemcpyAsync(dst[x], outs + x * n_pred, 8 * (size_t)n_pred, cudaMemcpyDefault, st));
    CU(cudaStreamSynchronize(st));
    return SMILER_OK;
}

extern "C" int smiler_index_envelope(smiler_index *idx, int32_t sensor, int32_t rho, void *U, void *L) {
    if (!idx) return fail(SMILER_EINVAL, "index is NULL");
    if (!U || !L) return fail(SMILER_EINVAL, "U/L is NULL");
    if (sensor < 0 || sensor >= (int)idx->sensors.size()) return fail(SMILER_EINVAL, "bad sensor %d", sensor);
    if (rho < 0) return fail(SMILER_EINVAL, "rho < 0");
    TRY(set_device(idx));
    void *dU, *dL;
    TRY(ensure_envelope(idx, rho, &dU, &dL));
    const SensorInfo &si = idx->sensors[sensor];
    const size_t es = esize(idx->dtype);
    CU(cudaMemcpyAsync(U, (char *)dU + si.off * es, si.n * es, cudaMemcpyDefault, idx->stream));
    CU(cudaMemcpyAsync(L, (char *)dL + si.off * es, si.n * es, cudaMemcpyDefault, idx->stream));
    CU(cudaStreamSynchronize(idx->stream));
    return SMILER_OK;
}

template <typename S>
static int dtw_impl(smiler_index *idx, int32_t sensor, const void *q, int32_t d, int32_t rho,
                    const int64_t *ts, int64_t n_t, void *dists) {
    using V = typename Tr<S>::V;
    const SensorInfo &si = idx->sensors[sensor];
    if (d < 1 || d > kMaxD || d > si.n) return fail(SMILER_EINVAL, "bad d = %d", d);
    if (std::is_same<S, int16_t>::value && d > kMaxDI16)
        return fail(SMILER_EINVAL, "I16: d = %d exceeds %d (int32 exactness, R17)", d, kMaxDI16);
    if (rho < 0) return fail(SMILER_EINVAL, "rho < 0");
    rho = std::min(rho, d - 1);
    // rho > kMaxRhoFast runs the anti-diagonal wavefront kernel
    if (n_t < 1 || n_t > INT32_MAX / 2) return fail(SMILER_EINVAL, "bad n_t");
    std::vector<int64_t> th(n_t);
    if (is_device_ptr(ts)) CU(cudaMemcpy(th.data(), ts, 8 * n_t, cudaMemcpyDeviceToHost));
    else memcpy(th.data(), ts, 8 * n_t);
    std::vector<int32_t> t32(n_t);
    for (int64_t x = 0; x < n_t; x++) {
        if (th[x] < 0 || th[x] > si.n - d) return fail(SMILER_EINVAL, "ts[%lld] = %lld out of range", (long long)x, (long long)th[x]);
        t32[x] = (int32_t)th[x];
    }
    MQMeta m;
    memset(&m, 0, sizeof(m));
    m.series_off = si.off;
    m.n = si.n;
    m.t_hi = si.n;
    TRY(idx->meta.ensure(sizeof(MQMeta)));
    TRY(idx->queries.ensure(sizeof(S) * d));
    TRY(idx->qv.ensure(sizeof(V) * d));
    TRY(idx->qtab.ensure(sizeof(typename Tr<S>::V4) * d));
    TRY(idx->tauc.ensure(4 * (size_t)n_t));
    TRY(idx->tauk.ensure(8 * (size_t)n_t));
    TRY(idx->taskoff.ensure(8));
    TRY(idx->out_d.ensure(4 * (size_t)n_t));
    CU(cudaMemcpyAsync(idx->meta.p, &m, sizeof(m), cudaMemcpyHostToDevice, idx->stream));
    CU(cudaMemcpyAsync(idx->queries.p, q, sizeof(S) * d, cudaMemcpyDefault, idx->stream));
    CU(cudaMemcpyAsync(idx->tauc.p, t32.data(), 4 * n_t, cudaMemcpyHostToDevice, idx->stream));
    query_prep_kernel<S><<<1, 256, 0, idx->stream>>>(idx->queries.as<S>(), d, 0, idx->qv.as<V>(),
                                                     idx->qtab.as<typename Tr<S>::V4>(), 0.f, nullptr,
                                                     idx->qflag_d, IQTab{}, 0, nullptr);
    CHECK_LAUNCH();
    Plan pl;
    pl.n_len = 1;
    pl.len = {d};
    pl.rho = {rho};
    TRY(run_dtw_list<S>(idx, pl, 0, 1, 0, idx->tauc.as<int32_t>(), (int)n_t, nullptr, idx->taskoff.as<int32_t>(),
                        idx->tauk.as<uint64_t>(), nullptr, nullptr, nullptr, idx->meta.as<MQMeta>(),
                        idx->qv.as<V>(), d));
    keys_to_dists_kernel<V><<<std::max<int64_t>(1, std::min<int64_t>((n_t + 255) / 256, 4096)), 256, 0,
                             idx->stream>>>(idx->tauk.as<uint64_t>(), n_t, idx->out_d.as<V>());
    CHECK_LAUNCH();
    CU(cudaMemcpyAsync(dists, idx->out_d.p, 4 * n_t, cudaMemcpyDefault, idx->stream));
    CU(cudaStreamSynchronize(idx->stream));
    return SMILER_OK;
}

extern "C" int smiler_dtw(smiler_index *idx, int32_t sensor, const void *q, int32_t d, int32_t rho,
                          const int64_t *ts, int64_t n_t, void *dists) {
    if (!idx) return fail(SMILER_EINVAL, "index is NULL");
    if (!q || !ts || !dists) return fail(SMILER_EINVAL, "NULL argument");
    if (sensor < 0 || sensor >= (int)idx->sensors.size()) return fail(SMILER_EINVAL, "bad sensor %d", sensor);
    TRY(set_device(idx));
    if (idx->dtype == SMILER_I16) return dtw_impl<int16_t>(idx, sensor, q, d, rho, ts, n_t, dists);
    return dtw_impl<float>(idx, sensor, q, d, rho, ts, n_t, dists);
}

extern "C" int smiler_merge_topk(const int64_t *ids_in, const void *dists_in, smiler_dtype dtype, int32_t G,
                                 int32_t rows, int32_t k, int64_t *ids_out, void *dists_out, int32_t device,
                                 void *cuda_stream) {
    if (!ids_in || !dists_in || !ids_out || !dists_out) return fail(SMILER_EINVAL, "NULL argument");
    if (G < 1 || rows < 1 || k < 1 || k > kMaxK || (int64_t)G * k > kSortCap)
        return fail(SMILER_EINVAL, "need G >= 1, rows >= 1, 1 <= k <= %d, G*k <= %d", kMaxK, kSortCap);
    if (dtype != SMILER_I16 && dtype != SMILER_F32) return fail(SMILER_EINVAL, "bad dtype");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return fail(SMILER_ECUDA, "no CUDA device available; there is no CPU fallback");
    }
    CU(cudaSetDevice(device));
    cudaStream_t st = (cudaStream_t)cuda_stream;
    const size_t nin = (size_t)G * rows * k, nout = (size_t)rows * k;
    const bool in_dev = is_device_ptr(ids_in) && is_device_ptr(dists_in);
    const bool out_dev = is_device_ptr(ids_out) && is_device_ptr(dists_out);
    struct Scratch {  // freed on every return path (after the stream has drained it)
        void *p = nullptr;
        cudaStream_t st;
        ~Scratch() {
            if (p) {
                cudaStreamSynchronize(st);
                cudaFree(p);
            }
        }
    } scratch{nullptr, st};
    const size_t need = (in_dev ? 0 : nin * 12) + (out_dev ? 0 : nout * 12);
    if (need) CU(cudaMalloc(&scratch.p, need));
    void *buf = scratch.p;
    const int64_t *di = ids_in;
    const void *dd = dists_in;
    char *cur = (char *)buf;
    if (!in_dev) {
        CU(cudaMemcpyAsync(cur, ids_in, nin * 8, cudaMemcpyHostToDevice, st));
        CU(cudaMemcpyAsync(cur + nin * 8, dists_in, nin * 4, cudaMemcpyHostToDevice, st));
        di = (const int64_t *)cur;
        dd = cur + nin * 8;
        cur += nin * 12;
    }
    int64_t *io = ids_out;
    void *doo = dists_out;
    if (!out_dev) {
        io = (int64_t *)cur;
        doo = cur + nout * 8;
    }
    if (dtype == SMILER_I16)
        merge_topk_kernel<int32_t><<<rows, 512, 0, st>>>(di, (const int32_t *)dd, G, rows, k, io,
                                                         (int32_t *)doo, 0x7FFFFFFF);
    else
        merge_topk_kernel<float><<<rows, 512, 0, st>>>(di, (const float *)dd, G, rows, k, io, (float *)doo,
                                                       INFINITY);
    CHECK_LAUNCH();
    if (!out_dev) {
        CU(cudaMemcpyAsync(ids_out, io, nout * 8, cudaMemcpyDeviceToHost, st));
        CU(cudaMemcpyAsync(dists_out, doo, nout * 4, cudaMemcpyDeviceToHost, st));
    }
    if (need) CU(cudaStreamSynchronize(st));
    return SMILER_OK;
}
