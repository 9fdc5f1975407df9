// predict.cu -- the predictors that consume the Suffix kNN result (SURVEY
// §8(f) NEXT-3; Sec. 5.2).  One CTA per predictor f_{i,j} (item
// query length d_i, k_j in EKV) of one master query:
//
//   kNN data   X = {c[t_a .. t_a+d)},  Y_h = {c[t_a + d - 1 + h]},  a < k_j
//              (the first k_j neighbours: multi-k by prefix, P:838-841;
//               h-step target)
//   AR         u~0 = sum_a y_a / k_j,  s~0^2 = sum_a (y_a - u~0)^2 / k_j    (Eq. 12-13)
//   GP         C_ab = th0^2 exp(-|x_a - x_b|^2 / (2 th1^2)) + delta_ab th2^2 (Eq. 18)
//              c0_a = th0^2 exp(-|x_a - x0|^2 / (2 th1^2)),  x0 = IQ_i
//              u0 = c0^T C^-1 Y,  s0^2 = th0^2 + th2^2 - c0^T C^-1 c0      (Eq. 16-17)
//
// All arithmetic in fp64 (the Gram of fp32/int16 inputs is exact in the
// differences).  C^-1 is applied through its Cholesky factor L (C = L L^T):
// with z = L^-1 c0 and w = L^-1 Y,  u0 = z.w and c0^T C^-1 c0 = z.z.  The
// k x k factor lives in shared memory (k_j <= kMaxPredK); the Gram streams
// the segments through shared memory 64 points at a time.  No tensor cores:
// k_j^2 d / 2 + k_j^3 / 3 fp64 flops per predictor (at most ~1.8 MFLOP at
// k = 128, d = 128), a latency-bound small dense problem per CTA.
#include <math.h>

#include "internal.h"

namespace smiler {

constexpr int kPredThreads = 256;
constexpr int kPredChunk = 64;  // segment points staged per Gram pass

struct PredSensor {
    int64_t off, n;
};

// staged points [kmax + 1][kPredChunk + 1] floats, rounded up to 16 bytes (int64 follow)
__host__ __device__ inline size_t pred_xs_bytes(int kmax) {
    return ((size_t)(kmax + 1) * (kPredChunk + 1) * sizeof(float) + 15) & ~(size_t)15;
}

__host__ __device__ inline size_t pred_smem_bytes(int kmax) {
    const int kp = kmax + 1;
    return (size_t)kp * kp * sizeof(double)                  // Gram / C / L (row-major, lower)
           + (size_t)4 * kp * sizeof(double)                 // c0, Y, z, w
           + pred_xs_bytes(kmax)                              // staged points (k_j segments + x0)
           + (size_t)kp * sizeof(int64_t) + 64;              // neighbour starts, flags
}

template <typename S>
__global__ void __launch_bounds__(kPredThreads) predict_kernel(
    const S *series, const PredSensor *sens, const int32_t *qsens, const S *queries, int D, const int32_t *lens,
    int n_len, const int64_t *ids, int k, const int32_t *ekv, int n_k, int h, const double *theta, int kmax,
    double *ar_mean, double *ar_var, double *gp_mean, double *gp_var) {
    extern __shared__ __align__(16) unsigned char pr_smem[];
    const int pred = blockIdx.x;
    const int j = pred % n_k, i = (pred / n_k) % n_len, m = pred / (n_k * n_len);
    const int kj = ekv[j], d = lens[i];
    const int kp = kmax + 1;
    double *G = reinterpret_cast<double *>(pr_smem);  // [kp][kp]
    double *c0 = G + (size_t)kp * kp;
    double *Yv = c0 + kp;
    double *z = Yv + kp;
    double *wv = z + kp;
    float *Xs = reinterpret_cast<float *>(wv + kp);  // [kj + 1][kPredChunk + 1]
    int64_t *ts = reinterpret_cast<int64_t *>(reinterpret_cast<unsigned char *>(Xs) + pred_xs_bytes(kmax));
    int *flag = reinterpret_cast<int *>(ts + kp);
    const int tid = threadIdx.x;
    const PredSensor sn = sens[qsens[m]];
    const S *c = series + sn.off;
    const S *x0 = queries + (int64_t)m * D + (D - d);  // IQ_i = last d points of the MQ
    const int64_t out = pred;

    if (tid == 0) *flag = 0;
    __syncthreads();
    for (int a = tid; a < kj; a += kPredThreads) {
        const int64_t t = ids[((int64_t)m * n_len + i) * k + a];
        ts[a] = t;
        if (t < 0 || t + d - 1 + h >= sn.n) atomicOr(flag, 1);  // no h-step-ahead value
        else Yv[a] = (double)c[t + d - 1 + h];
    }
    __syncthreads();
    if (*flag) {
        if (tid == 0) ar_mean[out] = ar_var[out] = gp_mean[out] = gp_var[out] = nan("");
        return;
    }
    // ---- AR (Eq. 12-13): two passes, warp 0 ----------------------------------
    if (tid < 32) {
        double s = 0;
        for (int a = tid; a < kj; a += 32) s += Yv[a];
#pragma unroll
        for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        const double u = s / kj;
        double v = 0;
        for (int a = tid; a < kj; a += 32) v += (Yv[a] - u) * (Yv[a] - u);
#pragma unroll
        for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (tid == 0) {
            ar_mean[out] = u;
            ar_var[out] = v / kj;
        }
    }
    // ---- Gram: G[a][b] = |x_a - x_b|^2 (a >= b), row kj = x0 -----------------
    const int np = kj + 1;
    const int npairs = np * (np + 1) / 2;
    for (int x = tid; x < npairs; x += kPredThreads) {
        // pair x -> (a, b), a >= b: a = floor((sqrt(8x+1)-1)/2)
        int a = (int)((sqrt(8.0 * x + 1.0) - 1.0) * 0.5);
        while ((a + 1) * (a + 2) / 2 <= x) a++;
        while (a * (a + 1) / 2 > x) a--;
        G[a * kp + (x - a * (a + 1) / 2)] = 0.0;
    }
    for (int p0 = 0; p0 < d; p0 += kPredChunk) {
        const int pn = min(kPredChunk, d - p0);
        __syncthreads();
        for (int x = tid; x < np * kPredChunk; x += kPredThreads) {
            const int a = x / kPredChunk, pp = x % kPredChunk;
            float v = 0.f;
            if (pp < pn) v = (float)(a < kj ? c[ts[a] + p0 + pp] : x0[p0 + pp]);
            Xs[a * (kPredChunk + 1) + pp] = v;
        }
        __syncthreads();
        for (int x = tid; x < npairs; x += kPredThreads) {
            int a = (int)((sqrt(8.0 * x + 1.0) - 1.0) * 0.5);
            while ((a + 1) * (a + 2) / 2 <= x) a++;
            while (a * (a + 1) / 2 > x) a--;
            const int b = x - a * (a + 1) / 2;
            if (a == b) continue;
            const float *xa = Xs + a * (kPredChunk + 1), *xb = Xs + b * (kPredChunk + 1);
            double acc = 0.0;
            for (int pp = 0; pp < pn; pp++) {
                const double df = (double)xa[pp] - (double)xb[pp];
                acc = fma(df, df, acc);
            }
            G[a * kp + b] += acc;
        }
    }
    __syncthreads();
    // ---- covariance (Eq. 18) ---------------------------------------------------
    const double* th = theta + out * 3;
    const double t0s = th[0] * th[0], inv2t1 = 0.5 / (th[1] * th[1]), t2s = th[2] * th[2];
    for (int x = tid; x < npairs; x += kPredThreads) {
        int a = (int)((sqrt(8.0 * x + 1.0) - 1.0) * 0.5);
        while ((a + 1) * (a + 2) / 2 <= x) a++;
        while (a * (a + 1) / 2 > x) a--;
        const int b = x - a * (a + 1) / 2;
        const double cv = t0s * exp(-G[a * kp + b] * inv2t1);
        if (a == kj) {
            if (b < kj) c0[b] = cv;  // c(x_b, x0): no delta term
        } else {
            G[a * kp + b] = cv + (a == b ? t2s : 0.0);
        }
    }
    __syncthreads();
    // ---- Cholesky C = L L^T (right-looking, lower, in place) ------------------
    for (int p = 0; p < kj; p++) {
        if (tid == 0) {
            const double piv = G[p * kp + p];
            if (!(piv > 0.0)) *flag = 1;
            G[p * kp + p] = sqrt(piv > 0.0 ? piv : 1.0);
        }
        __syncthreads();
        const double lpp = G[p * kp + p];
        for (int r = p + 1 + tid; r < kj; r += kPredThreads) G[r * kp + p] /= lpp;
        __syncthreads();
        const int nr = kj - p - 1;
        for (int x = tid; x < nr * nr; x += kPredThreads) {
            const int r = p + 1 + x / nr, cc = p + 1 + x % nr;
            if (cc <= r) G[r * kp + cc] -= G[r * kp + p] * G[cc * kp + p];
        }
        __syncthreads();
    }
    // ---- z = L^-1 c0, w = L^-1 Y (forward substitution, column-oriented) -------
    for (int a = tid; a < kj; a += kPredThreads) {
        z[a] = c0[a];
        wv[a] = Yv[a];
    }
    __syncthreads();
    for (int p = 0; p < kj; p++) {
        const double lpp = G[p * kp + p];
        const double zp = z[p] / lpp, wp = wv[p] / lpp;
        for (int r = p + 1 + tid; r < kj; r += kPredThreads) {
            const double l = G[r * kp + p];
            z[r] -= l * zp;
            wv[r] -= l * wp;
        }
        __syncthreads();
        if (tid == 0) {
            z[p] = zp;
            wv[p] = wp;
        }
    }
    __syncthreads();
    if (tid < 32) {
        double uw = 0, zz = 0;
        for (int a = tid; a < kj; a += 32) {
            uw += z[a] * wv[a];
            zz += z[a] * z[a];
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            uw += __shfl_xor_sync(0xffffffffu, uw, o);
            zz += __shfl_xor_sync(0xffffffffu, zz, o);
        }
        if (tid == 0) {
            const bool bad = *flag != 0;
            gp_mean[out] = bad ? nan("") : uw;
            gp_var[out] = bad ? nan("") : t0s + t2s - zz;
        }
    }
}

template <typename S>
int launch_predict(const void *series, const int64_t *soff_n, int n_sensors, const int32_t *qsens, const void *queries,
                   int D, const int32_t *lens, int n_len, const int64_t *ids, int k, const int32_t *ekv, int n_k,
                   int kmax, int h, const double *theta, int n_pred, double *ar_mean, double *ar_var,
                   double *gp_mean, double *gp_var, cudaStream_t st) {
    (void)n_sensors;
    const size_t smem = pred_smem_bytes(kmax);
    if (smem > 48 * 1024)
        cudaFuncSetAttribute(predict_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    predict_kernel<S><<<n_pred, kPredThreads, smem, st>>>(
        (const S *)series, reinterpret_cast<const PredSensor *>(soff_n), qsens, (const S *)queries, D, lens, n_len,
        ids, k, ekv, n_k, h, theta, kmax, ar_mean, ar_var, gp_mean, gp_var);
    return (int)cudaGetLastError();
}

template int launch_predict<int16_t>(const void *, const int64_t *, int, const int32_t *, const void *, int,
                                     const int32_t *, int, const int64_t *, int, const int32_t *, int, int, int,
                                     const double *, int, double *, double *, double *, double *, cudaStream_t);
template int launch_predict<float>(const void *, const int64_t *, int, const int32_t *, const void *, int,
                                   const int32_t *, int, const int64_t *, int, const int32_t *, int, int, int,
                                   const double *, int, double *, double *, double *, double *, cudaStream_t);

size_t predict_smem(int kmax) { return pred_smem_bytes(kmax); }

}  // namespace smiler
