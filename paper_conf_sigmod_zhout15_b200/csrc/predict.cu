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
// differences).  C^-1 is applied through C = L D L^T (unit lower L): with
// z = L^-1 c0 and w = L^-1 Y, u0 = sum z_a w_a / D_a and c0^T C^-1 c0 =
// sum z_a^2 / D_a; the forward solves ride along the elimination (c0 and Y
// are extra columns), one barrier per column.  The k x k matrix lives in
// shared memory (k_j <= kMaxPredK); the Gram uses 4 x 4 register tiles of
// pairs over points staged 32 at a time.  No tensor cores: 3 d k_j^2 / 2 +
// k_j^3 / 3 fp64 flops per predictor (~3.9 MFLOP at k = 128, d = 128), a
// small dense problem per CTA.
#include <math.h>

#include "internal.h"

namespace smiler {

constexpr int kPredThreads = 512;
constexpr int kPredChunk = 32;  // segment points staged per Gram pass
constexpr int kPredTile = 4;    // Gram register tile (4 x 4 pairs per thread task)

struct PredSensor {
    int64_t off, n;
};

// padded row length (doubles) of the point-major staging Xs[pp][a]
__host__ __device__ inline int pred_xs_stride(int kmax) { return ((kmax + 1 + kPredTile - 1) / kPredTile) * kPredTile + 2; }

__host__ __device__ inline size_t pred_smem_bytes(int kmax) {
    const int kp = kmax + 1;
    return (size_t)kp * kp * sizeof(double)                            // Gram / C / LDL^T (row-major, lower)
           + (size_t)3 * kp * sizeof(double)                           // c0, Y, D
           + (size_t)kPredChunk * pred_xs_stride(kmax) * sizeof(double)  // staged points
           + (size_t)kp * sizeof(int64_t) + 64;                        // neighbour starts, flag
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
    const int XS = pred_xs_stride(kmax);
    double *G = reinterpret_cast<double *>(pr_smem);  // [kp][kp]
    double *c0 = G + (size_t)kp * kp;
    double *Yv = c0 + kp;
    double *Dg = Yv + kp;
    double *Xs = Dg + kp;                                   // [kPredChunk][XS], point-major
    int64_t *ts = reinterpret_cast<int64_t *>(Xs + (size_t)kPredChunk * XS);
    int *flag = reinterpret_cast<int *>(ts + kp);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    constexpr int NW = kPredThreads / 32;
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
    if (warp == 0) {
        double sacc = 0;
        for (int a = lane; a < kj; a += 32) sacc += Yv[a];
#pragma unroll
        for (int o = 16; o; o >>= 1) sacc += __shfl_xor_sync(0xffffffffu, sacc, o);
        const double u = sacc / kj;
        double v = 0;
        for (int a = lane; a < kj; a += 32) v += (Yv[a] - u) * (Yv[a] - u);
#pragma unroll
        for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == 0) {
            ar_mean[out] = u;
            ar_var[out] = v / kj;
        }
    }
    // ---- Gram G[a][b] = |x_a - x_b|^2 (a > b; row kj is x0) in 4 x 4 register
    // tiles of pairs, points staged 32 at a time as doubles (exact differences)
    const int np = kj + 1;
    const int R = (np + kPredTile - 1) / kPredTile;
    const int T = R * (R + 1) / 2;  // lower-triangle tiles (ta >= tb)
    for (int x = tid; x < np * kp; x += kPredThreads) G[x] = 0.0;
    for (int p0 = 0; p0 < d; p0 += kPredChunk) {
        const int pn = min(kPredChunk, d - p0);
        __syncthreads();
        for (int x = tid; x < kPredChunk * R * kPredTile; x += kPredThreads) {
            const int pp = x / (R * kPredTile), a = x % (R * kPredTile);
            double v = 0.0;
            if (pp < pn && a < np) v = (double)(a < kj ? c[ts[a] + p0 + pp] : x0[p0 + pp]);
            Xs[pp * XS + a] = v;
        }
        __syncthreads();
        for (int tt = tid; tt < T; tt += kPredThreads) {
            // tile tt -> (ta, tb), ta >= tb (row-major over the lower triangle)
            int ta = (int)((sqrt(8.0 * tt + 1.0) - 1.0) * 0.5);
            while ((ta + 1) * (ta + 2) / 2 <= tt) ta++;
            while (ta * (ta + 1) / 2 > tt) ta--;
            const int tb = tt - ta * (ta + 1) / 2;
            double acc[kPredTile][kPredTile];
#pragma unroll
            for (int u = 0; u < kPredTile; u++)
#pragma unroll
                for (int v = 0; v < kPredTile; v++) acc[u][v] = 0.0;
            const double *xa = Xs + ta * kPredTile, *xb = Xs + tb * kPredTile;
            for (int pp = 0; pp < pn; pp++) {
                const double2 a01 = *reinterpret_cast<const double2 *>(xa + pp * XS);
                const double2 a23 = *reinterpret_cast<const double2 *>(xa + pp * XS + 2);
                const double2 b01 = *reinterpret_cast<const double2 *>(xb + pp * XS);
                const double2 b23 = *reinterpret_cast<const double2 *>(xb + pp * XS + 2);
                const double av[4] = {a01.x, a01.y, a23.x, a23.y}, bv[4] = {b01.x, b01.y, b23.x, b23.y};
#pragma unroll
                for (int u = 0; u < kPredTile; u++)
#pragma unroll
                    for (int v = 0; v < kPredTile; v++) {
                        const double df = av[u] - bv[v];
                        acc[u][v] = fma(df, df, acc[u][v]);
                    }
            }
#pragma unroll
            for (int u = 0; u < kPredTile; u++)
#pragma unroll
                for (int v = 0; v < kPredTile; v++) {
                    const int a = ta * kPredTile + u, b = tb * kPredTile + v;
                    if (a < np && b < a) G[a * kp + b] += acc[u][v];
                }
        }
    }
    __syncthreads();
    // ---- covariance (Eq. 18): C in the lower triangle, c0 = row kj ----------
    const double *th = theta + out * 3;
    const double t0s = th[0] * th[0], inv2t1 = 0.5 / (th[1] * th[1]), t2s = th[2] * th[2];
    for (int a = warp; a < np; a += NW)
        for (int b = lane; b <= a; b += 32) {
            const double cv = t0s * exp(-G[a * kp + b] * inv2t1);
            if (a == kj) {
                if (b < kj) c0[b] = cv;  // c(x_b, x0): no delta term
            } else {
                G[a * kp + b] = cv + (a == b ? t2s : 0.0);
            }
        }
    __syncthreads();
    // ---- C = L D L^T with the forward solves folded in: eliminating column p
    // also updates the right-hand sides c0 and Y, so afterwards c0 = L^-1 c0,
    // Y = L^-1 Y and c0^T C^-1 Y = sum_a c0_a Y_a / D_a (one barrier per column)
    for (int p = 0; p < kj; p++) {
        const double dp = G[p * kp + p];
        if (!(dp > 0.0)) {
            if (tid == 0) *flag = 1;
            break;  // uniform: every thread reads the same pivot
        }
        const double inv = 1.0 / dp;
        for (int r = p + 1 + warp; r < kj; r += NW) {
            const double lr = G[r * kp + p] * inv;
            for (int cc = p + 1 + lane; cc <= r; cc += 32) G[r * kp + cc] -= lr * G[cc * kp + p];
            if (lane == 0) {
                c0[r] -= lr * c0[p];
                Yv[r] -= lr * Yv[p];
            }
        }
        if (tid == 0) Dg[p] = dp;
        __syncthreads();
    }
    __syncthreads();
    if (warp == 0) {
        double uw = 0, zz = 0;
        for (int a = lane; a < kj; a += 32) {
            uw += c0[a] * Yv[a] / Dg[a];
            zz += c0[a] * c0[a] / Dg[a];
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            uw += __shfl_xor_sync(0xffffffffu, uw, o);
            zz += __shfl_xor_sync(0xffffffffu, zz, o);
        }
        if (lane == 0) {
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
