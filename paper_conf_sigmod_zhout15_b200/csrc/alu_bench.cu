// alu_bench.cu -- ALU issue-rate micro-benchmark that sets the
// ALU rooflines of the window-level LB kernel (a3) and the DTW kernel (a7).
// Not part of libsmiler.so; built as a standalone executable:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o alu_bench alu_bench.cu
// Prints one JSON object: per-SM per-clock rates of the exact instruction
// mixes of the hot loops, measured with clock64() over one full wave
// (one resident set of CTAs per SM), plus the SM clock seen.
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdint.h>
#include <stdlib.h>

constexpr int kIters = 4096;
constexpr int kChains = 8;
constexpr int kThreads = 256;

// DTW cell, f32: diff = q - c; m = min3(l, a, b); x = fma(diff, diff, m)
__global__ void __launch_bounds__(kThreads) dtw_f32_mix(float *out, long long *cyc, float q0) {
    float a[kChains], b[kChains];
    float c = threadIdx.x * 0.001f;
#pragma unroll
    for (int i = 0; i < kChains; i++) {
        a[i] = i * 0.5f + c;
        b[i] = i * 0.25f;
    }
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
        float q = q0 + it;
#pragma unroll
        for (int i = 0; i < kChains; i++) {
            float diff = q - a[i];
            float m = fminf(fminf(b[i], a[i]), c);
            a[i] = fmaf(diff, diff, m);
        }
    }
    long long t1 = clock64();
    float s = 0;
#pragma unroll
    for (int i = 0; i < kChains; i++) s += a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// DTW cell, int32: diff = q - c; m = min3; x = diff*diff + m (IADD, VIMNMX3,
// IMAD: the kernel's three ops; unsigned, so wrap-around is defined and no
// masking op is needed to keep the values bounded)
__global__ void __launch_bounds__(kThreads) dtw_i32_mix(unsigned *out, long long *cyc, unsigned q0) {
    unsigned a[kChains], b[kChains];
    unsigned c = threadIdx.x;
#pragma unroll
    for (int i = 0; i < kChains; i++) {
        a[i] = i * 3 + c;
        b[i] = i * 7;
    }
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
        unsigned q = q0 + it;
#pragma unroll
        for (int i = 0; i < kChains; i++) {
            unsigned diff = q - a[i];
            unsigned m = min(min(b[i], a[i]), c);
            a[i] = diff * diff + m;
        }
    }
    long long t1 = clock64();
    unsigned s = 0;
#pragma unroll
    for (int i = 0; i < kChains; i++) s += a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// LB term pair (a3): EQ: dd = v - min(max(v, L), U); acc = fma(dd, dd, acc); EC likewise.
__global__ void __launch_bounds__(kThreads) lbterm_f32_mix(float *out, long long *cyc, float q0) {
    float acc[kChains], v[kChains];
    float U = 0.5f + threadIdx.x * 1e-3f, L = -0.5f;
#pragma unroll
    for (int i = 0; i < kChains; i++) {
        acc[i] = 0;
        v[i] = i * 0.3f - 1.0f;
    }
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
        float q = q0 + it * 1e-4f;
#pragma unroll
        for (int i = 0; i < kChains; i++) {
            float d1 = v[i] - fminf(fmaxf(v[i], q), U);
            acc[i] = fmaf(d1, d1, acc[i]);
            float d2 = q - fminf(fmaxf(q, L), v[i]);
            acc[i] = fmaf(d2, d2, acc[i]);
        }
    }
    long long t1 = clock64();
    float s = 0;
#pragma unroll
    for (int i = 0; i < kChains; i++) s += acc[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// LB term pair as the kernels compute it: per term FADD, FADD, FMNMX3, FFMA
// (max(v - U, L - v, 0)^2, bit-identical to the clamp form).
__global__ void __launch_bounds__(kThreads) lbterm_max3_mix(float *out, long long *cyc, float q0) {
    // EQ term: series value v vs query envelope (q + 0.5, q - 0.5);
    // EC term: query value q vs series envelope (U2, L2): no shared subexpressions
    float acc[kChains], v[kChains], U2[kChains], L2[kChains];
#pragma unroll
    for (int i = 0; i < kChains; i++) {
        acc[i] = 0;
        v[i] = i * 0.3f - 1.0f;
        U2[i] = 0.5f + threadIdx.x * 1e-3f + i;
        L2[i] = -0.5f - i;
    }
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
        const float q = q0 + it * 1e-4f;
        const float uq = q + 0.5f, lq = q - 0.5f;
#pragma unroll
        for (int i = 0; i < kChains; i++) {
            float m1 = fmaxf(fmaxf(v[i] - uq, lq - v[i]), 0.0f);
            acc[i] = fmaf(m1, m1, acc[i]);
            float m2 = fmaxf(fmaxf(q - U2[i], L2[i] - q), 0.0f);
            acc[i] = fmaf(m2, m2, acc[i]);
        }
    }
    long long t1 = clock64();
    float s = 0;
#pragma unroll
    for (int i = 0; i < kChains; i++) s += acc[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

__global__ void __launch_bounds__(kThreads) lbterm_i32_mix(int *out, long long *cyc, int q0) {
    int acc[kChains], v[kChains];
    int U = 500 + threadIdx.x, L = -500;
#pragma unroll
    for (int i = 0; i < kChains; i++) {
        acc[i] = 0;
        v[i] = i * 37 - 100;
    }
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
        int q = q0 + (it & 1023);
#pragma unroll
        for (int i = 0; i < kChains; i++) {
            int d1 = v[i] - min(max(v[i], q), U);
            acc[i] += d1 * d1;
            int d2 = q - min(max(q, L), v[i]);
            acc[i] += d2 * d2;
        }
    }
    long long t1 = clock64();
    int s = 0;
#pragma unroll
    for (int i = 0; i < kChains; i++) s += acc[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// LB term pair with packed fp32x2 (sm_100), lb_diag_x2_kernel's form: per pair
// A = (c, L_C) - (U_Q, q), B = (q, L_Q) - (U_C, c) (two FADD2, the second operand
// negated), m = (max(A.x, B.y, 0), max(A.y, B.x, 0)) (two FMNMX3, each reading
// one even and one odd register), acc = fma(m, m, acc) (FFMA2).
__global__ void __launch_bounds__(kThreads) lbterm_f32x2_mix(float *out, long long *cyc, float q0) {
    float2 acc[kChains], cl[kChains], uc[kChains];
#pragma unroll
    for (int i = 0; i < kChains; i++) {
        acc[i] = make_float2(0.f, 0.f);
        cl[i] = make_float2(i * 0.3f - 1.0f, -0.5f - i);                         // (c, L_C)
        uc[i] = make_float2(0.5f + threadIdx.x * 1e-3f + i, i * 0.3f - 1.0f);    // (U_C, c)
    }
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
        // per-thread values (vector registers, as the kernel's LDS-broadcast window)
        const float q = q0 + it * 1e-4f + threadIdx.x * 1e-7f;
        const float2 uq = make_float2(q + 0.5f, q);   // (U_Q, q)
        const float2 ql = make_float2(q, q - 0.5f);   // (q, L_Q)
#pragma unroll
        for (int i = 0; i < kChains; i++) {
            const float2 a = __fadd2_rn(cl[i], make_float2(-uq.x, -uq.y));
            const float2 b = __fadd2_rn(ql, make_float2(-uc[i].x, -uc[i].y));
            const float2 m = make_float2(fmaxf(fmaxf(a.x, b.y), 0.f), fmaxf(fmaxf(a.y, b.x), 0.f));
            acc[i] = __ffma2_rn(m, m, acc[i]);
        }
    }
    long long t1 = clock64();
    float s = 0;
#pragma unroll
    for (int i = 0; i < kChains; i++) s += acc[i].x + acc[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// DTW cells, two candidates per thread with packed fp32x2: per 2 cells FADD2, FMNMX3 x2, FFMA2.
__global__ void __launch_bounds__(kThreads) dtw_f32x2_mix(float *out, long long *cyc, float q0) {
    float2 a[kChains], b[kChains], nc[kChains];
#pragma unroll
    for (int i = 0; i < kChains; i++) {
        a[i] = make_float2(i * 0.5f, i * 0.25f);
        b[i] = make_float2(i * 0.25f, i * 0.5f);
        nc[i] = make_float2(-threadIdx.x * 0.001f - i, -threadIdx.x * 0.002f + i);
    }
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
        const float q = q0 + it;
        const float2 qq = make_float2(q, q);
#pragma unroll
        for (int i = 0; i < kChains; i++) {
            float2 diff = __fadd2_rn(qq, nc[i]);
            float2 m = make_float2(fminf(fminf(b[i].x, a[i].x), b[i].y), fminf(fminf(b[i].y, a[i].y), b[i].x));
            b[i] = a[i];
            a[i] = __ffma2_rn(diff, diff, m);
        }
    }
    long long t1 = clock64();
    float s = 0;
#pragma unroll
    for (int i = 0; i < kChains; i++) s += a[i].x + a[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// fp64 FMA (the predictors' Gram / Cholesky arithmetic, smiler_predict):
// independent DFMA chains; unit = one DFMA (2 flops)
__global__ void __launch_bounds__(kThreads) dfma_mix(double *out, long long *cyc, double q0) {
    double a[kChains];
    const double c = 1.0 + threadIdx.x * 1e-9;
#pragma unroll
    for (int i = 0; i < kChains; i++) a[i] = i * 0.5 + q0;
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
#pragma unroll
        for (int i = 0; i < kChains; i++) a[i] = fma(a[i], c, -0.5);
    }
    long long t1 = clock64();
    double s = 0;
#pragma unroll
    for (int i = 0; i < kChains; i++) s += a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

struct Rate {
    double per_clk_sm;  // units per SM per SM clock
    double mhz;         // SM clock during the run (units per second / per-clock rate)
    double per_s;       // units per second, whole GPU
    int ctas_per_sm;    // resident CTAs per SM (one full wave is launched)
};

// Launch `kern` back to back for >= min_ms of device time (sustained clock).
// The grid is exactly one resident wave (occupancy of this kernel, at most
// per_sm CTAs per SM), so every CTA runs concurrently and the per-CTA clock64
// span is the per-SM time of the whole launch.
template <typename K, typename T>
static Rate run(K kern, T arg, int sms, int per_sm, double units_per_iter_chain, float min_ms) {
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kThreads, 0);
    if (occ < 1) occ = 1;
    if (occ > per_sm) occ = per_sm;
    int grid = sms * occ;
    T *out;
    long long *cyc;
    cudaMalloc(&out, sizeof(T) * grid * kThreads);
    cudaMalloc(&cyc, sizeof(long long) * grid);
    kern<<<grid, kThreads>>>(out, cyc, arg);  // warm
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    int reps = 1;
    float ms = 0;
    long long cycles = 0;
    while (true) {
        cudaEventRecord(e0);
        for (int r = 0; r < reps; r++) kern<<<grid, kThreads>>>(out, cyc, arg);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms >= min_ms || reps > (1 << 16)) break;
        reps *= 2;
    }
    long long *h = new long long[grid];
    cudaMemcpy(h, cyc, sizeof(long long) * grid, cudaMemcpyDeviceToHost);
    for (int i = 0; i < grid; i++) cycles = h[i] > cycles ? h[i] : cycles;  // last launch
    delete[] h;
    cudaFree(out);
    cudaFree(cyc);
    double units_launch = (double)grid * kThreads * kIters * kChains * units_per_iter_chain;
    Rate R;
    R.per_clk_sm = units_launch / sms / (double)cycles;
    R.per_s = units_launch * reps / (ms * 1e-3);
    R.mhz = R.per_s / (R.per_clk_sm * sms) / 1e6;
    R.ctas_per_sm = occ;
    return R;
}

int main(int argc, char **argv) {
    int dev = 0, sms = 0;
    cudaSetDevice(dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int per_sm = argc > 2 ? atoi(argv[2]) : 8;  // CTAs of 256 threads per SM (8 = 64 warps)
    const float min_ms = argc > 1 ? (float)atof(argv[1]) : 400.f;
    // interleaved, sustained: each mix twice, keep the second (steady clock)
    Rate r[8];
    for (int pass = 0; pass < 2; pass++) {
        r[0] = run(dtw_f32_mix, 1.0f, sms, per_sm, 1.0, min_ms);
        r[1] = run(dtw_f32x2_mix, 1.0f, sms, per_sm, 2.0, min_ms);
        r[2] = run(lbterm_f32_mix, 0.1f, sms, per_sm, 1.0, min_ms);
        r[3] = run(lbterm_f32x2_mix, 0.1f, sms, per_sm, 1.0, min_ms);
        r[4] = run(dtw_i32_mix, 1u, sms, per_sm, 1.0, min_ms);
        r[5] = run(lbterm_i32_mix, 1, sms, per_sm, 1.0, min_ms);
        r[6] = run(lbterm_max3_mix, 0.1f, sms, per_sm, 1.0, min_ms);
        r[7] = run(dfma_mix, 1.0, sms, per_sm, 1.0, min_ms);
    }
    cudaError_t e = cudaGetLastError();
    const char *names[8] = {"dtw_cell_f32", "dtw_cell_f32x2", "lbterm", "lbterm_f32x2", "dtw_cell_i32", "lbterm_i32",
                            "lbterm_max3", "dfma"};
    printf("{\"sms\": %d, \"ctas_per_sm\": %d, \"sustained_ms_per_mix\": %.0f", sms, per_sm, min_ms);
    for (int i = 0; i < 8; i++)
        printf(", \"%s_per_clk_sm\": %.3f, \"%s_mhz\": %.0f, \"%s_per_s\": %.4e, \"%s_ctas_per_sm\": %d", names[i],
               r[i].per_clk_sm, names[i], r[i].mhz, names[i], r[i].per_s, names[i], r[i].ctas_per_sm);
    printf(", \"note\": \"units per SM per SM clock and per second over back-to-back single full waves (the kernel's "
           "resident CTAs of 256 threads per SM, at most 8; 8 independent chains per thread), sustained for the stated "
           "time; dtw cell = FADD+FMNMX3+FFMA (f32), f32x2 = FADD2+2 FMNMX3+FFMA2 per 2 cells, i32 = IADD+VIMNMX3+IMAD; lbterm = one (SW,DW,j) EQ+EC "
           "term pair = 2x(FMNMX,FMNMX,FADD,FFMA), lbterm_max3 = 2x(FADD,FADD,FMNMX3,FFMA) (the kernels' form), f32x2 = FADD2,FADD2,FMNMX3,FMNMX3,FFMA2; dfma = one fp64 FMA (2 flops)\", \"cuda\": \"%s\"}\n",
           cudaGetErrorString(e));
    return e == cudaSuccess ? 0 : 1;
}
