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

// DTW cell, int32: diff = q - c; m = min3; x = diff*diff + m
__global__ void __launch_bounds__(kThreads) dtw_i32_mix(int *out, long long *cyc, int q0) {
    int a[kChains], b[kChains];
    int c = threadIdx.x;
#pragma unroll
    for (int i = 0; i < kChains; i++) {
        a[i] = i * 3 + c;
        b[i] = i * 7;
    }
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
        int q = q0 + it;
#pragma unroll
        for (int i = 0; i < kChains; i++) {
            int diff = q - a[i];
            int m = min(min(b[i], a[i]), c);
            a[i] = (diff * diff + m) & 0xFFFF;  // keep values small (the AND adds one ALU op)
        }
    }
    long long t1 = clock64();
    int s = 0;
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

// LB term pair with packed fp32x2 (sm_100): per pair FADD2, FADD2, FMNMX3 x2, FFMA2.
__global__ void __launch_bounds__(kThreads) lbterm_f32x2_mix(float *out, long long *cyc, float q0) {
    float2 acc[kChains], cc[kChains], ne[kChains];
#pragma unroll
    for (int i = 0; i < kChains; i++) {
        acc[i] = make_float2(0.f, 0.f);
        cc[i] = make_float2(i * 0.3f - 1.0f, i * 0.3f - 1.0f);
        ne[i] = make_float2(-0.5f - threadIdx.x * 1e-3f - i, 0.5f + i);
    }
    long long t0 = clock64();
    for (int it = 0; it < kIters; it++) {
        const float q = q0 + it * 1e-4f;
        const float2 nq = make_float2(-q, -q * 0.5f);
        const float2 qq = make_float2(q, q);
#pragma unroll
        for (int i = 0; i < kChains; i++) {
            float2 d1 = __fadd2_rn(cc[i], nq);
            float2 d2 = __fadd2_rn(qq, ne[i]);
            float2 m = make_float2(fmaxf(fmaxf(d1.x, -d1.y), 0.f), fmaxf(fmaxf(d2.x, -d2.y), 0.f));
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
    double mhz;         // effective SM clock during the run
    double per_s;       // units per second, whole GPU
};

// Launch `kern` back to back for >= min_ms of device time (sustained clock).
template <typename K, typename T>
static Rate run(K kern, T arg, int sms, int per_sm, double units_per_iter_chain, float min_ms) {
    int grid = sms * per_sm;
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
        r[4] = run(dtw_i32_mix, 1, sms, per_sm, 1.0, min_ms);
        r[5] = run(lbterm_i32_mix, 1, sms, per_sm, 1.0, min_ms);
        r[6] = run(lbterm_max3_mix, 0.1f, sms, per_sm, 1.0, min_ms);
        r[7] = run(dfma_mix, 1.0, sms, per_sm, 1.0, min_ms);
    }
    cudaError_t e = cudaGetLastError();
    const char *names[8] = {"dtw_cell_f32", "dtw_cell_f32x2", "lbterm", "lbterm_f32x2", "dtw_cell_i32", "lbterm_i32",
                            "lbterm_max3", "dfma"};
    printf("{\"sms\": %d, \"ctas_per_sm\": %d, \"sustained_ms_per_mix\": %.0f", sms, per_sm, min_ms);
    for (int i = 0; i < 8; i++)
        printf(", \"%s_per_clk_sm\": %.3f, \"%s_mhz\": %.0f, \"%s_per_s\": %.4e", names[i], r[i].per_clk_sm,
               names[i], r[i].mhz, names[i], r[i].per_s);
    printf(", \"note\": \"units per SM per SM clock and per second over back-to-back full waves (8 CTAs x 256 threads "
           "per SM, 8 independent chains per thread), sustained for the stated time; dtw cell = FADD+FMNMX3+FFMA (f32), "
           "f32x2 = FADD2+2 FMNMX3+FFMA2 per 2 cells, i32 = IADD+VIMNMX3+IMAD(+LOP); lbterm = one (SW,DW,j) EQ+EC "
           "term pair = 2x(FMNMX,FMNMX,FADD,FFMA), lbterm_max3 = 2x(FADD,FADD,FMNMX3,FFMA) (the kernels' form), f32x2 = FADD2,FADD2,FMNMX3,FMNMX3,FFMA2; dfma = one fp64 FMA (2 flops)\", \"cuda\": \"%s\"}\n",
           cudaGetErrorString(e));
    return e == cudaSuccess ? 0 : 1;
}
