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

template <typename K, typename T>
static double run(K kern, T arg, int sms, int per_sm, double units_per_iter_chain, double *mhz) {
    int grid = sms * per_sm;
    T *out;
    long long *cyc;
    cudaMalloc(&out, sizeof(T) * grid * kThreads);
    cudaMalloc(&cyc, sizeof(long long) * grid);
    kern<<<grid, kThreads>>>(out, cyc, arg);  // warm
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<<<grid, kThreads>>>(out, cyc, arg);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    long long *h = new long long[grid];
    cudaMemcpy(h, cyc, sizeof(long long) * grid, cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < grid; i++) mx = h[i] > mx ? h[i] : mx;
    delete[] h;
    cudaFree(out);
    cudaFree(cyc);
    // units per SM per clock: all per_sm CTAs of an SM run concurrently for ~mx cycles
    double units = (double)per_sm * kThreads * kIters * kChains * units_per_iter_chain;
    *mhz = mx / (ms * 1e3);
    return units / (double)mx;
}

int main() {
    int dev = 0, sms = 0;
    cudaSetDevice(dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int per_sm = 8;  // 64 warps per SM
    double mz1, mz2, mz3, mz4;
    double cf = run(dtw_f32_mix, 1.0f, sms, per_sm, 1.0, &mz1);
    double ci = run(dtw_i32_mix, 1, sms, per_sm, 1.0, &mz2);
    double lf = run(lbterm_f32_mix, 0.1f, sms, per_sm, 1.0, &mz3);
    double li = run(lbterm_i32_mix, 1, sms, per_sm, 1.0, &mz4);
    cudaError_t e = cudaGetLastError();
    printf("{\"sms\": %d, \"dtw_cell_f32_per_clk_sm\": %.3f, \"dtw_cell_i32_per_clk_sm\": %.3f, "
           "\"lbterm_per_clk_sm\": %.3f, \"lbterm_i32_per_clk_sm\": %.3f, \"sm_mhz_seen\": [%.0f, %.0f, %.0f, %.0f], "
           "\"note\": \"units per SM per SM-clock over one full wave (8 CTAs x 256 threads per SM, 8 independent "
           "chains per thread); dtw cell = FADD+FMNMX3+FFMA (f32) or IADD+VIMNMX3+IMAD(+LOP) (i32); lbterm = one "
           "(SW,DW,j) EQ+EC term pair = 2x(FMNMX,FMNMX,FADD,FFMA)\", \"cuda\": \"%s\"}\n",
           sms, cf, ci, lf, li, mz1, mz2, mz3, mz4, cudaGetErrorString(e));
    return e == cudaSuccess ? 0 : 1;
}
