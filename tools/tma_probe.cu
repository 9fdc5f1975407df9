// Probe: 2-D TMA loads of a w x 256 box (the ring-scan shape), descriptor in
// kernel-param space (__grid_constant__) vs global memory, several coordinates.
// nvcc -gencode arch=compute_100a,code=sm_100a -o tma_probe tools/tma_probe.cu -lcuda
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

__device__ __forceinline__ uint32_t su(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <bool GLOBAL>
__global__ void probe(const __grid_constant__ CUtensorMap tmap, const CUtensorMap *gmap, int col, int row0,
                      int rstep, int boxw, float *out) {
    extern __shared__ __align__(128) unsigned char sm[];
    __shared__ __align__(8) uint64_t bar;
    __half *t = (__half *)sm;
    const int row = row0 + blockIdx.x * rstep;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su(&bar)), "r"(1));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        const CUtensorMap *m = GLOBAL ? gmap : &tmap;
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&bar)), "r"(8 * boxw * 2)
                     : "memory");
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::
                "r"(su(t)),
            "l"(m), "r"(col), "r"(row), "r"(su(&bar))
            : "memory");
    }
    asm volatile(
        "{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
            su(&bar)),
        "r"(0)
        : "memory");
    for (int e = threadIdx.x; e < 8 * boxw; e += blockDim.x) out[(size_t)blockIdx.x * 2048 + e] = __half2float(t[e]);
}

int main(int argc, char **argv) {
    // args: global(0/1) boxw col promo(0 none, 1 256B) rowstart
    const int use_global = atoi(argv[1]), boxw = atoi(argv[2]), col = atoi(argv[3]), promo = atoi(argv[4]);
    const int row0 = atoi(argv[5]);
    const int ndw = 1500, pstride = 1504, rows = 1536;
    __half *g;
    cudaMalloc(&g, (size_t)rows * pstride * 2);
    __half *h = (__half *)malloc((size_t)rows * pstride * 2);
    for (int r = 0; r < rows; r++)
        for (int c = 0; c < pstride; c++) h[(size_t)r * pstride + c] = __float2half((float)((r * 7 + c) % 1000));
    cudaMemcpy(g, h, (size_t)rows * pstride * 2, cudaMemcpyHostToDevice);
    PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&encode, cudaEnableDefault, &q);
    alignas(64) CUtensorMap tm;
    const cuuint64_t gdim[2] = {(cuuint64_t)ndw, (cuuint64_t)rows};
    const cuuint64_t gstride[1] = {(cuuint64_t)pstride * 2};
    const cuuint32_t box[2] = {(cuuint32_t)boxw, 8};
    const cuuint32_t estr[2] = {1, 1};
    CUresult cr = encode(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, g, gdim, gstride, box, estr,
                         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                         promo ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B : CU_TENSOR_MAP_L2_PROMOTION_NONE,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    CUtensorMap *gm;
    cudaMalloc(&gm, sizeof(CUtensorMap));
    cudaMemcpy(gm, &tm, sizeof(tm), cudaMemcpyHostToDevice);
    float *out;
    const int nb = 8;
    cudaMalloc(&out, (size_t)nb * 2048 * 4);
    cudaMemset(out, 0, (size_t)nb * 2048 * 4);
    float *ho = (float *)malloc((size_t)nb * 2048 * 4);
    cudaFuncSetAttribute(probe<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8192);
    cudaFuncSetAttribute(probe<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8192);
    if (!use_global) probe<false><<<nb, 256, 4096>>>(tm, gm, col, row0, 190, boxw, out);
    else probe<true><<<nb, 256, 4096>>>(tm, gm, col, row0, 190, boxw, out);
    cudaError_t e = cudaDeviceSynchronize();
    printf("encode=%d global=%d boxw=%d col=%d promo=%d row0=%d: ", (int)cr, use_global, boxw, col, promo, row0);
    if (e != cudaSuccess) {
        printf("%s\n", cudaGetErrorString(e));
        return 1;
    }
    cudaMemcpy(ho, out, (size_t)nb * 2048 * 4, cudaMemcpyDeviceToHost);
    long bad = 0;
    for (int b = 0; b < nb; b++)
        for (int rr = 0; rr < 8; rr++)
            for (int x = 0; x < boxw; x++) {
                const int r = row0 + b * 190 + rr, c = col + x;
                const float want = (r < rows && c >= 0 && c < ndw) ? (float)((r * 7 + c) % 1000) : 0.f;
                bad += ho[(size_t)b * 2048 + rr * boxw + x] != want;
            }
    printf("%ld mismatches\n", bad);
    return 0;
}
