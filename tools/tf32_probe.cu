// tools/tf32_probe.cu -- how does tcgen05.mma kind::tf32 read a 32-bit operand, and is a
// 3-product split (x = hi + lo) accurate to fp32 level?  Feasibility aid for the fp32
// tensor-core path; not part of the library.
//
// Test 1: A[r][0] = 1 + 2^-11 + 2^-13 (bits below TF32's 10-bit mantissa), B = e_0:
//         D = 1.0 => the tensor core truncates the low 13 bits; 1 + 2^-10 => round-to-nearest.
// Test 2: D = A B^T (128 x 64 x 32, random fp32) as one tf32 product and as the split
//         hi_A hi_B + hi_A lo_B + lo_A hi_B with hi = raw x (hardware truncation) and
//         lo = x - trunc13(x); max error vs fp64.
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cstring>
#include <cuda_runtime.h>

#include "tc_common.cuh"

using namespace ftw::tc;

__host__ __device__ constexpr uint32_t idesc_tf32(int M, int N) {
    return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void mma_tf32(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                         uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc)
        : "memory");
}

// A [128][32] fp32 and B [64][32] fp32, K-major SW128 (32 fp32 = 128 B per row); `mode`:
// 0 = one product of the raw values, 1 = 3-product split
__global__ void kern(const float* A, const float* B, float* D, int mode) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t holder;
    __shared__ uint64_t bar;
    const int t = threadIdx.x, warp = t / 32;
    uint8_t* sA = smem;              // hi A  16 KB
    uint8_t* sB = smem + 16384;      // hi B   8 KB
    uint8_t* sAl = smem + 24576;     // lo A  16 KB
    uint8_t* sBl = smem + 40960;     // lo B   8 KB
    auto put = [&](uint8_t* base, int r, int k, float v) {
        const int c = k / 4, e = k % 4;
        *reinterpret_cast<float*>(base + r * 128 + ((c ^ (r & 7)) * 16) + e * 4) = v;
    };
    for (int i = t; i < 128 * 32; i += blockDim.x) {
        const float x = A[i];
        const float hi = __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
        put(sA, i / 32, i % 32, x);
        put(sAl, i / 32, i % 32, x - hi);
    }
    for (int i = t; i < 64 * 32; i += blockDim.x) {
        const float x = B[i];
        const float hi = __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
        put(sB, i / 32, i % 32, x);
        put(sBl, i / 32, i % 32, x - hi);
    }
    if (warp == 0) { tmem_alloc(&holder, 64); tmem_relinquish(); }
    if (t == 32) { mbar_init(&bar, 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tb = holder;
    if (t == 32) {
        const uint32_t id = idesc_tf32(128, 64);
        for (int kk = 0; kk < 4; ++kk) {   // K = 8 fp32 = 32 bytes per MMA
            const uint64_t a = sdesc_sw128(smem_u32(sA) + kk * 32, 16, 1024);
            const uint64_t b = sdesc_sw128(smem_u32(sB) + kk * 32, 16, 1024);
            mma_tf32(tb, a, b, id, kk != 0);
            if (mode == 1) {
                mma_tf32(tb, a, sdesc_sw128(smem_u32(sBl) + kk * 32, 16, 1024), id, 1);
                mma_tf32(tb, sdesc_sw128(smem_u32(sAl) + kk * 32, 16, 1024), b, id, 1);
            }
        }
        mma_commit(&bar);
    }
    __syncwarp();
    mbar_wait(&bar, 0);
    tc_fence_after();
    if (warp < 4) {
        uint32_t r0[32], r1[32];
        tmem_ld32(tb + ((uint32_t)(warp * 32) << 16), r0);
        tmem_ld32(tb + ((uint32_t)(warp * 32) << 16) + 32, r1);
        tmem_wait_ld();
        for (int j = 0; j < 32; ++j) {
            D[t * 64 + j] = __uint_as_float(r0[j]);
            D[t * 64 + 32 + j] = __uint_as_float(r1[j]);
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tb, 64); }
}

int main() {
    const int M = 128, N = 64, K = 32;
    static float hA[M * K], hB[N * K], hD[M * N];
    float *dA, *dB, *dD;
    cudaMalloc(&dA, sizeof(hA));
    cudaMalloc(&dB, sizeof(hB));
    cudaMalloc(&dD, sizeof(hD));
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    // test 1
    const float x = 1.0f + ldexpf(1.f, -11) + ldexpf(1.f, -13);
    for (int i = 0; i < M * K; ++i) hA[i] = (i % K == 0) ? x : 0.f;
    for (int i = 0; i < N * K; ++i) hB[i] = (i % K == 0) ? 1.f : 0.f;
    cudaMemcpy(dA, hA, sizeof(hA), cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB, sizeof(hB), cudaMemcpyHostToDevice);
    kern<<<1, 128, 64 * 1024>>>(dA, dB, dD, 0);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
    printf("test1 (%s): x = %.9g  D = %.9g  (trunc -> 1, RN -> %.9g)\n", cudaGetErrorString(e), x, hD[0],
           1.0 + ldexp(1.0, -10));
    // test 2
    unsigned s = 777;
    auto rnd = [&]() { s = s * 1664525u + 1013904223u; return ((s >> 8) & 0xFFFFFF) / 16777216.0 * 2 - 1; };
    for (int i = 0; i < M * K; ++i) hA[i] = (float)rnd();
    for (int i = 0; i < N * K; ++i) hB[i] = (float)rnd();
    cudaMemcpy(dA, hA, sizeof(hA), cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB, sizeof(hB), cudaMemcpyHostToDevice);
    for (int mode = 0; mode < 2; ++mode) {
        kern<<<1, 128, 64 * 1024>>>(dA, dB, dD, mode);
        e = cudaDeviceSynchronize();
        cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
        double maxe = 0, maxr = 0;
        for (int m = 0; m < M; ++m)
            for (int n = 0; n < N; ++n) {
                double r = 0;
                for (int k = 0; k < K; ++k) r += (double)hA[m * K + k] * hB[n * K + k];
                maxe = fmax(maxe, fabs(hD[m * N + n] - r));
                maxr = fmax(maxr, fabs(r));
            }
        printf("test2 mode %d (%s): max abs err %.3e  (max |ref| %.3f, rel %.3e)\n", mode,
               cudaGetErrorString(e), maxe, maxr, maxe / maxr);
    }
    return 0;
}
