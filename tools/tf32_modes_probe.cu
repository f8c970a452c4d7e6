// tools/tf32_modes_probe.cu -- which operand forms does tcgen05.mma kind::tf32 accept on sm_100a,
// and does the 3-product split x = hi + lo (hi = raw value, read truncated by the tensor core;
// lo = x - trunc13(x)) stay at fp32 accuracy in each?  Feasibility aid for the fp32 tensor-core
// path; not part of the library.
//   mode 0: SS, A and B K-major, one product            mode 1: SS K-major, 3 products
//   mode 2: SS, B MN-major (N contiguous), 3 products   mode 3: TS (A in TMEM), B K-major, 3 products
//   mode 4: TS, B MN-major, 3 products
// D[128 x 64] = A[128 x 32] B[64 x 32]^T, compared with a host fp64 product.
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cuda_runtime.h>

#include "tc_common.cuh"

using namespace ftw::tc;

__host__ __device__ constexpr uint32_t idesc_tf32(int M, int N, bool a_mn, bool b_mn) {
    return (1u << 4) | (2u << 7) | (2u << 10) | ((a_mn ? 1u : 0u) << 15) | ((b_mn ? 1u : 0u) << 16) |
           ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void mma_ss32(uint32_t d, uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d), "l"(a), "l"(b), "r"(id),
                 "r"(acc) : "memory");
}
__device__ __forceinline__ void mma_ts32(uint32_t d, uint32_t a, uint64_t b, uint32_t id, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d), "r"(a), "l"(b), "r"(id),
                 "r"(acc) : "memory");
}

__device__ __forceinline__ float lo_of(float x) { return x - __uint_as_float(__float_as_uint(x) & 0xFFFFE000u); }

__global__ void kern(const float* A, const float* B, float* D, int mode, uint32_t lbo, uint32_t sbo) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t holder;
    __shared__ uint64_t bar;
    const int t = threadIdx.x, warp = t / 32;
    uint8_t* sA = smem;              // A hi, K-major 128 rows x 128 B
    uint8_t* sAl = smem + 16384;     // A lo
    uint8_t* sB = smem + 32768;      // B hi: K-major 64 rows x 128 B, or MN-major 2 groups x 32 rows x 128 B
    uint8_t* sBl = smem + 40960;     // B lo
    const bool bmn = mode == 2 || mode == 4;
    const bool ts = mode >= 3;
    for (int i = t; i < 128 * 32; i += blockDim.x) {
        const int r = i / 32, k = i % 32, c = k / 4, e = k % 4;
        const uint32_t off = r * 128 + ((c ^ (r & 7)) * 16) + e * 4;
        *reinterpret_cast<float*>(sA + off) = A[i];
        *reinterpret_cast<float*>(sAl + off) = lo_of(A[i]);
    }
    for (int i = t; i < 64 * 32; i += blockDim.x) {
        const int n = i / 32, k = i % 32;
        uint32_t off;
        if (!bmn) {
            off = n * 128 + (((k / 4) ^ (n & 7)) * 16) + (k % 4) * 4;
        } else {   // row = k (32 rows of 128 B), 32 n per row, group g = n / 32 at g * 4096
            const int g = n / 32, e = n % 32;
            off = g * 4096 + k * 128 + (((e / 4) ^ (k & 7)) * 16) + (e % 4) * 4;
        }
        *reinterpret_cast<float*>(sB + off) = B[i];
        *reinterpret_cast<float*>(sBl + off) = lo_of(B[i]);
    }
    if (warp == 0) { tmem_alloc(&holder, 128); tmem_relinquish(); }
    if (t == 32) { mbar_init(&bar, 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tb = holder;
    if (ts && warp < 4) {   // A hi -> TMEM cols [64, 96), A lo -> [96, 128); lane = row
        uint32_t hi[16], lo[16];
        for (int h = 0; h < 2; ++h) {
            for (int j = 0; j < 16; ++j) {
                const float x = A[t * 32 + 16 * h + j];
                hi[j] = __float_as_uint(x);
                lo[j] = __float_as_uint(lo_of(x));
            }
            tmem_st16(tb + ((uint32_t)(warp * 32) << 16) + 64 + 16 * h, hi);
            tmem_st16(tb + ((uint32_t)(warp * 32) << 16) + 96 + 16 * h, lo);
        }
        tmem_wait_st();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (t == 32) {
        const uint32_t id = idesc_tf32(128, 64, false, bmn);
        for (int kk = 0; kk < 4; ++kk) {   // K = 8 per MMA
            const uint64_t b = bmn ? sdesc_sw128(smem_u32(sB) + kk * 1024, lbo, sbo)
                                   : sdesc_sw128(smem_u32(sB) + kk * 32, 16, 1024);
            const uint64_t bl = bmn ? sdesc_sw128(smem_u32(sBl) + kk * 1024, lbo, sbo)
                                    : sdesc_sw128(smem_u32(sBl) + kk * 32, 16, 1024);
            if (!ts) {
                const uint64_t a = sdesc_sw128(smem_u32(sA) + kk * 32, 16, 1024);
                const uint64_t al = sdesc_sw128(smem_u32(sAl) + kk * 32, 16, 1024);
                mma_ss32(tb, a, b, id, kk != 0);
                if (mode >= 1) { mma_ss32(tb, a, bl, id, 1); mma_ss32(tb, al, b, id, 1); }
            } else {
                const uint32_t a = tb + 64 + 8 * kk, al = tb + 96 + 8 * kk;
                mma_ts32(tb, a, b, id, kk != 0);
                mma_ts32(tb, a, bl, id, 1);
                mma_ts32(tb, al, b, id, 1);
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
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tb, 128); }
}

int main() {
    const int M = 128, N = 64, K = 32;
    static float hA[M * K], hB[N * K], hD[M * N];
    float *dA, *dB, *dD;
    cudaMalloc(&dA, sizeof(hA));
    cudaMalloc(&dB, sizeof(hB));
    cudaMalloc(&dD, sizeof(hD));
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    unsigned s = 777;
    auto rnd = [&]() { s = s * 1664525u + 1013904223u; return ((s >> 8) & 0xFFFFFF) / 16777216.0 * 2 - 1; };
    for (int i = 0; i < M * K; ++i) hA[i] = (float)rnd();
    for (int i = 0; i < N * K; ++i) hB[i] = (float)rnd();
    cudaMemcpy(dA, hA, sizeof(hA), cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB, sizeof(hB), cudaMemcpyHostToDevice);
    const uint32_t LB[7] = {16, 16, 4096, 16, 4096, 1024, 4096};
    const uint32_t SB[7] = {1024, 1024, 1024, 1024, 1024, 4096, 4096};
    for (int m7 = 0; m7 < 7; ++m7) {
        const int mode = m7 < 5 ? m7 : 2;
        cudaMemset(dD, 0, sizeof(hD));
        kern<<<1, 128, 64 * 1024>>>(dA, dB, dD, mode, LB[m7], SB[m7]);
        cudaError_t e = cudaDeviceSynchronize();
        cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
        double maxe = 0, maxr = 0;
        for (int m = 0; m < M; ++m)
            for (int n = 0; n < N; ++n) {
                double r = 0;
                for (int k = 0; k < K; ++k) r += (double)hA[m * K + k] * hB[n * K + k];
                maxe = fmax(maxe, fabs(hD[m * N + n] - r));
                maxr = fmax(maxr, fabs(r));
            }
        double e32 = 0;   // columns 0..31 only (first MN group)
        for (int m = 0; m < M; ++m)
            for (int n = 0; n < 32; ++n) {
                double r = 0;
                for (int k = 0; k < K; ++k) r += (double)hA[m * K + k] * hB[n * K + k];
                e32 = fmax(e32, fabs(hD[m * N + n] - r));
            }
        printf("mode %d lbo %u sbo %u (%s): max abs err %.3e (cols 0-31: %.3e) (max |ref| %.3f)  D[0][0..3] = %g %g %g %g\n",
               mode, LB[m7], SB[m7], cudaGetErrorString(e), maxe, e32, maxr, hD[0], hD[1], hD[2], hD[3]);
        if (e != cudaSuccess) return 1;
    }
    return 0;
}
