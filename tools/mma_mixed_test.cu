// tools/mma_mixed_test.cu -- does tcgen05.mma kind::f16 accept A = fp16 with B = bf16?
// D[128 x 64] = A[128 x 16] * B[64 x 16]^T, both K-major SWIZZLE_128B in smem; compares
// against a host fp64 product.  Profiling/feasibility aid, not part of the library.
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>

#include "tc_common.cuh"

using namespace ftw::tc;

__global__ void kern(const uint16_t* A, const uint16_t* B, float* D, uint32_t idesc) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t holder;
    __shared__ uint64_t bar;
    const int t = threadIdx.x, warp = t / 32;
    // SW128 K-major: row r at r*128, 16-byte chunk c at ((c ^ (r & 7)) * 16); K = 16 -> chunks 0,1
    for (int i = t; i < 128 * 16; i += blockDim.x) {
        const int r = i / 16, k = i % 16, c = k / 8, e = k % 8;
        *reinterpret_cast<uint16_t*>(smem + r * 128 + ((c ^ (r & 7)) * 16) + e * 2) = A[i];
    }
    for (int i = t; i < 64 * 16; i += blockDim.x) {
        const int r = i / 16, k = i % 16, c = k / 8, e = k % 8;
        *reinterpret_cast<uint16_t*>(smem + 16384 + r * 128 + ((c ^ (r & 7)) * 16) + e * 2) = B[i];
    }
    if (warp == 0) { tmem_alloc(&holder, 64); tmem_relinquish(); }
    if (t == 32) { mbar_init(&bar, 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tb = holder;
    if (t == 32) {
        mma_ss(tb, sdesc_sw128(smem_u32(smem), 16, 1024), sdesc_sw128(smem_u32(smem + 16384), 16, 1024), idesc, 0);
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
    const int M = 128, N = 64, K = 16;
    uint16_t hA[M * K], hB[N * K];
    double a[M * K], b[N * K];
    unsigned s = 12345;
    auto rnd = [&]() { s = s * 1664525u + 1013904223u; return ((s >> 8) & 0xFFFF) / 65536.0 * 2 - 1; };
    for (int i = 0; i < M * K; ++i) {
        const double x = rnd() * 37.0;                     // fp16 A with large magnitude
        __half h = __double2half(x);
        hA[i] = *reinterpret_cast<uint16_t*>(&h);
        a[i] = __half2float(h);
    }
    for (int i = 0; i < N * K; ++i) {
        const double x = rnd();
        __nv_bfloat16 h = __double2bfloat16(x);
        hB[i] = *reinterpret_cast<uint16_t*>(&h);
        b[i] = __bfloat162float(h);
    }
    uint16_t *dA, *dB;
    float* dD;
    cudaMalloc(&dA, sizeof(hA));
    cudaMalloc(&dB, sizeof(hB));
    cudaMalloc(&dD, M * N * 4);
    cudaMemcpy(dA, hA, sizeof(hA), cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB, sizeof(hB), cudaMemcpyHostToDevice);
    // a_format = 0 (F16), b_format = 1 (BF16), D = F32
    for (int variant = 0; variant < 2; ++variant) {
        uint32_t idesc = idesc_bf16(128, 64, false, false);
        if (variant == 1) idesc &= ~(7u << 7);   // a_format = F16
        cudaMemset(dD, 0, M * N * 4);
        kern<<<1, 128, 40 * 1024>>>(dA, dB, dD, idesc);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("variant %d: error %s\n", variant, cudaGetErrorString(e)); return 1; }
        static float hD[M * N];
        cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
        double maxerr = 0, maxref = 0;
        for (int i = 0; i < M; ++i)
            for (int j = 0; j < N; ++j) {
                double ref = 0;
                for (int k = 0; k < K; ++k) ref += a[i * K + k] * b[j * K + k];
                maxerr = fmax(maxerr, fabs(ref - hD[i * N + j]));
                maxref = fmax(maxref, fabs(ref));
            }
        printf("variant %s: max |err| %.3e, max |ref| %.3e\n",
               variant == 0 ? "A read as bf16 (expect garbage)" : "A=f16 B=bf16", maxerr, maxref);
    }
    return 0;
}
