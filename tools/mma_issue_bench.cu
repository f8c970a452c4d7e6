// tools/mma_issue_bench.cu -- cycles per tcgen05.mma (kind::f16, cta_group::1, K=16) when the
// issue loop is fully unrolled and warp-uniform (descriptors are compile-time offsets from a
// uniform base, so they live in uniform registers and no R2UR waterfall loop is emitted).
// Compares against the lane-0-only issue style.  Profiling aid, not part of the library.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//        -I paper_conf_pldi_tangzwjzyz22_b200/csrc tools/mma_issue_bench.cu -o /tmp/mib && /tmp/mib
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "tc_common.cuh"

using namespace ftw::tc;

__device__ __forceinline__ void mma_ss_el(uint32_t d, uint64_t a, uint64_t b, uint32_t id, int acc) {
    asm volatile("{\n\t.reg .pred p, e;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
                 :: "r"(d), "l"(a), "l"(b), "r"(id), "r"(acc) : "memory");
}
__device__ __forceinline__ void commit_el(uint64_t* bar) {
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
                 "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}"
                 :: "r"(smem_u32(bar)) : "memory");
}

// Four K=16 MMAs (one 64-wide K slice of SW128 K-major operands) in one asm block: the
// descriptors of steps 1-3 are formed inside the asm (+32 B start address = +2 in the
// descriptor), so each MMA gets its own registers.
__device__ __forceinline__ void mma_ss_x4(uint32_t d, uint64_t a, uint64_t b, uint32_t id, int acc) {
    asm volatile("{\n\t.reg .pred p;\n\t.reg .b64 a1, a2, a3, b1, b2, b3;\n\t"
                 "setp.ne.b32 p, %4, 0;\n\t"
                 "add.s64 a1, %1, 2;\n\tadd.s64 a2, %1, 4;\n\tadd.s64 a3, %1, 6;\n\t"
                 "add.s64 b1, %2, 2;\n\tadd.s64 b2, %2, 4;\n\tadd.s64 b3, %2, 6;\n\t"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], a1, b1, %3, 1;\n\t"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], a2, b2, %3, 1;\n\t"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], a3, b3, %3, 1;\n\t}"
                 :: "r"(d), "l"(a), "l"(b), "r"(id), "r"(acc) : "memory");
}

// STYLE 0: whole warp, elect inside asm.  STYLE 1: lane 0 only.  STYLE 2: lane 0, runtime
// (non-unrolled) descriptor arithmetic per MMA, as in the library's issue loops.  STYLE 3:
// lane 0, non-unrolled loop over 64-wide K slices, 4 MMAs per asm block (mma_ss_x4).
template <int N, int NACC, int STYLE, int M = 128>
__global__ void bench(int outer, unsigned long long* out, float* val) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t holder;
    __shared__ uint64_t bar;
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    for (int i = threadIdx.x; i < 96 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0x3F803F80u;   // bf16 1.0 pairs
    if (warp == 0) { tmem_alloc(&holder, 512); tmem_relinquish(); }
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tb = holder;
    if (warp == 1 && (STYLE == 0 || lane == 0)) {
        const unsigned long long t0 = clock64();
        const uint32_t sa = smem_u32(smem), sb = sa + 32768;
        constexpr uint32_t id = idesc_bf16(M, N, false, false);
        const uint64_t da = sdesc_sw128(sa, 16, 1024), db = sdesc_sw128(sb, 16, 1024);
        if (STYLE == 2) {
#pragma unroll 1
            for (int i = 0; i < outer * 16; ++i) {
                const int kk = i & 15;
                mma_ss(tb + (i % NACC) * N, sdesc_sw128(sa + (kk & 3) * 32 + (kk >> 2) * 8192, 16, 1024),
                       sdesc_sw128(sb + (kk & 3) * 32 + (kk >> 2) * 8192, 16, 1024), id, i != 0);
            }
        } else if (STYLE == 3) {
#pragma unroll 1
            for (int i = 0; i < outer * 4; ++i) {
                const int ks = i & 3;
                mma_ss_x4(tb + (i % NACC) * N, sdesc_sw128(sa + ks * 8192, 16, 1024),
                          sdesc_sw128(sb + ks * 8192, 16, 1024), id, i != 0);
            }
        } else if (STYLE == 4) {   // TS: A from TMEM (cols 256..), B MN-major (LBO 8192)
            constexpr uint32_t idT = idesc_bf16(M, N, false, true);
#pragma unroll 1
            for (int i = 0; i < outer * 4; ++i) {
                const int ks = i & 3;
                mma_ts_x4<8, 128>(tb + (i % NACC) * N, tb + 256 + 32 * ks, sdesc_sw128(sb + ks * 8192, 8192, 1024), idT, i != 0);
            }
        } else if (STYLE == 5) {   // latency: 4 SS MMAs + commit + wait, repeated
#pragma unroll 1
            for (int i = 0; i < outer; ++i) {
                mma_ss_x4<2, 2>(tb, da, db, id, 0);
                mma_commit(&bar);
                mbar_wait(&bar, i & 1);
            }
        } else
        for (int o = 0; o < outer; ++o) {
#pragma unroll
            for (int kk = 0; kk < 16; ++kk)
#pragma unroll
                for (int a = 0; a < NACC; ++a) {
                    const uint64_t off = (uint64_t)(((kk & 3) * 32 + (kk >> 2) * 8192) >> 4);
                    const int acc = (o | kk) != 0;
                    if (STYLE == 0) mma_ss_el(tb + a * N, da + off, db + off, id, acc);
                    else mma_ss(tb + a * N, da + off, db + off, id, acc);
                }
        }
        if (STYLE != 5) {
            if (STYLE == 0) commit_el(&bar); else mma_commit(&bar);
            mbar_wait(&bar, 0);
        }
        const unsigned long long t1 = clock64();
        if (lane == 0) out[blockIdx.x] = t1 - t0;   // the issuing thread times itself
    }
    __syncthreads();
    tc_fence_after();
    if (warp == 0) {   // accumulator check: every element = 16 * 16 * outer
        uint32_t r[32];
        tmem_ld32(tb, r);
        tmem_wait_ld();
        if (lane == 0 && blockIdx.x == 0) *val = __uint_as_float(r[0]);
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tb, 512); }
}

static float* g_val;
template <int N, int NACC, int STYLE, int M = 128>
void run(unsigned long long* d) {
    auto k = bench<N, NACC, STYLE, M>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    const int outer = 128;
    for (int rep = 0; rep < 2; ++rep) {
        cudaMemset(d, 0, 8 * 148);
        k<<<148, 128, 96 * 1024>>>(outer, d, g_val);
        cudaError_t e = cudaGetLastError();
        if (e == cudaSuccess) e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return; }
        unsigned long long h[148];
        float v = 0;
        cudaMemcpy(&v, g_val, 4, cudaMemcpyDeviceToHost);
        if (rep == 1) printf("acc[0]=%.0f (expect %d) ", v, 16 * 16 * outer);
        cudaMemcpy(h, d, 8 * 148, cudaMemcpyDeviceToHost);
        double mx = 0;
        for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
        const double n = STYLE == 5 ? (double)outer : (double)outer * 16 * (STYLE >= 2 ? 1 : NACC);
        if (rep == 1)
            printf("[h0=%llu] %s M=%d N=%3d chains=%d: %6.1f clk/MMA  %6.0f MAC/clk/SM\n", h[0],
                   STYLE == 0 ? "warp+elect" : STYLE == 1 ? "lane0     " : STYLE == 2 ? "lane0-rt  " : STYLE == 3 ? "lane0-x4  " : STYLE == 4 ? "TS-x4     " : "lat4+cmt  ", M, N, NACC, mx / n, (double)M * N * 16 * n / mx);
    }
}

int main() {
    unsigned long long* d;
    cudaMalloc(&d, 8 * 148);
    cudaMalloc(&g_val, 4);
    run<64, 1, 0>(d); run<128, 1, 0>(d); run<256, 1, 0>(d); run<192, 1, 0>(d);
    run<64, 1, 3>(d); run<128, 1, 3>(d); run<192, 1, 3>(d);
    run<64, 1, 4>(d); run<128, 1, 4>(d); run<64, 2, 4>(d);
    run<192, 1, 5>(d); run<64, 1, 5>(d);
    return 0;
}
