// tools/mma_microbench.cu -- cycles per tcgen05.mma (kind::f16, M=128, K=16) for the operand
// shapes the band kernels use.  Profiling aid, not part of the library.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_pldi_tangzwjzyz22_b200/csrc \
//        tools/mma_microbench.cu -o /tmp/mma_mb && /tmp/mma_mb
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "tc_common.cuh"

using namespace ftw::tc;
__device__ __forceinline__ uint32_t elect_one() {
    uint32_t e;
    asm volatile("{\n\t.reg .pred p;\n\telect.sync _|p, 0xffffffff;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(e));
    return e;
}


// whole-warp variants: all 32 lanes execute, one elected lane issues
__device__ __forceinline__ void mma_ss_w(uint32_t d, uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p, e;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
                 :: "r"(d), "l"(a), "l"(b), "r"(id), "r"(acc) : "memory");
}
__device__ __forceinline__ void mma_ts_w(uint32_t d, uint32_t a, uint64_t b, uint32_t id, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p, e;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}"
                 :: "r"(d), "r"(a), "l"(b), "r"(id), "r"(acc) : "memory");
}
__device__ __forceinline__ void commit_w(uint64_t* bar) {
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
                 "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}"
                 :: "r"(smem_u32(bar)) : "memory");
}

__global__ void bench_w(int mode, int N, int nacc, int iters, unsigned long long* out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t holder;
    __shared__ uint64_t bar;
    const int warp = threadIdx.x / 32;
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0;
    if (warp == 0) { tmem_alloc(&holder, 512); tmem_relinquish(); }
    if (threadIdx.x == 32) { mbar_init(&bar, 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tb = holder;
    if (warp == 1) {
        const uint32_t sa = smem_u32(smem), sb = sa + 16384;
        const uint32_t id = idesc_bf16(128, N, false, mode == 1);
        for (int i = 0; i < 16; ++i)
            for (int a = 0; a < nacc; ++a) {
                const uint32_t d = mode == 0 ? tb + (nacc > 2 ? 128 : 256) * a : tb + 128 + 128 * a;
                if (mode == 0) mma_ss_w(d, sdesc_sw128(sa, 16, 1024), sdesc_sw128(sb, 16, 1024), id, 1);
                else mma_ts_w(d, tb, sdesc_sw128(sb, 8192, 1024), id, 1);
            }
        commit_w(&bar);
        mbar_wait(&bar, 0);
        unsigned long long t0 = clock64();
        for (int i = 0; i < iters; ++i)
            for (int a = 0; a < nacc; ++a) {
                const uint32_t d = mode == 0 ? tb + (nacc > 2 ? 128 : 256) * a : tb + 128 + 128 * a;
                const int kk = i & 3;
                if (mode == 0)
                    mma_ss_w(d, sdesc_sw128(sa + kk * 32, 16, 1024), sdesc_sw128(sb + kk * 32, 16, 1024), id, 1);
                else
                    mma_ts_w(d, tb + kk * 8, sdesc_sw128(sb + kk * 2048, 8192, 1024), id, 1);
            }
        commit_w(&bar);
        mbar_wait(&bar, 1);
        unsigned long long t1 = clock64();
        if (threadIdx.x == 32) out[blockIdx.x] = t1 - t0;
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tb, 512); }
}

// mode 0: SS (A K-major smem, B K-major smem), mode 1: TS (A tmem, B MN-major smem)
__global__ void bench(int mode, int N, int nacc, int iters, unsigned long long* out, int M = 128) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t holder;
    __shared__ uint64_t bar;
    const int warp = threadIdx.x / 32;
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0;
    if (warp == 0) { tmem_alloc(&holder, 512); tmem_relinquish(); }
    if (threadIdx.x == 32) { mbar_init(&bar, 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tb = holder;
    if (threadIdx.x == 32) {
        const uint32_t sa = smem_u32(smem), sb = sa + 16384;
        const uint32_t id = idesc_bf16(M, N, false, mode == 1);
        // warm up
        for (int i = 0; i < 16; ++i)
            for (int a = 0; a < nacc; ++a) {
                const uint32_t d = mode == 0 ? tb + (nacc > 2 ? 128 : 256) * a : tb + 128 + 128 * a;
                if (mode == 0) mma_ss(d, sdesc_sw128(sa, 16, 1024), sdesc_sw128(sb, 16, 1024), id, 1);
                else mma_ts(d, tb, sdesc_sw128(sb, 8192, 1024), id, 1);
            }
        mma_commit(&bar);
        mbar_wait(&bar, 0);
        unsigned long long t0 = clock64();
        for (int i = 0; i < iters; ++i)
            for (int a = 0; a < nacc; ++a) {
                const uint32_t d = mode == 0 ? tb + (nacc > 2 ? 128 : 256) * a : tb + 128 + 128 * a;
                const int kk = i & 3;
                if (mode == 0)
                    mma_ss(d, sdesc_sw128(sa + kk * 32, 16, 1024), sdesc_sw128(sb + kk * 32, 16, 1024), id, 1);
                else
                    mma_ts(d, tb + kk * 8, sdesc_sw128(sb + kk * 2048, 8192, 1024), id, 1);
            }
        mma_commit(&bar);
        mbar_wait(&bar, 1);
        unsigned long long t1 = clock64();
        out[blockIdx.x] = t1 - t0;
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tb, 512); }
}

template <bool WW>
__global__ void bench_multi_t(int N, int nacc, int issuers, int iters, unsigned long long* out, int wstride = 1) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t holder;
    __shared__ uint64_t bar[4];
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0;
    if (warp == 0) { tmem_alloc(&holder, 512); tmem_relinquish(); }
    if (threadIdx.x == 0) { for (int i = 0; i < 4; ++i) mbar_init(&bar[i], 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tb = holder;
    unsigned long long t0 = clock64();
    if (warp % wstride == 0 && warp / wstride < issuers && (WW || lane == 0)) {
        const uint32_t sa = smem_u32(smem), sb = sa + 16384;
        const uint32_t id = idesc_bf16(128, N, false, false);
        for (int i = 0; i < iters; ++i)
            for (int a = 0; a < nacc; ++a) {
                const uint32_t d = tb + (uint32_t)(((warp / wstride) * nacc + a) * N);
                const int kk = i & 3;
                if (WW) { if (elect_one()) mma_ss(d, sdesc_sw128(sa + kk * 32, 16, 1024), sdesc_sw128(sb + kk * 32, 16, 1024), id, 1); }
                else mma_ss(d, sdesc_sw128(sa + kk * 32, 16, 1024), sdesc_sw128(sb + kk * 32, 16, 1024), id, 1);
            }
        if (WW) { if (elect_one()) mma_commit(&bar[warp / wstride]); }
        else mma_commit(&bar[warp / wstride]);
        mbar_wait(&bar[warp / wstride], 0);
    }
    __syncthreads();
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
    tc_fence_before();
    __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tb, 512); }
}

// Whole-warp issuer: all 32 lanes run the loop (descriptors warp-uniform, so they can
// live in uniform registers); one elected lane issues each MMA (elect.sync).
__device__ __forceinline__ void mma_ss_elect(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                             uint32_t idesc, uint32_t accumulate) {
    if (elect_one()) mma_ss(d_tmem, adesc, bdesc, idesc, accumulate);
}
__device__ __forceinline__ void commit_elect(uint64_t* bar) {
    if (elect_one()) mma_commit(bar);
}
__global__ void bench_warp(int N, int nacc, int iters, unsigned long long* out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t holder;
    __shared__ uint64_t bar;
    const int warp = threadIdx.x / 32;
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0;
    if (warp == 0) { tmem_alloc(&holder, 512); tmem_relinquish(); }
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tb = holder;
    unsigned long long t0 = clock64();
    if (warp == 1) {   // whole warp
        const uint32_t sa = smem_u32(smem), sb = sa + 16384;
        const uint32_t id = idesc_bf16(128, N, false, false);
        for (int i = 0; i < iters; ++i)
            for (int a = 0; a < nacc; ++a) {
                const int kk = i & 3;
                mma_ss_elect(tb + (uint32_t)(a * N), sdesc_sw128(sa + kk * 32, 16, 1024), sdesc_sw128(sb + kk * 32, 16, 1024), id, 1);
            }
        commit_elect(&bar);
        mbar_wait(&bar, 0);
    }
    __syncthreads();
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
    tc_fence_before();
    __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tb, 512); }
}

int main() {
    {
        unsigned long long* dd;
        cudaMalloc(&dd, 8 * 148);
        cudaFuncSetAttribute(bench_warp, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
        const int iters = 2048;
        for (int rep = 0; rep < 2; ++rep)
        for (int nacc : {1, 2, 4}) for (int N : {64, 128}) {
            bench_warp<<<148, 128, 96 * 1024>>>(N, nacc, iters, dd);
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) { printf("launch err %s\n", cudaGetErrorString(e)); return 1; }
            e = cudaDeviceSynchronize();
            if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
            unsigned long long h[148] = {0};
            cudaMemcpy(h, dd, 8 * 148, cudaMemcpyDeviceToHost);
            double mx = 0;
            for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
            printf("whole-warp issuer (elect.sync) N=%3d chains=%d: %6.1f clk/MMA\n", N, nacc, mx / ((double)iters * nacc));
        }
    }

    {
        unsigned long long* dd;
        cudaMalloc(&dd, 8 * 148);
        cudaFuncSetAttribute(bench_multi_t<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
        const int iters = 2048;
        struct M { int N, nacc, issuers; };
        cudaFuncSetAttribute(bench_multi_t<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
        for (M m : {M{128, 1, 1}, M{128, 2, 1}, M{128, 4, 1}, M{64, 2, 1}, M{128, 2, 2}}) {
            bench_multi_t<true><<<148, 128, 96 * 1024>>>(m.N, m.nacc, m.issuers, iters, dd);
            cudaDeviceSynchronize();
            unsigned long long h[148] = {0};
            cudaMemcpy(h, dd, 8 * 148, cudaMemcpyDeviceToHost);
            double mx = 0;
            for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
            const double total = (double)iters * m.nacc * m.issuers;
            printf("WHOLE-WARP issuer N=%3d chains/issuer=%d issuers=%d: %6.1f clk/MMA per issuer\n",
                   m.N, m.nacc, m.issuers, mx / (total / m.issuers));
        }
        for (int rep = 0; rep < 1; ++rep)
        for (M m : {M{128, 1, 1}, M{128, 2, 1}, M{128, 4, 1}, M{128, 1, 2}, M{128, 2, 2}, M{128, 1, 3},
                    M{256, 1, 1}, M{256, 1, 2}, M{256, 2, 2}, M{64, 1, 1}, M{64, 1, 2}, M{64, 1, 4}}) {
            bench_multi_t<false><<<148, 128, 96 * 1024>>>(m.N, m.nacc, m.issuers, iters, dd);
            unsigned long long h[148] = {0};
            cudaMemcpy(h, dd, 8 * 148, cudaMemcpyDeviceToHost);
            double mx = 0;
            for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
            const double total = (double)iters * m.nacc * m.issuers;
            printf("multi-issuer SS M=128 N=%3d chains/issuer=%d issuers=%d: %6.1f clk/MMA per issuer, %5.0f MAC/clk/SM\n",
                   m.N, m.nacc, m.issuers, mx / (total / m.issuers), 128.0 * m.N * 16 * total / mx);
        }
        for (M m : {M{64, 2, 2}, M{128, 2, 2}}) {   // issuers on warps 0 and 4: same SM sub-partition
            bench_multi_t<false><<<148, 256, 96 * 1024>>>(m.N, m.nacc, m.issuers, iters, dd, 4);
            unsigned long long h[148] = {0};
            cudaMemcpy(h, dd, 8 * 148, cudaMemcpyDeviceToHost);
            double mx = 0;
            for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
            const double total = (double)iters * m.nacc * m.issuers;
            printf("multi-issuer same-SMSP N=%3d acc/issuer=%d issuers=%d: %6.1f clk per MMA, %5.0f MAC/clk/SM\n",
                   m.N, m.nacc, m.issuers, mx / total, 128.0 * m.N * 16 * total / mx);
        }
    }

    unsigned long long* d;
    cudaMalloc(&d, 8 * 148);
    cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    cudaFuncSetAttribute(bench_w, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    const int iters = 2048;
    for (int N : {64, 128, 256})
        for (int nacc : {1, 2, 4}) {
            if (N == 256 && nacc == 4) continue;
            bench<<<148, 128, 96 * 1024>>>(0, N, nacc, iters, d, 64);
            unsigned long long h[148] = {0};
            cudaMemcpy(h, d, 8 * 148, cudaMemcpyDeviceToHost);
            double mx = 0;
            for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
            const double per = mx / (iters * nacc);
            printf("lane0 SS M= 64 N=%3d acc=%d grid=148: %6.1f clk/MMA  %5.0f MAC/clk/SM\n", N, nacc, per,
                   64.0 * N * 16 / per);
        }
    struct Cfg { int variant, mode, N, nacc, grid; };
    Cfg cfgs[] = {
        {0, 0, 64, 1, 1}, {0, 0, 64, 4, 1}, {0, 0, 128, 1, 1}, {0, 0, 128, 4, 1},
        {0, 0, 256, 1, 1}, {0, 0, 256, 1, 148}, {0, 0, 128, 4, 148}, {0, 0, 64, 4, 148},
        {1, 0, 256, 1, 148}, {1, 0, 128, 4, 148}, {0, 1, 64, 2, 148}, {0, 1, 128, 2, 148},
        {0, 1, 256, 1, 148},
    };
    for (const Cfg& c : cfgs) {
        if (c.variant == 0) bench<<<c.grid, 128, 96 * 1024>>>(c.mode, c.N, c.nacc, iters, d);
        else bench_w<<<c.grid, 128, 96 * 1024>>>(c.mode, c.N, c.nacc, iters, d);
        unsigned long long h[148] = {0};
        cudaError_t e = cudaMemcpy(h, d, 8 * c.grid, cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        double mx = 0;
        for (int i = 0; i < c.grid; ++i) mx = h[i] > mx ? h[i] : mx;
        const double per = mx / (iters * c.nacc);
        printf("%s %s M=128 N=%3d acc=%d grid=%3d: %6.1f clk/MMA (floor %3d) %5.0f MAC/clk/SM\n",
               c.variant == 0 ? "lane0" : "warp ", c.mode == 0 ? "SS" : "TS", c.N, c.nacc, c.grid,
               per, 128 * c.N / 256, 128.0 * c.N * 16 / per);
    }
    return 0;
}
