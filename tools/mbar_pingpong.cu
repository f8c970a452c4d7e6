// tools/mbar_pingpong.cu -- round-trip latency of an mbarrier handoff between two warps
// (warp 0 arrives on A, warp 1 waits A then arrives on B, warp 0 waits B) with three wait
// flavours: try_wait (no hint), try_wait with a 10 ms suspend hint, test_wait spin.
// Also: tcgen05.commit -> mbarrier -> waiter latency with no MMA in flight.  Profiling aid.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define FT_MBAR_SUSPEND_NS 0
#include "tc_common.cuh"
using namespace ftw::tc;
__device__ __forceinline__ bool tw_hint(uint64_t* bar, uint32_t par) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(par), "r"(10000000u) : "memory");
    return ok;
}
__device__ __forceinline__ bool tw_plain(uint64_t* bar, uint32_t par) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(par) : "memory");
    return ok;
}
__device__ __forceinline__ bool test_w(uint64_t* bar, uint32_t par) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(par) : "memory");
    return ok;
}
template <int MODE>
__device__ __forceinline__ void wt(uint64_t* bar, uint32_t par) {
    if (MODE == 0) while (!tw_plain(bar, par)) {}
    else if (MODE == 1) while (!tw_hint(bar, par)) {}
    else while (!test_w(bar, par)) {}
}
template <int MODE>
__global__ void pingpong(int iters, unsigned long long* out) {
    __shared__ uint64_t A, B;
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (threadIdx.x == 0) { mbar_init(&A, 1); mbar_init(&B, 1); fence_barrier_init(); }
    __syncthreads();
    unsigned long long t0 = clock64();
    if (lane == 0) {
        if (warp == 0) {
            for (int i = 0; i < iters; ++i) { mbar_arrive(&A); wt<MODE>(&B, i & 1); }
        } else if (warp == 1) {
            for (int i = 0; i < iters; ++i) { wt<MODE>(&A, i & 1); mbar_arrive(&B); }
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) out[blockIdx.x] = (clock64() - t0) / iters;
}
// warp 0 lane 0: tcgen05.commit -> A (no MMA); warp 1 waits A then arrives B; warp 0 waits B
template <int MODE>
__global__ void commitpong(int iters, unsigned long long* out) {
    __shared__ uint64_t A, B;
    __shared__ uint32_t holder;
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (warp == 0) { tmem_alloc(&holder, 32); tmem_relinquish(); }
    if (threadIdx.x == 32) { mbar_init(&A, 1); mbar_init(&B, 1); fence_barrier_init(); }
    tc_fence_before(); __syncthreads(); tc_fence_after();
    unsigned long long t0 = clock64();
    if (lane == 0) {
        if (warp == 0) {
            for (int i = 0; i < iters; ++i) { mma_commit(&A); wt<MODE>(&B, i & 1); }
        } else if (warp == 1) {
            for (int i = 0; i < iters; ++i) { wt<MODE>(&A, i & 1); mbar_arrive(&B); }
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) out[blockIdx.x] = (clock64() - t0) / iters;
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(holder, 32); }
}
int main() {
    unsigned long long* d; cudaMalloc(&d, 8 * 148);
    unsigned long long h[148];
    const char* names[3] = {"try_wait (no hint)", "try_wait (10ms hint)", "test_wait spin"};
    for (int m = 0; m < 3; ++m) {
        if (m == 0) pingpong<0><<<148, 64>>>(20000, d);
        if (m == 1) pingpong<1><<<148, 64>>>(20000, d);
        if (m == 2) pingpong<2><<<148, 64>>>(20000, d);
        cudaDeviceSynchronize();
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        printf("arrive->wait round trip, %-22s: %llu clk\n", names[m], h[0]);
    }
    for (int m = 0; m < 3; ++m) {
        if (m == 0) commitpong<0><<<148, 64>>>(20000, d);
        if (m == 1) commitpong<1><<<148, 64>>>(20000, d);
        if (m == 2) commitpong<2><<<148, 64>>>(20000, d);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        printf("tcgen05.commit->wait->arrive->wait, %-22s: %llu clk\n", names[m], h[0]);
    }
    return 0;
}
