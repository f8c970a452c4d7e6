// tools/mma_major_bench.cu -- cycles per tcgen05.mma (kind::f16, cta_group::1, M=128, K=16) for
// K-major vs MN-major SW128 smem operands (profiling aid for csrc/tc_narrow_fused.cu, whose
// dK/dV products take both operands MN-major).  One CTA per SM, one issuing thread, a chain of
// NMMA MMAs into one accumulator, timed from the first issue to the commit's mbarrier.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//        -I paper_conf_pldi_tangzwjzyz22_b200/csrc tools/mma_major_bench.cu -o /tmp/mmb && /tmp/mmb
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "tc_common.cuh"

using namespace ftw::tc;

constexpr int NMMA = 512;

// A: 32 KB region (two 16 KB halves), B: 16 KB.  Per step: K-major advances 32 B within the
// 128-B row (+2), MN-major advances 2 K-row groups (2048 B, +128).
template <int N, bool AMN, bool BMN>
__global__ void bench(unsigned long long* out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t holder;
    __shared__ uint64_t bar;
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    for (int i = threadIdx.x; i < 96 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0x3C003C00u;
    if (warp == 0) { tmem_alloc(&holder, 512); tmem_relinquish(); }
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tb = holder;
    if (warp == 1 && lane == 0) {
        const uint32_t sa = smem_u32(smem), sb = sa + 32768;
        constexpr uint32_t id = idesc_f16(128, N, AMN, BMN);
        const uint64_t ad = AMN ? sdesc_sw128(sa, 16384, 1024) : sdesc_sw128(sa, 16, 1024);
        const uint64_t bd = BMN ? sdesc_sw128(sb, 8192, 1024) : sdesc_sw128(sb, 16, 1024);
        const unsigned long long t0 = clock64();
        for (int it = 0; it < NMMA / 4; ++it) {
            if (AMN && BMN) mma_ss_x4<128, 128>(tb, ad, bd, id, it > 0);
            else if (AMN) mma_ss_x4<128, 2>(tb, ad, bd, id, it > 0);
            else if (BMN) mma_ss_x4<2, 128>(tb, ad, bd, id, it > 0);
            else mma_ss_x4<2, 2>(tb, ad, bd, id, it > 0);
        }
        mma_commit(&bar);
        mbar_wait(&bar, 0);
        const unsigned long long t1 = clock64();
        if (blockIdx.x == 0) out[0] = t1 - t0;
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tb, 512); }
}

template <int N, bool AMN, bool BMN>
void run(const char* name) {
    unsigned long long* d;
    cudaMalloc(&d, 8);
    auto k = bench<N, AMN, BMN>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    k<<<148, 128, 100 * 1024>>>(d);
    k<<<148, 128, 100 * 1024>>>(d);
    unsigned long long h = 0;
    cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
    printf("%-28s N=%3d  %6.1f clk/MMA  (%s)\n", name, N, (double)h / NMMA, cudaGetErrorString(cudaGetLastError()));
    cudaFree(d);
}

int main() {
    run<64, false, false>("A K-major,  B K-major");
    run<64, false, true>("A K-major,  B MN-major");
    run<64, true, false>("A MN-major, B K-major");
    run<64, true, true>("A MN-major, B MN-major");
    run<128, false, false>("A K-major,  B K-major");
    run<128, true, true>("A MN-major, B MN-major");
    run<192, false, false>("A K-major,  B K-major");
    return 0;
}
