// tools/bwd_step_bench.cu -- the wide-window dQ kernel's second-pass softmax step in isolation:
// per warp, tcgen05.ld of 32 S and 32 dP columns, P = exp2(S - lse), dS = P (dP - D), bf16
// hi/lo split, two tcgen05.st.  8 warps (2 per SM sub-partition), optionally with 8 more
// warps parked in mbarrier try_wait loops (like idle issuers / epilogue).  Profiling aid.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include "tc_common.cuh"
using namespace ftw::tc;
__device__ __forceinline__ float fast_exp2(float x) { float y; asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__device__ __forceinline__ void split_bf16x2(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    __nv_bfloat162 h = __floats2bfloat162_rn(x0, x1);
    const float2 hf = __bfloat1622float2(h);
    hi = *reinterpret_cast<uint32_t*>(&h);
    lo = pack_bf16x2(x0 - hf.x, x1 - hf.y);
}
__global__ void kern(int iters, int spinners, int pass2, unsigned long long* cyc, float* out) {
    __shared__ uint32_t holder;
    __shared__ uint64_t never;
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (warp == 0) { tmem_alloc(&holder, 512); tmem_relinquish(); }
    if (threadIdx.x == 0) { mbar_init(&never, 1); fence_barrier_init(); }
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const uint32_t tb = holder;
    __shared__ volatile int done;
    if (threadIdx.x == 0) done = 0;
    __syncthreads();
    unsigned long long t0 = clock64();
    float D = 0.3f, lse2 = 1.f, acc = 0.f;
    if (warp < 8) {
        const int wq = warp & 3, hf = warp >> 2;
        const uint32_t row = tb + ((uint32_t)(wq * 32) << 16);
        for (int it = 0; it < iters; ++it) {
            const uint32_t xs = row + (uint32_t)((it % 6) * 64 + 32 * hf);
            const uint32_t xd = row + (uint32_t)(((it + 1) % 6) * 64 + 32 * hf);
            uint32_t rs[32], rd[32];
            tmem_ld32(xs, rs);
            tmem_ld32(xd, rd);
            tmem_wait_ld();
            if (pass2) {
                uint32_t ph[16], pl[16];
#pragma unroll
                for (int e = 0; e < 32; e += 2) {
                    const float p0 = fast_exp2(fmaf(__uint_as_float(rs[e]), 1.4426950408889634f, -lse2));
                    const float p1 = fast_exp2(fmaf(__uint_as_float(rs[e + 1]), 1.4426950408889634f, -lse2));
                    split_bf16x2(p0 * (__uint_as_float(rd[e]) - D), p1 * (__uint_as_float(rd[e + 1]) - D), ph[e / 2], pl[e / 2]);
                }
                tmem_st16(xs, ph);
                tmem_st16(xs + 16, pl);
                tmem_wait_st();
            } else {
                float d2[2] = {0.f, 0.f};
#pragma unroll
                for (int e = 0; e < 32; ++e) {
                    const float pv = fast_exp2(fmaf(__uint_as_float(rs[e]), 1.4426950408889634f, -lse2));
                    d2[e & 1] = fmaf(pv, __uint_as_float(rd[e]), d2[e & 1]);
                }
                acc += d2[0] + d2[1];
            }
        }
        if (lane == 0) atomicAdd((int*)&done, 1);
    } else if (warp < 8 + spinners) {
        while (done < 8) { mbar_try_wait(&never, 0); }
    }
    __syncthreads();
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    if (acc == 1234.5f) out[0] = acc;
    tc_fence_before(); __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tb, 512); }
}
int main() {
    unsigned long long* c; float* o;
    cudaMalloc(&c, 8 * 148); cudaMalloc(&o, 4);
    const int iters = 2000;
    for (int pass2 = 0; pass2 < 2; ++pass2)
        for (int sp : {0, 8}) {
            kern<<<148, 512>>>(iters, sp, pass2, c, o);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
            unsigned long long h[148];
            cudaMemcpy(h, c, sizeof(h), cudaMemcpyDeviceToHost);
            double mx = 0; for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
            printf("dQ softmax step (%s), 8 warps, %d spinning warps: %.0f clk per 32-column step per warp\n",
                   pass2 ? "pass 2" : "pass 1", sp, mx / iters);
        }
    return 0;
}
