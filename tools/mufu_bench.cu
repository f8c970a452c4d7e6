// tools/mufu_bench.cu -- MUFU.EX2 (ex2.approx.ftz.f32) throughput per SM on this GPU, with
// 1 / 2 / 4 warps per SM sub-partition.  Profiling aid, not part of the library.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void kern(int nwarps, int iters, float* out, unsigned long long* cyc) {
    const int warp = threadIdx.x / 32;
    float x[8];
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x * 1e-3f + i * 1e-4f;
    __syncthreads();
    unsigned long long t0 = clock64();
    if (warp < nwarps) {
        for (int it = 0; it < iters; ++it) {
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                float y;
                asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x[i]));
                x[i] = y * -0.5f;
            }
        }
    }
    __syncthreads();
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    float s = 0.f;
    for (int i = 0; i < 8; ++i) s += x[i];
    if (s == 1234.5f) out[0] = s;
}
int main() {
    float* o; unsigned long long* c;
    cudaMalloc(&o, 4); cudaMalloc(&c, 8 * 148);
    const int iters = 4096;
    for (int nw : {4, 8, 16}) {
        kern<<<148, 512>>>(nw, iters, o, c);
        cudaDeviceSynchronize();
        unsigned long long h[148];
        cudaMemcpy(h, c, sizeof(h), cudaMemcpyDeviceToHost);
        double mx = 0; for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
        const double ex = (double)nw * 32 * iters * 8;
        printf("ex2.approx: %2d warps/SM: %.2f ex2 per clk per SM (%.1f clk per warp-instruction per SMSP)\n",
               nw, ex / mx, mx / ((double)nw / 4 * iters * 8));
    }
    return 0;
}
