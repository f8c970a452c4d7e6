// tma_fill_bench.cu -- TMA ring fill rate of the fp32 band kernels' access pattern (profiling aid).
//
// Each persistent CTA walks C2a-shaped tiles (8 units x 10000 rows x 512 fp32, 128-row tiles,
// 192-row halo) slice by slice, like tc_band32.cu's score phase: per ring slot an A box set of
// 128 rows and a B box set of 192 rows covering `cs` columns, loaded with TMA into a ring of
// `ns` slots; one consumer thread waits for each slot, spins `work` clocks (stand-in for the
// conversion and MMAs) and frees it.  Reports the aggregate L2 -> SM rate and the slot period.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_pldi_tangzwjzyz22_b200/csrc \
//        tools/tma_fill_bench.cu -lcuda -o /tmp/tma_fill_bench && /tmp/tma_fill_bench
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include "tc_common.cuh"
#include "tmap.h"

using namespace ftw;
using namespace ftw::tc;

struct P {
    CUtensorMap a, b;
    int bc, cs, ns, work, tiles_per_unit, units, d;
    unsigned slot_bytes;
    unsigned long long* clk;   // per CTA: total clocks
};

__global__ void __launch_bounds__(64, 1) fill_kernel(const __grid_constant__ P p) {
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + p.ns * p.slot_bytes);
    uint64_t* empty = full + 16;
    if (threadIdx.x == 0) {
        for (int i = 0; i < p.ns; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
        fence_barrier_init();
    }
    __syncthreads();
    const int total = p.units * p.tiles_per_unit, nsl = p.d / p.cs, nb = p.cs / p.bc;
    const unsigned long long t0 = clock64();
    if (threadIdx.x == 0) {   // producer
        int st = 0; uint32_t ph = 0;
        for (int tau = blockIdx.x; tau < total; tau += gridDim.x) {
            const int u = tau / p.tiles_per_unit, m0 = (tau % p.tiles_per_unit) * 128;
            for (int s = 0; s < nsl; ++s) {
                mbar_wait(&empty[st], ph ^ 1u);
                uint8_t* sp = smem + (size_t)st * p.slot_bytes;
                mbar_arrive_expect_tx(&full[st], (uint32_t)nb * (128 + 192) * p.bc * 4);
                for (int h = 0; h < nb; ++h) {
                    tma_load_3d(sp + h * 128 * p.bc * 4, &p.a, &full[st], p.cs * s + p.bc * h, m0, u);
                    tma_load_3d(sp + nb * 128 * p.bc * 4 + h * 192 * p.bc * 4, &p.b, &full[st], p.cs * s + p.bc * h, m0 - 32, u);
                }
                if (++st == p.ns) { st = 0; ph ^= 1u; }
            }
        }
    } else if (threadIdx.x == 32) {   // consumer
        int st = 0; uint32_t ph = 0;
        for (int tau = blockIdx.x; tau < total; tau += gridDim.x)
            for (int s = 0; s < nsl; ++s) {
                mbar_wait(&full[st], ph);
                const unsigned long long w0 = clock64();
                while (clock64() - w0 < (unsigned long long)p.work) {}
                mbar_arrive(&empty[st]);
                if (++st == p.ns) { st = 0; ph ^= 1u; }
            }
        p.clk[blockIdx.x] = clock64() - t0;
    }
}

int main(int argc, char** argv) {
    const int U = 8, L = 10000, D = 512;
    float *x, *y;
    cudaMalloc(&x, (size_t)U * L * D * 4);
    cudaMalloc(&y, (size_t)U * L * D * 4);
    cudaMemset(x, 0, (size_t)U * L * D * 4);
    cudaMemset(y, 0, (size_t)U * L * D * 4);
    unsigned long long* clk;
    cudaMalloc(&clk, 1024 * 8);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaFuncSetAttribute(fill_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    struct Cfg { int bc, cs, ns, work, grid; };
    const Cfg cfgs[] = {
        {16, 32, 5, 0, sms}, {32, 32, 5, 0, sms}, {32, 64, 2, 0, sms},
        {16, 32, 5, 1100, sms}, {32, 32, 5, 1100, sms}, {32, 64, 2, 2200, sms},
        {16, 32, 5, 0, sms / 2}, {32, 32, 5, 0, sms / 2}, {16, 32, 5, 0, 16}, {32, 32, 5, 0, 16},
        {16, 32, 3, 0, sms}, {16, 32, 4, 0, sms}, {32, 32, 3, 0, sms}, {32, 32, 4, 0, sms},
    };
    printf("%4s %4s %3s %6s %5s %10s %10s %10s\n", "bc", "cs", "ns", "work", "grid", "us", "GB/s", "clk/slot");
    for (const Cfg& c : cfgs) {
        P p;
        p.bc = c.bc; p.cs = c.cs; p.ns = c.ns; p.work = c.work; p.units = U; p.tiles_per_unit = (L + 127) / 128; p.d = D;
        p.slot_bytes = (unsigned)((128 + 192) * c.cs * 4);
        p.clk = clk;
        if (!make_residue_map_f32(&p.a, x, L, D, U, 1, 0, 128, c.bc) || !make_residue_map_f32(&p.b, y, L, D, U, 1, 0, 192, c.bc)) {
            printf("tmap failed\n");
            return 1;
        }
        const size_t smem = 1024 + (size_t)c.ns * p.slot_bytes + 512;
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0); cudaEventCreate(&e1);
        float best = 1e30f;
        for (int rep = 0; rep < 5; ++rep) {
            cudaEventRecord(e0);
            fill_kernel<<<c.grid, 64, smem>>>(p);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        cudaError_t err = cudaGetLastError();
        if (err != cudaSuccess) { printf("error %s\n", cudaGetErrorString(err)); return 1; }
        const double slots = (double)U * p.tiles_per_unit * (D / c.cs);
        const double bytes = slots * p.slot_bytes;
        const double slots_per_cta = slots / c.grid;
        printf("%4d %4d %3d %6d %5d %10.1f %10.1f %10.0f\n", c.bc, c.cs, c.ns, c.work, c.grid, best * 1e3,
               bytes / (best * 1e-3) / 1e9, best * 1e-3 * 1.965e9 / slots_per_cta);
    }
    return 0;
}
