// tests/helpers/early_trigger.cu -- a "foreign" producer kernel for the stream-order test
// (tests/test_gpu_parity.py::test_stream_order_aliasing): it executes
// griddepcontrol.launch_dependents first, as CUTLASS / cuBLASLt-style kernels may, then waits
// ~delay_ns and only then writes dst = src.  A consumer launched after it with programmatic
// dependent launch could start reading dst before it is written; ft_winattn's calls must not.
#include <cuda_runtime.h>
#include <stdint.h>

__global__ void early_trigger_copy(const uint4* src, uint4* dst, long long n, long long delay_ns) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    uint64_t t0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    for (;;) {
        uint64_t t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        if ((long long)(t - t0) >= delay_ns) break;
    }
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        dst[i] = src[i];
}

extern "C" int early_trigger_copy_launch(const void* src, void* dst, long long bytes, long long delay_ns,
                                         void* stream) {
    early_trigger_copy<<<148, 256, 0, (cudaStream_t)stream>>>((const uint4*)src, (uint4*)dst, bytes / 16, delay_ns);
    return (int)cudaGetLastError();
}
