// tc_common.cuh -- thin inline-PTX wrappers for the sm_100a features the tensor-core
// window-attention kernels use: mbarriers, TMA (cp.async.bulk.tensor), tcgen05 MMA /
// TMEM alloc / ld / st / commit, and the UMMA shared-memory + instruction descriptors.
//
// Descriptor bit layouts follow the PTX ISA "tcgen05 matrix descriptors" (as mirrored
// by CUTLASS's cute/arch/mma_sm100_desc.hpp, read as a format reference only):
//   smem desc: [0,14) start>>4, [16,30) LBO>>4, [32,46) SBO>>4, [46,48) version=1,
//              [49,52) base offset, [52] lbo mode, [61,64) layout (2 = SWIZZLE_128B)
//   instr desc (kind::f16): [4,6) D fmt (1=f32), [7,10) A fmt (1=bf16), [10,13) B fmt,
//              [15] A major (1=MN), [16] B major, [17,23) N>>3, [24,29) M>>4
#pragma once
#include <stdlib.h>
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <stdint.h>

namespace ftw {
namespace tc {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ------------------------------------------------------------------ mbarrier
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_barrier_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}
// try_wait suspends the waiting thread until the phase completes or the hint (ns) elapses,
// so warps parked on a barrier do not take issue slots from the working warps.
#ifndef FT_MBAR_SUSPEND_NS
#define FT_MBAR_SUSPEND_NS 0x989680u
#endif
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
#if FT_MBAR_SUSPEND_NS > 0
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity), "r"(FT_MBAR_SUSPEND_NS)
        : "memory");
#else
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
#endif
    return ok != 0;
}
// Watchdog: a protocol bug must end the kernel with an error (cudaErrorLaunchFailure), not hang
// the GPU.  No legitimate wait in these kernels lasts more than milliseconds; after
// FT_WATCHDOG_NS of global time (checked every 256 polls) the waiting thread traps.
#ifndef FT_WATCHDOG_NS
#define FT_WATCHDOG_NS 4000000000ull
#endif
#ifndef FT_WATCHDOG_SPINS
#define FT_WATCHDOG_SPINS (1u << 28)
#endif
__device__ __forceinline__ uint64_t global_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// The timer is read only once a wait has polled 4096 times, so handoffs on the critical path
// never pay for it.
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    uint32_t spins = 0;
    uint64_t t0 = 0;
    while (!mbar_try_wait(bar, parity)) {
        if (++spins < 4096u || (spins & 255u) != 0) continue;
        const uint64_t now = global_ns();
        if (t0 == 0) t0 = now;
        else if (now - t0 > FT_WATCHDOG_NS) __trap();
    }
}

// Always-suspending wait (a suspend-time hint even where FT_MBAR_SUSPEND_NS is 0): for a warp
// that would otherwise spin for thousands of cycles on an SM sub-partition another role needs
// (the narrow backward's softmax waiting for the converter warps' scale table).
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
    uint32_t ok = 0, spins = 0;
    uint64_t t0 = 0;
    for (;;) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(smem_u32(bar)), "r"(parity), "r"(0x989680u)
            : "memory");
        if (ok) return;
        if (++spins < 4096u || (spins & 255u) != 0) continue;
        const uint64_t now = global_ns();
        if (t0 == 0) t0 = now;
        else if (now - t0 > FT_WATCHDOG_NS) __trap();
    }
}

// Non-blocking probe (mbarrier.test_wait): for an issuer that polls several hand-offs and
// serves whichever completes first.
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

// Spin variant (no suspend-time hint): for single-thread MMA issuers whose handoffs are on the
// critical path -- the hinted wait compiles to NANOSLEEP.SYNCS, whose wake-up after the phase
// completes cost the fused backward's issuers ~200 clk per wait (tools/trace_fused.py).
__device__ __forceinline__ bool mbar_try_wait_spin(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait_spin(uint64_t* bar, uint32_t parity) {
    uint32_t spins = 0;
    uint64_t t0 = 0;
    while (!mbar_try_wait_spin(bar, parity)) {
        if (++spins < 65536u || (spins & 1023u) != 0) continue;
        const uint64_t now = global_ns();
        if (t0 == 0) t0 = now;
        else if (now - t0 > FT_WATCHDOG_NS) __trap();
    }
}

// One arrival per warp on a barrier whose count is in warps: per-thread arrivals of 128-512
// threads on one mbarrier serialise in the shared-memory atomic unit and delay the SM's other
// barrier and MMA traffic (fused backward: 0.626 -> 0.593 ms).  Every lane must have completed
// (and fenced) its own work before the call; the call must be warp-uniform.
__device__ __forceinline__ void warp_arrive(uint64_t* bar) {
    __syncwarp();
    if ((threadIdx.x & 31u) == 0) mbar_arrive(bar);
}

// ------------------------------------------------------------------ fences / barriers
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ void tc_fence_before() {
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}

// ------------------------------------------------------------------ TMA
__device__ __forceinline__ void tma_prefetch(const CUtensorMap* m) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(m)) : "memory");
}
__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* m, uint64_t* bar,
                                            int c0, int c1, int c2) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(m)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2)
        : "memory");
}
__device__ __forceinline__ void tma_load_4d(void* dst, const CUtensorMap* m, uint64_t* bar,
                                            int c0, int c1, int c2, int c3) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5, %6}], [%2];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(m)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
        : "memory");
}
// Prefetch a tensor box into L2 (no smem, no barrier).
__device__ __forceinline__ void tma_prefetch_l2_3d(const CUtensorMap* m, int c0, int c1, int c2) {
    asm volatile("cp.async.bulk.prefetch.tensor.3d.L2.global.tile [%0, {%1, %2, %3}];" ::"l"(
                     reinterpret_cast<uint64_t>(m)),
                 "r"(c0), "r"(c1), "r"(c2)
                 : "memory");
}
__device__ __forceinline__ void tma_store_3d(const CUtensorMap* m, const void* src, int c0, int c1,
                                             int c2) {
    asm volatile(
        "cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
            reinterpret_cast<uint64_t>(m)),
        "r"(smem_u32(src)), "r"(c0), "r"(c1), "r"(c2)
        : "memory");
}
__device__ __forceinline__ void tma_store_commit() {
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void tma_store_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
template <int N>
__device__ __forceinline__ void tma_store_wait_all() {
    asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}

// 4-byte asynchronous global -> shared copy (LDGSTS); src_bytes = 0 writes zero.  No register
// receives the value, so a prefetch issued a tile ahead never stalls the issuing thread.
__device__ __forceinline__ void cp_async4(void* dst, const void* src, uint32_t src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(smem_u32(dst)),
                 "l"(reinterpret_cast<uint64_t>(src)), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// ------------------------------------------------------------------ TMEM
__device__ __forceinline__ void tmem_alloc(uint32_t* dst_smem, uint32_t ncols) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(dst_smem)),
                 "r"(ncols)
                 : "memory");
}
__device__ __forceinline__ void tmem_relinquish() {
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t ncols) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols)
                 : "memory");
}

// 32 lanes x 32 consecutive 32-bit columns: thread t of the warp gets lane (base_lane + t).
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,"
        "%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
          "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]),
          "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]),
          "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,"
        "%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
          "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,"
        "%14,%15,%16};" ::"r"(taddr),
        "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
        "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]),
        "r"(r[15])
        : "memory");
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t* r) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr),
        "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7])
        : "memory");
}
__device__ __forceinline__ void tmem_wait_ld() {
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_wait_st() {
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

// ------------------------------------------------------------------ MMA
// D[tmem] (+)= A[smem] * B[smem]^T  (kind::f16, bf16 in, fp32 accumulate)
__device__ __forceinline__ void mma_ss(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                       uint32_t idesc, uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}
// D[tmem] (+)= A[tmem] * B[smem]  (A is M lanes x K, bf16 packed 2 per 32-bit column)
__device__ __forceinline__ void mma_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t bdesc,
                                       uint32_t idesc, uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}
// Four K=16 steps in one asm block.  Step k adds k*ASTEP to the A operand (descriptor units,
// bytes >> 4, for smem; columns for TMEM) and k*BSTEP to the B descriptor; the per-step
// operands are formed inside the asm, so ptxas gives each MMA its own uniform registers and
// the issuing thread does not wait for the previous MMA to release them
// (tools/mma_issue_bench.cu: ~58 clk per N=64 MMA issued this way vs ~89 with per-MMA
// descriptor arithmetic in C; N >= 128 runs at the tensor-pipe rate either way).
template <int ASTEP, int BSTEP>
__device__ __forceinline__ void mma_ss_x4(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                          uint32_t idesc, uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t.reg .b64 a1, a2, a3, b1, b2, b3;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "add.s64 a1, %1, %5;\n\tadd.s64 a2, %1, %6;\n\tadd.s64 a3, %1, %7;\n\t"
        "add.s64 b1, %2, %8;\n\tadd.s64 b2, %2, %9;\n\tadd.s64 b3, %2, %10;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], a1, b1, %3, 1;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], a2, b2, %3, 1;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], a3, b3, %3, 1;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate), "n"(ASTEP), "n"(2 * ASTEP),
        "n"(3 * ASTEP), "n"(BSTEP), "n"(2 * BSTEP), "n"(3 * BSTEP)
        : "memory");
}
template <int ASTEP, int BSTEP>
__device__ __forceinline__ void mma_ts_x4(uint32_t d_tmem, uint32_t a_tmem, uint64_t bdesc,
                                          uint32_t idesc, uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t.reg .b32 a1, a2, a3;\n\t.reg .b64 b1, b2, b3;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "add.u32 a1, %1, %5;\n\tadd.u32 a2, %1, %6;\n\tadd.u32 a3, %1, %7;\n\t"
        "add.s64 b1, %2, %8;\n\tadd.s64 b2, %2, %9;\n\tadd.s64 b3, %2, %10;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [a1], b1, %3, 1;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [a2], b2, %3, 1;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [a3], b3, %3, 1;\n\t}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(bdesc), "r"(idesc), "r"(accumulate), "n"(ASTEP), "n"(2 * ASTEP),
        "n"(3 * ASTEP), "n"(BSTEP), "n"(2 * BSTEP), "n"(3 * BSTEP)
        : "memory");
}
// Four TS steps with arbitrary TMEM column offsets of A (packed operands interleave hi / lo
// or two 32-key halves) and a uniform B step.
template <int A1, int A2, int A3, int BSTEP>
__device__ __forceinline__ void mma_ts_x4o(uint32_t d_tmem, uint32_t a_tmem, uint64_t bdesc,
                                           uint32_t idesc, uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t.reg .b32 a1, a2, a3;\n\t.reg .b64 b1, b2, b3;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "add.u32 a1, %1, %5;\n\tadd.u32 a2, %1, %6;\n\tadd.u32 a3, %1, %7;\n\t"
        "add.s64 b1, %2, %8;\n\tadd.s64 b2, %2, %9;\n\tadd.s64 b3, %2, %10;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [a1], b1, %3, 1;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [a2], b2, %3, 1;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [a3], b3, %3, 1;\n\t}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(bdesc), "r"(idesc), "r"(accumulate), "n"(A1), "n"(A2), "n"(A3),
        "n"(BSTEP), "n"(2 * BSTEP), "n"(3 * BSTEP)
        : "memory");
}
// Arrive on an mbarrier when all prior tcgen05.mma of this thread complete.
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    asm volatile(
        "tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
            smem_u32(bar))
        : "memory");
}

// ------------------------------------------------------------------ descriptors
// SWIZZLE_128B smem descriptor.  K-major: SBO = 1024 (8 rows x 128 B), LBO unused (1).
// MN-major: LBO = byte stride between 64-element MN groups, SBO = 1024 (8 K-rows x 128 B).
__device__ __forceinline__ uint64_t sdesc_sw128(uint32_t saddr, uint32_t lbo_bytes,
                                                uint32_t sbo_bytes) {
    uint64_t desc = 0;
    desc |= (uint64_t)((saddr >> 4) & 0x3FFFu);
    desc |= (uint64_t)((lbo_bytes >> 4) & 0x3FFFu) << 16;
    desc |= (uint64_t)((sbo_bytes >> 4) & 0x3FFFu) << 32;
    desc |= (uint64_t)1 << 46;   // version (sm_100)
    desc |= (uint64_t)2 << 61;   // SWIZZLE_128B
    return desc;
}

__host__ __device__ constexpr uint32_t idesc_bf16(int M, int N, bool a_mn, bool b_mn) {
    return (1u << 4) | (1u << 7) | (1u << 10) | ((a_mn ? 1u : 0u) << 15) |
           ((b_mn ? 1u : 0u) << 16) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

// kind::f16 with fp16 A and B (format code 0)
__host__ __device__ constexpr uint32_t idesc_f16(int M, int N, bool a_mn, bool b_mn) {
    return (1u << 4) | ((a_mn ? 1u : 0u) << 15) | ((b_mn ? 1u : 0u) << 16) |
           ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
// Blackwell packed fp32 pairs (one FFMA2 / FADD2 instruction for two lanes of work):
// (r0, r1) = (a0 b + c, a1 b + c) and (s0, s1) += (a0, a1)
__device__ __forceinline__ void ffma2_bc(float a0, float a1, float b, float c, float& r0, float& r1) {
    asm("{\n\t.reg .b64 aa, bb, cc, rr;\n\t"
        "mov.b64 aa, {%2, %3};\n\tmov.b64 bb, {%4, %4};\n\tmov.b64 cc, {%5, %5};\n\t"
        "fma.rn.f32x2 rr, aa, bb, cc;\n\tmov.b64 {%0, %1}, rr;\n\t}"
        : "=f"(r0), "=f"(r1)
        : "f"(a0), "f"(a1), "f"(b), "f"(c));
}
__device__ __forceinline__ void fadd2_acc(float& s0, float& s1, float a0, float a1) {
    asm("{\n\t.reg .b64 ss, aa;\n\t"
        "mov.b64 ss, {%0, %1};\n\tmov.b64 aa, {%2, %3};\n\t"
        "add.rn.f32x2 ss, ss, aa;\n\tmov.b64 {%0, %1}, ss;\n\t}"
        : "+f"(s0), "+f"(s1)
        : "f"(a0), "f"(a1));
}
// general packed pairs: (r0, r1) = (a0 b0 + c0, a1 b1 + c1), (a0 b0, a1 b1), (a0 + b0, a1 + b1)
__device__ __forceinline__ void ffma2(float a0, float a1, float b0, float b1, float c0, float c1, float& r0,
                                      float& r1) {
    asm("{\n\t.reg .b64 aa, bb, cc, rr;\n\t"
        "mov.b64 aa, {%2, %3};\n\tmov.b64 bb, {%4, %5};\n\tmov.b64 cc, {%6, %7};\n\t"
        "fma.rn.f32x2 rr, aa, bb, cc;\n\tmov.b64 {%0, %1}, rr;\n\t}"
        : "=f"(r0), "=f"(r1)
        : "f"(a0), "f"(a1), "f"(b0), "f"(b1), "f"(c0), "f"(c1));
}
__device__ __forceinline__ void fmul2(float a0, float a1, float b0, float b1, float& r0, float& r1) {
    asm("{\n\t.reg .b64 aa, bb, rr;\n\t"
        "mov.b64 aa, {%2, %3};\n\tmov.b64 bb, {%4, %5};\n\t"
        "mul.rn.f32x2 rr, aa, bb;\n\tmov.b64 {%0, %1}, rr;\n\t}"
        : "=f"(r0), "=f"(r1)
        : "f"(a0), "f"(a1), "f"(b0), "f"(b1));
}
// (x0, x1) -> hi = bf16x2 RN of (x0, x1), lo = bf16x2 RN of (x0, x1) - hi, the subtraction as one
// packed f32x2 instruction (x0 in the low halves)
__device__ __forceinline__ void split_bf16x2_p(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    asm("{\n\t.reg .b32 h0, h1, r0, r1;\n\t.reg .b64 xx, hh, rr;\n\t"
        "cvt.rn.bf16x2.f32 %0, %3, %2;\n\t"
        "shl.b32 h0, %0, 16;\n\tand.b32 h1, %0, 0xffff0000;\n\t"
        "mov.b64 xx, {%2, %3};\n\tmov.b64 hh, {h0, h1};\n\t"
        "sub.rn.f32x2 rr, xx, hh;\n\t"
        "mov.b64 {r0, r1}, rr;\n\t"
        "cvt.rn.bf16x2.f32 %1, r1, r0;\n\t}"
        : "=r"(hi), "=r"(lo)
        : "f"(x0), "f"(x1));
}
__device__ __forceinline__ uint32_t pack_f16x2(float lo, float hi) {
    __half2 h = __floats2half2_rn(lo, hi);   // .x = lo (low 16 bits)
    return *reinterpret_cast<uint32_t*>(&h);
}

__device__ __forceinline__ uint32_t pack_bf16x2(float lo, float hi) {
    __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);   // .x = lo (low 16 bits), .y = hi
    return *reinterpret_cast<uint32_t*>(&h);
}

__device__ __forceinline__ uint32_t elect_lane0() { return (threadIdx.x & 31u) == 0u; }
// One lane of a converged warp (elect.sync).  Whole-warp MMA issuers run their loop on all
// 32 lanes -- descriptors stay warp-uniform (uniform registers) -- and issue through the
// elected lane: ~1.5x the MMA issue rate of a lane-0-only issuer when several accumulator
// chains are in flight (tools/mma_microbench.cu).
__device__ __forceinline__ uint32_t elect_one() {
    uint32_t e;
    asm volatile("{\n\t.reg .pred p;\n\telect.sync _|p, 0xffffffff;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(e));
    return e;
}

// ---- D hand-off between the two kernels of a split backward (dQ kernel -> dK/dV kernel).
// The dQ kernel's CTAs first mark the D rows of their tiles D_UNSET, then trigger the
// programmatic dependent launch; the dK/dV kernel, launched with PDL, reads each D row with
// ld_D_ready as soon as it is stored, so its first tiles overlap the dQ kernel's last ones.
// Arithmetic never produces D_UNSET: a NaN from the FP units is the canonical 0x7FFFFFFF.
constexpr uint32_t D_UNSET = 0xFFFFFFFFu;
__device__ __forceinline__ float ld_D_ready(const float* ptr) {
    // D is stored by the dQ kernel of the same call, which is resident (the dependent grid
    // launches only after every dQ CTA triggered): a protocol bug traps instead of hanging
    uint32_t x;
    uint64_t t0 = 0;
    for (;;) {
        asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(x) : "l"(ptr) : "memory");
        if (x != D_UNSET) break;
        if (t0 == 0) t0 = global_ns();
        else if (global_ns() - t0 > FT_WATCHDOG_NS) __trap();
        __nanosleep(128);
    }
    return __uint_as_float(x);
}

// Tile flags of the dS tape (tc_band32.cu): the dQ kernel clears them before triggering the dependent
// launch and releases 1 once a tile's tape rows are stored; the dK/dV kernel acquires them.
__device__ __forceinline__ void wait_flag(const uint32_t* ptr) {
    uint32_t x;
    uint64_t t0 = 0;
    for (;;) {
        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(x) : "l"(ptr) : "memory");
        if (x != 0u) break;
        if (t0 == 0) t0 = global_ns();
        else if (global_ns() - t0 > FT_WATCHDOG_NS) __trap();
        __nanosleep(256);
    }
}
__device__ __forceinline__ void st_release_gpu(uint32_t* ptr, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(ptr), "r"(v) : "memory");
}

// one relaxed load (no memory clobber: a thread's loads of a halo issue back to back; the
// few still D_UNSET are then re-read with ld_D_ready)
__device__ __forceinline__ float ld_D_first(const float* ptr) {
    uint32_t x;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(x) : "l"(ptr));
    return __uint_as_float(x);
}

// lse hand-off (forward band kernel -> dQ kernel): the forward's CTAs mark their lse rows
// D_UNSET before triggering.  Unlike D, lse is a caller's buffer that may hold any bits when
// the preceding grid is not that forward, so the poll is bounded: after ~1 ms it waits for
// the preceding grid to complete (griddepcontrol.wait) and takes the value as stored;
// `settled` remembers that wait, after which every value is final and read once.
__device__ __forceinline__ float ld_lse_ready(const float* ptr, bool& settled) {
    uint32_t x;
    for (int i = 0; i < (settled ? 1 : 8192); ++i) {
        asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(x) : "l"(ptr) : "memory");
        if (x != D_UNSET) return __uint_as_float(x);
        __nanosleep(128);
    }
    if (settled) return __uint_as_float(x);
    asm volatile("griddepcontrol.wait;" ::: "memory");
    settled = true;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(x) : "l"(ptr) : "memory");
    return __uint_as_float(x);
}

// The hand-off pays only when the forward's last partial wave is a visible share of it: with
// many tiles per SM the forward's marking pass costs more than the overlap gains (narrow
// C5_w32, 110 tiles per SM: forward 0.176 -> 0.194 ms).  Used by both sides of a call.
inline bool lsepoll_worth(int64_t tiles, int sms) { return tiles < 8 * (int64_t)sms; }

}  // namespace tc
}  // namespace ftw
