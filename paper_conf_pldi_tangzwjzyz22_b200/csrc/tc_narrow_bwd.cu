// tc_narrow_bwd.cu -- backward of banded window attention for head dim d = 64 and w <= 32 on
// sm_100a (the HBM-bound C5 shape).  Two modes of one persistent
// kernel, each owning 128-row tiles of one (unit, residue) band problem and the 192-row halo
// m0-w .. m0-w+191 of the other operand (the cached window of PAPER.md Fig. 14, 402-423):
//
//   NQ   rows = queries.  S = Q K_h^T, dP = dO V_h^T;  P = exp(S - lse) recomputed from the
//        saved lse (selective materialization);  D = sum_j P dP (exact,
//        reading R1, -> workspace);  dS = P (dP - D) -> bf16 in TMEM;  dQ = dS K_h.
//   NKV  rows = keys (tile ownership: each dk/dv row has one writer, no atomics -- the
//        parallel reduction of PAPER.md Fig. 13(d) rather than 13(e)).  S^T = K Q_h^T,
//        dP^T = V dO_h^T;  P^T = exp(S^T - lse_col), dS^T = P^T (dP^T - D_col) -> bf16 in
//        TMEM;  dV = P^T dO_h,  dK = dS^T Q_h.
// (the gradient program of PAPER.md:447-453).
//
// Pipelining.  A tile's two 128 x 192 fp32 score matrices fill 384 of the 512 TMEM columns,
// so tiles cannot be double-buffered whole.  Instead the two 192-column regions alternate
// roles: tile j puts S in region j&1 and dP in region (j+1)&1; the softmax writes the bf16
// MMA operand (dS, or P^T | dS^T) over S in place.  S(j+1) can then start as soon as the
// softmax of j has read dP(j), and dP(j+1) right after the output MMAs of j were issued
// (tcgen05.mma executes in issue order).  Per tile the tensor pipe runs S(j+1), out(j),
// dP(j+1) while the softmax warps drain tile j's accumulator.
//
// dS enters its output MMA as fp16 (11-bit significand) with power-of-two scales, so the
// result does not depend on the magnitude of the inputs (reading A10): the converter warp
// turns the bf16 halo the dS GEMM multiplies (K_h for dQ, Q_h for dK) into fp16 row by row,
// each row c scaled by 2^f_c so that its largest |value| lands in [2^14, 2^15), once the
// score GEMM has read it, and publishes 2^-f_c; the softmax forms dS'_rc = dS_rc 2^-f_c,
// scales its row r by 2^e_r (largest |dS'| in [2^14, 2^15); NQ: an upper bound of it, so one
// exchange between the row's column halves suffices) and stores it as fp16.  The MMA
// then accumulates 2^e_r sum_c dS_rc x_c exactly up to fp16 rounding of the two operands, and
// the drain multiplies the row by 2^-e_r.  Powers of two are exact, so a gradient scaled by
// 2^16 (loss scaling) or 2^-24 gives the same relative error, with no overflow to inf and no
// fp16 subnormals (tests/test_gpu_parity.py::test_scale_equivariance).  A single bf16 dS
// failed the 2e-2 / 1e-2 bound at one element of 8.4 M (16 x 8192 case); the bf16 hi + lo
// pair of the band kernels would need a second operand, which does not fit (NQ: smem; NKV:
// the P^T | dS^T pair fills the 192 columns over S^T).
//
// Roles (320 threads): warps 0-7 softmax -- warp w reads TMEM lanes 32*(w%4).. (thread <->
// row) and column half h = w/4 of the row's 96-column band range; warp 8 TMA producer +
// TMEM allocator; warp 9 MMA issuer.  TMEM: R0 = [0,192), R1 = [192,384), accumulators at
// [384,512) (NQ: dQ at 384; NKV: dV at 384, dK at 448).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>

#include "internal.h"
#include "tc_common.cuh"
#include "tile_sched.cuh"
#include "tmap.h"

namespace ftw {
namespace {

using namespace tc;

enum { NQ = 0, NKV = 1 };

constexpr int BM = 128;
constexpr int D = 64;
constexpr int NK = 192;
constexpr int NSTAGE = 2;
constexpr int NTHREADS = 384;   // + converter warps 10, 11
constexpr int RES_PER_LAUNCH = 8;
static_assert(RES_PER_LAUNCH <= SCHED_MAX_RES, "residue table of the tile cursor");
constexpr uint32_t ABYTES = BM * D * 2;      // 16 KB: a 128-row tile
constexpr uint32_t HBYTES = NK * D * 2;      // 24 KB: a 192-row halo
constexpr uint32_t STAGE = 2 * ABYTES + 2 * HBYTES;   // {A1, A2, B1, B2}
constexpr uint32_t STG = 32 * 128;
constexpr uint32_t XBYTES = 3 * 16384;      // NQ: dS operand (fp16, 128 x 192); NKV: 8 x STG staging
// per-tile scratch: NKV [2][2][NK] column lse / D; NQ [2][2][BM] D halves + [2][256] row lse
constexpr int SCRATCH_FLOATS = 2 * 2 * BM + 2 * 256 > 2 * 2 * NK ? 2 * 2 * BM + 2 * 256 : 2 * 2 * NK;
// halo row scales 2^-f_c [2][NK] and the two halves' row maxima [2][2][BM] (NKV: of |dS'|; NQ:
// of P 2^-f |dP|, then of P 2^-f [2][2][BM])
constexpr int SCALE_FLOATS = 2 * NK + 2 * 2 * 2 * BM;
constexpr size_t SMEM_BYTES = 1024 + (size_t)NSTAGE * STAGE + XBYTES + (SCRATCH_FLOATS + SCALE_FLOATS) * 4 + 256;
static_assert(SMEM_BYTES <= 232448, "shared memory plan");
constexpr float LOG2E = 1.4426950408889634f;
constexpr uint32_t TACC = 384;

// a1/b1: first score GEMM (A: 128 rows at m0, B: halo at m0-w); a2/b2: second; o1/o2: outputs.
struct BMaps {
    CUtensorMap a1, a2, b1, b2, o1, o2;
};
struct BParams {
    BMaps maps[RES_PER_LAUNCH];
    const float* lse;
    float* D;      // NQ: written; NKV: read
    uint16_t* o1;  // NQ: dq (written with direct 16-byte stores)
    int64_t L;
    int w, dil;
    SchedParams sc;
    unsigned long long* trace;   // optional phase trace (ft_winattn_debug_trace, modes 1 / 2)
    int dpoll;                   // D hand-off by row polling (tc_common.cuh ld_D_ready)
    int lsepoll;                 // lse hand-off from the narrow forward (ld_lse_ready)
};

// Phase trace: per CTA and local tile j < 8, clock64 stamps (tools/trace_narrow.py).
// MMA: 0 iteration start, 1 S(j) issued, 2 out(j-1) issued, 3 dP(j) issued.  Softmax warp 0:
// 4 s_full seen, 5 S/dP loaded, 6 operand buffer free, 7 pair barrier passed, 8 p_done
// arrived, 9 accumulator seen, 10 drained.  Producer: 11 loads of tile j issued.
// Converter: 12 halo converted.
__device__ __forceinline__ void trace_ev(const BParams& p, int j, int ev) {
    if (p.trace && j >= 0 && j < 8) p.trace[((size_t)blockIdx.x * 8 + j) * 48 + ev] = clock64();
}

using Tile = SchedTile;
using TileCursor = SchedCursor<BM>;

// f with max|x| * 2^f in [2^14, 2^15) for a biased binary exponent E of max|x| (fp32 and bf16
// share the field), clamped so that 2^f and 2^-f are both normal floats
__device__ __forceinline__ int pow2_exp_fp16(int E) { return min(126, max(-126, 141 - E)); }
// 2^e and 2^-e of a row whose largest |value| is mx (e = 0 for an all-zero row)
__device__ __forceinline__ void row_pow2(float mx, float& up, float& down) {
    const int f = mx > 0.f ? pow2_exp_fp16(int(__float_as_uint(mx) >> 23) & 0xFF) : 0;
    up = __uint_as_float((uint32_t)(127 + f) << 23);
    down = __uint_as_float((uint32_t)(127 - f) << 23);
}

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// rows 32*wq .. +31 of a 64-column accumulator -> bf16 -> this warp's staging -> TMA store
// (the accumulator is released on `freed` as soon as it is in registers)
__device__ __forceinline__ void drain_store(uint32_t tacc, uint8_t* stg, const CUtensorMap* m, int row0,
                                           int u, int lane, uint64_t* freed, float scale) {
    uint32_t ov[2][32];
    tmem_ld32(tacc, ov[0]);
    tmem_ld32(tacc + 32, ov[1]);
    tmem_wait_ld();
    tc_fence_before();
    warp_arrive(freed);
    if (lane == 0) tma_store_wait_read<0>();
    __syncwarp();
#pragma unroll
    for (int q = 0; q < 8; ++q) {
        const uint32_t* src = &ov[q >> 2][(q & 3) * 8];
        uint4 val;
        const float* f = reinterpret_cast<const float*>(src);
        val.x = pack_bf16x2(f[0] * scale, f[1] * scale);
        val.y = pack_bf16x2(f[2] * scale, f[3] * scale);
        val.z = pack_bf16x2(f[4] * scale, f[5] * scale);
        val.w = pack_bf16x2(f[6] * scale, f[7] * scale);
        *reinterpret_cast<uint4*>(stg + lane * 128 + ((q ^ (lane & 7)) * 16)) = val;
    }
    fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) {
        tma_store_3d(m, stg, 0, row0, u);
        tma_store_commit();
    }
}

template <int MODE>
__global__ void __launch_bounds__(NTHREADS, 1) tc_narrow_bwd_kernel(const __grid_constant__ BParams p) {
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);
    if (MODE == NQ && p.dpoll) {   // this CTA's D rows: unset, before NKV may launch
        TileCursor cr(p.sc);
        Tile T;
        while (cr.next(p.sc, T)) {
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;
            for (int i = threadIdx.x; i < BM && T.m0 + i < T.Lr; i += NTHREADS)
                reinterpret_cast<uint32_t*>(p.D)[rowbase + (int64_t)(T.m0 + i) * p.dil] = D_UNSET;
        }
        __threadfence();
        __syncthreads();
    }
    if (MODE == NQ) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    uint8_t* stages = smem;                                        // [NSTAGE] {A1, A2, B1, B2}
    uint8_t* xbuf = smem + (size_t)NSTAGE * STAGE;                 // NQ: dS operand; NKV: staging
    float* colv = reinterpret_cast<float*>(xbuf + XBYTES);         // NKV [2][2][NK]: lse, D of columns
    float* dx = colv;                                              // NQ [2][2][BM]: D halves, then [2][256] lse
    float* hscale = colv + SCRATCH_FLOATS;                         // [2][NK] 2^-f of the halo rows
    float* mxh = hscale + 2 * NK;                                  // [2][2][BM] row max halves
    uint64_t* bars = reinterpret_cast<uint64_t*>(colv + SCRATCH_FLOATS + SCALE_FLOATS);
    uint64_t* full1 = bars;                 // [NSTAGE] A1 + B1
    uint64_t* full2 = bars + NSTAGE;        // [NSTAGE] A2 + B2
    uint64_t* empty = bars + 2 * NSTAGE;    // [NSTAGE]
    uint64_t* s_full = bars + 3 * NSTAGE;   // S and dP of the tile done
    uint64_t* dp_free = s_full + 1;         // softmax holds S and dP in registers
    uint64_t* p_done = s_full + 2;          // the softmax warps wrote the tile's operands
    uint64_t* acc_full = s_full + 3;        // [2]
    uint64_t* acc_free = s_full + 5;        // [2]
    uint64_t* hs_full = s_full + 7;         // [2] halo row scales of tile j published
    uint64_t* s_full2 = s_full + 9;         // [2] S and dP of tile j done, for the converters (which
                                            // may lag the softmax by a tile: a single-phase barrier
                                            // would let its parity wrap)
    // [2] the converter warps converted tile j's dS halo.  Its own barrier, by tile parity: the
    // converters may run a tile ahead of the softmax warps (they need only the tile's score GEMMs,
    // which start once the softmax holds the previous tile's S and dP in registers), and sharing
    // p_done let their arrivals for tile j+1 complete tile j's phase before the last softmax pair
    // had written its rows of dS(j) -- 32 rows of dq / dk read a stale operand (~1-2 % of runs).
    uint64_t* cv_done = s_full + 11;
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(s_full + 13);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int w = p.w;

    if (warp == 8) {
        if (lane == 0) {
            for (int i = 0; i < NSTAGE; ++i) {
                mbar_init(&full1[i], 1);
                mbar_init(&full2[i], 1);
                mbar_init(&empty[i], 1);
            }
            mbar_init(s_full, 1);
            mbar_init(dp_free, 8);
            mbar_init(p_done, 8);
            mbar_init(&cv_done[0], 2);
            mbar_init(&cv_done[1], 2);
            for (int b = 0; b < 2; ++b) {
                mbar_init(&acc_full[b], 1);
                mbar_init(&acc_free[b], 8);
                mbar_init(&hs_full[b], 64);
                mbar_init(&s_full2[b], 1);
            }
            fence_barrier_init();
            for (int i = 0; i < p.sc.nr; ++i) {
                const BMaps& m = p.maps[i];
                tma_prefetch(&m.a1); tma_prefetch(&m.a2); tma_prefetch(&m.b1); tma_prefetch(&m.b2);
                if (MODE == NKV) { tma_prefetch(&m.o1); tma_prefetch(&m.o2); }
            }
        }
        __syncwarp();
        tmem_alloc(tmem_holder, 512);
        tmem_relinquish();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tbase = *tmem_holder;

    if (warp == 8) {
        if (lane == 0) {   // ---------------------------------------------------- TMA producer
            TileCursor cur(p.sc);
            Tile T;
            for (int j = 0; cur.next(p.sc, T); ++j) {
                const int s = j % NSTAGE;
                if (j >= NSTAGE) mbar_wait(&empty[s], ((j / NSTAGE) - 1) & 1);
                uint8_t* st = stages + (size_t)s * STAGE;
                const BMaps& mp = p.maps[T.rl];
                trace_ev(p, j, 11);
                mbar_arrive_expect_tx(&full1[s], ABYTES + HBYTES);
                tma_load_3d(st, &mp.a1, &full1[s], 0, T.m0, T.u);
                tma_load_3d(st + 2 * ABYTES, &mp.b1, &full1[s], 0, T.m0 - w, T.u);
                mbar_arrive_expect_tx(&full2[s], ABYTES + HBYTES);
                tma_load_3d(st + ABYTES, &mp.a2, &full2[s], 0, T.m0, T.u);
                tma_load_3d(st + 2 * ABYTES + HBYTES, &mp.b2, &full2[s], 0, T.m0 - w, T.u);
            }
        }
    } else if (warp == 10 || warp == 11) {   // ----------------------------- halo converters
        // the halo of the dS GEMM (NQ: K_h, NKV: Q_h) to fp16 in place.  Lane l of converter warp
        // cw owns halo rows 64 i + 32 cw + l, i < 3 (whole 128-byte rows: no shuffles).  As soon
        // as the TMA landed it reduces each row's largest |value| and publishes 2^-f (hs_full);
        // once the score GEMM has read the bf16 halo (s_full2) it rewrites the rows times 2^f as
        // fp16; the output MMAs read them after cv_done.  The row loops stay rolled and the
        // second pass re-reads its rows from shared memory: holding all three rows in registers
        // unrolled this role to ~880 instructions, which pushed the kernel's steady-state code
        // past the 32 KB instruction cache (ncu: no_inst the top stall reason of every role).
        const int cw = warp - 10;
        constexpr int NR = NK / 64;     // rows per lane
        TileCursor cur(p.sc);
        Tile T;
        for (int j = 0; cur.next(p.sc, T); ++j) {
            mbar_wait(&full1[j % NSTAGE], (j / NSTAGE) & 1);
            if (lane == 0 && cw == 0) trace_ev(p, j, 14);
            uint8_t* hb = stages + (size_t)(j % NSTAGE) * STAGE + 2 * ABYTES;
            float* tab = hscale + (j & 1) * NK;
#pragma unroll 1
            for (int i = 0; i < NR; ++i) {
                const int r = 64 * i + 32 * cw + lane;
                uint4 v[8];
#pragma unroll
                for (int x = 0; x < 8; ++x)
                    v[x] = *reinterpret_cast<const uint4*>(hb + r * 128 + ((x ^ (r & 7)) << 4));
                uint32_t m = 0;
#pragma unroll
                for (int x = 0; x < 8; ++x)
                    m = __vmaxu2(m, __vmaxu2(__vmaxu2(v[x].x & 0x7FFF7FFFu, v[x].y & 0x7FFF7FFFu),
                                             __vmaxu2(v[x].z & 0x7FFF7FFFu, v[x].w & 0x7FFF7FFFu)));
                m = max(m & 0xFFFFu, m >> 16);   // bf16 bits of the row's max |x|
                const int f = m == 0 ? 0 : pow2_exp_fp16(int(m >> 7));
                tab[r] = __uint_as_float((uint32_t)(127 - f) << 23);
            }
            mbar_arrive(&hs_full[j & 1]);   // every lane releases its own table entries
            if (lane == 0 && cw == 0) trace_ev(p, j, 17);
            mbar_wait(&s_full2[j & 1], (j >> 1) & 1);   // the score GEMM has read the bf16 halo
#pragma unroll 1
            for (int i = 0; i < NR; ++i) {
                const int r = 64 * i + 32 * cw + lane;
                const float sc = __uint_as_float((254u << 23) - __float_as_uint(tab[r]));   // 2^f
                uint4 v[8];
#pragma unroll
                for (int x = 0; x < 8; ++x)
                    v[x] = *reinterpret_cast<const uint4*>(hb + r * 128 + ((x ^ (r & 7)) << 4));
#pragma unroll
                for (int x = 0; x < 8; ++x) {
                    uint32_t* wv = reinterpret_cast<uint32_t*>(&v[x]);
#pragma unroll
                    for (int y = 0; y < 4; ++y) {
                        const float2 f2 = __bfloat1622float2(*reinterpret_cast<__nv_bfloat162*>(&wv[y]));
                        wv[y] = pack_f16x2(f2.x * sc, f2.y * sc);
                    }
                    *reinterpret_cast<uint4*>(hb + r * 128 + ((x ^ (r & 7)) << 4)) = v[x];
                }
            }
            fence_proxy_async_smem();
            warp_arrive(&cv_done[j & 1]);
            if (lane == 0 && cw == 0) trace_ev(p, j, 12);
        }
    } else if (warp == 9) {
        if (lane == 0) {   // ------------------------------------------------------ MMA issuer
            constexpr uint32_t idS = idesc_bf16(BM, NK, false, false);
            constexpr uint32_t idO = idesc_bf16(BM, D, false, true);
            constexpr uint32_t idH = idesc_f16(BM, D, false, true);
            // output MMAs of tile i (B = a halo as MN-major SW128, 2048 B per 16-key step):
            //   NQ:  dQ = dS K_h, A = dS in smem (K-major SW128: 64-key atoms of 16 KB), -> acc[i&1]
            //   NKV: dV = P^T dO_h, dK = dS^T Q_h, A = packed operands over S^T in TMEM region
            //        i&1 (8 columns per step) -> acc (dV at 384, dK at 448)
            auto acc_free_phase = [&](int i) -> int { return (MODE == NQ ? (i - 2) >> 1 : i - 1) & 1; };
            auto acc_free_needed = [&](int i) -> bool { return MODE == NQ ? i >= 2 : i >= 1; };
            // all of out(i)'s hand-offs complete (non-blocking)
            auto out_ready = [&](int i) -> bool {
                return mbar_test(p_done, i & 1) && mbar_test(&cv_done[i & 1], (i >> 1) & 1) &&
                       (!acc_free_needed(i) || mbar_test(&acc_free[MODE == NQ ? (i & 1) : 0], acc_free_phase(i)));
            };
            auto out_issue = [&](int i) {
                const int s = i % NSTAGE, b = MODE == NQ ? (i & 1) : 0;
                const uint32_t st = smem_u32(stages + (size_t)s * STAGE);
                tc_fence_after();
                if (MODE == NQ) {
                    const uint32_t sb = st + 2 * ABYTES, sa = smem_u32(xbuf);
#pragma unroll
                    for (int g = 0; g < 3; ++g)
                        mma_ss_x4<2, 128>(tbase + TACC + 64u * b, sdesc_sw128(sa + 16384u * g, 16, 1024),
                                          sdesc_sw128(sb + 8192u * g, 8192, 1024), idH, g);
                } else {
                    const uint32_t tR = tbase + 192u * (i & 1);
                    const uint32_t sq = st + 2 * ABYTES, sdo = sq + HBYTES;
#pragma unroll
                    for (int g = 0; g < 3; ++g) {
                        mma_ts_x4<8, 128>(tbase + TACC, tR + 32u * g, sdesc_sw128(sdo + 8192u * g, 8192, 1024), idO, g);
                        mma_ts_x4<8, 128>(tbase + TACC + 64, tR + 96u + 32u * g, sdesc_sw128(sq + 8192u * g, 8192, 1024), idH, g);
                    }
                }
                mma_commit(&acc_full[b]);
                mma_commit(&empty[s]);
            };
            auto out = [&](int i) {
                mbar_wait(p_done, i & 1);
                mbar_wait(&cv_done[i & 1], (i >> 1) & 1);
                if (acc_free_needed(i)) mbar_wait(&acc_free[MODE == NQ ? (i & 1) : 0], acc_free_phase(i));
                out_issue(i);
            };
            TileCursor cur(p.sc);
            Tile T;
            int j = 0;
            for (; cur.next(p.sc, T); ++j) {
                const int s = j % NSTAGE, ph = (j / NSTAGE) & 1;
                const uint32_t st = smem_u32(stages + (size_t)s * STAGE);
                // NQ: S in [0,192), dP in [192,384) every tile (the dS operand is in smem), so
                // both score GEMMs of j run while the softmax of j-1 computes.
                // NKV: S(j) in region j&1 (which held dP(j-1)), dP(j) in region (j+1)&1 (the
                // operands of j-1, read by out(j-1) first: tcgen05.mma executes in issue order)
                const uint32_t rS = MODE == NQ ? tbase : tbase + 192u * (j & 1);
                const uint32_t rP = MODE == NQ ? tbase + 192u : tbase + 192u * ((j + 1) & 1);
                trace_ev(p, j, 0);
                if (j >= 1) mbar_wait(dp_free, (j - 1) & 1);
                // S(j) and out(j-1) in whichever order their inputs complete: out(j-1)'s
                // completion frees the ring slot tile j+1 loads into, so it must not queue behind
                // tile j's loads, and S(j) must not wait for the softmax of j-1 (dP(j) goes after
                // both: in NKV it overwrites the operands out(j-1) reads)
                {
                    bool od = j == 0, sd = false;
                    uint32_t spins = 0;
                    uint64_t t0 = 0;
                    while (!(od && sd)) {
                        if (!od && out_ready(j - 1)) {
                            out_issue(j - 1);
                            od = true;
                            trace_ev(p, j, 2);
                        }
                        if (!sd && mbar_test(&full1[s], ph)) {
                            tc_fence_after();
                            mma_ss_x4<2, 2>(rS, sdesc_sw128(st, 16, 1024), sdesc_sw128(st + 2 * ABYTES, 16, 1024),
                                            idS, 0);
                            sd = true;
                            trace_ev(p, j, 1);
                        }
                        if (++spins < 4096u || (spins & 255u) != 0) continue;
                        const uint64_t now = global_ns();
                        if (t0 == 0) t0 = now;
                        else if (now - t0 > FT_WATCHDOG_NS) __trap();
                    }
                }
                mbar_wait(&full2[s], ph);
                tc_fence_after();
                mma_ss_x4<2, 2>(rP, sdesc_sw128(st + ABYTES, 16, 1024),
                                sdesc_sw128(st + 2 * ABYTES + HBYTES, 16, 1024), idS, 0);
                mma_commit(s_full);
                mma_commit(&s_full2[j & 1]);
                trace_ev(p, j, 3);
                if (p.trace && j < 8) {   // debug only: when did the score GEMMs complete?
                    mbar_wait(s_full, j & 1);
                    trace_ev(p, j, 13);
                }
            }
            if (j >= 1) out(j - 1);
        }
    } else if (warp < 8) {   // ------------------------------------------------- softmax warps
        const int wq = warp & 3, h = warp >> 2;
        const int t = wq * 32 + lane;
        const uint32_t lane_off = (uint32_t)(wq * 32) << 16;
        const int c0 = 32 * wq + 48 * h;         // first of this warp's 48 score columns
        const uint32_t pc = 16u * wq + 24u * h;  // NKV: its packed operand columns
        uint32_t zero16[16];
#pragma unroll
        for (int e = 0; e < 16; ++e) zero16[e] = 0u;
        // NKV: 48 packed columns of an operand at TMEM base (+ zeros on the columns outside
        // every band column of this row: h = 0 writes the ones before, h = 1 the ones after)
        auto st_operand = [&](uint32_t base, const uint32_t (&pk)[24]) {
            tmem_st16(base + pc, *reinterpret_cast<const uint32_t(*)[16]>(&pk[0]));
            tmem_st8(base + pc + 16, &pk[16]);
            if (h == 0) {
                for (int c = 0; c < wq; ++c) tmem_st16(base + 16u * c, zero16);
            } else {
                for (int c = wq + 3; c < NK / 32; ++c) tmem_st16(base + 16u * c, zero16);
            }
        };
        // NQ: dS row t in smem (K-major SW128, 64-key atoms of 128 rows x 128 B): keys
        // c .. c+7 are 16-byte granule ((c % 64) / 8) ^ (t % 8) of row t in atom c / 64
        auto ds_granule = [&](int c) -> uint4* {
            return reinterpret_cast<uint4*>(xbuf + (c >> 6) * 16384 + t * 128 + ((((c & 63) >> 3) ^ (t & 7)) << 4));
        };
        if (MODE == NQ) {   // keys outside every band column of this row stay zero
            const uint4 z = make_uint4(0u, 0u, 0u, 0u);
            if (h == 0) for (int c = 0; c < 32 * wq; c += 8) *ds_granule(c) = z;
            else for (int c = 32 * wq + 96; c < NK; c += 8) *ds_granule(c) = z;
        }
        // per-tile values from HBM are copied one tile ahead into shared memory with cp.async
        // (NQ: this row's lse -> lpre[b][threadIdx.x]; NKV: lse and D of halo column
        // threadIdx.x -> colv[b]), so their latency hides behind the previous tile
        float* lpre = colv + (MODE == NQ ? 2 * 2 * BM : 0);   // NQ [2][256]
        TileCursor cur(p.sc), nxt(p.sc);
        Tile T, Tn;
        bool hn = nxt.next(p.sc, Tn);
        bool lse_settled = false;   // ld_lse_ready fell back to griddepcontrol.wait
        bool first_store = true;    // NQ launched early: wait for the preceding grid first
        // NKV with the D hand-off: D is stored by the NQ grid, which this grid does not wait for
        // (no griddepcontrol.wait), so it is read with ld.relaxed.gpu (at the coherence point,
        // never from a possibly stale L1 line) one tile ahead and kept in a register until setup
        float dnext = 0.f, lnext = 0.f;   // (lse likewise while the forward may still run: lsepoll)
        auto prefetch = [&](const Tile& X, int jx) {
            const int64_t rb = (int64_t)X.u * p.L + X.r;
            if (MODE == NKV) {
                if (threadIdx.x < NK) {
                    const int mc = X.m0 - w + (int)threadIdx.x;
                    const bool ok = mc >= 0 && mc < X.Lr;
                    const int64_t off = ok ? rb + (int64_t)mc * p.dil : 0;
                    float* cl = colv + (jx & 1) * 2 * NK;
                    if (p.lsepoll) lnext = ok ? ld_D_first(p.lse + off) : 0.f;
                    else cp_async4(cl + threadIdx.x, p.lse + off, ok ? 4u : 0u);
                    if (p.dpoll) dnext = ok ? ld_D_first(p.D + off) : 0.f;
                    else cp_async4(cl + NK + threadIdx.x, p.D + off, ok ? 4u : 0u);
                }
            } else {
                const int mrow = X.m0 + t;
                const bool ok = mrow < X.Lr;
                if (p.lsepoll) lnext = ok ? ld_D_first(p.lse + rb + (int64_t)mrow * p.dil) : 0.f;
                else cp_async4(lpre + (jx & 1) * 256 + threadIdx.x, p.lse + (ok ? rb + (int64_t)mrow * p.dil : 0),
                               ok ? 4u : 0u);
            }
            cp_async_commit();
        };
        if (hn) prefetch(Tn, 0);
        // per-tile state, set up for tile j+1 as soon as tile j's operands are written
        struct St {
            int Lr, m0, kb, u, rl;
            int64_t rowbase;
            float lse2;
            uint64_t bits;
            float rsc;   // 2^-e of this row's dS (NQ: dq row; NKV: dk row), set by the softmax
        };
        auto setup = [&](const Tile& X, int jx) -> St {
            St c;
            c.rsc = 1.f;
            c.Lr = X.Lr; c.m0 = X.m0; c.kb = X.m0 - w; c.u = X.u; c.rl = X.rl;
            c.rowbase = (int64_t)X.u * p.L + X.r;
            cp_async_wait_all();   // this tile's values (copied a tile ago)
            if (p.lsepoll) {   // lse rows the forward had not stored yet
                if (MODE == NQ) {
                    float* cl = lpre + (jx & 1) * 256 + threadIdx.x;
                    *cl = lnext;
                    if (__float_as_uint(*cl) == D_UNSET)
                        *cl = ld_lse_ready(p.lse + c.rowbase + (int64_t)(c.m0 + t) * p.dil, lse_settled);
                } else if (threadIdx.x < NK) {
                    float* cl = colv + (jx & 1) * 2 * NK + threadIdx.x;
                    *cl = lnext;
                    if (__float_as_uint(*cl) == D_UNSET)
                        *cl = ld_lse_ready(p.lse + c.rowbase + (int64_t)(c.kb + (int)threadIdx.x) * p.dil, lse_settled);
                }
            }
            if (MODE == NKV && p.dpoll && threadIdx.x < NK) {   // D rows NQ had not stored yet
                float* cd = colv + (jx & 1) * 2 * NK + NK + threadIdx.x;
                *cd = dnext;
                if (__float_as_uint(*cd) == D_UNSET)
                    *cd = ld_D_ready(p.D + c.rowbase + (int64_t)(c.kb + (int)threadIdx.x) * p.dil);
            }
            c.lse2 = MODE == NQ ? lpre[(jx & 1) * 256 + threadIdx.x] * LOG2E : 0.f;
            if (MODE == NKV) named_bar_sync(5, 256);   // every thread's columns landed
            hn = nxt.next(p.sc, Tn);
            if (hn) prefetch(Tn, jx + 1);
            // band columns of this row: n in [t, t+2w] within the sequence
            const int lo = max(t, -c.kb) - c0, hi = min(t + 2 * w, c.Lr - 1 - c.kb) - c0;
            const int l0 = max(lo, 0), h0 = min(hi, 47);
            c.bits = h0 < l0 ? 0ull : ((~0ull >> (63 - h0)) & (~0ull << l0));
            return c;
        };
        // NQ: drain dQ of tile i (columns 32h .. 32h+31 of this row) with direct 16-byte
        // stores; NKV: dV (h = 0) or dK (h = 1) of tile i through staging + TMA store
        auto drain = [&](int i, const St& c) {
            const int b = MODE == NQ ? (i & 1) : 0;
            mbar_wait(&acc_full[b], MODE == NQ ? (i >> 1) & 1 : i & 1);
            tc_fence_after();
            if (threadIdx.x == 0) trace_ev(p, i, 9);
            if (MODE == NQ && p.lsepoll && first_store) {
                asm volatile("griddepcontrol.wait;" ::: "memory");
                first_store = false;
            }
            if (MODE == NQ) {
                uint32_t ov[32];
                tmem_ld32(tbase + lane_off + TACC + 64u * b + 32u * h, ov);
                tmem_wait_ld();
                if (threadIdx.x == 0) trace_ev(p, i, 16);
                tc_fence_before();
                warp_arrive(&acc_free[b]);
                const int mrow = c.m0 + t;
                if (mrow < c.Lr) {
                    uint4* dst = reinterpret_cast<uint4*>(p.o1 + (c.rowbase + (int64_t)mrow * p.dil) * D + 32 * h);
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const float* o = reinterpret_cast<const float*>(&ov[8 * q]);
                        const float r = c.rsc;
                        dst[q] = make_uint4(pack_bf16x2(o[0] * r, o[1] * r), pack_bf16x2(o[2] * r, o[3] * r),
                                            pack_bf16x2(o[4] * r, o[5] * r), pack_bf16x2(o[6] * r, o[7] * r));
                    }
                }
            } else {
                const BMaps& mp = p.maps[c.rl];
                drain_store(tbase + lane_off + TACC + 64u * h, xbuf + warp * STG, h == 0 ? &mp.o1 : &mp.o2,
                            c.m0 + 32 * wq, c.u, lane, &acc_free[0], h == 0 ? 1.f : c.rsc);
            }
            if (threadIdx.x == 0) trace_ev(p, i, 10);
        };
        bool have = cur.next(p.sc, T);
        St cs = have ? setup(T, 0) : St{};
        St prev = cs;
        int j = 0;
        for (; have; ++j) {
            const int Lr = cs.Lr, m0 = cs.m0;
            const int64_t rowbase = cs.rowbase;
            const float lse2 = cs.lse2;
            const uint64_t bits = cs.bits;
            const uint32_t tS = MODE == NQ ? tbase + lane_off : tbase + lane_off + 192u * (j & 1);
            const uint32_t tP = MODE == NQ ? tbase + lane_off + 192u : tbase + lane_off + 192u * ((j + 1) & 1);
            const float* cl = colv + (j & 1) * 2 * NK;   // NKV: this tile's column lse*log2e and D
            const bool tr = threadIdx.x == 0;
            mbar_wait(s_full, j & 1);
            tc_fence_after();
            if (tr) trace_ev(p, j, 4);
            uint32_t rs[48], rd[48];
            tmem_ld16(tS + c0, *reinterpret_cast<uint32_t(*)[16]>(&rs[0]));
            tmem_ld16(tS + c0 + 16, *reinterpret_cast<uint32_t(*)[16]>(&rs[16]));
            tmem_ld16(tS + c0 + 32, *reinterpret_cast<uint32_t(*)[16]>(&rs[32]));
            tmem_ld16(tP + c0, *reinterpret_cast<uint32_t(*)[16]>(&rd[0]));
            tmem_ld16(tP + c0 + 16, *reinterpret_cast<uint32_t(*)[16]>(&rd[16]));
            tmem_ld16(tP + c0 + 32, *reinterpret_cast<uint32_t(*)[16]>(&rd[32]));
            tmem_wait_ld();
            tc_fence_before();
            warp_arrive(dp_free);
            if (tr) trace_ev(p, j, 5);
            uint32_t pk[24], pk2[24];
            if (MODE == NQ) {
                // One exchange between the row's two column halves: the D parts, and for the row
                // scale the bound max_c |dS'_c| <= max_c P 2^-f_c |dP_c| + max_c P 2^-f_c |D| (dS' =
                // P (dP - D) 2^-f_c).  The bound can exceed the true maximum (by cancellation in
                // dP - D), which only moves the fp16 values down by powers of two: a normal fp16
                // value keeps its 11 bits (a second exchange for the exact maximum cost more).
                mbar_wait_sleep(&hs_full[j & 1], (j >> 1) & 1);
                const float* tab = hscale + (j & 1) * NK + c0;
                float dpart[4] = {0.f, 0.f, 0.f, 0.f};
                float am = 0.f, bm = 0.f;
#pragma unroll
                for (int e = 0; e < 48; e += 2) {   // packed f32x2 pairs (FFMA2)
                    float a0, a1;
                    ffma2_bc(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, -lse2, a0, a1);
                    const float p0 = ((bits >> e) & 1ull) ? fast_exp2(a0) : 0.f;
                    const float p1 = ((bits >> (e + 1)) & 1ull) ? fast_exp2(a1) : 0.f;
                    const int q = e & 2;
                    ffma2(p0, p1, __uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), dpart[q], dpart[q + 1],
                          dpart[q], dpart[q + 1]);
                    float t0, t1;
                    fmul2(p0, p1, tab[e], tab[e + 1], t0, t1);   // exact: 2^-f_c
                    rs[e] = __float_as_uint(t0);
                    rs[e + 1] = __float_as_uint(t1);
                    am = fmaxf(am, fmaxf(t0 * fabsf(__uint_as_float(rd[e])), t1 * fabsf(__uint_as_float(rd[e + 1]))));
                    bm = fmaxf(bm, fmaxf(t0, t1));
                }
                float* dxb = dx + (j & 1) * 2 * BM;
                float* mxb = mxh + (j & 1) * 2 * BM;
                float* mbb = mxh + 2 * 2 * BM + (j & 1) * 2 * BM;
                dxb[h * BM + t] = (dpart[0] + dpart[1]) + (dpart[2] + dpart[3]);
                mxb[h * BM + t] = am;
                mbb[h * BM + t] = bm;
                named_bar_sync(1 + wq, 64);   // both halves posted their parts
                if (tr) trace_ev(p, j, 7);
                const float Dv = dxb[t] + dxb[BM + t];
                float up, down;
                row_pow2(fmaxf(mxb[t], mxb[BM + t]) + fmaxf(mbb[t], mbb[BM + t]) * fabsf(Dv), up, down);
                cs.rsc = down;
#pragma unroll
                for (int e = 0; e < 48; e += 2) {   // dS' 2^e = (P 2^-f_c) (dP - D) 2^e
                    float q0, q1, r0, r1;
                    ffma2_bc(__uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), 1.f, -Dv, q0, q1);
                    fmul2(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), q0, q1, r0, r1);
                    fmul2(r0, r1, up, up, r0, r1);
                    pk[e / 2] = pack_f16x2(r0, r1);
                }
                // the dS buffer is free once out(j-1) completed
                if (j >= 1) mbar_wait(&acc_full[(j - 1) & 1], ((j - 1) >> 1) & 1);
                if (tr) trace_ev(p, j, 6);
#pragma unroll
                for (int g = 0; g < 6; ++g)
                    *ds_granule(c0 + 8 * g) = make_uint4(pk[4 * g], pk[4 * g + 1], pk[4 * g + 2], pk[4 * g + 3]);
                fence_proxy_async_smem();
                const int mrow = m0 + t;
                if (h == 0 && mrow < Lr) p.D[rowbase + (int64_t)mrow * p.dil] = Dv;
            } else {
                const float4* cL = reinterpret_cast<const float4*>(cl + c0);
                const float4* cD = reinterpret_cast<const float4*>(cl + NK + c0);
                mbar_wait_sleep(&hs_full[j & 1], (j >> 1) & 1);
                const float* tab = hscale + (j & 1) * NK + c0;   // 2^-f of the Q_h rows (columns)
                float mx = 0.f;
#pragma unroll
                for (int e4 = 0; e4 < 12; ++e4) {
                    const float4 l4 = cL[e4], d4 = cD[e4];
                    const float lv[4] = {l4.x * LOG2E, l4.y * LOG2E, l4.z * LOG2E, l4.w * LOG2E};
                    const float dvv[4] = {d4.x, d4.y, d4.z, d4.w};
                    float pv[4];
#pragma unroll
                    for (int x = 0; x < 4; x += 2) {   // packed f32x2 pairs
                        const int e = 4 * e4 + x;
                        float a0, a1, q0, q1, r0, r1;
                        ffma2(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, LOG2E, -lv[x], -lv[x + 1], a0, a1);
                        pv[x] = ((bits >> e) & 1ull) ? fast_exp2(a0) : 0.f;
                        pv[x + 1] = ((bits >> (e + 1)) & 1ull) ? fast_exp2(a1) : 0.f;
                        ffma2(__uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), 1.f, 1.f, -dvv[x], -dvv[x + 1], q0, q1);
                        fmul2(pv[x], pv[x + 1], q0, q1, r0, r1);
                        fmul2(r0, r1, tab[e], tab[e + 1], r0, r1);
                        rd[e] = __float_as_uint(r0);
                        rd[e + 1] = __float_as_uint(r1);
                        mx = fmaxf(mx, fmaxf(fabsf(r0), fabsf(r1)));
                    }
                    pk[2 * e4] = pack_bf16x2(pv[0], pv[1]);
                    pk[2 * e4 + 1] = pack_bf16x2(pv[2], pv[3]);
                }
                float* mxb = mxh + (j & 1) * 2 * BM;
                mxb[h * BM + t] = mx;
                named_bar_sync(1 + wq, 64);   // both halves read S^T / dP^T and posted their row max
                if (tr) trace_ev(p, j, 7);
                float up, down;
                row_pow2(fmaxf(mxb[t], mxb[BM + t]), up, down);
                cs.rsc = down;
#pragma unroll
                for (int e = 0; e < 48; e += 2) {
                    float r0, r1;
                    fmul2(__uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), up, up, r0, r1);
                    pk2[e / 2] = pack_f16x2(r0, r1);
                }
                // P^T (bf16) | dS^T (fp16) over S^T
                st_operand(tS, pk);
                st_operand(tS + 96, pk2);
                tmem_wait_st();
            }
            tc_fence_before();
            warp_arrive(p_done);
            if (tr) trace_ev(p, j, 8);
            const St done = cs;
            have = cur.next(p.sc, T);
            if (have) cs = setup(T, j + 1);
            if (tr) trace_ev(p, j, 15);
            // NQ: the accumulator of the previous tile (out(j-1) completed before dS(j) was
            // written); NKV: this tile's, once out(j) completed
            if (MODE == NQ) {
                if (j >= 1) drain(j - 1, prev);
            } else {
                drain(j, done);
            }
            prev = done;
        }
        if (MODE == NQ && j >= 1) drain(j - 1, prev);
        if (MODE == NKV && lane == 0) tma_store_wait_all<0>();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 8) {
        tc_fence_after();
        tmem_dealloc(tbase, 512);
    }
}

int num_sms_nb() {
    static int n = 0;
    static std::once_flag once;
    std::call_once(once, [] {
        int dev = 0;
        cudaGetDevice(&dev);
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0)
            n = 148;
    });
    return n;
}

template <int MODE>
cudaError_t launch_nb(const void* a1, const void* a2, const void* b1, const void* b2, void* o1,
                      void* o2, const float* lse, float* Dws, int64_t B, int64_t H, int64_t L,
                      int64_t w, int64_t dil, cudaStream_t st, int* launches) {
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_narrow_bwd_kernel<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)SMEM_BYTES);
    });
    const int64_t wc = w < L ? w : L;
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    int n = 0;
    for (int64_t r0 = 0; r0 < nres; r0 += RES_PER_LAUNCH) {
        BParams p;
        memset(&p, 0, sizeof(p));
        const int nr = (int)(nres - r0 < RES_PER_LAUNCH ? nres - r0 : RES_PER_LAUNCH);
        for (int i = 0; i < nr; ++i) {
            const int64_t r = r0 + i;
            BMaps& m = p.maps[i];
            bool ok = make_residue_map(&m.a1, a1, L, D, units, dil, r, BM) &&
                      make_residue_map(&m.a2, a2, L, D, units, dil, r, BM) &&
                      make_residue_map(&m.b1, b1, L, D, units, dil, r, NK) &&
                      make_residue_map(&m.b2, b2, L, D, units, dil, r, NK) &&
                      make_residue_map(&m.o1, o1, L, D, units, dil, r, 32);
            if (ok && o2) ok = make_residue_map(&m.o2, o2, L, D, units, dil, r, 32);
            if (!ok) return cudaErrorInvalidValue;
        }
        p.lse = lse;
        p.D = Dws;
        p.o1 = static_cast<uint16_t*>(o1);
        p.L = L;
        p.w = (int)wc;
        p.dil = (int)dil;

        p.trace = (unsigned long long*)trace_buffer(MODE == NQ ? 1 : 2);
        const int64_t Lr0 = ceil_div(L - r0, dil);
        const int tiles = (int)ceil_div(Lr0, BM);
        const int64_t total = units * nr * tiles;
        dim3 grid((unsigned)(total < num_sms_nb() ? total : num_sms_nb()));
        sched_init(p.sc, L, dil, r0, nr, units, tiles, (int)grid.x);
        p.dpoll = dpoll_enabled();
        p.lsepoll = r0 == 0 && lsepoll_enabled() && lsepoll_worth(total, num_sms_nb());
        if (r0 == 0 && ((MODE == NKV && p.dpoll) || (MODE == NQ && p.lsepoll))) {
            // NKV directly follows this call's last NQ launch: programmatic dependent launch,
            // D handed over row by row
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = grid;
            cfg.blockDim = dim3(NTHREADS);
            cfg.dynamicSmemBytes = SMEM_BYTES;
            cfg.stream = st;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            at[0].val.programmaticStreamSerializationAllowed = 1;
            cfg.attrs = at;
            cfg.numAttrs = 1;
            cudaLaunchKernelEx(&cfg, tc_narrow_bwd_kernel<MODE>, p);
        } else {
            tc_narrow_bwd_kernel<MODE><<<grid, NTHREADS, SMEM_BYTES, st>>>(p);
        }
        prof_mark(st);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        ++n;
    }
    if (launches) *launches += n;
    return cudaSuccess;
}

}  // namespace

cudaError_t tc_narrow_bwd(const void* q, const void* k, const void* v, const float* lse,
                          const void* dout, void* dq, void* dk, void* dv, float* Dws, int64_t B,
                          int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st,
                          int* launches) {
    (void)d;
    // NQ: S = Q K_h^T (a1 = q, b1 = k), dP = dO V_h^T (a2 = dout, b2 = v), dQ = dS K_h (b1)
    cudaError_t e = launch_nb<NQ>(q, dout, k, v, dq, nullptr, lse, Dws, B, H, L, w, dil, st, launches);
    if (e != cudaSuccess) return e;
    // NKV: S^T = K Q_h^T (a1 = k, b1 = q), dP^T = V dO_h^T (a2 = v, b2 = dout);
    //      dV = P^T dO_h (b2) -> o1 = dv, dK = dS^T Q_h (b1) -> o2 = dk
    return launch_nb<NKV>(k, v, q, dout, dv, dk, lse, Dws, B, H, L, w, dil, st, launches);
}

}  // namespace ftw
