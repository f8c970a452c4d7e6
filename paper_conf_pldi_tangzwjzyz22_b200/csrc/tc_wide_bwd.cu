// tc_wide_bwd.cu -- tcgen05/TMEM backward kernels of banded window attention for WIDE
// windows (128 + 2w > 256 halo rows, i.e. w > 64), bf16 storage, fp32 math, d in {64, 128}.
//
// Two persistent kernels, one owner per output row (no atomics; the tile-ownership choice of
// PAPER.md Fig. 13(d) over 13(e)), over 128-row tiles of one (unit, residue) band problem
// and the halo of the other operand streamed in KC = 64-row chunks (the cached a[i:i+m]
// window of PAPER.md Fig. 14):
//
//   WQ   rows = queries.  pass 1 per chunk: S = Q K_c^T, dP = dO V_c^T (TMEM);
//        P = exp(S - lse) (recomputed from the saved lse: selective materialization,
//        PAPER.md:489-497); D += rowsum(P dP) (exact; written to the workspace).
//        pass 2: S, dP again; dS = P (dP - D) as bf16 hi + lo (over S in TMEM);
//        dQ_hi += dS_hi K_c, dQ_lo += dS_lo K_c.
//   WKV  rows = keys, one pass.  S^T = K Q_c^T, dP^T = V dO_c^T; P^T = exp(S^T - lse_col)
//        (bf16, over S^T), dS^T = P^T (dP^T - D_col) (bf16 hi + lo, over dP^T);
//        dV += P^T dO_c, dK += dS^T Q_c.
//
// TMEM rotation: the accumulators take the first ACC columns; the rest is nreg 64-column
// regions.  Step k (global over the CTA) writes S into region (2k) mod nreg and dP into
// (2k+1) mod nreg, so region uses are numbered m = 2k (+1) and use m waits until use
// m - nreg has been freed (rfree[region], phase (m / nreg - 1) & 1).  With nreg = 4..6 the
// score GEMMs of the next 2-3 steps are in flight while the softmax works on this one -- a
// dependent tcgen05.mma chain costs ~350 cycles per instruction (tools/mma_microbench.cu), so
// the score latency must be hidden behind other steps, not waited for.
//
// Roles (512 threads): softmax warps 0-7 (warps w and w+4 share rows 32w.. -- TMEM lane
// quarter w -- and take the two 32-column halves of every step); epilogue warps 8-11;
// warp 12 TMA producer + TMEM allocator; issuers: warp 13 A (S / S^T), warp 14 B (dP / dP^T),
// warp 15 C (the output GEMMs once the softmax of a step is done: dQ, or dV and dK -- B issuing
// dV(k-1) behind dP^T(k) held dV, and with it the S^T region, behind dP^T's region wait).
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

enum { WQ = 0, WKV = 1 };

constexpr int BM = 128;
constexpr int KC = 64;
constexpr int NTHREADS = 512;
constexpr int RES_PER_LAUNCH = 4;
static_assert(RES_PER_LAUNCH <= SCHED_MAX_RES, "residue table of the tile cursor");
constexpr int MAX_RING = 8;
constexpr int MAX_NKT = 4096;          // halo columns per tile (smem column arrays)
constexpr uint32_t ABOX = 128 * 128;   // 128-row x 64-col bf16 box (row operands)
constexpr uint32_t HBOX = 64 * 128;    // 64-row x 64-col bf16 box (halo chunks)
constexpr uint32_t STG = 32 * 128;     // one epilogue warp's 32-row x 64-col staging slice
constexpr float LOG2E = 1.4426950408889634f;
constexpr size_t SMEM_LIMIT = 227 * 1024;

struct BMaps {
    CUtensorMap a1, a2, b1, b2, o1, o2;
};
struct BParams {
    BMaps maps[RES_PER_LAUNCH];
    const float* lse;
    float* D;       // WQ: written; WKV: read
    int64_t L;
    int d, w, dil, nkc;
    SchedParams sc;
    int na, n1, n2;   // row-operand buffers, ring-1 / ring-2 slots
    int wqc;          // WQ in one pass with the D correction (see the header); 0: two passes
    const uint16_t* dout;   // WQ (wqc): raw dout / out rows for D~ = dout . out
    const uint16_t* out;
    unsigned long long* trace;   // optional phase trace (ft_winattn_debug_trace, mode 1 / 2)
    int dpoll;                   // D hand-off by row polling (tc_common.cuh ld_D_ready)
};

// Phase trace, per CTA and local tile j < 8, 48 uint64 slots (ns sums over the tile):
// softmax warp 0: 0 tile start, 1 S/dP wait, 2 compute, 6 tile end; issuer A: 10 region
// wait, 11 ring wait; issuer B: 14 region wait, 15 ring wait; issuer C: 20 p_full wait,
// 21 o_empty wait; epilogue: 30 o_full seen, 31 done.
__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ void trace_put(const BParams& p, int j, int slot, unsigned long long v) {
    if (p.trace && j < 8) p.trace[((size_t)blockIdx.x * 8 + j) * 48 + slot] = v;
}

using Tile = SchedTile;
using TileCursor = SchedCursor<BM>;
struct Ring {
    int s = 0;
    uint32_t ph = 0;
    __device__ void adv(int n) { if (++s == n) { s = 0; ph ^= 1u; } }
};

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ void split_bf16x2(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    split_bf16x2_p(x0, x1, hi, lo);   // tc_common.cuh: one packed subtraction
}

// WQ: dQ + with wqc the PK = sum_j P_ij k_j accumulator (at column d); WKV: dV, dK (at d).  The
// hi and lo products of dS share one accumulator (d = 64 had them in two partials, which cost a
// 64-column TMEM region: 5 instead of 6 regions of score-GEMM lookahead)
template <int MODE> __host__ __device__ inline int acc_cols(int d, int wqc) {
    return MODE == WQ ? d + (wqc ? d : 0) : 2 * d;
}
template <int MODE> __host__ __device__ inline int n_regions(int d, int wqc) { return (512 - acc_cols<MODE>(d, wqc)) / 64; }
__host__ __device__ inline uint32_t row_bytes(int d) { return (uint32_t)(d / 64) * ABOX; }
__host__ __device__ inline uint32_t slot_bytes(int d) { return (uint32_t)(d / 64) * HBOX; }
template <int MODE> inline size_t fixed_bytes(int d, int nkc) {
    return 1024 + 4 * (size_t)(d / 64) * STG + (MODE == WKV ? 2 * (size_t)nkc * KC * sizeof(float) : 0) +
           6 * 128 * sizeof(float) + 1024;
}

template <int MODE>
__global__ void __launch_bounds__(NTHREADS, 1) tc_wide_bwd_kernel(const __grid_constant__ BParams p) {
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int d = p.d, w = p.w, nkc = p.nkc, nds = d / 64;
    const bool wqc = MODE == WQ && p.wqc;
    const int ACC = acc_cols<MODE>(d, p.wqc), NREG = n_regions<MODE>(d, p.wqc);
    if (MODE == WQ && p.dpoll) {   // this CTA's D rows: unset, before WKV may launch
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
    if (MODE == WQ) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int nsteps = (MODE == WQ && !wqc ? 2 : 1) * nkc;   // steps per tile
    const uint32_t RB = row_bytes(d), SB = slot_bytes(d);
    const int NKt = nkc * KC;

    uint8_t* sA = smem;                                   // [na][a1, a2] row operands
    uint8_t* sR1 = sA + (size_t)p.na * 2 * RB;            // ring 1 (K_c / Q_c)
    uint8_t* sR2 = sR1 + (size_t)p.n1 * SB;               // ring 2 (V_c / dO_c)
    uint8_t* ostg = sR2 + (size_t)p.n2 * SB;              // [4 warps][nds] staging
    float* colLse = reinterpret_cast<float*>(ostg + 4 * nds * STG);   // WKV [NKt] (log2 units)
    float* colD = colLse + (MODE == WKV ? NKt : 0);                   // WKV [NKt]
    float* Dx = colD + (MODE == WKV ? NKt : 0);                       // WQ [2 halves][128]
    float* Dt = Dx + 2 * 128;                                         // WQ [2 tiles][128]: D~
    float* dlt = Dt + 2 * 128;                                        // WQ [2 tiles][128]: D - D~
    uint64_t* bars = reinterpret_cast<uint64_t*>(dlt + 2 * 128);
    uint64_t* a_full = bars;                  // [2]
    uint64_t* a_empty = bars + 2;             // [2]
    uint64_t* r1_full = bars + 4;             // [MAX_RING]
    uint64_t* r1_empty = r1_full + MAX_RING;
    uint64_t* r2_full = r1_empty + MAX_RING;
    uint64_t* r2_empty = r2_full + MAX_RING;
    uint64_t* s_full = r2_empty + MAX_RING;   // [4] S of step gk (slot gk & 3)
    uint64_t* dp_full = s_full + 4;           // [4] dP of step gk
    uint64_t* p_full = dp_full + 4;           // [4] softmax done with step gk (256)
    uint64_t* rfree = p_full + 4;             // [8] TMEM region freed
    uint64_t* o_full = rfree + 8;             // accumulators complete
    uint64_t* o_empty = o_full + 1;           // accumulators drained (128)
    uint64_t* d_full = o_empty + 1;           // [2] WQ (wqc): D - D~ of the tile published (256)
    uint64_t* dt_full = d_full + 2;           // [2] WQ (wqc): D~ of the tile published (128)
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(dt_full + 2);

    if (warp == 12) {
        if (lane == 0) {
            for (int i = 0; i < 2; ++i) { mbar_init(&a_full[i], 1); mbar_init(&a_empty[i], 2); }
            for (int i = 0; i < MAX_RING; ++i) {
                mbar_init(&r1_full[i], 1);
                mbar_init(&r1_empty[i], 2);   // issuer A (score GEMM) and C (output GEMM)
                mbar_init(&r2_full[i], 1);
                mbar_init(&r2_empty[i], 1);   // issuer B
            }
            for (int i = 0; i < 4; ++i) {
                mbar_init(&s_full[i], 1);
                mbar_init(&dp_full[i], 1);
                mbar_init(&p_full[i], 256);
            }
            for (int i = 0; i < 8; ++i) mbar_init(&rfree[i], 1);
            mbar_init(o_full, 1);
            mbar_init(o_empty, 128);
            mbar_init(&d_full[0], 256);
            mbar_init(&d_full[1], 256);
            mbar_init(&dt_full[0], 128);
            mbar_init(&dt_full[1], 128);
            fence_barrier_init();
            for (int i = 0; i < p.sc.nr; ++i) {
                const BMaps& m = p.maps[i];
                tma_prefetch(&m.a1); tma_prefetch(&m.a2); tma_prefetch(&m.b1); tma_prefetch(&m.b2);
                tma_prefetch(&m.o1);
                if (MODE == WKV) tma_prefetch(&m.o2);
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
    // region of use m (m = 2 gk for S, 2 gk + 1 for dP); wait for use m - NREG to be freed
    auto region_col = [&](int m) -> uint32_t { return (uint32_t)(ACC + (m % NREG) * 64); };
    auto wait_region = [&](int m) {
        if (m >= NREG) {
            mbar_wait(&rfree[m % NREG], ((m / NREG) - 1) & 1);
            tc_fence_after();
        }
    };
    // halo chunk c of a tile spans residue rows m0 - w + 64c ..
    const uint32_t idS = idesc_bf16(128, KC, false, false);
    const uint32_t idO = idesc_bf16(128, d, false, true);

    if (warp == 12) {
        if (lane == 0) {   // ------------------------------------------------ TMA producer
            Ring r1, r2;
            int j = 0;
            TileCursor cur(p.sc);
            Tile T;
            while (cur.next(p.sc, T)) {
                const BMaps& mp = p.maps[T.rl];
                const int ab = j % p.na;
                if (j >= p.na) mbar_wait(&a_empty[ab], ((j / p.na) - 1) & 1);
                mbar_arrive_expect_tx(&a_full[ab], 2 * RB);
                uint8_t* a = sA + (size_t)ab * 2 * RB;
                for (int s = 0; s < nds; ++s) {
                    tma_load_3d(a + s * ABOX, &mp.a1, &a_full[ab], s * 64, T.m0, T.u);
                    tma_load_3d(a + RB + s * ABOX, &mp.a2, &a_full[ab], s * 64, T.m0, T.u);
                }
                for (int k = 0; k < nsteps; ++k) {
                    const int row = T.m0 - w + (k % nkc) * KC;
                    mbar_wait(&r1_empty[r1.s], r1.ph ^ 1u);
                    mbar_arrive_expect_tx(&r1_full[r1.s], SB);
                    for (int s = 0; s < nds; ++s)
                        tma_load_3d(sR1 + (size_t)r1.s * SB + s * HBOX, &mp.b1, &r1_full[r1.s], s * 64, row, T.u);
                    r1.adv(p.n1);
                    mbar_wait(&r2_empty[r2.s], r2.ph ^ 1u);
                    mbar_arrive_expect_tx(&r2_full[r2.s], SB);
                    for (int s = 0; s < nds; ++s)
                        tma_load_3d(sR2 + (size_t)r2.s * SB + s * HBOX, &mp.b2, &r2_full[r2.s], s * 64, row, T.u);
                    r2.adv(p.n2);
                }
                ++j;
            }
        }
    } else if (warp == 13 || warp == 14) {
        if (lane == 0) {   // ------------------------------- issuers A (S) and B (dP, dV)
            const bool isA = warp == 13;
            Ring rr;   // ring 1 (A) or ring 2 (B)
            int j = 0, gk = 0;
            TileCursor cur(p.sc);
            Tile T;
            while (cur.next(p.sc, T)) {
                const int ab = j % p.na;
                mbar_wait(&a_full[ab], (j / p.na) & 1);
                tc_fence_after();
                const uint32_t sa = smem_u32(sA + (size_t)ab * 2 * RB + (isA ? 0 : RB));
                const bool tr = p.trace && j < 8;
                unsigned long long wr = 0, wf = 0, t0 = 0;
                for (int k = 0; k < nsteps; ++k, ++gk) {
                    const int m = 2 * gk + (isA ? 0 : 1);
                    if (tr) t0 = gtime();
                    wait_region(m);
                    if (tr) { wr += gtime() - t0; t0 = gtime(); }
                    uint64_t* fullb = isA ? r1_full : r2_full;
                    mbar_wait(&fullb[rr.s], rr.ph);
                    tc_fence_after();
                    if (tr) wf += gtime() - t0;
                    const uint32_t sb = smem_u32((isA ? sR1 : sR2) + (size_t)rr.s * SB);
                    const uint32_t td = tbase + region_col(m);
                    for (int s = 0; s < nds; ++s)
                        mma_ss_x4<2, 2>(td, sdesc_sw128(sa + s * ABOX, 16, 1024),
                                        sdesc_sw128(sb + s * HBOX, 16, 1024), idS, s != 0);
                    mma_commit(isA ? &s_full[gk & 3] : &dp_full[gk & 3]);
                    if (isA) mma_commit(&r1_empty[rr.s]);
                    else if (MODE == WQ) mma_commit(&r2_empty[rr.s]);
                    rr.adv(isA ? p.n1 : p.n2);
                }
                mma_commit(&a_empty[ab]);
                if (tr) { trace_put(p, j, isA ? 10 : 14, wr); trace_put(p, j, isA ? 11 : 15, wf); }
                ++j;
            }
        }
    } else if (warp == 15) {
        if (lane == 0) {   // ------------------------------------------------ issuer C: dQ / dK
            Ring r1;
            int j = 0, gk = 0;
            TileCursor cur(p.sc);
            Tile T;
            // dQ (WQ, dS hi/lo over S) or dK (WKV, dS^T hi/lo over dP^T): hi and lo products
            // into one accumulator at column 0 (+ d for dK)
            const uint32_t acc_hi = MODE == WQ ? 0u : (uint32_t)d;
            const uint32_t acc_lo = acc_hi;
            Ring rv;   // WKV: ring 2 (dO_c), read again here by dV = P^T dO_c after issuer B's dP^T
            while (cur.next(p.sc, T)) {
                int outk = 0;   // output steps issued in this tile
                const bool tr = p.trace && j < 8;
                unsigned long long wp = 0, wo = 0, t0 = 0;
                for (int k = 0; k < nsteps; ++k, ++gk) {
                    if (tr) t0 = gtime();
                    mbar_wait(&p_full[gk & 3], (gk >> 2) & 1);
                    tc_fence_after();
                    if (tr) wp += gtime() - t0;
                    const bool out = MODE == WKV || wqc || k >= nkc;
                    const int mS = 2 * gk, mD = 2 * gk + 1;
                    if (!out) {   // WQ pass 1: the softmax only read S and dP
                        mbar_arrive(&rfree[mS % NREG]);
                        mbar_arrive(&rfree[mD % NREG]);
                        mbar_arrive(&r1_empty[r1.s]);
                        r1.adv(p.n1);
                        continue;
                    }
                    if (tr) t0 = gtime();
                    if (outk == 0 && j > 0) { mbar_wait(o_empty, (j - 1) & 1); tc_fence_after(); }
                    if (tr) wo += gtime() - t0;
                    if (MODE == WKV) {   // dV += P^T dO_c, P^T packed bf16 in the S region
                        mbar_wait(&r2_full[rv.s], rv.ph);   // (landed long ago: issuer B's dP^T read it)
                        tc_fence_after();
                        const uint32_t sv = smem_u32(sR2 + (size_t)rv.s * SB);
                        mma_ts_x4o<8, 32, 40, 128>(tbase, tbase + region_col(mS), sdesc_sw128(sv, HBOX, 1024), idO,
                                                   outk == 0 ? 0u : 1u);
                        mma_commit(&rfree[mS % NREG]);
                        mma_commit(&r2_empty[rv.s]);
                        rv.adv(p.n2);
                    }
                    const uint32_t xa = region_col(MODE == WQ ? mS : mD);   // dS (hi/lo) region
                    const uint32_t sb = smem_u32(sR1 + (size_t)r1.s * SB);
                    {   // K-steps kk = 0..3 of the 64-key chunk: A columns 0, 8, 32, 40 (hi;
                        // lo at +16), B rows 16 kk (2048 B = 128 descriptor units per step)
                        const uint64_t bd = sdesc_sw128(sb, HBOX, 1024);
                        const uint32_t ta = tbase + xa;
                        const uint32_t acc = outk == 0 ? 0u : 1u;
                        mma_ts_x4o<8, 32, 40, 128>(tbase + acc_hi, ta, bd, idO, acc);
                        mma_ts_x4o<8, 32, 40, 128>(tbase + acc_lo, ta + 16, bd, idO, 1u);
                        if (wqc)   // PK += P K_c, P (bf16) packed over dP
                            mma_ts_x4o<8, 32, 40, 128>(tbase + (uint32_t)d, tbase + region_col(mD), bd, idO, acc);
                    }
                    mma_commit(&rfree[(MODE == WQ ? mS : mD) % NREG]);
                    if (MODE == WQ) {
                        if (wqc) mma_commit(&rfree[mD % NREG]);   // P read by the PK MMAs
                        else mbar_arrive(&rfree[mD % NREG]);      // dP only read by the softmax
                    }
                    mma_commit(&r1_empty[r1.s]);
                    r1.adv(p.n1);
                    ++outk;
                }
                mma_commit(o_full);
                if (tr) { trace_put(p, j, 20, wp); trace_put(p, j, 21, wo); }
                ++j;
            }
        }
    } else if (warp < 8) {   // ------------------------------------------- softmax warps
        const int wq = warp & 3, hf = warp >> 2;   // lane quarter; 32-column half of a step
        const int t = wq * 32 + lane;
        const uint32_t lrow = (uint32_t)(wq * 32) << 16;
        int j = 0, gk = 0;
        TileCursor cur(p.sc);
        Tile T;
        const int hlo = 32 * wq;   // warp-uniform band extent of rows 32*wq..: [hlo, hlo+31+2w]
        while (cur.next(p.sc, T)) {
            const int Lr = T.Lr, m0 = T.m0, mrow = m0 + t, kb = m0 - w;
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;
            float lse2 = 0.f, D = 0.f;
            if (MODE == WKV) {   // per-column lse (log2 units) and D of this tile's halo
                named_bar_sync(1, 256);   // every softmax warp is done with the previous tile
                for (int n = warp * 32 + lane; n < NKt; n += 256) {
                    const int mc = kb + n;
                    const bool ok = mc >= 0 && mc < Lr;
                    colLse[n] = ok ? p.lse[rowbase + (int64_t)mc * p.dil] * LOG2E : 0.f;
                    colD[n] = !ok ? 0.f
                              : p.dpoll ? ld_D_first(p.D + rowbase + (int64_t)mc * p.dil)
                                        : p.D[rowbase + (int64_t)mc * p.dil];
                }
                if (p.dpoll)   // rows whose WQ tile had not stored D yet
                    for (int n = warp * 32 + lane; n < NKt; n += 256)
                        if (__float_as_uint(colD[n]) == D_UNSET)
                            colD[n] = ld_D_ready(p.D + rowbase + (int64_t)(kb + n) * p.dil);
                named_bar_sync(1, 256);
            } else {
                lse2 = mrow < Lr ? p.lse[rowbase + (int64_t)mrow * p.dil] * LOG2E : 0.f;
            }
            float Dtil = 0.f, Dex = 0.f;   // wqc: D~ (from the epilogue warps), exact D
            const bool tr = p.trace && j < 8 && warp == 0 && lane == 0;
            unsigned long long ws = 0, wc = 0, t0 = 0, t1 = 0;
            if (tr) trace_put(p, j, 0, gtime());
            for (int k = 0; k < nsteps; ++k, ++gk) {
                const int c = k % nkc;
                const bool pass2 = MODE == WQ && (wqc || k >= nkc);
                if (MODE == WQ && !wqc && k == nkc) {   // end of pass 1: D of the whole row
                    Dx[hf * 128 + t] = D;
                    named_bar_sync(1 + wq, 64);
                    D = Dx[t] + Dx[128 + t];
                    if (hf == 0 && mrow < Lr) p.D[rowbase + (int64_t)mrow * p.dil] = D;
                }
                const uint32_t xs = tbase + lrow + region_col(2 * gk) + 32u * hf;
                const uint32_t xd = tbase + lrow + region_col(2 * gk + 1) + 32u * hf;
                if (tr) t0 = gtime();
                mbar_wait(&s_full[gk & 3], (gk >> 2) & 1);
                mbar_wait(&dp_full[gk & 3], (gk >> 2) & 1);
                tc_fence_after();
                if (tr) { t1 = gtime(); ws += t1 - t0; t0 = t1; }
                const int h0 = c * KC + 32 * hf;   // first halo column of my 32
                if (wqc && k == 0) {   // D~ = dout_i . out_i, computed by the epilogue warps
                    mbar_wait(&dt_full[j & 1], (j >> 1) & 1);
                    Dtil = Dt[(j & 1) * 128 + t];
                }
                uint32_t rs[32], rd[32];
                tmem_ld32(xs, rs);
                tmem_ld32(xd, rd);
                tmem_wait_ld();
                // columns outside this row's band or the sequence -> score -inf (P = 0)
                const bool inner = h0 >= hlo + 31 && h0 + 31 <= hlo + 2 * w && kb + h0 >= 0 && kb + h0 + 31 < Lr;
                if (!inner) {
                    const int lo = max(max(t - h0, -kb - h0), 0);
                    const int hi = min(min(t + 2 * w - h0, Lr - 1 - kb - h0), 31);
                    const uint32_t bits = hi < lo ? 0u : ((0xffffffffu >> (31 - hi)) & (0xffffffffu << lo));
#pragma unroll
                    for (int e = 0; e < 32; ++e)
                        if (!((bits >> e) & 1u)) rs[e] = 0xff800000u;
                }
                if (MODE == WQ && !pass2) {
                    float d2[2] = {0.f, 0.f};
#pragma unroll
                    for (int e = 0; e < 32; ++e) {
                        const float pv = fast_exp2(fmaf(__uint_as_float(rs[e]), LOG2E, -lse2));
                        d2[e & 1] = fmaf(pv, __uint_as_float(rd[e]), d2[e & 1]);
                    }
                    D += d2[0] + d2[1];
                } else if (MODE == WQ) {
                    // two-pass: dS = P (dP - D) with the exact D of pass 1.  wqc: dS~ = P (dP - D~),
                    // the exact D accumulated on the way, and P (bf16) over dP for PK
                    const float Dsub = wqc ? Dtil : D;
                    uint32_t ph[16], pl[16], pp[16];
                    float dd[2] = {0.f, 0.f};
#pragma unroll
                    for (int e = 0; e < 32; e += 2) {   // packed f32x2 pairs: FFMA2 / FMUL2
                        const float dp0 = __uint_as_float(rd[e]), dp1 = __uint_as_float(rd[e + 1]);
                        float a0, a1;
                        ffma2_bc(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, -lse2, a0, a1);
                        const float p0 = fast_exp2(a0), p1 = fast_exp2(a1);
                        if (wqc) {
                            ffma2(p0, p1, dp0, dp1, dd[0], dd[1], dd[0], dd[1]);
                            pp[e / 2] = pack_bf16x2(p0, p1);
                        }
                        float q0, q1, r0, r1;
                        ffma2_bc(dp0, dp1, 1.f, -Dsub, q0, q1);   // dP - D (exact: a single rounding)
                        fmul2(p0, p1, q0, q1, r0, r1);
                        split_bf16x2(r0, r1, ph[e / 2], pl[e / 2]);
                    }
                    if (wqc) Dex += dd[0] + dd[1];
                    tmem_st16(xs, ph);
                    tmem_st16(xs + 16, pl);
                    if (wqc) tmem_st16(xd, pp);
                } else {   // WKV: P^T over S^T, dS^T hi/lo over dP^T
                    uint32_t pk[16], ph[16], pl[16];
#pragma unroll
                    for (int e = 0; e < 32; e += 2) {
                        const float4 cl = *reinterpret_cast<const float4*>(&colLse[h0 + (e & ~3)]);
                        const float4 cd = *reinterpret_cast<const float4*>(&colD[h0 + (e & ~3)]);
                        const float l0 = (e & 2) ? cl.z : cl.x, l1 = (e & 2) ? cl.w : cl.y;
                        const float dd0 = (e & 2) ? cd.z : cd.x, dd1 = (e & 2) ? cd.w : cd.y;
                        float a0, a1, q0, q1, r0, r1;
                        ffma2(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, LOG2E, -l0, -l1, a0, a1);
                        const float p0 = fast_exp2(a0), p1 = fast_exp2(a1);
                        pk[e / 2] = pack_bf16x2(p0, p1);
                        ffma2(__uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), 1.f, 1.f, -dd0, -dd1, q0, q1);
                        fmul2(p0, p1, q0, q1, r0, r1);
                        split_bf16x2(r0, r1, ph[e / 2], pl[e / 2]);
                    }
                    tmem_st16(xs, pk);
                    tmem_st16(xd, ph);
                    tmem_st16(xd + 16, pl);
                }
                if (MODE == WKV || pass2) tmem_wait_st();
                tc_fence_before();
                mbar_arrive(&p_full[gk & 3]);
                if (tr) wc += gtime() - t0;
            }
            if (wqc) {   // exact D of the row; the epilogue subtracts (D - D~) PK from dQ~
                Dx[hf * 128 + t] = Dex;
                named_bar_sync(1 + wq, 64);
                const float Dfull = Dx[t] + Dx[128 + t];
                if (hf == 0) {
                    dlt[(j & 1) * 128 + t] = Dfull - Dtil;
                    if (mrow < Lr) p.D[rowbase + (int64_t)mrow * p.dil] = Dfull;
                }
                mbar_arrive(&d_full[j & 1]);
            }
            if (tr) { trace_put(p, j, 1, ws); trace_put(p, j, 2, wc); trace_put(p, j, 6, gtime()); }
            ++j;
        }
    } else if (warp < 12) {   // ----------------------------------------- epilogue warps
        const int ew = warp - 8;
        const uint32_t trow = tbase + ((uint32_t)(ew * 32) << 16);
        uint8_t* mystg = ostg + ew * nds * STG;
        int j = 0;
        // wqc: D~_i = dout_i . out_i of a tile's rows (thread <-> row), published one tile
        // ahead of the softmax warps that need it at the tile's first step
        auto publish_dtil = [&](const Tile& X, int jx) {
            const int mr = X.m0 + ew * 32 + lane;
            float acc = 0.f;
            if (mr < X.Lr) {
                const int64_t off = ((int64_t)X.u * p.L + X.r + (int64_t)mr * p.dil) * d;
                const uint4* dr = reinterpret_cast<const uint4*>(p.dout + off);
                const uint4* orr = reinterpret_cast<const uint4*>(p.out + off);
                for (int v = 0; v < d / 8; v += 4) {
                    uint4 a4[4], b4[4];
#pragma unroll
                    for (int x = 0; x < 4; ++x) { a4[x] = dr[v + x]; b4[x] = orr[v + x]; }
#pragma unroll
                    for (int x = 0; x < 4; ++x) {
                        const uint32_t* aw = reinterpret_cast<const uint32_t*>(&a4[x]);
                        const uint32_t* bw = reinterpret_cast<const uint32_t*>(&b4[x]);
#pragma unroll
                        for (int y = 0; y < 4; ++y) {
                            const float2 fa = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&aw[y]));
                            const float2 fb = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&bw[y]));
                            acc = fmaf(fa.x, fb.x, fmaf(fa.y, fb.y, acc));
                        }
                    }
                }
            }
            Dt[(jx & 1) * 128 + ew * 32 + lane] = acc;
            mbar_arrive(&dt_full[jx & 1]);
        };
        TileCursor cur(p.sc), nxt(p.sc);
        Tile T, Tn;
        if (wqc && nxt.next(p.sc, Tn)) publish_dtil(Tn, 0);
        while (cur.next(p.sc, T)) {
            const BMaps& mp = p.maps[T.rl];
            if (wqc && nxt.next(p.sc, Tn)) publish_dtil(Tn, j + 1);
            mbar_wait(o_full, j & 1);
            tc_fence_after();
            float dl = 0.f;   // wqc: D - D~ of this row
            if (wqc) {
                mbar_wait(&d_full[j & 1], (j >> 1) & 1);
                dl = dlt[(j & 1) * 128 + ew * 32 + lane];
            }
            if (ew == 0 && lane == 0) trace_put(p, j, 30, gtime());
            if (lane == 0) tma_store_wait_read<0>();   // staging of the previous tile read
            __syncwarp();
            // WQ: dQ = [0, d);  WKV: dV = [0, d), dK = [d, 2d)
            const int nout = MODE == WKV ? 2 : 1;
            for (int o = 0; o < nout; ++o) {
                const uint32_t c0 = MODE == WQ ? 0u : (o == 0 ? 0u : (uint32_t)d);
                const bool two = false;
                const CUtensorMap* om = o == 0 ? &mp.o1 : &mp.o2;
                for (int s = 0; s < nds; ++s) {
                    uint8_t* stg = mystg + s * STG;
                    if (o == 1) {   // staging reuse within the tile
                        if (lane == 0) tma_store_wait_read<0>();
                        __syncwarp();
                    }
#pragma unroll 1
                    for (int hh = 0; hh < 2; ++hh) {
                        uint32_t v0[32], v1[32], v2[32];
                        const uint32_t col = c0 + (uint32_t)(s * 64 + hh * 32);
                        tmem_ld32(trow + col, v0);
                        if (two) tmem_ld32(trow + col + (uint32_t)d, v1);
                        if (wqc) tmem_ld32(trow + (uint32_t)d + col, v2);   // PK
                        tmem_wait_ld();
                        float acc[32];
#pragma unroll
                        for (int e = 0; e < 32; ++e) {
                            acc[e] = __uint_as_float(v0[e]) + (two ? __uint_as_float(v1[e]) : 0.f);
                            if (wqc) acc[e] = fmaf(-dl, __uint_as_float(v2[e]), acc[e]);
                        }
                        if (o == nout - 1 && s == nds - 1 && hh == 1) {
                            tc_fence_before();
                            mbar_arrive(o_empty);
                        }
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            uint4 val;
                            val.x = pack_bf16x2(acc[8 * q + 0], acc[8 * q + 1]);
                            val.y = pack_bf16x2(acc[8 * q + 2], acc[8 * q + 3]);
                            val.z = pack_bf16x2(acc[8 * q + 4], acc[8 * q + 5]);
                            val.w = pack_bf16x2(acc[8 * q + 6], acc[8 * q + 7]);
                            const int gq = hh * 4 + q;
                            *reinterpret_cast<uint4*>(stg + lane * 128 + ((gq ^ (lane & 7)) * 16)) = val;
                        }
                    }
                    fence_proxy_async_smem();
                    __syncwarp();
                    if (lane == 0) {
                        tma_store_3d(om, stg, s * 64, T.m0 + 32 * ew, T.u);
                        tma_store_commit();
                    }
                }
            }
            if (ew == 0 && lane == 0) trace_put(p, j, 31, gtime());
            ++j;
        }
        if (lane == 0) tma_store_wait_all<0>();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 12) {
        tc_fence_after();
        tmem_dealloc(tbase, 512);
    }
}

int num_sms_b() {
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

// Buffers: two row-operand sets when they fit, then ring slots split evenly (>= 2 each).
template <int MODE>
bool plan(int d, int nkc, int& na, int& n1, int& n2) {
    if (nkc * KC > MAX_NKT) return false;
    const size_t RB = row_bytes(d), SB = slot_bytes(d);
    const size_t fixed = fixed_bytes<MODE>(d, nkc);
    if (fixed >= SMEM_LIMIT) return false;
    const size_t avail = SMEM_LIMIT - fixed;
    for (na = 2; na >= 1; --na) {
        if (avail < (size_t)na * 2 * RB + 4 * SB) continue;
        int n = (int)((avail - (size_t)na * 2 * RB) / SB);
        if (na == 2 && n < 6) continue;   // prefer deeper rings over a second row buffer
        if (n > 2 * MAX_RING) n = 2 * MAX_RING;
        n1 = (n + 1) / 2;
        n2 = n - n1;
        if (n1 > MAX_RING) n1 = MAX_RING;
        if (n2 > MAX_RING) n2 = MAX_RING;
        return true;
    }
    return false;
}

template <int MODE>
cudaError_t launch(const void* a1, const void* a2, const void* b1, const void* b2, void* o1,
                   void* o2, const float* lse, float* D, int64_t B, int64_t H, int64_t L,
                   int64_t d, int64_t w, int64_t dil, int wqc, const void* dout, const void* out,
                   cudaStream_t st, int* launches) {
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_wide_bwd_kernel<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)SMEM_LIMIT);
    });
    const int64_t wc = w < L ? w : L;
    const int nkc = (int)ceil_div(BM + 2 * wc, KC);
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    int na, n1, n2;
    if (!plan<MODE>((int)d, nkc, na, n1, n2)) return cudaErrorInvalidConfiguration;
    int n = 0;
    for (int64_t r0 = 0; r0 < nres; r0 += RES_PER_LAUNCH) {
        BParams p;
        memset(&p, 0, sizeof(p));
        const int nr = (int)(nres - r0 < RES_PER_LAUNCH ? nres - r0 : RES_PER_LAUNCH);
        for (int i = 0; i < nr; ++i) {
            const int64_t r = r0 + i;
            BMaps& m = p.maps[i];
            bool ok = make_residue_map(&m.a1, a1, L, d, units, dil, r, BM) &&
                      make_residue_map(&m.a2, a2, L, d, units, dil, r, BM) &&
                      make_residue_map(&m.b1, b1, L, d, units, dil, r, KC) &&
                      make_residue_map(&m.b2, b2, L, d, units, dil, r, KC) &&
                      make_residue_map(&m.o1, o1, L, d, units, dil, r, 32);
            if (ok && o2) ok = make_residue_map(&m.o2, o2, L, d, units, dil, r, 32);
            if (!ok) return cudaErrorInvalidValue;
        }
        p.lse = lse;
        p.D = D;
        p.L = L;
        p.d = (int)d;
        p.w = (int)wc;
        p.dil = (int)dil;
        p.nkc = nkc;
        p.na = na;
        p.n1 = n1;
        p.n2 = n2;
        p.trace = (unsigned long long*)trace_buffer(MODE == WQ ? 1 : 2);
        p.wqc = MODE == WQ ? wqc : 0;
        p.dout = static_cast<const uint16_t*>(dout);
        p.out = static_cast<const uint16_t*>(out);
        const int64_t Lr0 = ceil_div(L - r0, dil);
        const int tiles = (int)ceil_div(Lr0, BM);
        const int64_t total = units * nr * tiles;
        dim3 grid((unsigned)(total < num_sms_b() ? total : num_sms_b()));
        sched_init(p.sc, L, dil, r0, nr, units, tiles, (int)grid.x);
        const size_t smem = fixed_bytes<MODE>((int)d, nkc) + (size_t)na * 2 * row_bytes((int)d) +
                            (size_t)(n1 + n2) * slot_bytes((int)d);
        p.dpoll = dpoll_enabled();
        if (MODE == WKV && r0 == 0 && p.dpoll) {
            // WKV directly follows this call's last WQ launch on the stream: programmatic
            // dependent launch, D handed over row by row
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = grid;
            cfg.blockDim = dim3(NTHREADS);
            cfg.dynamicSmemBytes = smem;
            cfg.stream = st;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            at[0].val.programmaticStreamSerializationAllowed = 1;
            cfg.attrs = at;
            cfg.numAttrs = 1;
            cudaLaunchKernelEx(&cfg, tc_wide_bwd_kernel<MODE>, p);
        } else {
            tc_wide_bwd_kernel<MODE><<<grid, NTHREADS, smem, st>>>(p);
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

bool tc_wide_bwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    const int64_t wc = w < L ? w : L;
    const int nkc = (int)ceil_div(BM + 2 * wc, KC);
    int na, n1, n2;
    return (d == 64 || d == 128) && dil <= 256 && units * ((L + 127) / 128) < (1 << 30) &&
           plan<WQ>((int)d, nkc, na, n1, n2) && plan<WKV>((int)d, nkc, na, n1, n2);
}

cudaError_t tc_wide_bwd(const void* q, const void* k, const void* v, const void* out,
                        const float* lse, const void* dout, void* dq, void* dk, void* dv, float* Dws,
                        int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                        cudaStream_t st, int* launches) {
    // WQ in one pass with the D correction (reading R1)
    const int wqc = 1;
    // WQ: rows Q (a1) / dO (a2), halo K (b1) / V (b2) -> dQ;  WKV: rows K / V, halo Q / dO -> dV, dK
    cudaError_t e = launch<WQ>(q, dout, k, v, dq, nullptr, lse, Dws, B, H, L, d, w, dil, wqc, dout, out, st,
                               launches);
    if (e != cudaSuccess) return e;
    return launch<WKV>(k, v, q, dout, dv, dk, lse, Dws, B, H, L, d, w, dil, 0, dout, out, st, launches);
}

}  // namespace ftw
