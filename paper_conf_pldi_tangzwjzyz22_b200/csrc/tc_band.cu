// tc_band.cu -- tcgen05/TMEM tensor-core kernels of banded window attention for sm_100a
// (bf16 storage; fp32 scores, softmax statistics and accumulators).
//
// One kernel template, three modes.  A CTA owns BM = 128 rows m0..m0+127 of one
// (unit, residue) band problem and the NK = round_up(128 + 2w, 32) <= 256-row halo
// m0-w .. m0+127+w of the other operand: the cached a[i:i+m] window of PAPER.md Fig. 14
// (lines 402-423), staged by TMA instead of the (2w+1)-fold as_strided copy of Q that the
// operator baseline makes (Fig. 1c).
//
//   FWD   rows = queries.  S = Q K_h^T -> row max, exp, row sum (the fused dot/max of
//         Fig. 10 and dot_norm/softmax of Fig. 8), lse -> HBM,
//         P (bf16) -> TMEM;  O_n = P V_h,n  (n = 64-column d-slices), scaled by 1/l.
//   BWDQ  rows = queries.  S = Q K_h^T, dP = dO V_h^T;  P = exp(S - lse) (recomputed from the
//         saved lse: selective materialization);  D = sum_j P dP (exact,
//         written to the workspace);  dS = P (dP - D) (bf16) -> TMEM;  dQ_n = dS K_h,n.
//   BWDKV rows = keys (tile ownership: each dk/dv row has exactly one writer, no atomics;
//         the parallel-reduction choice of PAPER.md Fig. 13(d) over 13(e)).  S^T = K Q_h^T,
//         dP^T = V dO_h^T;  P^T = exp(S^T - lse_col), dS^T = P^T (dP^T - D_col);
//         dV_n = P^T dO_h,n,  dK_n = dS^T Q_h,n.
//
// Roles (192 threads): warps 0-3 softmax + epilogue (thread t <-> row m0+t <-> TMEM lane t),
// warp 4 TMA producer + TMEM allocator, warp 5 MMA issuer (one elected thread).
// The band geometry: column n of the halo is residue row m0 - w + n, and
// |m_col - m_row| <= w  <=>  0 <= n - t <= 2w, so one mask serves all three modes.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include <mutex>

#include "internal.h"
#include "tc_common.cuh"
#include "tmap.h"

namespace ftw {
namespace {

using namespace tc;

enum { FWD = 0, BWDQ = 1, BWDKV = 2 };

constexpr int BM = 128;

constexpr int RES_PER_LAUNCH = 4;
constexpr uint32_t ABYTES = BM * 128;   // one 128-row x 64-col bf16 slice (SW128)
constexpr float LOG2E = 1.4426950408889634f;
constexpr float LN2 = 0.6931471805599453f;

// TMEM layout (columns).  Score accumulators: S at 0 and dP at 256 (FWD: S of tile j in
// region 256*(j&1), so the next tile's QK^T runs while this tile's softmax + epilogue do).
// The bf16 A operands of the output GEMMs overwrite the scores as they are consumed:
// "compact" = 16 columns per 32-column score chunk, at 16c; "split" = hi/lo bf16 pair
// (x = hi + lo, lo = bf16(x - hi)) in place of chunk c: hi at 32c, lo at 32c+16.  dS is
// split because at large d its entries reach O(10) and one bf16 rounding (2^-9) of them
// would dominate the dq/dk error budget.  Output accumulators (64-column slices) sit outside
// the score regions when NK <= 192 ("out-of-region"), so the next tile's score GEMMs can
// run while the epilogue drains them; otherwise inside, and the next tile waits (tile_done).
template <int MODE> struct Cfg {
    static constexpr int NA = MODE == FWD ? 1 : 2;       // score GEMMs (S, and dP)
    static constexpr int NO = MODE == BWDKV ? 2 : 1;     // output GEMMs per d-slice
    static constexpr int NR = MODE == FWD ? 2 : 1;       // TMEM score regions
    static constexpr int LA = MODE == FWD ? 1 : 0;       // score-GEMM tile lookahead
    static constexpr uint32_t TCOLS = 512;
    static constexpr bool SPLIT0 = MODE == BWDQ;         // A of output GEMM 0 split?
    static constexpr bool SPLIT1 = MODE == BWDKV;        // A of output GEMM 1 split?
    static constexpr int OBUFS = MODE == BWDKV ? 1 : 2;  // TMEM output buffers per output
};

// Column of output accumulator `o`, buffer `b`, for a tile in score region R.
template <int MODE>
__device__ __forceinline__ uint32_t out_col(int o, int b, int R, bool outside) {
    if (MODE == FWD) return 256u * R + 128u + 64u * b;
    if (MODE == BWDQ) return outside ? (b == 0 ? 192u : 448u) : 256u + 64u * b;
    return outside ? (o == 0 ? 192u : 448u) : (o == 0 ? 128u : 192u);   // BWDKV
}

__device__ __forceinline__ uint32_t a_col(bool split, int kk) {
    return split ? 32u * (kk >> 1) + 8u * (kk & 1) : 8u * kk;
}
__device__ __forceinline__ void split_bf16x2(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    __nv_bfloat162 h = __floats2bfloat162_rn(x0, x1);
    const float2 hf = __bfloat1622float2(h);
    hi = *reinterpret_cast<uint32_t*>(&h);
    lo = pack_bf16x2(x0 - hf.x, x1 - hf.y);
}
__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// a1/b1: first score GEMM (A rows m0.., B halo rows m0-w..), a2/b2: second (or, in FWD,
// b2 = V for the output GEMM); o1/o2: outputs (TMA boxes of 32 rows: one per epilogue warp).
struct Maps {
    CUtensorMap a1, b1, a2, b2, o1, o2;
};
struct Params {
    Maps maps[RES_PER_LAUNCH];
    float* lse;   // FWD: written; BWD: read
    float* D;     // BWDQ: written; BWDKV: read
    int64_t L;
    int d, w, dil, r0, nr, NK, nsl, nst, units, tiles;
    unsigned long long* trace;   // optional: [grid][TRACE_TILES][TRACE_EV] globaltimer stamps
};

// Optional phase trace (ft_winattn_debug_trace): per CTA and local tile j < TRACE_TILES,
// globaltimer stamps of: 0 producer first score-GEMM load, 1 producer last output load,
// 2 MMA score GEMM first stage ready, 3 MMA s_full commit, 4 MMA p_full seen,
// 5 MMA last output MMA issued, 6 softmax s_full seen, 7 softmax p_full arrive,
// 8 epilogue first o_full seen, 9 epilogue done.
constexpr int TRACE_TILES = 8, TRACE_EV = 48;
// per-slice (n < 8): 10+n MMA stage-full seen, 18+n MMA o_empty seen, 26+n epilogue o_full
// seen, 34+n epilogue store issued (epilogue warp 0)
__device__ __forceinline__ void trace_ev(const Params& p, int j, int ev) {
    if (p.trace && j < TRACE_TILES) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        p.trace[((size_t)blockIdx.x * TRACE_TILES + j) * TRACE_EV + ev] = t;
    }
}

constexpr int NTHREADS = 320;    // warps 0-3 softmax, 4-7 epilogue, 8 producer, 9 MMA
constexpr uint32_t STG = 32 * 128;   // one warp's 32-row x 64-col bf16 staging slice
constexpr int NSTG = 2;              // staging slices per epilogue warp

template <int MODE>
__host__ __device__ inline uint32_t stage_bytes(int NK) {
    return Cfg<MODE>::NA * (ABYTES + (uint32_t)NK * 128u);
}
template <int MODE>
inline size_t fixed_smem_bytes() {
    return 1024 + 4 * NSTG * STG + 2 * 256 * sizeof(float) + 2 * 128 * sizeof(float) + 512;
}
constexpr int MAX_NST = 8;
constexpr size_t SMEM_LIMIT = 227 * 1024;

template <int MODE>
inline int pick_nst(int NK) {
    const size_t avail = SMEM_LIMIT - fixed_smem_bytes<MODE>();
    int n = (int)(avail / stage_bytes<MODE>(NK));
    return n < MAX_NST ? n : MAX_NST;
}

__device__ __forceinline__ bool band_ok(int n, int t, int w, int mcol, int Lr) {
    return (unsigned)(n - t) <= (unsigned)(2 * w) && mcol >= 0 && mcol < Lr;
}

struct Tile {
    int u, rl, r, Lr, m0;
};
// Tile tau -> (unit, residue, row block); t fastest so concurrently running CTAs work on
// neighbouring row blocks and share their K/V halos through L2.
__device__ __forceinline__ bool decode_tile(const Params& p, int tau, Tile& T) {
    const int t = tau % p.tiles;
    const int rest = tau / p.tiles;
    T.rl = rest % p.nr;
    T.u = rest / p.nr;
    T.r = p.r0 + T.rl;
    T.Lr = (int)((p.L - T.r + p.dil - 1) / p.dil);
    T.m0 = t * BM;
    return T.m0 < T.Lr;
}
// Iterates this CTA's valid tiles in order (static round robin over the grid).
struct TileCursor {
    int tau;
    __device__ explicit TileCursor(int start) : tau(start - (int)gridDim.x) {}
    __device__ bool next(const Params& p, int total, Tile& T) {
        for (tau += gridDim.x; tau < total; tau += gridDim.x)
            if (decode_tile(p, tau, T)) return true;
        return false;
    }
};

template <int MODE>
__global__ void __launch_bounds__(NTHREADS, 1) tc_band_kernel(const __grid_constant__ Params p) {
    using C = Cfg<MODE>;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int NK = p.NK, nsl = p.nsl, w = p.w, NST = p.nst;
    const int total = p.units * p.nr * p.tiles;
    const uint32_t SB = stage_bytes<MODE>(NK);
    const uint32_t HB = (uint32_t)NK * 128u;   // one halo slice
    const bool outside = MODE != FWD && NK <= 192;
    const bool wait_region = !outside;          // next score GEMM must wait for the epilogue

    uint8_t* ostg = smem + NST * SB;                                       // [4 warps][NSTG]
    float* colLse = reinterpret_cast<float*>(ostg + 4 * NSTG * STG);       // BWDKV
    float* colD = colLse + 256;
    float* rowScale = colD + 256;                                          // FWD [2][128]
    uint64_t* bars = reinterpret_cast<uint64_t*>(rowScale + 256);
    uint64_t* full = bars;
    uint64_t* empty = bars + MAX_NST;
    uint64_t* s_full = bars + 2 * MAX_NST;   // [NR]
    uint64_t* p_full = s_full + 2;           // [NR]
    uint64_t* o_full = s_full + 4;           // [2]
    uint64_t* o_empty = s_full + 6;          // [2]
    uint64_t* tile_done = s_full + 8;        // [NR]
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(s_full + 10);

    if (warp == 8) {
        if (lane == 0) {
            for (int i = 0; i < NST; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
            for (int i = 0; i < 2; ++i) {
                mbar_init(&s_full[i], 1);
                mbar_init(&p_full[i], 128);
                mbar_init(&o_full[i], 1);
                mbar_init(&o_empty[i], 128);
                mbar_init(&tile_done[i], 128);
            }
            fence_barrier_init();
            for (int i = 0; i < p.nr; ++i) {
                const Maps& mp = p.maps[i];
                tma_prefetch(&mp.a1); tma_prefetch(&mp.b1); tma_prefetch(&mp.b2); tma_prefetch(&mp.o1);
                if (C::NA == 2) tma_prefetch(&mp.a2);
                if (C::NO == 2) tma_prefetch(&mp.o2);
            }
        }
        __syncwarp();
        tmem_alloc(tmem_holder, C::TCOLS);
        tmem_relinquish();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tbase = *tmem_holder;

    if (warp == 8) {
        if (lane == 0) {   // ------------------------------------------------ TMA producer
            // Load order = MMA consumption order: G(0..LA-1), then per step i: G(i+LA), O(i).
            int st = 0;
            uint32_t ph = 0;
            TileCursor cg(blockIdx.x), co(blockIdx.x);
            Tile Tg, To;
            bool hg = cg.next(p, total, Tg), ho = co.next(p, total, To);
            int jg = 0, jo = 0;
            auto load_g = [&](const Tile& T) {
                const Maps& mp = p.maps[T.rl];
                for (int s = 0; s < nsl; ++s) {
                    mbar_wait(&empty[st], ph ^ 1u);
                    if (s == 0) trace_ev(p, jg, 0);
                    uint8_t* sp = smem + st * SB;
                    mbar_arrive_expect_tx(&full[st], SB);
                    tma_load_3d(sp, &mp.a1, &full[st], s * 64, T.m0, T.u);
                    tma_load_3d(sp + ABYTES, &mp.b1, &full[st], s * 64, T.m0 - w, T.u);
                    if (C::NA == 2) {
                        tma_load_3d(sp + ABYTES + HB, &mp.a2, &full[st], s * 64, T.m0, T.u);
                        tma_load_3d(sp + 2 * ABYTES + HB, &mp.b2, &full[st], s * 64, T.m0 - w, T.u);
                    }
                    if (++st == NST) { st = 0; ph ^= 1u; }
                }
            };
            auto load_o = [&](const Tile& T) {
                const Maps& mp = p.maps[T.rl];
                for (int n = 0; n < nsl; ++n) {
                    mbar_wait(&empty[st], ph ^ 1u);
                    uint8_t* sp = smem + st * SB;
                    mbar_arrive_expect_tx(&full[st], C::NO * HB);
                    // output-GEMM B operands: FWD V (b2), BWDQ K (b1), BWDKV dO (b2) then Q (b1)
                    const CUtensorMap* m_first = MODE == BWDQ ? &mp.b1 : &mp.b2;
                    tma_load_3d(sp, m_first, &full[st], n * 64, T.m0 - w, T.u);
                    if (C::NO == 2) tma_load_3d(sp + HB, &mp.b1, &full[st], n * 64, T.m0 - w, T.u);
                    if (++st == NST) { st = 0; ph ^= 1u; }
                }
                trace_ev(p, jo, 1);
            };
            for (int la = 0; la < C::LA && hg; ++la) { load_g(Tg); ++jg; hg = cg.next(p, total, Tg); }
            while (ho) {
                if (hg) { load_g(Tg); ++jg; hg = cg.next(p, total, Tg); }
                load_o(To); ++jo; ho = co.next(p, total, To);
            }
        }
    } else if (warp == 9) {
        if (lane == 0) {   // ------------------------------------------------ MMA issuer
            const uint32_t idS = idesc_bf16(128, NK, false, false);
            const uint32_t idO = idesc_bf16(128, 64, false, true);
            int st = 0, g = 0;
            uint32_t ph = 0;
            TileCursor cg(blockIdx.x), co(blockIdx.x);
            Tile Tg, To;
            bool hg = cg.next(p, total, Tg), ho = co.next(p, total, To);
            int jg = 0, jo = 0;
            auto mma_g = [&]() {   // score GEMM(s) of local tile jg into its region
                const int R = jg % C::NR;
                const uint32_t tR = tbase + 256u * R;
                if (wait_region && jg >= C::NR) {
                    mbar_wait(&tile_done[R], ((jg / C::NR) - 1) & 1);
                    tc_fence_after();
                }
                for (int s = 0; s < nsl; ++s) {
                    mbar_wait(&full[st], ph);
                    tc_fence_after();
                    if (s == 0) trace_ev(p, jg, 2);
                    const uint32_t a1 = smem_u32(smem + st * SB), b1 = a1 + ABYTES;
                    const uint32_t a2 = b1 + HB, b2 = a2 + ABYTES;
                    // S and dP are independent accumulators: interleave their K-steps so the
                    // tensor core always has two chains in flight
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk) {
                        mma_ss(tR, sdesc_sw128(a1 + kk * 32, 16, 1024),
                               sdesc_sw128(b1 + kk * 32, 16, 1024), idS, (s | kk) != 0);
                        if (C::NA == 2)
                            mma_ss(tbase + 256, sdesc_sw128(a2 + kk * 32, 16, 1024),
                                   sdesc_sw128(b2 + kk * 32, 16, 1024), idS, (s | kk) != 0);
                    }
                    mma_commit(&empty[st]);
                    if (++st == NST) { st = 0; ph ^= 1u; }
                }
                mma_commit(&s_full[R]);
                trace_ev(p, jg, 3);
            };
            auto mma_o = [&]() {   // output GEMMs of local tile jo, 64-column slices
                const int R = jo % C::NR;
                const uint32_t tR = tbase + 256u * R;
                mbar_wait(&p_full[R], (jo / C::NR) & 1);
                tc_fence_after();
                trace_ev(p, jo, 4);
                // Slices are issued in pairs (n, n+1) when both TMEM buffers exist, with
                // their K-steps interleaved: consecutive MMAs then target independent
                // accumulators instead of serialising on one (BWDKV interleaves dV / dK).
                const int pair = C::OBUFS == 2 ? 2 : 1;
                for (int n = 0; n < nsl; n += pair) {
                    const int cnt = min(pair, nsl - n);
                    uint32_t bbs[2], tDs[2][2];
                    int sts[2];
                    for (int q = 0; q < cnt; ++q) {
                        const int gq = g + q, buf = gq % C::OBUFS;
                        if (gq >= C::OBUFS) {
                            mbar_wait(&o_empty[buf], ((gq / C::OBUFS) - 1) & 1);
                            tc_fence_after();
                        }
                        if (n + q < 8) trace_ev(p, jo, 18 + n + q);
                        mbar_wait(&full[st], ph);
                        tc_fence_after();
                        if (n + q < 8) trace_ev(p, jo, 10 + n + q);
                        bbs[q] = smem_u32(smem + st * SB);
                        sts[q] = st;
                        for (int o = 0; o < C::NO; ++o) tDs[q][o] = tbase + out_col<MODE>(o, buf, R, outside);
                        if (++st == NST) { st = 0; ph ^= 1u; }
                    }
                    for (int kk = 0; kk < NK / 16; ++kk) {
                        for (int q = 0; q < cnt; ++q) {
#pragma unroll
                            for (int o = 0; o < C::NO; ++o) {
                                const bool split = o == 0 ? C::SPLIT0 : C::SPLIT1;
                                const uint32_t tA = tR + (o == 0 ? 0u : 256u) + a_col(split, kk);
                                const uint64_t bd = sdesc_sw128(bbs[q] + o * HB + kk * 2048, HB, 1024);
                                mma_ts(tDs[q][o], tA, bd, idO, kk != 0);
                                if (split) mma_ts(tDs[q][o], tA + 16, bd, idO, 1);
                            }
                        }
                    }
                    for (int q = 0; q < cnt; ++q) {
                        mma_commit(&empty[sts[q]]);
                        mma_commit(&o_full[(g + q) % C::OBUFS]);
                    }
                    g += cnt;
                }
                trace_ev(p, jo, 5);
            };
            for (int la = 0; la < C::LA && hg; ++la) { mma_g(); ++jg; hg = cg.next(p, total, Tg); }
            while (ho) {
                if (hg) { mma_g(); ++jg; hg = cg.next(p, total, Tg); }
                mma_o(); ++jo; ho = co.next(p, total, To);
            }
        }
    } else if (warp < 4) {   // ------------------------------------------- softmax warps
        const int t = warp * 32 + lane;
        const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
        const int nch = NK / 32;
        // chunks holding any column of this warp's band rows (warp-uniform): rows
        // 32*warp..32*warp+31 need columns [32*warp, 32*warp + 31 + 2w]
        const int c_lo = warp, c_hi = min(nch - 1, (32 * warp + 31 + 2 * w) / 32);
        TileCursor cur(blockIdx.x);
        Tile T;
        int j = 0;
        while (cur.next(p, total, T)) {
            const int R = j % C::NR;
            const uint32_t trow = tbase + lane_off + 256u * R;   // score region of this tile
            const uint32_t trow0 = tbase + lane_off;
            const int Lr = T.Lr, m0 = T.m0;
            const int mrow = m0 + t;
            const int kb = m0 - w;   // residue index of halo column 0
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;   // flat row of m = 0

            if (MODE == BWDKV) {
                named_bar_sync(1, 128);   // everyone is done with the previous tile's columns
                for (int n = t; n < NK; n += 128) {
                    const int mc = kb + n;
                    const bool ok = mc >= 0 && mc < Lr;
                    colLse[n] = ok ? p.lse[rowbase + (int64_t)mc * p.dil] * LOG2E : 0.f;
                    colD[n] = ok ? p.D[rowbase + (int64_t)mc * p.dil] : 0.f;
                }
                named_bar_sync(1, 128);
            }
            mbar_wait(&s_full[R], (j / C::NR) & 1);
            tc_fence_after();
            if (t == 0) trace_ev(p, j, 6);
            uint32_t zero16[16];
#pragma unroll
            for (int e = 0; e < 16; ++e) zero16[e] = 0u;

            if (MODE == FWD) {
                float mx = -INFINITY;
                for (int c = c_lo; c <= c_hi; ++c) {
                    uint32_t rr[32];
                    tmem_ld32(trow + c * 32, rr);
                    tmem_wait_ld();
#pragma unroll
                    for (int e = 0; e < 32; ++e) {
                        const int n = c * 32 + e;
                        if (band_ok(n, t, w, kb + n, Lr)) mx = fmaxf(mx, __uint_as_float(rr[e]));
                    }
                }
                if (mx == -INFINITY) mx = 0.f;   // only rows beyond the sequence (never stored)
                const float mxs = mx * LOG2E;
                float sum = 0.f;
                for (int c = 0; c < nch; ++c) {
                    if (c < c_lo || c > c_hi) { tmem_st16(trow + c * 16, zero16); continue; }
                    uint32_t rr[32], pk[16];
                    tmem_ld32(trow + c * 32, rr);
                    tmem_wait_ld();
#pragma unroll
                    for (int e = 0; e < 32; e += 2) {
                        float pv[2];
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
                            const int n = c * 32 + e + h;
                            pv[h] = band_ok(n, t, w, kb + n, Lr)
                                        ? fast_exp2(fmaf(__uint_as_float(rr[e + h]), LOG2E, -mxs))
                                        : 0.f;
                            sum += pv[h];
                        }
                        pk[e / 2] = pack_bf16x2(pv[0], pv[1]);
                    }
                    tmem_st16(trow + c * 16, pk);
                }
                rowScale[R * 128 + t] = 1.f / sum;
                tmem_wait_st();
                tc_fence_before();
                mbar_arrive(&p_full[R]);
                if (mrow < Lr) p.lse[rowbase + (int64_t)mrow * p.dil] = (mxs + log2f(sum)) * LN2;
            } else if (MODE == BWDQ) {
                const float lse2 = mrow < Lr ? p.lse[rowbase + (int64_t)mrow * p.dil] * LOG2E : 0.f;
                float D = 0.f;
                for (int c = c_lo; c <= c_hi; ++c) {   // pass 1: D = sum_j P_ij dP_ij
                    uint32_t rs[32], rd[32];
                    tmem_ld32(trow + c * 32, rs);
                    tmem_ld32(trow0 + 256 + c * 32, rd);
                    tmem_wait_ld();
#pragma unroll
                    for (int e = 0; e < 32; ++e) {
                        const int n = c * 32 + e;
                        const float pv = band_ok(n, t, w, kb + n, Lr)
                                             ? fast_exp2(fmaf(__uint_as_float(rs[e]), LOG2E, -lse2))
                                             : 0.f;
                        D = fmaf(pv, __uint_as_float(rd[e]), D);
                    }
                }
                for (int c = 0; c < nch; ++c) {   // pass 2: dS = P (dP - D) -> TMEM (bf16 hi/lo)
                    if (c < c_lo || c > c_hi) {
                        tmem_st16(trow + c * 32, zero16);
                        tmem_st16(trow + c * 32 + 16, zero16);
                        continue;
                    }
                    uint32_t rs[32], rd[32], pk[16], pl[16];
                    tmem_ld32(trow + c * 32, rs);
                    tmem_ld32(trow0 + 256 + c * 32, rd);
                    tmem_wait_ld();
#pragma unroll
                    for (int e = 0; e < 32; e += 2) {
                        float dv[2];
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
                            const int n = c * 32 + e + h;
                            const float pv = band_ok(n, t, w, kb + n, Lr)
                                                 ? fast_exp2(fmaf(__uint_as_float(rs[e + h]), LOG2E, -lse2))
                                                 : 0.f;
                            dv[h] = pv * (__uint_as_float(rd[e + h]) - D);
                        }
                        split_bf16x2(dv[0], dv[1], pk[e / 2], pl[e / 2]);
                    }
                    tmem_st16(trow + c * 32, pk);
                    tmem_st16(trow + c * 32 + 16, pl);
                }
                tmem_wait_st();
                tc_fence_before();
                mbar_arrive(&p_full[R]);
                if (mrow < Lr) p.D[rowbase + (int64_t)mrow * p.dil] = D;
            } else {   // BWDKV: rows are keys, columns are halo queries
                for (int c = 0; c < nch; ++c) {
                    if (c < c_lo || c > c_hi) {
                        tmem_st16(trow + c * 16, zero16);
                        tmem_st16(trow0 + 256 + c * 32, zero16);
                        tmem_st16(trow0 + 256 + c * 32 + 16, zero16);
                        continue;
                    }
                    uint32_t rs[32], rd[32], pk[16], dk[16], dl[16];
                    tmem_ld32(trow + c * 32, rs);
                    tmem_ld32(trow0 + 256 + c * 32, rd);
                    tmem_wait_ld();
#pragma unroll
                    for (int e = 0; e < 32; e += 2) {
                        float pv[2], dv[2];
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
                            const int n = c * 32 + e + h;
                            pv[h] = band_ok(n, t, w, kb + n, Lr)
                                        ? fast_exp2(fmaf(__uint_as_float(rs[e + h]), LOG2E, -colLse[n]))
                                        : 0.f;
                            dv[h] = pv[h] * (__uint_as_float(rd[e + h]) - colD[n]);
                        }
                        pk[e / 2] = pack_bf16x2(pv[0], pv[1]);
                        split_bf16x2(dv[0], dv[1], dk[e / 2], dl[e / 2]);
                    }
                    tmem_st16(trow + c * 16, pk);
                    tmem_st16(trow0 + 256 + c * 32, dk);
                    tmem_st16(trow0 + 256 + c * 32 + 16, dl);
                }
                tmem_wait_st();
                tc_fence_before();
                mbar_arrive(&p_full[R]);
            }
            if (t == 0) trace_ev(p, j, 7);
            ++j;
        }
    } else if (warp < 8) {   // ------------------------------------------ epilogue warps
        const int ew = warp - 4;   // TMEM lanes 32*ew .. 32*ew+31  (warp % 4 == ew)
        const uint32_t trow0 = tbase + ((uint32_t)(ew * 32) << 16);
        uint8_t* mystg = ostg + ew * NSTG * STG;
        TileCursor cur(blockIdx.x);
        Tile T;
        int j = 0, g = 0, sidx = 0;
        while (cur.next(p, total, T)) {
            const Maps& mp = p.maps[T.rl];
            const int R = j % C::NR;
            float scale = 1.f;
            if (MODE == FWD) {   // 1/l of this row, published before p_full
                mbar_wait(&p_full[R], (j / C::NR) & 1);
                scale = rowScale[R * 128 + ew * 32 + lane];
            }
            for (int n = 0; n < nsl; ++n, ++g) {
                const int buf = g % C::OBUFS;
                mbar_wait(&o_full[buf], (g / C::OBUFS) & 1);
                tc_fence_after();
                if (lane == 0 && ew == 0 && n == 0) trace_ev(p, j, 8);
                if (lane == 0 && ew == 0 && n < 8) trace_ev(p, j, 26 + n);
#pragma unroll
                for (int o = 0; o < C::NO; ++o) {
                    uint32_t ov[64];
                    const uint32_t tcol = out_col<MODE>(o, buf, R, outside);
                    tmem_ld32(trow0 + tcol, *reinterpret_cast<uint32_t(*)[32]>(&ov[0]));
                    tmem_ld32(trow0 + tcol + 32, *reinterpret_cast<uint32_t(*)[32]>(&ov[32]));
                    tmem_wait_ld();
                    if (o == C::NO - 1) {
                        tc_fence_before();
                        mbar_arrive(&o_empty[buf]);
                        if (n == nsl - 1) mbar_arrive(&tile_done[R]);
                    }
                    uint8_t* stg = mystg + (sidx % NSTG) * STG;
                    if (lane == 0 && sidx >= NSTG) tma_store_wait_read<NSTG - 1>();
                    __syncwarp();
#pragma unroll
                    for (int c = 0; c < 8; ++c) {
                        uint4 val;
                        val.x = pack_bf16x2(__uint_as_float(ov[8 * c + 0]) * scale, __uint_as_float(ov[8 * c + 1]) * scale);
                        val.y = pack_bf16x2(__uint_as_float(ov[8 * c + 2]) * scale, __uint_as_float(ov[8 * c + 3]) * scale);
                        val.z = pack_bf16x2(__uint_as_float(ov[8 * c + 4]) * scale, __uint_as_float(ov[8 * c + 5]) * scale);
                        val.w = pack_bf16x2(__uint_as_float(ov[8 * c + 6]) * scale, __uint_as_float(ov[8 * c + 7]) * scale);
                        *reinterpret_cast<uint4*>(stg + lane * 128 + ((c ^ (lane & 7)) * 16)) = val;
                    }
                    fence_proxy_async_smem();
                    __syncwarp();
                    if (lane == 0) {
                        tma_store_3d(o == 1 ? &mp.o2 : &mp.o1, stg, n * 64, T.m0 + 32 * ew, T.u);
                        tma_store_commit();
                        if (ew == 0 && n < 8 && o == C::NO - 1) trace_ev(p, j, 34 + n);
                    }
                    ++sidx;
                }
            }
            if (lane == 0 && ew == 0) trace_ev(p, j, 9);
            ++j;
        }
        if (lane == 0) tma_store_wait_all<0>();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 8) {
        tc_fence_after();
        tmem_dealloc(tbase, C::TCOLS);
    }
}

template <int MODE>
void set_attr_once() {
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_band_kernel<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             227 * 1024);
    });
}

int num_sms() {
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

int halo_rows(int64_t L, int64_t w) {
    const int64_t wc = w < L ? w : L;
    return (int)(((BM + 2 * wc) + 31) / 32 * 32);
}

// maps: per residue, (a1, b1, a2, b2, o1, o2) tensors; box rows BM for a/o, NK for b.
template <int MODE>
cudaError_t launch(const void* a1, const void* b1, const void* a2, const void* b2, void* o1,
                   void* o2, float* lse, float* D, int64_t B, int64_t H, int64_t L, int64_t d,
                   int64_t w, int64_t dil, cudaStream_t st, int* launches) {
    const int64_t wc = w < L ? w : L;
    const int NK = halo_rows(L, w);
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    set_attr_once<MODE>();
    int n = 0;
    for (int64_t r0 = 0; r0 < nres; r0 += RES_PER_LAUNCH) {
        Params p;
        memset(&p, 0, sizeof(p));
        const int nr = (int)(nres - r0 < RES_PER_LAUNCH ? nres - r0 : RES_PER_LAUNCH);
        for (int i = 0; i < nr; ++i) {
            const int64_t r = r0 + i;
            Maps& m = p.maps[i];
            bool ok = make_residue_map(&m.a1, a1, L, d, units, dil, r, BM) &&
                      make_residue_map(&m.b1, b1, L, d, units, dil, r, NK) &&
                      make_residue_map(&m.b2, b2, L, d, units, dil, r, NK) &&
                      make_residue_map(&m.o1, o1, L, d, units, dil, r, 32);
            if (ok && a2) ok = make_residue_map(&m.a2, a2, L, d, units, dil, r, BM);
            if (ok && o2) ok = make_residue_map(&m.o2, o2, L, d, units, dil, r, 32);
            if (!ok) return cudaErrorInvalidValue;
        }
        p.lse = lse;
        p.D = D;
        p.L = L;
        p.d = (int)d;
        p.w = (int)wc;
        p.dil = (int)dil;
        p.r0 = (int)r0;
        p.NK = NK;
        p.nsl = (int)(d / 64);
        const int64_t Lr0 = ceil_div(L - r0, dil);   // longest residue of this group
        p.nr = nr;
        p.trace = (unsigned long long*)trace_buffer(MODE);
        p.units = (int)units;
        p.tiles = (int)ceil_div(Lr0, BM);
        const int64_t total = (int64_t)p.units * p.nr * p.tiles;
        dim3 grid((unsigned)(total < num_sms() ? total : num_sms()));
        const int nst = pick_nst<MODE>(NK);
        p.nst = nst;
        const size_t smem = fixed_smem_bytes<MODE>() + (size_t)nst * stage_bytes<MODE>(NK);
        tc_band_kernel<MODE><<<grid, NTHREADS, smem, st>>>(p);
        prof_mark(st);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        ++n;
    }
    if (launches) *launches += n;
    return cudaSuccess;
}

bool band_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    const int64_t wc = w < L ? w : L;
    return d % 64 == 0 && d <= 512 && wc <= 64 && dil <= 256 && units * ((L + 127) / 128) < (1 << 30);
}

int band_launches(int64_t L, int64_t dil) {
    const int64_t nres = dil < L ? dil : L;
    return (int)ceil_div(nres, RES_PER_LAUNCH);
}

}  // namespace

bool tc_fwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    return halo_rows(L, w) <= 256 ? band_supported(units, L, d, w, dil)
                                  : tc_chunk_supported(units, L, d, w, dil);
}
bool tc_bwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    return tc_fwd_supported(units, L, d, w, dil);
}
int tc_fwd_launches(int64_t L, int64_t d, int64_t w, int64_t dil) {
    (void)d;
    return halo_rows(L, w) <= 256 ? band_launches(L, dil) : tc_chunk_launches(L, dil);
}
int tc_bwd_launches(int64_t L, int64_t d, int64_t w, int64_t dil) {
    return 2 * tc_fwd_launches(L, d, w, dil);
}

cudaError_t tc_fwd(const void* q, const void* k, const void* v, void* out, float* lse, int64_t B,
                   int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st,
                   int* launches) {
    if (launches) *launches = 0;
    if (halo_rows(L, w) > 256)
        return tc_chunk_fwd(q, k, v, out, lse, B, H, L, d, w, dil, st, launches);
    return launch<FWD>(q, k, nullptr, v, out, nullptr, lse, nullptr, B, H, L, d, w, dil, st,
                       launches);
}

cudaError_t tc_bwd(const void* q, const void* k, const void* v, const void* out,
                   const float* lse, const void* dout, void* dq, void* dk, void* dv, float* Dws,
                   int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                   cudaStream_t st, int* launches) {
    (void)out;   // D_i is recomputed exactly as sum_j P_ij dP_ij by the BWDQ kernel
    if (launches) *launches = 0;
    if (halo_rows(L, w) > 256)
        return tc_chunk_bwd(q, k, v, lse, dout, dq, dk, dv, Dws, B, H, L, d, w, dil, st, launches);
    cudaError_t e = launch<BWDQ>(q, k, dout, v, dq, nullptr, const_cast<float*>(lse), Dws, B, H,
                                 L, d, w, dil, st, launches);
    if (e != cudaSuccess) return e;
    return launch<BWDKV>(k, q, v, dout, dv, dk, const_cast<float*>(lse), Dws, B, H, L, d, w, dil,
                         st, launches);
}

}  // namespace ftw
