// tc_chunk.cu -- tcgen05/TMEM kernels of banded window attention for WIDE windows
// (128 + 2w > 256 halo rows, i.e. w > 64), bf16 storage, fp32 math, d in {64, 128}.
//
// A CTA owns BM = 128 rows m0.. of one (unit, residue) band problem.  The halo
// m0-w .. m0+127+w (128 + 2w rows) is streamed in key chunks of KC = 128 rows; the rows'
// operands (Q, or K/V in BWDKV) stay resident in shared memory for the whole tile.  This
// is the cache a[i:i+m] of PAPER.md Fig. 14 (lines 402-423) applied chunk by chunk.
//
//   FWD   pass 1: S_c = Q K_c^T; running row max / sum (the fused dot/max of Fig. 10)
//                 -> lse (written);  pass 2: S_c again, P_c = exp(S_c - lse) (exact, so O
//                 needs no rescaling: the dot_max dependence of P:239 is resolved by the
//                 first pass), O += P_c V_c in TMEM.
//   BWDQ  pass 1: S_c, dP_c = dO V_c^T -> D = sum P dP (exact, written);  pass 2: dS_c =
//                 P (dP - D) as bf16 hi/lo -> dQ += dS_c K_c.
//   BWDKV one pass (rows = keys): S^T_c = K Q_c^T, dP^T_c = V dO_c^T; P^T, dS^T with the
//                 per-column lse and D;  dV += P^T dO_c, dK += dS^T Q_c.
// Each output row has one writer (no atomics), as in tc_band.cu.
//
// Roles (192 threads): warps 0-3 softmax + epilogue (thread t <-> row t <-> TMEM lane t),
// warp 4 TMA producer + TMEM allocator, warp 5 MMA issuer.
// TMEM (512 columns): score buffers S at 0 / 128 (FWD: double-buffered, BWD: S at 0 and
// dP at 128), output accumulators at 256 (+d for BWDKV's dK).
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

enum { CFWD = 0, CBWDQ = 1, CBWDKV = 2 };

constexpr int BM = 128;
constexpr int KC = 128;
constexpr int NTHREADS = 192;
constexpr int RES_PER_LAUNCH = 4;
constexpr int MAX_NST = 8;
constexpr uint32_t BOX = 128 * 128;   // one 128-row x 64-col bf16 box (SW128)
constexpr float LOG2E = 1.4426950408889634f;
constexpr float LN2 = 0.6931471805599453f;
constexpr size_t SMEM_LIMIT = 227 * 1024;

template <int MODE> struct CCfg {
    static constexpr int NA = MODE == CFWD ? 1 : 2;        // resident row operands
    static constexpr int PASSES = MODE == CBWDKV ? 1 : 2;
    static constexpr int NO = MODE == CBWDKV ? 2 : 1;      // output accumulators
    static constexpr int NB = MODE == CFWD ? 2 : 1;        // score buffers
};

struct CMaps {
    CUtensorMap a1, b1, a2, b2, o1, o2;
};
struct CParams {
    CMaps maps[RES_PER_LAUNCH];
    float* lse;
    float* D;
    int64_t L;
    int d, w, dil, r0, nr, nkc, nst, units, tiles;
};

struct Tile {
    int u, rl, r, Lr, m0;
};
__device__ __forceinline__ bool decode_tile(const CParams& p, int tau, Tile& T) {
    const int t = tau % p.tiles;
    const int rest = tau / p.tiles;
    T.rl = rest % p.nr;
    T.u = rest / p.nr;
    T.r = p.r0 + T.rl;
    T.Lr = (int)((p.L - T.r + p.dil - 1) / p.dil);
    T.m0 = t * BM;
    return T.m0 < T.Lr;
}
struct TileCursor {
    int tau;
    __device__ explicit TileCursor(int start) : tau(start - (int)gridDim.x) {}
    __device__ bool next(const CParams& p, int total, Tile& T) {
        for (tau += gridDim.x; tau < total; tau += gridDim.x)
            if (decode_tile(p, tau, T)) return true;
        return false;
    }
};

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ void split_bf16x2(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    __nv_bfloat162 h = __floats2bfloat162_rn(x0, x1);
    const float2 hf = __bfloat1622float2(h);
    hi = *reinterpret_cast<uint32_t*>(&h);
    lo = pack_bf16x2(x0 - hf.x, x1 - hf.y);
}
// halo column hn of row t is in the band and inside the sequence
__device__ __forceinline__ bool band_ok(int hn, int t, int w, int mcol, int Lr) {
    return (unsigned)(hn - t) <= (unsigned)(2 * w) && mcol >= 0 && mcol < Lr;
}

template <int MODE> __host__ __device__ inline uint32_t a_bytes(int d) { return CCfg<MODE>::NA * (d / 64) * BOX; }
__host__ __device__ inline uint32_t stage_bytes(int d) { return 2u * (d / 64) * BOX; }
inline size_t fixed_bytes(int d, int nkc) {
    return 1024 + 4 * (size_t)(d / 64) * 32 * 128 + 2 * (size_t)nkc * KC * sizeof(float) + 512;
}

template <int MODE>
__global__ void __launch_bounds__(NTHREADS, 1) tc_chunk_kernel(const __grid_constant__ CParams p) {
    using C = CCfg<MODE>;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int d = p.d, w = p.w, nkc = p.nkc, NST = p.nst, nds = d / 64;
    const int total = p.units * p.nr * p.tiles;
    const uint32_t AB = a_bytes<MODE>(d), SB = stage_bytes(d);
    const int NKt = nkc * KC;

    uint8_t* sA = smem;                       // resident row operands: a1 boxes, then a2
    uint8_t* sStage = smem + AB;              // ring of NST stages: b1 boxes, then b2 boxes
    uint8_t* ostg = sStage + (size_t)NST * SB;                         // [4 warps][nds][4 KB]
    float* colLse = reinterpret_cast<float*>(ostg + 4 * nds * 32 * 128);
    float* colD = colLse + NKt;
    uint64_t* bars = reinterpret_cast<uint64_t*>(colD + NKt);
    uint64_t* full = bars;
    uint64_t* empty = bars + MAX_NST;
    uint64_t* s_full = bars + 2 * MAX_NST;    // [2]
    uint64_t* p_full = s_full + 2;            // [2]
    uint64_t* a_full = s_full + 4;
    uint64_t* a_empty = s_full + 5;
    uint64_t* acc_full = s_full + 6;
    uint64_t* acc_empty = s_full + 7;
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(s_full + 8);

    if (warp == 4) {
        if (lane == 0) {
            for (int i = 0; i < NST; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
            for (int i = 0; i < 2; ++i) { mbar_init(&s_full[i], 1); mbar_init(&p_full[i], 128); }
            mbar_init(a_full, 1);
            mbar_init(a_empty, 1);
            mbar_init(acc_full, 1);
            mbar_init(acc_empty, 128);
            fence_barrier_init();
        }
        __syncwarp();
        tmem_alloc(tmem_holder, 512);
        tmem_relinquish();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tbase = *tmem_holder;

    if (warp == 4) {
        if (lane == 0) {   // ------------------------------------------------ TMA producer
            int st = 0, j = 0;
            uint32_t ph = 0;
            TileCursor cur(blockIdx.x);
            Tile T;
            while (cur.next(p, total, T)) {
                const CMaps& mp = p.maps[T.rl];
                mbar_wait(a_empty, (j & 1) ^ 1u);
                mbar_arrive_expect_tx(a_full, AB);
                for (int s = 0; s < nds; ++s) {
                    tma_load_3d(sA + s * BOX, &mp.a1, a_full, s * 64, T.m0, T.u);
                    if (C::NA == 2) tma_load_3d(sA + (nds + s) * BOX, &mp.a2, a_full, s * 64, T.m0, T.u);
                }
                for (int pass = 0; pass < C::PASSES; ++pass) {
                    // FWD pass 1 needs only K; every other step needs both halo operands
                    const bool two = !(MODE == CFWD && pass == 0);
                    for (int c = 0; c < nkc; ++c) {
                        mbar_wait(&empty[st], ph ^ 1u);
                        uint8_t* sp = sStage + (size_t)st * SB;
                        mbar_arrive_expect_tx(&full[st], (two ? 2u : 1u) * nds * BOX);
                        const int row = T.m0 - w + c * KC;
                        for (int s = 0; s < nds; ++s) {
                            tma_load_3d(sp + s * BOX, &mp.b1, &full[st], s * 64, row, T.u);
                            if (two) tma_load_3d(sp + (nds + s) * BOX, &mp.b2, &full[st], s * 64, row, T.u);
                        }
                        if (++st == NST) { st = 0; ph ^= 1u; }
                    }
                }
                ++j;
            }
        }
    } else if (warp == 5) {
        if (lane == 0) {   // ------------------------------------------------ MMA issuer
            const uint32_t idS = idesc_bf16(128, KC, false, false);
            const uint32_t idO = idesc_bf16(128, d, false, true);
            int st = 0, j = 0, gs = 0;   // gs: global score-step counter (buffer phases)
            uint32_t ph = 0;
            TileCursor cur(blockIdx.x);
            Tile T;
            while (cur.next(p, total, T)) {
                mbar_wait(a_full, j & 1);
                tc_fence_after();
                const uint32_t sa = smem_u32(sA);
                bool first_out = true;
                const int nsteps = C::PASSES * nkc;
                // score GEMMs for step k into buffer (gs+k) % NB; FWD issues step k+1's
                // scores before waiting for step k's softmax (the buffers alternate).
                auto issue_scores = [&](int k) {
                    const int gk = gs + k, buf = gk % C::NB;
                    mbar_wait(&full[(st + k) % NST], (ph ^ (uint32_t)(((st + k) / NST) & 1)));
                    tc_fence_after();
                    const uint32_t sb = smem_u32(sStage + (size_t)((st + k) % NST) * SB);
                    const uint32_t tS = tbase + 128u * buf;
                    for (int s = 0; s < nds; ++s) {
#pragma unroll
                        for (int kk = 0; kk < 4; ++kk) {
                            const uint32_t off = s * BOX + kk * 32;
                            mma_ss(tS, sdesc_sw128(sa + off, 16, 1024), sdesc_sw128(sb + off, 16, 1024),
                                   idS, (s | kk) != 0);
                            if (C::NA == 2)   // dP (or dP^T) = A2 B2^T into column 128
                                mma_ss(tbase + 128, sdesc_sw128(sa + nds * BOX + off, 16, 1024),
                                       sdesc_sw128(sb + nds * BOX + off, 16, 1024), idS, (s | kk) != 0);
                        }
                    }
                    mma_commit(&s_full[buf]);
                };
                int issued = 0;
                issue_scores(0);
                issued = 1;
                for (int k = 0; k < nsteps; ++k) {
                    if (C::NB == 2 && issued < nsteps) { issue_scores(issued); ++issued; }
                    const int gk = gs + k, buf = gk % C::NB;
                    mbar_wait(&p_full[buf], (gk / C::NB) & 1);
                    tc_fence_after();
                    const int pass = k / nkc;
                    const int sk = (st + k) % NST;
                    const bool out = pass == C::PASSES - 1;
                    if (out) {
                        if (first_out) {
                            if (j > 0) { mbar_wait(acc_empty, (j - 1) & 1); tc_fence_after(); }
                        }
                        const uint32_t sb = smem_u32(sStage + (size_t)sk * SB);
                        for (int kk = 0; kk < KC / 16; ++kk) {
                            const uint32_t acc = (first_out && kk == 0) ? 0u : 1u;
                            if (MODE == CFWD) {        // O += P V : P compact over S buffer
                                mma_ts(tbase + 256, tbase + 128u * buf + 8u * kk,
                                       sdesc_sw128(sb + nds * BOX + kk * 2048, BOX, 1024), idO, acc);
                            } else if (MODE == CBWDQ) { // dQ += dS K : dS hi/lo over S
                                const uint32_t tA = tbase + 32u * (kk >> 1) + 8u * (kk & 1);
                                const uint64_t bd = sdesc_sw128(sb + kk * 2048, BOX, 1024);
                                mma_ts(tbase + 256, tA, bd, idO, acc);
                                mma_ts(tbase + 256, tA + 16, bd, idO, 1);
                            } else {                   // dV += P^T dO ; dK += dS^T Q
                                mma_ts(tbase + 256, tbase + 8u * kk,
                                       sdesc_sw128(sb + nds * BOX + kk * 2048, BOX, 1024), idO, acc);
                                const uint32_t tA = tbase + 128 + 32u * (kk >> 1) + 8u * (kk & 1);
                                const uint64_t bd = sdesc_sw128(sb + kk * 2048, BOX, 1024);
                                mma_ts(tbase + 256 + d, tA, bd, idO, acc);
                                mma_ts(tbase + 256 + d, tA + 16, bd, idO, 1);
                            }
                        }
                        first_out = false;
                    }
                    mma_commit(&empty[sk]);
                    if (C::NB == 1 && k + 1 < nsteps) { issue_scores(k + 1); ++issued; }
                }
                mma_commit(acc_full);
                mma_commit(a_empty);
                // advance the stage ring by this tile's steps
                const int adv = st + nsteps;
                ph ^= (uint32_t)((adv / NST) & 1);
                st = adv % NST;
                gs += nsteps;
                ++j;
            }
        }
    } else {   // --------------------------------------------------------- softmax + epilogue
        const int t = warp * 32 + lane;
        const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
        const uint32_t trow = tbase + lane_off;
        uint8_t* mystg = ostg + warp * nds * 32 * 128;
        int j = 0, gs = 0;
        TileCursor cur(blockIdx.x);
        Tile T;
        uint32_t zero16[16];
#pragma unroll
        for (int e = 0; e < 16; ++e) zero16[e] = 0u;
        while (cur.next(p, total, T)) {
            const CMaps& mp = p.maps[T.rl];
            const int Lr = T.Lr, m0 = T.m0, mrow = m0 + t, kb = m0 - w;
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;
            if (MODE == CBWDKV) {
                named_bar_sync(1, 128);
                for (int n = t; n < NKt; n += 128) {
                    const int mc = kb + n;
                    const bool ok = mc >= 0 && mc < Lr;
                    colLse[n] = ok ? p.lse[rowbase + (int64_t)mc * p.dil] * LOG2E : 0.f;
                    colD[n] = ok ? p.D[rowbase + (int64_t)mc * p.dil] : 0.f;
                }
                named_bar_sync(1, 128);
            }
            // per-row running state
            float m2 = -INFINITY, l = 0.f;   // FWD pass 1 (log2 domain)
            float lse2 = 0.f, D = 0.f;
            if (MODE == CBWDQ) lse2 = mrow < Lr ? p.lse[rowbase + (int64_t)mrow * p.dil] * LOG2E : 0.f;
            const int nsteps = C::PASSES * nkc;
            // warp-uniform band extent in halo columns: [32*warp, 32*warp + 31 + 2w]
            const int hlo = 32 * warp, hhi = 32 * warp + 31 + 2 * w;
            for (int k = 0; k < nsteps; ++k) {
                const int gk = gs + k, buf = gk % C::NB;
                const int pass = k / nkc, c = k % nkc;
                const uint32_t tS = trow + 128u * buf;
                mbar_wait(&s_full[buf], (gk / C::NB) & 1);
                tc_fence_after();
                for (int sc = 0; sc < 4; ++sc) {   // 32-column sub-chunks
                    const int h0 = c * KC + sc * 32;
                    const bool live = h0 + 31 >= hlo && h0 <= hhi;
                    if (MODE == CFWD) {
                        if (pass == 0) {
                            if (!live) continue;
                            uint32_t rr[32];
                            tmem_ld32(tS + sc * 32, rr);
                            tmem_wait_ld();
                            float cm = -INFINITY;
#pragma unroll
                            for (int e = 0; e < 32; ++e)
                                if (band_ok(h0 + e, t, w, kb + h0 + e, Lr)) cm = fmaxf(cm, __uint_as_float(rr[e]) * LOG2E);
                            if (cm > m2) { l *= fast_exp2(m2 - cm); m2 = cm; }
                            if (cm != -INFINITY) {
#pragma unroll
                                for (int e = 0; e < 32; ++e)
                                    if (band_ok(h0 + e, t, w, kb + h0 + e, Lr))
                                        l += fast_exp2(fmaf(__uint_as_float(rr[e]), LOG2E, -m2));
                            }
                        } else {
                            if (!live) { tmem_st16(tS + sc * 16, zero16); continue; }
                            uint32_t rr[32], pk[16];
                            tmem_ld32(tS + sc * 32, rr);
                            tmem_wait_ld();
#pragma unroll
                            for (int e = 0; e < 32; e += 2) {
                                float pv[2];
#pragma unroll
                                for (int h = 0; h < 2; ++h) {
                                    const int hn = h0 + e + h;
                                    pv[h] = band_ok(hn, t, w, kb + hn, Lr)
                                                ? fast_exp2(fmaf(__uint_as_float(rr[e + h]), LOG2E, -lse2))
                                                : 0.f;
                                }
                                pk[e / 2] = pack_bf16x2(pv[0], pv[1]);
                            }
                            tmem_st16(tS + sc * 16, pk);
                        }
                    } else if (MODE == CBWDQ) {
                        if (pass == 0 && !live) continue;
                        if (pass == 1 && !live) {
                            tmem_st16(trow + sc * 32, zero16);
                            tmem_st16(trow + sc * 32 + 16, zero16);
                            continue;
                        }
                        uint32_t rs[32], rd[32];
                        tmem_ld32(trow + sc * 32, rs);
                        tmem_ld32(trow + 128 + sc * 32, rd);
                        tmem_wait_ld();
                        if (pass == 0) {
#pragma unroll
                            for (int e = 0; e < 32; ++e) {
                                const int hn = h0 + e;
                                const float pv = band_ok(hn, t, w, kb + hn, Lr)
                                                     ? fast_exp2(fmaf(__uint_as_float(rs[e]), LOG2E, -lse2))
                                                     : 0.f;
                                D = fmaf(pv, __uint_as_float(rd[e]), D);
                            }
                        } else {
                            uint32_t pk[16], pl[16];
#pragma unroll
                            for (int e = 0; e < 32; e += 2) {
                                float dv[2];
#pragma unroll
                                for (int h = 0; h < 2; ++h) {
                                    const int hn = h0 + e + h;
                                    const float pv = band_ok(hn, t, w, kb + hn, Lr)
                                                         ? fast_exp2(fmaf(__uint_as_float(rs[e + h]), LOG2E, -lse2))
                                                         : 0.f;
                                    dv[h] = pv * (__uint_as_float(rd[e + h]) - D);
                                }
                                split_bf16x2(dv[0], dv[1], pk[e / 2], pl[e / 2]);
                            }
                            tmem_st16(trow + sc * 32, pk);
                            tmem_st16(trow + sc * 32 + 16, pl);
                        }
                    } else {   // CBWDKV
                        if (!live) {
                            tmem_st16(trow + sc * 16, zero16);
                            tmem_st16(trow + 128 + sc * 32, zero16);
                            tmem_st16(trow + 128 + sc * 32 + 16, zero16);
                            continue;
                        }
                        uint32_t rs[32], rd[32], pk[16], dk[16], dl[16];
                        tmem_ld32(trow + sc * 32, rs);
                        tmem_ld32(trow + 128 + sc * 32, rd);
                        tmem_wait_ld();
#pragma unroll
                        for (int e = 0; e < 32; e += 2) {
                            float pv[2], dv[2];
#pragma unroll
                            for (int h = 0; h < 2; ++h) {
                                const int hn = h0 + e + h;
                                pv[h] = band_ok(hn, t, w, kb + hn, Lr)
                                            ? fast_exp2(fmaf(__uint_as_float(rs[e + h]), LOG2E, -colLse[hn]))
                                            : 0.f;
                                dv[h] = pv[h] * (__uint_as_float(rd[e + h]) - colD[hn]);
                            }
                            pk[e / 2] = pack_bf16x2(pv[0], pv[1]);
                            split_bf16x2(dv[0], dv[1], dk[e / 2], dl[e / 2]);
                        }
                        tmem_st16(trow + sc * 16, pk);
                        tmem_st16(trow + 128 + sc * 32, dk);
                        tmem_st16(trow + 128 + sc * 32 + 16, dl);
                    }
                }
                tmem_wait_st();
                tc_fence_before();
                mbar_arrive(&p_full[buf]);
                if (MODE == CFWD && k == nkc - 1) {   // end of pass 1: lse
                    lse2 = m2 + log2f(l);
                    if (!(l > 0.f)) lse2 = 0.f;       // rows beyond the sequence only
                    if (mrow < Lr) p.lse[rowbase + (int64_t)mrow * p.dil] = lse2 * LN2;
                }
                if (MODE == CBWDQ && k == nkc - 1 && mrow < Lr) p.D[rowbase + (int64_t)mrow * p.dil] = D;
            }
            gs += nsteps;

            // ------------------------------------------------------------ epilogue
            mbar_wait(acc_full, j & 1);
            tc_fence_after();
            for (int o = 0; o < C::NO; ++o) {
                const CUtensorMap* om = o == 0 ? &mp.o1 : &mp.o2;
                for (int s = 0; s < nds; ++s) {
                    uint32_t ov[64];
                    const uint32_t col = 256u + o * d + s * 64;
                    tmem_ld32(trow + col, *reinterpret_cast<uint32_t(*)[32]>(&ov[0]));
                    tmem_ld32(trow + col + 32, *reinterpret_cast<uint32_t(*)[32]>(&ov[32]));
                    tmem_wait_ld();
                    if (o == C::NO - 1 && s == nds - 1) {
                        tc_fence_before();
                        mbar_arrive(acc_empty);
                    }
                    uint8_t* stg = mystg + s * 32 * 128;
                    if (lane == 0) tma_store_wait_read<0>();
                    __syncwarp();
#pragma unroll
                    for (int q = 0; q < 8; ++q) {
                        uint4 val;
                        val.x = pack_bf16x2(__uint_as_float(ov[8 * q + 0]), __uint_as_float(ov[8 * q + 1]));
                        val.y = pack_bf16x2(__uint_as_float(ov[8 * q + 2]), __uint_as_float(ov[8 * q + 3]));
                        val.z = pack_bf16x2(__uint_as_float(ov[8 * q + 4]), __uint_as_float(ov[8 * q + 5]));
                        val.w = pack_bf16x2(__uint_as_float(ov[8 * q + 6]), __uint_as_float(ov[8 * q + 7]));
                        *reinterpret_cast<uint4*>(stg + lane * 128 + ((q ^ (lane & 7)) * 16)) = val;
                    }
                    fence_proxy_async_smem();
                    __syncwarp();
                    if (lane == 0) {
                        tma_store_3d(om, stg, s * 64, m0 + 32 * warp, T.u);
                        tma_store_commit();
                    }
                }
            }
            ++j;
        }
        if (lane == 0) tma_store_wait_all<0>();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 4) {
        tc_fence_after();
        tmem_dealloc(tbase, 512);
    }
}

int num_sms_c() {
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
void set_attr_once() {
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_chunk_kernel<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             227 * 1024);
    });
}

template <int MODE>
cudaError_t launch(const void* a1, const void* b1, const void* a2, const void* b2, void* o1,
                   void* o2, float* lse, float* D, int64_t B, int64_t H, int64_t L, int64_t d,
                   int64_t w, int64_t dil, cudaStream_t st, int* launches) {
    const int64_t wc = w < L ? w : L;
    const int nkc = (int)ceil_div(BM + 2 * wc, KC);
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    set_attr_once<MODE>();
    const size_t fixed = fixed_bytes((int)d, nkc) + a_bytes<MODE>((int)d);
    int nst = (int)((SMEM_LIMIT - fixed) / stage_bytes((int)d));
    if (nst > MAX_NST) nst = MAX_NST;
    if (nst < 2) return cudaErrorInvalidConfiguration;
    int n = 0;
    for (int64_t r0 = 0; r0 < nres; r0 += RES_PER_LAUNCH) {
        CParams p;
        memset(&p, 0, sizeof(p));
        const int nr = (int)(nres - r0 < RES_PER_LAUNCH ? nres - r0 : RES_PER_LAUNCH);
        for (int i = 0; i < nr; ++i) {
            const int64_t r = r0 + i;
            CMaps& m = p.maps[i];
            bool ok = make_residue_map(&m.a1, a1, L, d, units, dil, r, BM) &&
                      make_residue_map(&m.b1, b1, L, d, units, dil, r, KC) &&
                      make_residue_map(&m.b2, b2, L, d, units, dil, r, KC) &&
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
        p.nr = nr;
        p.nkc = nkc;
        p.nst = nst;
        p.units = (int)units;
        const int64_t Lr0 = ceil_div(L - r0, dil);
        p.tiles = (int)ceil_div(Lr0, BM);
        const int64_t total = (int64_t)p.units * p.nr * p.tiles;
        dim3 grid((unsigned)(total < num_sms_c() ? total : num_sms_c()));
        const size_t smem = fixed + (size_t)nst * stage_bytes((int)d);
        tc_chunk_kernel<MODE><<<grid, NTHREADS, smem, st>>>(p);
        prof_mark(st);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        ++n;
    }
    if (launches) *launches += n;
    return cudaSuccess;
}

}  // namespace

bool tc_chunk_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    const int64_t wc = w < L ? w : L;
    const int nkc = (int)ceil_div(BM + 2 * wc, KC);
    return (d == 64 || d == 128) && dil <= 256 && units * ((L + 127) / 128) < (1 << 30) &&
           fixed_bytes((int)d, nkc) + a_bytes<CBWDQ>((int)d) + 2 * stage_bytes((int)d) <= SMEM_LIMIT;
}

cudaError_t tc_chunk_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                         int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                         cudaStream_t st, int* launches) {
    return launch<CFWD>(q, k, nullptr, v, out, nullptr, lse, nullptr, B, H, L, d, w, dil, st,
                        launches);
}

cudaError_t tc_chunk_bwd(const void* q, const void* k, const void* v, const float* lse,
                         const void* dout, void* dq, void* dk, void* dv, float* Dws, int64_t B,
                         int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st,
                         int* launches) {
    cudaError_t e = launch<CBWDQ>(q, k, dout, v, dq, nullptr, const_cast<float*>(lse), Dws, B, H,
                                  L, d, w, dil, st, launches);
    if (e != cudaSuccess) return e;
    return launch<CBWDKV>(k, q, v, dout, dv, dk, const_cast<float*>(lse), Dws, B, H, L, d, w, dil,
                          st, launches);
}

int tc_chunk_launches(int64_t L, int64_t dil) {
    const int64_t nres = dil < L ? dil : L;
    return (int)ceil_div(nres, RES_PER_LAUNCH);
}

}  // namespace ftw
