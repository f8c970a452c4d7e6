// tc_wide.cu -- tcgen05/TMEM forward kernel of banded window attention for WIDE windows
// (128 + 2w > 256 halo rows, i.e. w > 64), bf16 storage, fp32 math, d in {64, 128}.
//
// A CTA owns BM = 128 query rows m0.. of one (unit, residue) band problem at a time
// (persistent, static round robin over tiles).  The key/value halo m0-w .. m0+127+w is
// streamed once, in KC = 128-row chunks -- the cached a[i:i+m] window of PAPER.md Fig. 14
// (lines 402-423) applied chunk by chunk.  Per chunk c:
//
//   S_c = Q K_c^T (fp32, TMEM; issuer A)
//   softmax: chunk max -> running row max m (log2 domain); P_c = exp2(S_c - m) (bf16),
//            l += rowsum P_c  (the dot/max/exp fusion of Fig. 10)
//   O_0, O_1 += P_c V_c  (K-steps 0-3 / 4-7: two partial accumulators; issuer B)
//   end of tile: lse = ln 2 * (m + log2 l);  O = (O_0 + O_1) / l  (epilogue)
//
// Lazy rescaling (as in FlashAttention-4): m only moves when a chunk max exceeds it by more
// than RESCALE_LOG2 = 20, so P_c <= 2^20 (exact range for bf16 P and the fp32 sums); when it
// does move, the softmax warp multiplies its rows of the O partials (after O_{c-1} has
// completed) and l by 2^(m_old - m_new) before handing P_c over.  The final O / l and lse
// are exact whatever m was used.  Chunks are visited starting from the middle one, which is
// inside every row's band, so the first estimate of m is a 128-column max and rescales are
// rare (a row near a tile edge would otherwise see only a few band columns first).
//
// Why this shape (profiles/README.md, tools/mma_microbench.cu): a dependent tcgen05.mma
// chain advances one instruction per ~350 cycles whatever N is, and one issuing thread
// sustains ~1 instruction per 115-230 cycles.  The output GEMM of a wide window has a long
// reduction (128 + 2w keys = 40 K-steps at w = 256) but only N = d columns, so it is split
// over two partial accumulators; score and output GEMMs come from two warps; and a
// single pass over the halo halves the score GEMMs, the S reads and the handoffs of a
// two-pass (max, then exp) scheme, which the deletion experiments of profiles/README.md
// showed to be handoff-latency bound.
//
// P_c: for d = 64 (PSM) a double-buffered bf16 smem operand, so S_c's TMEM buffer is free
// as soon as the softmax has read it; for d = 128 (no smem to spare) P_c is packed over S_c
// in TMEM (TS operand) and the buffer is free once O_c has completed.
//
// Roles (480 threads): softmax warps 0-7 -- warps w and w+4 share rows 32w.. (TMEM lane
// quarter w) and split every chunk's 128 columns in halves (one warp per sub-partition
// cannot hide the exp / add latencies), exchanging chunk maxima through smem so that
// both make the same rescale decisions; warps 8-11 epilogue; warp 12 TMA producer + TMEM
// allocator; warp 13 issuer A (S GEMMs, K ring); warp 14 issuer B (O GEMMs, V ring).  TMEM: S double buffer at [0,128) / [128,256); the
// two O partials of tile j at 256 + (j % NOB) * 2d (NOB = 2 for d = 64: the next tile's
// O GEMMs do not wait for this tile's epilogue drain; NOB = 1 for d = 128).
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

constexpr int BM = 128;
constexpr int KC = 128;
constexpr int NTHREADS = 480;
constexpr int RES_PER_LAUNCH = 4;
static_assert(RES_PER_LAUNCH <= SCHED_MAX_RES, "residue table of the tile cursor");
constexpr int MAX_RING = 8;
constexpr uint32_t BOX = 128 * 128;   // one 128-row x 64-col bf16 box (SW128)
constexpr uint32_t STG = 32 * 128;    // one epilogue warp's 32-row x 64-col staging slice
constexpr float LOG2E = 1.4426950408889634f;
constexpr float LN2 = 0.6931471805599453f;
constexpr size_t SMEM_LIMIT = 227 * 1024;
constexpr float RESCALE_LOG2 = 20.f;  // lazy rescaling threshold (log2 units): P <= 2^20

struct WMaps {
    CUtensorMap q, k, v, o;
};
struct WParams {
    WMaps maps[RES_PER_LAUNCH];
    float* lse;
    int64_t L;
    int d, w, dil, nkc;
    SchedParams sc;
    int nq, nks, nvs;   // Q buffers, K ring slots, V ring slots
    unsigned long long* trace;   // optional phase trace (ft_winattn_debug_trace, mode 0)
};

// Phase trace, per CTA and local tile j < 8, 48 uint64 slots (ns): softmax 0 tile start,
// 1 S wait, 2 P-buffer wait, 3 compute, 4 rescales (count), 6 tile end; issuer A 10 start,
// 11 buffer-free wait, 12 K wait, 13 last S commit; issuer B 20 p_full wait, 21 o_empty
// wait, 22 V wait, 23 o_full commit; epilogue 30 o_full seen, 31 done.
__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ void trace_put(const WParams& p, int j, int slot, unsigned long long v) {
    if (p.trace && j < 8) p.trace[((size_t)blockIdx.x * 8 + j) * 48 + slot] = v;
}

using Tile = SchedTile;
using TileCursor = SchedCursor<BM>;

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
// halo column h of row t is in the band and inside the sequence
__device__ __forceinline__ bool band_ok(int h, int t, int w, int mcol, int Lr) {
    return (unsigned)(h - t) <= (unsigned)(2 * w) && mcol >= 0 && mcol < Lr;
}

struct Ring {   // slot index + phase of one side of a TMA ring
    int s = 0;
    uint32_t ph = 0;
    __device__ void adv(int n) { if (++s == n) { s = 0; ph ^= 1u; } }
};

__host__ __device__ inline uint32_t tile_bytes(int d) { return (uint32_t)(d / 64) * BOX; }
constexpr uint32_t PBUF = BM * KC * 2;   // one P_c buffer (two 64-key SW128 atoms)
inline bool psm_for(int d) { return d == 64; }
inline size_t fixed_bytes(int d) {
    return 1024 + (psm_for(d) ? 2 * (size_t)PBUF : 0) + 4 * (size_t)(d / 64) * STG +
           8 * 128 * sizeof(float) + 512;
}

// P_c row t, 32-key sub-chunk sc (16 packed words) -> K-major SW128 A operand.
__device__ __forceinline__ void st_p_sub(uint8_t* P, int t, int sc, const uint32_t (&pk)[16]) {
    uint8_t* row = P + (sc >> 1) * (BM * 128) + t * 128;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int g = (sc & 1) * 4 + q;
        *reinterpret_cast<uint4*>(row + ((g ^ (t & 7)) * 16)) =
            make_uint4(pk[4 * q], pk[4 * q + 1], pk[4 * q + 2], pk[4 * q + 3]);
    }
}

template <bool PSM>
__global__ void __launch_bounds__(NTHREADS, 1) tc_wide_fwd_kernel(const __grid_constant__ WParams p) {
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int d = p.d, w = p.w, nkc = p.nkc, nds = d / 64;
    const int NOB = 128 / d;                          // O buffers (tiles in flight)
    const int mid = nkc / 2;                          // first chunk visited (in every band)
    const uint32_t TB = tile_bytes(d);

    uint8_t* sQ = smem;                               // [nq] Q tiles
    uint8_t* sK = sQ + (size_t)p.nq * TB;             // [nks] K chunks
    uint8_t* sV = sK + (size_t)p.nks * TB;            // [nvs] V chunks
    uint8_t* sP = sV + (size_t)p.nvs * TB;            // PSM: [2] P_c buffers
    uint8_t* ostg = sP + (PSM ? 2 * (size_t)PBUF : 0); // [4 warps][nds] staging
    float* rowScale = reinterpret_cast<float*>(ostg + 4 * nds * STG);   // [2][128]
    float* cmx = rowScale + 2 * 128;   // softmax pair exchange: chunk max [2 slots][2 halves][128]
    float* lsx = cmx + 4 * 128;        // row sum [2 halves][128]
    uint64_t* bars = reinterpret_cast<uint64_t*>(lsx + 2 * 128);
    // per-slot barriers (slot j % 2 / j % NOB): a barrier never runs two phases ahead
    uint64_t* q_full = bars;                 // [2]
    uint64_t* q_empty = bars + 2;            // [2]
    uint64_t* k_full = bars + 4;             // [MAX_RING]
    uint64_t* k_empty = k_full + MAX_RING;
    uint64_t* v_full = k_empty + MAX_RING;
    uint64_t* v_empty = v_full + MAX_RING;
    uint64_t* s_full = v_empty + MAX_RING;   // [2] S_c in buffer b (issuer A)
    uint64_t* p_full = s_full + 2;           // [2] softmax done with step on buffer b (128)
    uint64_t* s_free = s_full + 4;           // [2] O of the step on buffer b completed
    uint64_t* o_full = s_full + 6;           // [2] O buffer complete (issuer B)
    uint64_t* o_empty = s_full + 8;          // [2] O buffer drained (epilogue, 128)
    uint64_t* st_full = s_full + 10;         // [2] 1/l of tile slot published (softmax, 128)
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(s_full + 12);

    if (warp == 12) {
        if (lane == 0) {
            for (int i = 0; i < 2; ++i) {
                mbar_init(&q_full[i], 1);
                mbar_init(&q_empty[i], 1);
                mbar_init(&s_full[i], 1);
                mbar_init(&p_full[i], 256);
                mbar_init(&s_free[i], 1);
            }
            for (int i = 0; i < MAX_RING; ++i) {
                mbar_init(&k_full[i], 1);
                mbar_init(&k_empty[i], 1);
                mbar_init(&v_full[i], 1);
                mbar_init(&v_empty[i], 1);
            }
            for (int i = 0; i < 2; ++i) {
                mbar_init(&o_full[i], 1);
                mbar_init(&o_empty[i], 128);
                mbar_init(&st_full[i], 128);
            }
            fence_barrier_init();
            for (int i = 0; i < p.sc.nr; ++i) {
                tma_prefetch(&p.maps[i].q); tma_prefetch(&p.maps[i].k);
                tma_prefetch(&p.maps[i].v); tma_prefetch(&p.maps[i].o);
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

    if (warp == 12) {
        if (lane == 0) {   // ------------------------------------------------ TMA producer
            // Order = consumption order: Q(j), then K_c / V_c per chunk.
            Ring kr, vr;
            int j = 0;
            TileCursor cur(p.sc);
            Tile T;
            while (cur.next(p.sc, T)) {
                const WMaps& mp = p.maps[T.rl];
                const int qb = j % p.nq;
                if (j >= p.nq) mbar_wait(&q_empty[qb], ((j / p.nq) - 1) & 1);
                mbar_arrive_expect_tx(&q_full[qb], TB);
                for (int s = 0; s < nds; ++s)
                    tma_load_3d(sQ + (size_t)qb * TB + s * BOX, &mp.q, &q_full[qb], s * 64, T.m0, T.u);
                for (int i = 0; i < nkc; ++i) {
                    const int c = (mid + i) % nkc, row = T.m0 - w + c * KC;
                    mbar_wait(&k_empty[kr.s], kr.ph ^ 1u);
                    mbar_arrive_expect_tx(&k_full[kr.s], TB);
                    for (int s = 0; s < nds; ++s)
                        tma_load_3d(sK + (size_t)kr.s * TB + s * BOX, &mp.k, &k_full[kr.s], s * 64, row, T.u);
                    kr.adv(p.nks);
                    mbar_wait(&v_empty[vr.s], vr.ph ^ 1u);
                    mbar_arrive_expect_tx(&v_full[vr.s], TB);
                    for (int s = 0; s < nds; ++s)
                        tma_load_3d(sV + (size_t)vr.s * TB + s * BOX, &mp.v, &v_full[vr.s], s * 64, row, T.u);
                    vr.adv(p.nvs);
                }
                ++j;
            }
        }
    } else if (warp == 13) {
        if (lane == 0) {   // ------------------------------------------------ issuer A: S
            const uint32_t idS = idesc_bf16(128, KC, false, false);
            Ring kr;
            int j = 0, gk = 0;   // gk: global chunk-step counter (S buffer gk & 1)
            TileCursor cur(p.sc);
            Tile T;
            while (cur.next(p.sc, T)) {
                const int qb = j % p.nq;
                mbar_wait(&q_full[qb], (j / p.nq) & 1);
                tc_fence_after();
                const bool tr = p.trace && j < 8;
                unsigned long long w_free = 0, w_k = 0, t0 = tr ? gtime() : 0;
                trace_put(p, j, 10, t0);
                const uint32_t sa = smem_u32(sQ + (size_t)qb * TB);
                for (int i = 0; i < nkc; ++i, ++gk) {
                    const int b = gk & 1;
                    if (gk >= 2) {   // step gk-2 is done with buffer b
                        if (tr) t0 = gtime();
                        mbar_wait(PSM ? &p_full[b] : &s_free[b], ((gk >> 1) - 1) & 1);
                        tc_fence_after();
                        if (tr) w_free += gtime() - t0;
                    }
                    if (tr) t0 = gtime();
                    mbar_wait(&k_full[kr.s], kr.ph);
                    tc_fence_after();
                    if (tr) w_k += gtime() - t0;
                    const uint32_t sb = smem_u32(sK + (size_t)kr.s * TB);
                    for (int s = 0; s < nds; ++s)
                        mma_ss_x4<2, 2>(tbase + 128u * b, sdesc_sw128(sa + s * BOX, 16, 1024),
                                        sdesc_sw128(sb + s * BOX, 16, 1024), idS, s != 0);
                    mma_commit(&k_empty[kr.s]);
                    kr.adv(p.nks);
                    mma_commit(&s_full[b]);
                }
                mma_commit(&q_empty[qb]);
                if (tr) { trace_put(p, j, 11, w_free); trace_put(p, j, 12, w_k); trace_put(p, j, 13, gtime()); }
                ++j;
            }
        }
    } else if (warp == 14) {
        if (lane == 0) {   // ------------------------------------------------ issuer B: O
            const uint32_t idO = idesc_bf16(128, d, false, true);
            Ring vr;
            int j = 0, gk = 0;
            TileCursor cur(p.sc);
            Tile T;
            while (cur.next(p.sc, T)) {
                const bool tr = p.trace && j < 8;
                unsigned long long w_p = 0, w_o = 0, w_v = 0, t0 = 0;
                const int ob = j % NOB;
                for (int i = 0; i < nkc; ++i, ++gk) {
                    const int b = gk & 1;
                    if (tr) t0 = gtime();
                    mbar_wait(&p_full[b], (gk >> 1) & 1);   // P_c ready (and any rescale done)
                    tc_fence_after();
                    if (tr) { w_p += gtime() - t0; t0 = gtime(); }
                    if (i == 0 && j >= NOB) {   // this O buffer's previous tile drained
                        mbar_wait(&o_empty[ob], ((j / NOB) - 1) & 1);
                        tc_fence_after();
                    }
                    if (tr) { w_o += gtime() - t0; t0 = gtime(); }
                    mbar_wait(&v_full[vr.s], vr.ph);
                    tc_fence_after();
                    if (tr) w_v += gtime() - t0;
                    const uint32_t sb = smem_u32(sV + (size_t)vr.s * TB);
                    // K-steps 0-3 and 4-7 go to the two partials (two 4-deep chains per
                    // chunk); the first chunk visited initialises them.
                    const uint32_t tO0 = tbase + 256u + (uint32_t)(ob * 2 * d);
                    const uint32_t tO1 = tO0 + (uint32_t)d;
                    const uint32_t sPa = smem_u32(sP + (size_t)b * PBUF);
                    {   // 4 K-steps per partial, one asm block each
                        const uint32_t acc = i > 0 ? 1u : 0u;
                        if (PSM) {   // P_c from smem: 64-key atoms of 16 KB, 32 B per step
                            mma_ss_x4<2, 128>(tO0, sdesc_sw128(sPa, 16, 1024), sdesc_sw128(sb, BOX, 1024), idO, acc);
                            mma_ss_x4<2, 128>(tO1, sdesc_sw128(sPa + BM * 128, 16, 1024),
                                              sdesc_sw128(sb + 4 * 2048, BOX, 1024), idO, acc);
                        } else {     // P_c packed bf16 over S_c: 8 columns per step
                            mma_ts_x4<8, 128>(tO0, tbase + 128u * b, sdesc_sw128(sb, BOX, 1024), idO, acc);
                            mma_ts_x4<8, 128>(tO1, tbase + 128u * b + 32u, sdesc_sw128(sb + 4 * 2048, BOX, 1024), idO, acc);
                        }
                    }
                    mma_commit(&v_empty[vr.s]);
                    vr.adv(p.nvs);
                    mma_commit(&s_free[b]);
                }
                mma_commit(&o_full[ob]);
                if (tr) { trace_put(p, j, 20, w_p); trace_put(p, j, 21, w_o); trace_put(p, j, 22, w_v); trace_put(p, j, 23, gtime()); }
                ++j;
            }
        }
    } else if (warp < 8) {   // ------------------------------------------- softmax warps
        const int wq = warp & 3, hf = warp >> 2;   // lane quarter, column half
        const int t = wq * 32 + lane;
        const uint32_t trow = tbase + ((uint32_t)(wq * 32) << 16);
        const int sp = 2 * hf;   // this warp's 32-column sub-chunks sp, sp+1 of every chunk
        int j = 0, gk = 0, xc = 0;   // xc: pair exchanges so far (slot xc & 1)
        uint32_t zero16[16];
#pragma unroll
        for (int e = 0; e < 16; ++e) zero16[e] = 0u;
        TileCursor cur(p.sc);
        Tile T;
        // warp-uniform band extent of rows 32*wq.. in halo columns
        const int hlo = 32 * wq, hhi = 32 * wq + 31 + 2 * w;
        // chunk-max exchange with the partner warp (same rows, other half): both get the
        // row max of the whole chunk
        auto xmax = [&](float mine) -> float {
            float* slot = cmx + (xc & 1) * 256;
            slot[hf * 128 + t] = mine;
            named_bar_sync(1 + wq, 64);
            ++xc;
            return fmaxf(slot[t], slot[128 + t]);
        };
        while (cur.next(p.sc, T)) {
            const int Lr = T.Lr, m0 = T.m0, mrow = m0 + t, kb = m0 - w;
            const bool tr = p.trace && j < 8 && t == 0 && hf == 0;
            unsigned long long acc_t[4] = {0, 0, 0, 0}, t0 = 0, t1 = 0;
            unsigned long long fine[5] = {0, 0, 0, 0, 0};
            if (tr) trace_put(p, j, 0, gtime());
            float ms = -INFINITY;   // running row max, log2 domain (-inf: nothing seen yet)
            float l = 0.f;          // this half's row sum at the running max
            const uint32_t tOb = trow + 256u + (uint32_t)((j % NOB) * 2 * d);   // this tile's O partials
            for (int i = 0; i < nkc; ++i, ++gk) {
                const int b = gk & 1, c = (mid + i) % nkc;
                const uint32_t tS = trow + 128u * b;
                uint8_t* Pb = sP + (size_t)b * PBUF;
                if (tr) t0 = gtime();
                // PSM: O of step gk-2 has read P buffer b
                if (PSM && gk >= 2) mbar_wait(&s_free[b], ((gk >> 1) - 1) & 1);
                if (tr) { t1 = gtime(); acc_t[1] += t1 - t0; t0 = t1; }
                mbar_wait(&s_full[b], (gk >> 1) & 1);
                tc_fence_after();
                if (tr) { t1 = gtime(); acc_t[0] += t1 - t0; t0 = t1; }
                // Live: some row of the warp has band columns in sub-chunk sc (warp-uniform);
                // inner: every row / column of it is in the band and the sequence.
                auto live = [&](int sc) { const int h0 = c * KC + sc * 32; return h0 + 31 >= hlo && h0 <= hhi; };
                auto inner = [&](int sc) {
                    const int h0 = c * KC + sc * 32;
                    return h0 >= hlo + 31 && h0 + 31 <= hlo + 2 * w && kb + h0 >= 0 && kb + h0 + 31 < Lr;
                };
                const bool any_live = live(sp) || live(sp + 1);
                // Load my half (two sub-chunks) of S_c; columns outside this row's band or the
                // sequence become -inf (exp2 -> 0, ignored by max).  One compact code path:
                // the kernel is instruction-fetch bound when the softmax is unrolled per case.
                uint32_t rr[2][32];
                auto load_half = [&]() {
                    tmem_ld32(tS + sp * 32, rr[0]);
                    tmem_ld32(tS + sp * 32 + 32, rr[1]);
                    tmem_wait_ld();
#pragma unroll
                    for (int x = 0; x < 2; ++x) {
                        const int sc = sp + x;
                        if (inner(sc)) continue;   // warp-uniform
                        const int h0 = c * KC + sc * 32;
                        // valid e: t <= h0+e <= t+2w and 0 <= kb+h0+e < Lr
                        const int lo = max(max(t - h0, -kb - h0), 0);
                        const int hi = min(min(t + 2 * w - h0, Lr - 1 - kb - h0), 31);
                        const uint32_t bits = (!live(sc) || hi < lo) ? 0u
                                              : ((0xffffffffu >> (31 - hi)) & (0xffffffffu << lo));
#pragma unroll
                        for (int e = 0; e < 32; ++e)
                            if (!((bits >> e) & 1u)) rr[x][e] = 0xff800000u;   // -inf
                    }
                };
                // max of my half of S_c (log2 domain)
                // (reload = false: from the registers of the last load -- once P is packed over S in
                // TMEM, d = 128, S can no longer be read back)
                auto half_max = [&](bool reload) -> float {
                    float m4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
                    if (any_live) {
                        if (reload) load_half();
#pragma unroll
                        for (int x = 0; x < 2; ++x)
#pragma unroll
                            for (int e = 0; e < 32; ++e) m4[e & 3] = fmaxf(m4[e & 3], __uint_as_float(rr[x][e]));
                    }
                    return fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3])) * LOG2E;
                };
                // P = exp2(S - mref) for my half -> operand; returns my half's row sum.  Per pair
                // of entries: one FFMA2 (s log2e - mref), two ex2, one FADD2 (the two partial
                // sums), one pack -- no running max: the rescale test below uses the row sum
                // (every P <= the sum of the chunk's P).
                auto exp_sweep = [&](float mref, bool reload) -> float {
                    float lc[2] = {0.f, 0.f};
                    if (!PSM && reload) {
                        // P goes over S in TMEM, and this warp's packed P columns [16 sp, 16 sp + 32)
                        // hold S of the partner warp's half when hf = 1: both warps must have read
                        // their S halves before either stores
                        if (any_live) load_half();
                        named_bar_sync(1 + wq, 64);
                    }
                    if (!any_live) {
                        if (PSM) { st_p_sub(Pb, t, sp, zero16); st_p_sub(Pb, t, sp + 1, zero16); }
                        else { tmem_st16(tS + sp * 16, zero16); tmem_st16(tS + sp * 16 + 16, zero16); }
                    } else {
                        unsigned long long q0 = tr ? gtime() : 0;
                        if (PSM && reload) load_half();
                        if (tr) fine[0] += gtime() - q0;
#pragma unroll
                        for (int x = 0; x < 2; ++x) {
                            uint32_t pk[16];
#pragma unroll
                            for (int e = 0; e < 32; e += 2) {
                                float a0, a1;
                                ffma2_bc(__uint_as_float(rr[x][e]), __uint_as_float(rr[x][e + 1]), LOG2E, -mref, a0, a1);
                                const float p0 = fast_exp2(a0), p1 = fast_exp2(a1);
                                fadd2_acc(lc[0], lc[1], p0, p1);
                                pk[e / 2] = pack_bf16x2(p0, p1);
                            }
                            if (PSM) st_p_sub(Pb, t, sp + x, pk);
                            else tmem_st16(tS + (sp + x) * 16, pk);
                        }
                    }
                    return lc[0] + lc[1];
                };
                // row sum of the whole chunk (both halves), exchanged with the partner warp
                auto xsum = [&](float mine) -> float {
                    float* slot = cmx + (xc & 1) * 256;
                    slot[hf * 128 + t] = mine;
                    named_bar_sync(1 + wq, 64);
                    ++xc;
                    return slot[t] + slot[128 + t];
                };
                // move the running max of rows whose chunk max exceeds it by more than the
                // threshold; where such a row has already accumulated, the half-0 warp rescales
                // its rows of the O partials (after O_{c-1} -- and every earlier O MMA --
                // completed) and both warps rescale their half of l
                auto move_max = [&](float cmf) {
                    const bool mv = cmf > ms + RESCALE_LOG2;
                    if (__any_sync(0xffffffffu, mv && ms != -INFINITY)) {
                        const float f = (mv && ms != -INFINITY) ? fast_exp2(ms - cmf) : 1.f;
                        if (tr) acc_t[3] += 1;
                        if (hf == 0) {
                            if (i > 0) mbar_wait(&s_free[(gk - 1) & 1], ((gk - 1) >> 1) & 1);
                            tc_fence_after();
#pragma unroll 1
                            for (int h = 0; h < 2 * d; h += 16) {   // both partials
                                uint32_t ov[16];
                                tmem_ld16(tOb + (uint32_t)h, ov);
                                tmem_wait_ld();
#pragma unroll
                                for (int e = 0; e < 16; ++e) ov[e] = __float_as_uint(__uint_as_float(ov[e]) * f);
                                tmem_st16(tOb + (uint32_t)h, ov);
                            }
                            tmem_wait_st();
                        }
                        l *= f;
                    }
                    if (mv) ms = cmf;
                };
                // rows without a running max yet (the first chunk): exact chunk max first
                if (__any_sync(0xffffffffu, ms == -INFINITY)) move_max(xmax(half_max(true)));
                // optimistic sweep at the running max.  If some row's chunk sum exceeds
                // 2^(RESCALE_LOG2 - 6) -- only then can one of its P exceed the threshold -- both
                // warps take the chunk's exact max, move the running max where it exceeds it by
                // more than the threshold, and redo the chunk (rare: m starts at the middle
                // chunk's exact max)
                float lc;
                unsigned long long q1 = tr ? gtime() : 0, q2 = 0;
                lc = exp_sweep(ms == -INFINITY ? 0.f : ms, true);
                if (tr) q2 = gtime();
                const float rowsum = xsum(lc);
                if (__any_sync(0xffffffffu, !(rowsum <= exp2f(RESCALE_LOG2 - 6.f)))) {   // (NaN: check)
                    const float cm = xmax(half_max(PSM));
                    if (__any_sync(0xffffffffu, cm > ms + RESCALE_LOG2)) {
                        move_max(cm);
                        lc = exp_sweep(ms == -INFINITY ? 0.f : ms, PSM);
                    }
                }
                if (tr) { fine[1] += q2 - q1; fine[2] += gtime() - q2; }
                l += lc;
                unsigned long long q3 = tr ? gtime() : 0;
                if (PSM) fence_proxy_async_smem();   // P (generic stores) -> tensor core
                else tmem_wait_st();
                tc_fence_before();
                mbar_arrive(&p_full[b]);
                if (tr) { fine[3] += gtime() - q3; acc_t[2] += gtime() - t0; }
            }
            if (tr) { trace_put(p, j, 1, acc_t[0]); trace_put(p, j, 2, acc_t[1]); trace_put(p, j, 3, acc_t[2]); trace_put(p, j, 4, acc_t[3]);
                      for (int f = 0; f < 4; ++f) trace_put(p, j, 40 + f, fine[f]); }
            lsx[hf * 128 + t] = l;
            named_bar_sync(1 + wq, 64);
            if (hf == 0) {
                l = lsx[t] + lsx[128 + t];
                // slot j & 1 was read by the epilogue of tile j-2 before its o_empty, which
                // precedes O(j) -- and P / S buffer reuse in this tile waits for O(j)'s chunks
                rowScale[(j & 1) * 128 + t] = l > 0.f ? 1.f / l : 0.f;
                mbar_arrive(&st_full[j & 1]);
                if (mrow < Lr) p.lse[(int64_t)T.u * p.L + T.r + (int64_t)mrow * p.dil] = (ms + log2f(l)) * LN2;
                if (tr) trace_put(p, j, 6, gtime());
            }
            ++j;
        }
    } else if (warp < 12) {   // ----------------------------------------- epilogue warps
        const int ew = warp - 8;   // TMEM lanes 32*ew.. (warp % 4 == ew)
        const uint32_t trow = tbase + ((uint32_t)(ew * 32) << 16);
        uint8_t* mystg = ostg + ew * nds * STG;
        int j = 0;
        TileCursor cur(p.sc);
        Tile T;
        while (cur.next(p.sc, T)) {
            const WMaps& mp = p.maps[T.rl];
            const int ob = j % NOB;
            mbar_wait(&st_full[j & 1], (j >> 1) & 1);
            const float scale = rowScale[(j & 1) * 128 + ew * 32 + lane];
            mbar_wait(&o_full[ob], (j / NOB) & 1);
            tc_fence_after();
            if (ew == 0 && lane == 0) trace_put(p, j, 30, gtime());
            if (lane == 0) tma_store_wait_read<0>();   // staging of the previous tile read
            __syncwarp();
            for (int s = 0; s < nds; ++s) {
                uint8_t* stg = mystg + s * STG;
#pragma unroll 1
                for (int hf = 0; hf < 2; ++hf) {   // 32-column halves of the 64-column slice
                    float acc[32];
                    {
                        uint32_t o0[32], o1[32];
                        const uint32_t col = 256u + (uint32_t)(ob * 2 * d + s * 64 + hf * 32);
                        tmem_ld32(trow + col, o0);
                        tmem_ld32(trow + col + (uint32_t)d, o1);
                        tmem_wait_ld();
#pragma unroll
                        for (int e = 0; e < 32; ++e) acc[e] = __uint_as_float(o0[e]) + __uint_as_float(o1[e]);
                    }
                    if (s == nds - 1 && hf == 1) {   // every partial column is in registers
                        tc_fence_before();
                        mbar_arrive(&o_empty[ob]);
                    }
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        uint4 val;
                        val.x = pack_bf16x2(acc[8 * q + 0] * scale, acc[8 * q + 1] * scale);
                        val.y = pack_bf16x2(acc[8 * q + 2] * scale, acc[8 * q + 3] * scale);
                        val.z = pack_bf16x2(acc[8 * q + 4] * scale, acc[8 * q + 5] * scale);
                        val.w = pack_bf16x2(acc[8 * q + 6] * scale, acc[8 * q + 7] * scale);
                        const int gq = hf * 4 + q;
                        *reinterpret_cast<uint4*>(stg + lane * 128 + ((gq ^ (lane & 7)) * 16)) = val;
                    }
                }
                fence_proxy_async_smem();
                __syncwarp();
                if (lane == 0) {
                    tma_store_3d(&mp.o, stg, s * 64, T.m0 + 32 * ew, T.u);
                    tma_store_commit();
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

int num_sms_w() {
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

// Ring sizes: two Q buffers when they fit, then K / V slots split evenly (>= 2 each).
bool plan_rings(int d, int& nq, int& nks, int& nvs) {
    const size_t TB = tile_bytes(d);
    const size_t avail = SMEM_LIMIT - fixed_bytes(d);
    for (nq = 2; nq >= 1; --nq) {
        if (avail < (size_t)(nq + 4) * TB) continue;
        int n = (int)((avail - nq * TB) / TB);
        if (n > 2 * MAX_RING) n = 2 * MAX_RING;
        nks = (n + 1) / 2;
        nvs = n - nks;
        if (nks > MAX_RING) nks = MAX_RING;
        if (nvs > MAX_RING) nvs = MAX_RING;
        return true;
    }
    return false;
}

}  // namespace

bool tc_wide_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    (void)w;
    int nq, nks, nvs;
    return (d == 64 || d == 128) && dil <= 256 && units * ((L + 127) / 128) < (1 << 30) &&
           plan_rings((int)d, nq, nks, nvs);
}

int tc_wide_launches(int64_t L, int64_t dil) {
    const int64_t nres = dil < L ? dil : L;
    return (int)ceil_div(nres, RES_PER_LAUNCH);
}

cudaError_t tc_wide_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                        int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                        cudaStream_t st, int* launches) {
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_wide_fwd_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)SMEM_LIMIT);
        cudaFuncSetAttribute(tc_wide_fwd_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)SMEM_LIMIT);
    });
    const int64_t wc = w < L ? w : L;
    const int nkc = (int)ceil_div(BM + 2 * wc, KC);
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    int nq, nks, nvs;
    if (!plan_rings((int)d, nq, nks, nvs)) return cudaErrorInvalidConfiguration;
    int n = 0;
    for (int64_t r0 = 0; r0 < nres; r0 += RES_PER_LAUNCH) {
        WParams p;
        memset(&p, 0, sizeof(p));
        const int nr = (int)(nres - r0 < RES_PER_LAUNCH ? nres - r0 : RES_PER_LAUNCH);
        for (int i = 0; i < nr; ++i) {
            const int64_t r = r0 + i;
            WMaps& m = p.maps[i];
            if (!(make_residue_map(&m.q, q, L, d, units, dil, r, BM) &&
                  make_residue_map(&m.k, k, L, d, units, dil, r, KC) &&
                  make_residue_map(&m.v, v, L, d, units, dil, r, KC) &&
                  make_residue_map(&m.o, out, L, d, units, dil, r, 32)))
                return cudaErrorInvalidValue;
        }
        p.lse = lse;
        p.L = L;
        p.d = (int)d;
        p.w = (int)wc;
        p.dil = (int)dil;
        p.nkc = nkc;
        p.nq = nq;
        p.nks = nks;
        p.nvs = nvs;
        p.trace = (unsigned long long*)trace_buffer(0);
        const int64_t Lr0 = ceil_div(L - r0, dil);
        const int tiles = (int)ceil_div(Lr0, BM);
        const int64_t total = units * nr * tiles;
        dim3 grid((unsigned)(total < num_sms_w() ? total : num_sms_w()));
        sched_init(p.sc, L, dil, r0, nr, units, tiles, (int)grid.x);
        const size_t smem = fixed_bytes((int)d) + (size_t)(nq + nks + nvs) * tile_bytes((int)d);
        if (psm_for((int)d)) tc_wide_fwd_kernel<true><<<grid, NTHREADS, smem, st>>>(p);
        else tc_wide_fwd_kernel<false><<<grid, NTHREADS, smem, st>>>(p);
        prof_mark(st);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        ++n;
    }
    if (launches) *launches += n;
    return cudaSuccess;
}

}  // namespace ftw
