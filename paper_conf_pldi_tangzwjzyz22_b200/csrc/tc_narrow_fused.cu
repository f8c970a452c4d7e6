// tc_narrow_fused.cu -- ONE-kernel backward of banded window attention for head dim d = 64 and
// w <= 32 on sm_100a (the HBM-bound C5 shape; SURVEY.md §8(a) rows B0-B5 in a single pass).
//
// The split backward (tc_narrow_bwd.cu: NQ then NKV) reads q, k, v and dout twice, 11de + 16
// bytes per row.  This kernel reads each of them once and writes dq, dk, dv once: 7de + 4 bytes
// per row (lse in; no D workspace, no out), the materialization-free gradient program of
// PAPER.md:447-453 with P recomputed from the saved lse (selective materialization,
// PAPER.md:489-497, reading A6).
//
// Query-major, so D_i = sum_j P_ij dP_ij stays exact and row-local (reading R1): a CTA takes a
// 128-query tile t (rows m0 = 128 t ..), computes S = Q_t K_h^T and dP = dO_t V_h^T over the
// 192-key halo m0-w .. m0-w+191 (the cached window of PAPER.md Fig. 14),
// P = exp(S - lse), D, dS = P (dP - D), and
//     dQ_t             = dS K_h                     (final: every key of a query's band is here)
//     dK/dV of keys     = dS^T Q_t,  P^T dO_t        (partial: a key's band spans two tiles)
// Key blocks are shifted by w against the query tiles, A_t = keys [128 t - w, 128 t + 128 - w):
// tile t adds into A_t (halo columns 0..127) and A_{t+1} (columns 128..191), and A_t is complete
// after tile t.  So each CTA walks a CONTIGUOUS strip of tiles and keeps two dK|dV accumulator
// blocks in TMEM, draining A_t after tile t -- every dk/dv row has exactly one writer and no
// atomics are used (Fig. 13(d), the parallel reduction, rather than 13(e)).  A strip
// that starts inside a (unit, residue) problem first runs a "warm-up" tile t0-1 whose only
// output is A_{t0}'s left part; the last tile of a problem also drains A_{t+1} (the tail).
//
// Consecutive tiles share 64 halo rows, so K and V are staged by TMA in 64-row blocks through
// rings (K: 5 slots, V: 4) and each tile loads two new blocks of each.  dS enters its MMAs as
// fp16 (reading A10), so the operands it multiplies (Q_t, the K blocks) are converted to fp16
// in place by a converter warp as soon as they land, and the score GEMM S = Q K^T runs in fp16
// too (dP = dO V^T stays bf16).
//
// P (bf16) and dS (fp16) go to shared memory (from registers: thread <-> query row) and serve
// as MN-major A operands for the transposed products (M = keys).  Their 64-key atoms are
// stored compressed -- a query row t only has band columns [t, t+2w] within [32(t/32),
// 32(t/32)+96), so atom 0 (columns 0..63) is empty for rows >= 64 and atom 2 for rows < 64 --
// and the zero halves are one shared 8 KB block reached through the descriptors' strides.
//
// TMEM (512 columns): S then dP of the tile share [0,192) (the softmax holds S in registers
// before dP is issued); dQ at [192,256); dK|dV blocks X[0] = [256,384), X[1] = [384,512);
// tile j uses X[j&1] as A_t and X[(j+1)&1] as A_{t+1}.
//
// Measured (C5_w32, tools/trace_fused.py): ~9000 clk per tile, bound by the serial handoffs of
// that chain (MMA issue at ~60-90 clk per N = 64 MMA, 36 output MMAs per tile; mbarrier
// handoffs; the 48 KB drain), not by HBM (~5100 clk per tile at the measured peak).
//
// Roles (640 threads): warps 0-15 softmax + drains (warp w: TMEM lanes 32*(w%4).., columns
// 24*(w/4).. of the row's 96-column band window); warp 16 TMA producer + TMEM allocator; warps
// 17 and 19 MMA issuers (S, dP, dQ | dK, dV); warp 18 fp16 converter.  Per tile the MMA chain is
// S(j) -> softmax -> dP(j) -> softmax -> out(j); the drain of tile j-1 runs while dP(j) does.
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
constexpr int D = 64;
constexpr int KB = 64;                       // rows per K / V ring block
constexpr int RK = 5, RV = 4;                // ring slots
constexpr int NTHREADS = 640;
constexpr int NSM = 512;                     // softmax threads (warps 0-15)
constexpr int RES_PER_LAUNCH = 8;
static_assert(RES_PER_LAUNCH <= SCHED_MAX_RES, "residue table");
constexpr uint32_t TILE = BM * D * 2;        // 16 KB
constexpr uint32_t BLK = KB * D * 2;         // 8 KB
constexpr uint32_t QO = 2 * TILE;            // Q_t | dO_t of one tile
// operand region: [dS0][Z][dS2][dS1][P0][P1][P2][ZB]; X0 / X2 hold query rows 0..63 / 64..127
constexpr uint32_t O_DS0 = 0, O_Z = 8192, O_DS2 = 16384, O_DS1 = 24576;
constexpr uint32_t O_P0 = 40960, O_P1 = 49152, O_P2 = 65536, O_ZB = 73728, OPS = 81920;
constexpr uint32_t OFF_QO = 0, OFF_K = 2 * QO, OFF_V = OFF_K + RK * BLK, OFF_OPS = OFF_V + RV * BLK;
constexpr uint32_t OFF_SCR = OFF_OPS + OPS;
constexpr int SCR_FLOATS = 2 * 4 * BM + 2 * NSM;   // D parts [2][4][BM], row lse [2][NSM]
constexpr uint32_t OFF_BAR = OFF_SCR + SCR_FLOATS * 4;
constexpr int NBAR = 40;
constexpr size_t SMEM_BYTES = 1024 + OFF_BAR + NBAR * 8 + 16;
static_assert(SMEM_BYTES <= 232448, "shared memory plan");
static_assert(OFF_OPS % 1024 == 0 && OFF_K % 1024 == 0 && OFF_V % 1024 == 0, "SW128 atoms");
constexpr float LOG2E = 1.4426950408889634f;
constexpr uint32_t T_DQ = 192, T_X = 256;

struct FMaps {
    CUtensorMap q, dout, k, v;   // q, dout: 128-row boxes; k, v: 64-row boxes
};
struct FParams {
    FMaps maps[RES_PER_LAUNCH];
    const float* lse;
    uint16_t* dq;
    uint16_t* dk;
    uint16_t* dv;
    int64_t L;
    int w, dil;
    int tiles, nr, r0;
    int Lr[SCHED_MAX_RES];
    long long ntau;   // units * nr * tiles
    unsigned long long* trace;   // optional phase trace (ft_winattn_debug_trace mode 1)
};

// Phase trace (tools/trace_fused.py): clock64 stamps of items 8..15 of every CTA.
__device__ __forceinline__ void trace_ev(const FParams& p, int j, int ev) {
    if (p.trace && j >= 8 && j < 16) p.trace[((size_t)blockIdx.x * 8 + (j - 8)) * 48 + ev] = clock64();
}

// One unit of work of a CTA: tile m0 of (unit u, residue r0 + rl).  warm: only its A_{t+1}
// contribution is kept; cont: the previous item was tile t-1 of the same problem (shares the
// first K / V block and A_t); tail: last tile of the problem (A_{t+1} drained too); bseq:
// ring sequence number of its first K / V block.
struct FItem {
    int u, rl, Lr, m0, bseq;
    int64_t rowbase;
    bool warm, cont, tail;
};

// The CTA's strip: tau in [c N / G, (c+1) N / G) over tau = (u * nr + rl) * tiles + t.
struct FCursor {
    int t, rl, u;
    long long left;
    bool have_prev;
    int pu, prl, pt, pb;
    __device__ explicit FCursor(const FParams& p) {
        const long long G = gridDim.x, c = blockIdx.x;
        const long long t0 = c * p.ntau / G, t1 = (c + 1) * p.ntau / G;
        left = t1 - t0;
        t = (int)(t0 % p.tiles);
        const long long rest = t0 / p.tiles;
        rl = (int)(rest % p.nr);
        u = (int)(rest / p.nr);
        have_prev = false;
        pu = prl = pt = -1;
        pb = 0;
    }
    __device__ __forceinline__ void adv(const FParams& p) {
        if (++t == p.tiles) {
            t = 0;
            if (++rl == p.nr) { rl = 0; ++u; }
        }
        --left;
    }
    __device__ bool next(const FParams& p, FItem& it) {
        for (;;) {
            if (left <= 0) return false;
            const int Lr = p.Lr[rl];
            if (t * BM >= Lr) { adv(p); continue; }
            const bool warm = !have_prev && t > 0;
            const int tt = warm ? t - 1 : t;
            it.u = u;
            it.rl = rl;
            it.Lr = Lr;
            it.m0 = tt * BM;
            it.warm = warm;
            it.cont = have_prev && pu == u && prl == rl && pt == tt - 1;
            it.tail = (tt + 1) * BM >= Lr;
            it.bseq = have_prev ? pb + (it.cont ? 2 : 3) : 0;
            it.rowbase = (int64_t)u * p.L + (p.r0 + rl);
            have_prev = true;
            pu = u; prl = rl; pt = tt; pb = it.bseq;
            if (!warm) adv(p);
            return true;
        }
    }
};

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// A warp's 32 rows (lane = row row0 + lane) x 16 fp32 columns (part pq of d = 64) -> bf16 in HBM.
// Lane pairs swap one 16-byte chunk (shfl.xor 1), so each of the two store instructions covers
// 16 rows x 32 contiguous bytes instead of 32 rows x 16 B: per-row direct stores put so many LSU
// transactions in flight that they stalled the whole SM sub-partition, MMA issue and mbarrier
// polls included (tools/trace_fused.py).
__device__ __forceinline__ void store_rows16(uint16_t* t, int64_t rowbase, int dil, int row0, int Lr, int pq,
                                             int lane, const uint32_t (&v)[16]) {
    uint32_t c[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) c[i] = pack_bf16x2(__uint_as_float(v[2 * i]), __uint_as_float(v[2 * i + 1]));
    const bool hi = (lane & 1) != 0;
#pragma unroll
    for (int x = 0; x < 4; ++x) {
        const uint32_t send = hi ? c[x] : c[4 + x];
        const uint32_t recv = __shfl_xor_sync(0xffffffffu, send, 1);
        if (hi) c[x] = recv;
        else c[4 + x] = recv;
    }
    const int pr = lane >> 1, ch = lane & 1;
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int row = row0 + 2 * pr + q;
#ifdef FT_EXPERIMENT_NO_DRAIN_STORES   // A/B experiment only: drops the results
        if (row < -1000000)
#else
        if (row >= 0 && row < Lr)
#endif
            *reinterpret_cast<uint4*>(t + (rowbase + (int64_t)row * dil) * D + 16 * pq + 8 * ch) =
                make_uint4(c[4 * q], c[4 * q + 1], c[4 * q + 2], c[4 * q + 3]);
    }
}

__device__ __forceinline__ void tmem_ld8(uint32_t taddr, uint32_t* r) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                 : "r"(taddr));
}

// bf16 at src -> fp16 at dst (may alias), `bytes`, by the converter warp
__device__ __forceinline__ void to_f16(const uint8_t* src, uint8_t* dst, uint32_t bytes, int ct) {
    const uint4* b = reinterpret_cast<const uint4*>(src);
    uint4* o = reinterpret_cast<uint4*>(dst);
#pragma unroll 8
    for (int i = ct; i < (int)(bytes / 16); i += 32) {
        uint4 v4 = b[i];
        uint32_t* wv = reinterpret_cast<uint32_t*>(&v4);
#pragma unroll
        for (int x = 0; x < 4; ++x) {
            const float2 f = __bfloat1622float2(*reinterpret_cast<__nv_bfloat162*>(&wv[x]));
            wv[x] = pack_f16x2(f.x, f.y);
        }
        o[i] = v4;
    }
}

__global__ void __launch_bounds__(NTHREADS, 1) tc_narrow_fused_kernel(const __grid_constant__ FParams p) {
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);
    uint8_t* ops = smem + OFF_OPS;
    float* scr = reinterpret_cast<float*>(smem + OFF_SCR);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + OFF_BAR);
    uint64_t* qo_full = bars;          // [2]
    uint64_t* qo_empty = bars + 2;     // [2]
    uint64_t* kfull = bars + 4;        // [RK]
    uint64_t* kempty = bars + 9;       // [RK]
    uint64_t* vfull = bars + 14;       // [RV]
    uint64_t* vempty = bars + 18;      // [RV]
    uint64_t* s_full = bars + 22;      // [2] S(j) done (softmax, converters)
    uint64_t* s_free = bars + 24;      // softmax holds S in registers
    uint64_t* dp_full = bars + 25;     // dP(j) done (and every earlier MMA)
    uint64_t* dp_free = bars + 26;     // softmax holds dP in registers
    uint64_t* p_done = bars + 27;      // P and dS of the tile are in smem
    uint64_t* oq_full = bars + 28;     // [2] dQ MMAs of the tile done (issuer 1)
    uint64_t* accfree = bars + 30;     // [2] dK|dV block drained
    uint64_t* dqfree = bars + 32;      // dQ drained
    uint64_t* opfree = bars + 33;      // the output MMAs of the tile (both issuers) read P / dS
    uint64_t* convB = bars + 34;       // [2] Q_t and the tile's K blocks landed and are fp16
    uint64_t* okv_full = bars + 36;    // [2] dK|dV MMAs of the tile done (issuer 2)
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bars + 38);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int w = p.w;

    // the compressed P / dS atoms rely on zeros outside the band windows
    for (int i = threadIdx.x; i < (int)(OPS / 16); i += NTHREADS)
        reinterpret_cast<uint4*>(ops)[i] = make_uint4(0u, 0u, 0u, 0u);
    fence_proxy_async_smem();
    if (warp == 16) {
        if (lane == 0) {
            for (int i = 0; i < 2; ++i) {
                mbar_init(&qo_full[i], 1);
                mbar_init(&qo_empty[i], 2);
                mbar_init(&s_full[i], 1);
                mbar_init(&oq_full[i], 1);
                mbar_init(&okv_full[i], 1);
                mbar_init(&accfree[i], NSM / 32);
                mbar_init(&convB[i], 1);
            }
            for (int i = 0; i < RK; ++i) { mbar_init(&kfull[i], 1); mbar_init(&kempty[i], 1); }
            for (int i = 0; i < RV; ++i) { mbar_init(&vfull[i], 1); mbar_init(&vempty[i], 1); }
            mbar_init(s_free, NSM / 32);
            mbar_init(dp_full, 1);
            mbar_init(dp_free, NSM / 32);
            mbar_init(p_done, NSM / 32);
            mbar_init(dqfree, NSM / 32);
            mbar_init(opfree, 2);
            fence_barrier_init();
            for (int i = 0; i < p.nr; ++i) {
                tma_prefetch(&p.maps[i].q); tma_prefetch(&p.maps[i].dout);
                tma_prefetch(&p.maps[i].k); tma_prefetch(&p.maps[i].v);
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

    if (warp == 16) {
        if (lane == 0) {   // ---------------------------------------------------- TMA producer
            FCursor cur(p);
            FItem it;
            for (int j = 0; cur.next(p, it); ++j) {
                const FMaps& mp = p.maps[it.rl];
                uint8_t* qo = smem + OFF_QO + (j & 1) * QO;
                if (j >= 2) mbar_wait(&qo_empty[j & 1], ((j >> 1) - 1) & 1);
                trace_ev(p, j, 8);
                mbar_arrive_expect_tx(&qo_full[j & 1], QO);
                tma_load_3d(qo, &mp.q, &qo_full[j & 1], 0, it.m0, it.u);
                tma_load_3d(qo + TILE, &mp.dout, &qo_full[j & 1], 0, it.m0, it.u);
                for (int i = it.cont ? 1 : 0; i < 3; ++i) {
                    const int seq = it.bseq + i, sk = seq % RK;
                    if (seq >= RK) mbar_wait(&kempty[sk], ((seq / RK) - 1) & 1);
                    mbar_arrive_expect_tx(&kfull[sk], BLK);
                    tma_load_3d(smem + OFF_K + sk * BLK, &mp.k, &kfull[sk], 0, it.m0 - w + KB * i, it.u);
                }
                trace_ev(p, j, 9);
                for (int i = it.cont ? 1 : 0; i < 3; ++i) {
                    const int seq = it.bseq + i, sv = seq % RV;
                    if (seq >= RV) mbar_wait(&vempty[sv], ((seq / RV) - 1) & 1);
                    mbar_arrive_expect_tx(&vfull[sv], BLK);
                    tma_load_3d(smem + OFF_V + sv * BLK, &mp.v, &vfull[sv], 0, it.m0 - w + KB * i, it.u);
                }
                trace_ev(p, j, 10);
            }
        }
    } else if (warp == 18) {   // ---------------------------------------------- fp16 converter
        // Q_t and the tile's new K blocks to fp16 in place as soon as they land: dS enters its
        // MMAs as fp16, so the operands it multiplies (Q for dK, K for dQ) and therefore the score
        // GEMM S = Q K^T run in fp16 (exact for bf16 values of magnitude 6.1e-5 .. 65504)
        FCursor cur(p);
        FItem I;
        for (int j = 0; cur.next(p, I); ++j) {
            mbar_wait(&qo_full[j & 1], (j >> 1) & 1);
            if (lane == 0) trace_ev(p, j, 11);
            to_f16(smem + OFF_QO + (j & 1) * QO, smem + OFF_QO + (j & 1) * QO, TILE, lane);
            for (int i = I.cont ? 1 : 0; i < 3; ++i) {
                const int seq = I.bseq + i;
                mbar_wait(&kfull[seq % RK], (seq / RK) & 1);
                uint8_t* blk = smem + OFF_K + (seq % RK) * BLK;
                to_f16(blk, blk, BLK, lane);
            }
            fence_proxy_async_smem();
            warp_arrive(&convB[j & 1]);
            if (lane == 0) trace_ev(p, j, 13);
        }
    } else if (warp == 17 || warp == 19) {
        // Two MMA issuers.  Issuer 1 (warp 17): S(j), dP(j), then dQ(j) once the softmax wrote
        // dS.  Issuer 2 (warp 19): the dK / dV products of tile j.  One thread cannot issue the
        // ~50 MMAs of a tile (N = 64: ~48 clk each in the pipe, 60-90 clk each to issue) and wait
        // on their barriers fast enough (tools/trace_fused.py).
        constexpr uint32_t idS64 = idesc_f16(BM, 64, false, false);      // S: fp16 Q and K
        constexpr uint32_t idS128 = idesc_f16(BM, 128, false, false);
        constexpr uint32_t idS192 = idesc_f16(BM, 192, false, false);
        constexpr uint32_t idP64 = idesc_bf16(BM, 64, false, false);     // dP: bf16 dO and V
        constexpr uint32_t idP128 = idesc_bf16(BM, 128, false, false);
        constexpr uint32_t idP192 = idesc_bf16(BM, 192, false, false);
        constexpr uint32_t idV = idesc_bf16(BM, D, true, true);    // P^T (MN) x dO (MN)
        constexpr uint32_t idK = idesc_f16(BM, D, true, true);     // dS^T (MN) x Q (MN), fp16
        constexpr uint32_t idQ = idesc_f16(BM, D, false, true);    // dS (K) x K_h (MN), fp16
        const uint32_t opsa = smem_u32(ops);
        const uint32_t kring = smem_u32(smem + OFF_K), vring = smem_u32(smem + OFF_V);
        FCursor cur(p), nx(p);
        FItem I, N;
        bool have = cur.next(p, I);
        nx.next(p, N);   // nx runs one item ahead of cur
        if (warp == 17 && lane == 0) {   // ----------------------------------------- issuer 1
            // C[0..192) = A (128 x 64, K-major) x three consecutive ring blocks (K-major), split
            // into contiguous runs of slots
            auto score = [&](uint32_t a_addr, uint32_t ring, int R, int s0, bool f16) {
                const uint64_t ad = sdesc_sw128(a_addr, 16, 1024);
                const uint32_t i64 = f16 ? idS64 : idP64, i128 = f16 ? idS128 : idP128, i192 = f16 ? idS192 : idP192;
                if (s0 + 2 < R) {
                    mma_ss_x4<2, 2>(tbase, ad, sdesc_sw128(ring + s0 * BLK, 16, 1024), i192, 0);
                } else if (s0 + 1 < R) {
                    mma_ss_x4<2, 2>(tbase, ad, sdesc_sw128(ring + s0 * BLK, 16, 1024), i128, 0);
                    mma_ss_x4<2, 2>(tbase + 128, ad, sdesc_sw128(ring, 16, 1024), i64, 0);
                } else {
                    mma_ss_x4<2, 2>(tbase, ad, sdesc_sw128(ring + s0 * BLK, 16, 1024), i64, 0);
                    mma_ss_x4<2, 2>(tbase + 64, ad, sdesc_sw128(ring, 16, 1024), i128, 0);
                }
            };
            int dq_req = 0;
            // dQ(i) = dS K_h: A = dS K-major atoms [dS0|Z], dS1, [Z|dS2].  Issued after S(i+1), so
            // the next tile's score GEMM runs while the softmax finishes tile i
            auto dq_issue = [&](int i, const FItem& X, bool cn) {
                mbar_wait_spin(p_done, i & 1);
                trace_ev(p, i, 15);
                if (!X.warm) {
                    if (dq_req >= 1) mbar_wait_spin(dqfree, (dq_req - 1) & 1);
                    tc_fence_after();
                    const uint32_t k2 = kring + ((X.bseq + 2) % RK) * BLK;
                    mma_ss_x4<2, 128>(tbase + T_DQ, sdesc_sw128(opsa + O_DS0, 16, 1024),
                                      sdesc_sw128(kring + (X.bseq % RK) * BLK, 8192, 1024), idQ, 0);
                    mma_ss_x4<2, 128>(tbase + T_DQ, sdesc_sw128(opsa + O_DS1, 16, 1024),
                                      sdesc_sw128(kring + ((X.bseq + 1) % RK) * BLK, 8192, 1024), idQ, 1);
                    mma_ss_x4<2, 128>(tbase + T_DQ, sdesc_sw128(opsa + O_Z, 16, 1024),
                                      sdesc_sw128(k2, 8192, 1024), idQ, 1);
                    ++dq_req;
                }
                mma_commit(&oq_full[i & 1]);
                mma_commit(opfree);
                for (int g = 0; g < (cn ? 2 : 3); ++g) mma_commit(&kempty[(X.bseq + g) % RK]);
                trace_ev(p, i, 2);
            };
            FItem Pv;
            int j = 0;
            for (; have; ++j) {
                const bool hnext = nx.next(p, N);   // N = item j+1
                const bool cn = hnext && N.cont;
                trace_ev(p, j, 0);
                // a tile that does not continue the previous one loads three fresh K blocks, one
                // of them into the slot the previous tile's dQ frees: its dQ must go first
                if (j >= 1 && !I.cont) dq_issue(j - 1, Pv, false);
                if (j >= 1) mbar_wait_spin(dp_free, (j - 1) & 1);
                const uint32_t qa = smem_u32(smem + OFF_QO + (j & 1) * QO);
                trace_ev(p, j, 25);
                mbar_wait_spin(&convB[j & 1], (j >> 1) & 1);   // Q_j and its K blocks landed, fp16
                trace_ev(p, j, 26);
                tc_fence_after();
                score(qa, kring, RK, I.bseq % RK, true);
                mma_commit(&s_full[j & 1]);
                trace_ev(p, j, 1);
                if (j >= 1 && I.cont) dq_issue(j - 1, Pv, true);
                mbar_wait_spin(s_free, j & 1);
                trace_ev(p, j, 16);
                for (int g = 0; g < 3; ++g) mbar_wait_spin(&vfull[(I.bseq + g) % RV], ((I.bseq + g) / RV) & 1);
                trace_ev(p, j, 23);
                tc_fence_after();
                score(qa + TILE, vring, RV, I.bseq % RV, false);
                trace_ev(p, j, 24);
                mma_commit(dp_full);
                trace_ev(p, j, 3);
                for (int g = 0; g < (cn ? 2 : 3); ++g) mma_commit(&vempty[(I.bseq + g) % RV]);
                mma_commit(&qo_empty[j & 1]);
                Pv = I;
                I = N;
                have = hnext;
            }
            if (j >= 1) dq_issue(j - 1, Pv, false);
        } else if (warp == 19 && lane == 0) {   // ----------------------------------- issuer 2
            int x_req[2] = {0, 0}, x_wait[2] = {0, 0};
            auto wait_x = [&](int b) {
                if (x_req[b] > x_wait[b]) {
                    mbar_wait_spin(&accfree[b], x_wait[b] & 1);
                    ++x_wait[b];
                }
            };
            for (int i = 0; have; ++i) {
                const FItem& X = I;
                mbar_wait_spin(p_done, i & 1);
                trace_ev(p, i, 18);
                const uint32_t qa = smem_u32(smem + OFF_QO + (i & 1) * QO), da = qa + TILE;
                const int a = i & 1, b = a ^ 1;
                const uint32_t XA = tbase + T_X + 128u * a, XB = tbase + T_X + 128u * b;
                if (!X.warm) {
                    if (!X.cont) wait_x(a);
                    tc_fence_after();
                    const uint32_t acc = X.cont ? 1u : 0u;
                    // A_t (halo columns 0..127): queries 0..63 see atoms 0 and 1, queries 64..127
                    // only atom 1 (atom 0 is the zero block Z for them)
                    mma_ss_x4<128, 128>(XA + 64, sdesc_sw128(opsa + O_P0, O_P1 - O_P0, 1024),
                                        sdesc_sw128(da, 8192, 1024), idV, acc);
                    mma_ss_x4<128, 128>(XA + 64, sdesc_sw128(opsa + O_Z, O_P1 + 8192 - O_Z, 1024),
                                        sdesc_sw128(da + 8192, 8192, 1024), idV, 1);
                    mma_ss_x4<128, 128>(XA, sdesc_sw128(opsa + O_DS0, O_DS1 - O_DS0, 1024),
                                        sdesc_sw128(qa, 8192, 1024), idK, acc);
                    mma_ss_x4<128, 128>(XA, sdesc_sw128(opsa + O_Z, O_DS1 + 8192 - O_Z, 1024),
                                        sdesc_sw128(qa + 8192, 8192, 1024), idK, 1);
                }
                trace_ev(p, i, 12);
                // A_{t+1} (columns 128..191, then the zero block): only queries 64..127 reach it
                wait_x(b);
                trace_ev(p, i, 14);
                tc_fence_after();
                mma_ss_x4<128, 128>(XB + 64, sdesc_sw128(opsa + O_P2, O_ZB - O_P2, 1024),
                                    sdesc_sw128(da + 8192, 8192, 1024), idV, 0);
                mma_ss_x4<128, 128>(XB, sdesc_sw128(opsa + O_DS2, O_ZB - O_DS2, 1024),
                                    sdesc_sw128(qa + 8192, 8192, 1024), idK, 0);
                mma_commit(&okv_full[i & 1]);
                mma_commit(opfree);
                mma_commit(&qo_empty[i & 1]);
                trace_ev(p, i, 20);
                if (!X.warm) ++x_req[a];
                if (X.tail) ++x_req[b];
                const bool hnext = nx.next(p, N);
                I = N;
                have = hnext;
            }
        }
    } else {   // ----------------------------------------------------------- softmax warps 0-15
        // warp w: TMEM lanes 32*(w%4).. (thread <-> query row t), columns 24*(w/4) .. +23 of the
        // row's 96-column band window; four warps per row exchange their parts of D in smem
        const int wq = warp & 3, pq = warp >> 2;
        const int t = wq * 32 + lane;
        const uint32_t lane_off = (uint32_t)(wq * 32) << 16;
        const int c0 = 32 * wq + 24 * pq;  // first of this thread's 24 halo columns
        float* dx = scr;                   // [2][4][BM]
        float* lpre = scr + 2 * 4 * BM;    // [2][NSM]
        // 16-byte granule of row t, columns c .. c+7, in the compressed operand atoms
        auto gran = [&](uint32_t o0, uint32_t o1, uint32_t o2, int c) -> uint4* {
            const int a = c >> 6;
            const uint32_t base = a == 0 ? o0 + t * 128 : a == 1 ? o1 + t * 128 : o2 + (t - 64) * 128;
            return reinterpret_cast<uint4*>(ops + base + ((((c & 63) >> 3) ^ (t & 7)) << 4));
        };
        auto prefetch = [&](const FItem& X, int jx) {
            const int mrow = X.m0 + t;
            const bool ok = mrow < X.Lr;
            cp_async4(lpre + (jx & 1) * NSM + threadIdx.x, p.lse + (ok ? X.rowbase + (int64_t)mrow * p.dil : 0),
                      ok ? 4u : 0u);
            cp_async_commit();
        };
        // accumulators of tile i -> HBM: this warp's 32 rows x 16 columns of dQ, dK, dV
        auto drain = [&](int i, const FItem& X) {
            uint32_t va[16], vb[16];
            if (!X.warm) {
                mbar_wait(&oq_full[i & 1], (i >> 1) & 1);
                tc_fence_after();
                tmem_ld16(tbase + lane_off + T_DQ + 16u * pq, va);
                tmem_wait_ld();
                tc_fence_before();
                warp_arrive(dqfree);
                if (threadIdx.x == 0) trace_ev(p, i + 1, 21);
                store_rows16(p.dq, X.rowbase, p.dil, X.m0 + 32 * wq, X.Lr, pq, lane, va);
                mbar_wait(&okv_full[i & 1], (i >> 1) & 1);
                tc_fence_after();
                const uint32_t xa = tbase + lane_off + T_X + 128u * (i & 1);
                tmem_ld16(xa + 16u * pq, va);
                tmem_ld16(xa + 64u + 16u * pq, vb);
                tmem_wait_ld();
                tc_fence_before();
                warp_arrive(&accfree[i & 1]);
                if (threadIdx.x == 0) trace_ev(p, i + 1, 22);
                store_rows16(p.dk, X.rowbase, p.dil, X.m0 - w + 32 * wq, X.Lr, pq, lane, va);
                store_rows16(p.dv, X.rowbase, p.dil, X.m0 - w + 32 * wq, X.Lr, pq, lane, vb);
            }
            if (X.tail) {
                mbar_wait(&okv_full[i & 1], (i >> 1) & 1);
                tc_fence_after();
                const uint32_t xb = tbase + lane_off + T_X + 128u * ((i + 1) & 1);
                tmem_ld16(xb + 16u * pq, va);
                tmem_ld16(xb + 64u + 16u * pq, vb);
                tmem_wait_ld();
                tc_fence_before();
                warp_arrive(&accfree[(i + 1) & 1]);
                store_rows16(p.dk, X.rowbase, p.dil, X.m0 - w + BM + 32 * wq, X.Lr, pq, lane, va);
                store_rows16(p.dv, X.rowbase, p.dil, X.m0 - w + BM + 32 * wq, X.Lr, pq, lane, vb);
            }
        };
        FCursor cur(p), nx(p);
        FItem I, In, Pv;
        bool hn = nx.next(p, In);
        if (hn) prefetch(In, 0);
        int j = 0;
        for (; cur.next(p, I); ++j) {
            cp_async_wait_all();
            const float lse2 = lpre[(j & 1) * NSM + threadIdx.x] * LOG2E;
            hn = nx.next(p, In);
            if (hn) prefetch(In, j + 1);
            // band columns of row t: n in [t, t+2w], keys inside the sequence, query inside too
            const int kb = I.m0 - w;
            const int lo = max(t, -kb) - c0;
            const int hi = (I.m0 + t < I.Lr) ? min(t + 2 * w, I.Lr - 1 - kb) - c0 : -1;
            const int l0 = max(lo, 0), h0 = min(hi, 23);
            const uint32_t bits = h0 < l0 ? 0u : ((~0u >> (31 - h0)) & (~0u << l0));

            mbar_wait(&s_full[j & 1], (j >> 1) & 1);
            tc_fence_after();
            const bool tr = threadIdx.x == 0;
            if (tr) trace_ev(p, j, 4);
            uint32_t rs[24], rd[24];
            tmem_ld16(tbase + lane_off + c0, *reinterpret_cast<uint32_t(*)[16]>(&rs[0]));
            tmem_ld8(tbase + lane_off + c0 + 16, &rs[16]);
            tmem_wait_ld();
            tc_fence_before();
            warp_arrive(s_free);
            uint32_t pk[12];
#pragma unroll
            for (int e = 0; e < 24; e += 2) {
                const float p0 = ((bits >> e) & 1u) ? fast_exp2(fmaf(__uint_as_float(rs[e]), LOG2E, -lse2)) : 0.f;
                const float p1 = ((bits >> (e + 1)) & 1u) ? fast_exp2(fmaf(__uint_as_float(rs[e + 1]), LOG2E, -lse2)) : 0.f;
                rs[e] = __float_as_uint(p0);
                rs[e + 1] = __float_as_uint(p1);
                pk[e / 2] = pack_bf16x2(p0, p1);
            }
            // while dP(j) runs: P to smem and the accumulators of tile j-1 to HBM, both once
            // tile j-1's output MMAs completed
            if (j >= 1) mbar_wait(opfree, (j - 1) & 1);
#pragma unroll
            for (int g = 0; g < 3; ++g)
                *gran(O_P0, O_P1, O_P2, c0 + 8 * g) = make_uint4(pk[4 * g], pk[4 * g + 1], pk[4 * g + 2], pk[4 * g + 3]);
            if (j >= 1) drain(j - 1, Pv);
            if (tr) trace_ev(p, j, 7);
            mbar_wait(dp_full, j & 1);
            tc_fence_after();
            if (tr) trace_ev(p, j, 5);
            tmem_ld16(tbase + lane_off + c0, *reinterpret_cast<uint32_t(*)[16]>(&rd[0]));
            tmem_ld8(tbase + lane_off + c0 + 16, &rd[16]);
            tmem_wait_ld();
            tc_fence_before();
            warp_arrive(dp_free);
            float dpart[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
            for (int e = 0; e < 24; ++e) dpart[e & 3] = fmaf(__uint_as_float(rs[e]), __uint_as_float(rd[e]), dpart[e & 3]);
            float* dxb = dx + (j & 1) * 4 * BM;
            dxb[pq * BM + t] = (dpart[0] + dpart[1]) + (dpart[2] + dpart[3]);
            named_bar_sync(1 + wq, 128);   // all four parts of the row posted their part of D
            if (tr) trace_ev(p, j, 17);
            const float Dv = (dxb[t] + dxb[BM + t]) + (dxb[2 * BM + t] + dxb[3 * BM + t]);
#pragma unroll
            for (int e = 0; e < 24; e += 2) {
                const float d0 = __uint_as_float(rs[e]) * (__uint_as_float(rd[e]) - Dv);
                const float d1 = __uint_as_float(rs[e + 1]) * (__uint_as_float(rd[e + 1]) - Dv);
                pk[e / 2] = pack_f16x2(d0, d1);
            }
#pragma unroll
            for (int g = 0; g < 3; ++g)
                *gran(O_DS0, O_DS1, O_DS2, c0 + 8 * g) = make_uint4(pk[4 * g], pk[4 * g + 1], pk[4 * g + 2], pk[4 * g + 3]);
            fence_proxy_async_smem();
            warp_arrive(p_done);
            if (tr) trace_ev(p, j, 6);
            Pv = I;
        }
        if (j >= 1) drain(j - 1, Pv);
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 16) {
        tc_fence_after();
        tmem_dealloc(tbase, 512);
    }
}

int num_sms_nf() {
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

}  // namespace

bool tc_narrow_fused_ok(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    // Default from ~4 tiles per SM (C5_w32: 0.620 vs 0.648 ms for NQ + NKV, same box);
    // FT_WINATTN_FUSED=0 selects the split kernels (A/B timing), =2 forces it (tests).
    const char* e = getenv("FT_WINATTN_FUSED");
    const int mode = e ? atoi(e) : 1;
    if (mode != 1 && mode != 2) return false;
    if (!tc_narrow_bwd_supported(units, L, d, w, dil)) return false;
    const int64_t nres = dil < L ? dil : L;
    const int64_t tiles = ceil_div(ceil_div(L, dil), BM);
    // each strip pays one warm-up tile: worth it from ~4 tiles per CTA
    return mode == 2 || units * nres * tiles >= 4 * (int64_t)num_sms_nf();
}

int tc_narrow_fused_launches(int64_t L, int64_t dil) {
    const int64_t nres = dil < L ? dil : L;
    return (int)ceil_div(nres, RES_PER_LAUNCH);
}

cudaError_t tc_narrow_fused_bwd(const void* q, const void* k, const void* v, const float* lse,
                                const void* dout, void* dq, void* dk, void* dv, int64_t B, int64_t H,
                                int64_t L, int64_t w, int64_t dil, cudaStream_t st, int* launches) {
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_narrow_fused_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)SMEM_BYTES);
    });
    const int64_t wc = w < L ? w : L;
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    int n = 0;
    for (int64_t r0 = 0; r0 < nres; r0 += RES_PER_LAUNCH) {
        FParams p;
        memset(&p, 0, sizeof(p));
        const int nr = (int)(nres - r0 < RES_PER_LAUNCH ? nres - r0 : RES_PER_LAUNCH);
        for (int i = 0; i < nr; ++i) {
            const int64_t r = r0 + i;
            FMaps& m = p.maps[i];
            if (!(make_residue_map(&m.q, q, L, D, units, dil, r, BM) &&
                  make_residue_map(&m.dout, dout, L, D, units, dil, r, BM) &&
                  make_residue_map(&m.k, k, L, D, units, dil, r, KB) &&
                  make_residue_map(&m.v, v, L, D, units, dil, r, KB)))
                return cudaErrorInvalidValue;
            p.Lr[i] = (int)ceil_div(L - r, dil);
        }
        p.lse = lse;
        p.dq = static_cast<uint16_t*>(dq);
        p.dk = static_cast<uint16_t*>(dk);
        p.dv = static_cast<uint16_t*>(dv);
        p.L = L;
        p.w = (int)wc;
        p.dil = (int)dil;
        p.tiles = (int)ceil_div(p.Lr[0], BM);
        p.nr = nr;
        p.r0 = (int)r0;
        p.ntau = (long long)units * nr * p.tiles;
        p.trace = (unsigned long long*)trace_buffer(1);
        dim3 grid((unsigned)(p.ntau < num_sms_nf() ? p.ntau : num_sms_nf()));
        tc_narrow_fused_kernel<<<grid, NTHREADS, SMEM_BYTES, st>>>(p);
        prof_mark(st);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        ++n;
    }
    if (launches) *launches += n;
    return cudaSuccess;
}

}  // namespace ftw
