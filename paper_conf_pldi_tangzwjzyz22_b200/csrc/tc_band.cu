// tc_band.cu -- tcgen05/TMEM tensor-core kernels of banded window attention for sm_100a
// (bf16 storage; fp32 scores, softmax statistics and accumulators), windows with
// 128 + 2w <= 256 halo rows (w <= 64).  Wider windows: tc_chunk.cu.
//
// One persistent kernel template, three modes.  A CTA owns BM = 128 rows m0..m0+127 of one
// (unit, residue) band problem at a time, and the NK = round_up(128 + 2w, 64) <= 256-row
// halo m0-w .. of the other operand: the cached a[i:i+m] window of PAPER.md Fig. 14
// (lines 402-423), staged by TMA instead of the (2w+1)-fold as_strided copy of Q that the
// operator baseline makes (Fig. 1c).
//
//   FWD   rows = queries.  S = Q K_h^T -> row max, exp, row sum (the fused dot/max of
//         Fig. 10 and dot_norm/softmax of Fig. 8), lse -> HBM,
//         P (bf16) -> smem;  O_c = P V_h,c  (c = 256-column output chunks), scaled by 1/l.
//   BWDQ  rows = queries.  S = Q K_h^T, dP = dO V_h^T;  P = exp(S - lse) (recomputed from the
//         saved lse: selective materialization);  D = sum_j P dP (exact,
//         written to the workspace);  dS = P (dP - D) (bf16 hi/lo) -> TMEM;  dQ_c = dS K_h,c.
//   BWDKV rows = keys (tile ownership: each dk/dv row has exactly one writer, no atomics;
//         the parallel-reduction choice of PAPER.md Fig. 13(d) over 13(e)).  S^T = K Q_h^T,
//         dP^T = V dO_h^T;  P^T = exp(S^T - lse_col) -> smem, dS^T = P^T (dP^T - D_col)
//         (bf16 hi/lo) -> TMEM;  dV_c = P^T dO_h,c,  dK_c = dS^T Q_h,c.
//
// Instruction economy (profiles/README.md, tools/mma_microbench.cu): a 1-SM tcgen05.mma
// costs ~150-300 cycles whatever its N, so output GEMMs use N = 256-column chunks whose B
// operand (V, K, dO or Q of the halo) is streamed in 64-row key blocks, and FWD issues the
// next tile's QK^T right after this tile's first output chunk.
//
// Roles (320 threads): warps 0-3 softmax (thread t <-> row m0+t <-> TMEM lane t), warps 4-7
// epilogue (TMEM -> bf16 -> smem -> warp-local TMA store), warp 8 TMA producer + TMEM
// allocator, warp 9 MMA issuer.  Halo column n is residue row m0 - w + n, and
// |m_col - m_row| <= w  <=>  0 <= n - t <= 2w, so one mask serves all three modes.
//
// TMEM (512 columns): S (or S^T) at [0, NK), dP (dP^T) at [256, 256+NK); dS / dS^T bf16
// hi/lo overwrite S in place; the output accumulator is [256, 256 + chunk) once the
// scores are consumed.
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

enum { FWD = 0, BWDQ = 1, BWDKV = 2 };

constexpr int BM = 128;
constexpr int KB = 64;                   // key-block rows of an output-GEMM B operand
constexpr int RES_PER_LAUNCH = 8;        // residues per launch (8 tensor maps each; kernel params up to 32 KB)
static_assert(RES_PER_LAUNCH <= SCHED_MAX_RES, "residue table of the tile cursor");
constexpr uint32_t ABYTES = BM * 128;    // one 128-row x 64-col bf16 slice (SW128)
constexpr uint32_t OBOX = KB * 128;      // one 64-row x 64-col bf16 box
constexpr uint32_t STG = 32 * 128;       // one warp's 32-row x 64-col staging slice
constexpr int NSTG = 1;                  // staging slices per epilogue warp
constexpr int NTHREADS = 352;
constexpr int MAX_NST = 8;
constexpr size_t SMEM_LIMIT = 227 * 1024;
constexpr float LOG2E = 1.4426950408889634f;
constexpr float LN2 = 0.6931471805599453f;

template <int MODE> struct Cfg {
    static constexpr int NA = MODE == FWD ? 1 : 2;       // score GEMMs; also slots per G slice
    static constexpr int NOUT = MODE == BWDKV ? 2 : 1;   // output tensors per chunk
    static constexpr bool PSMEM = MODE != BWDQ;          // P / P^T staged in smem
};

// a1/b1, a2/b2: score-GEMM operands (A: rows m0.., box 128; B: halo rows m0-w.., box NK);
// ob1/ob2: output-GEMM B operands (halo, box 64 rows); o1/o2: outputs (box 32 rows).
struct Maps {
    CUtensorMap a1, b1, a2, b2, ob1, ob2, o1, o2;
    CUtensorMap tp, ts;   // BWDKV with the dS tape (xt): P / dS planes, boxes of trows rows
};
struct Params {
    Maps maps[RES_PER_LAUNCH];
    float* lse;   // FWD: written; BWD: read
    float* D;     // BWDQ: written; BWDKV: read
    int64_t L;
    int d, w, dil, NK, nsl, nst;
    SchedParams sc;
    unsigned long long* trace;   // optional phase trace (ft_winattn_debug_trace)
    int two;                     // 1: two MMA issuers (warps 9, 10); 0: warp 9 issues all
    int dpoll;                   // BWDKV: poll D row by row instead of waiting for all of BWDQ
    int lsepoll;                 // FWD -> BWDQ lse hand-off: FWD marks its lse rows unset and
                                 // triggers; BWDQ (PDL) and BWDKV poll lse rows
    float* tape;                 // optional score tape (ft_winattn_fwd_tape / _bwd_tape): fp32
                                 // [rows][2w + 1], entry (row i, k + w) = s_ij, key j = i + k dil
                                 // (the materialized `dot` of Fig. 8).  FWD writes it; BWDQ / BWDKV
                                 // read s from it and skip the score GEMM S = Q K^T (selective
                                 // materialization)
    int tstride;                 // tape row stride, elements (2w + 1)
    // dS tape between BWDQ and BWDKV (ftw::DsTape, internal.h; the fp32 kernels' scheme,
    // tc_band32.cu): BWDQ stores P and dS of every band entry and releases a flag per tile;
    // BWDKV (xt) loads them instead of running the S^T and dP^T GEMMs.
    int xt, tsw, trows;          // trows: tape rows per ring slot (both planes; boxes of trows + 1)
    int64_t grows;               // tape granule stride (rows)
    uint32_t* flags;
    float* tP;
    float* tS;
};


// Phase trace: per CTA and local tile j < TRACE_TILES, clock64 stamps (SM cycles) of
// 0 producer first score-GEMM load, 1 producer last output load, 2 MMA score GEMM first
// stage ready, 3 MMA s_full commit, 4 MMA p_full seen, 5 MMA last output MMA issued,
// 6 softmax s_full seen, 7 softmax p_full arrive, 8 epilogue first o_full, 9 epilogue done.
constexpr int TRACE_TILES = 8, TRACE_EV = 48;
__device__ __forceinline__ void trace_ev(const Params& p, int j, int ev) {
    if (p.trace && j < TRACE_TILES) {
        p.trace[((size_t)blockIdx.x * TRACE_TILES + j) * TRACE_EV + ev] = clock64();   // SM cycles
    }
}

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ void split_bf16x2(float x0, float x1, uint32_t& hi, uint32_t& lo) {
    split_bf16x2_p(x0, x1, hi, lo);   // tc_common.cuh: one packed subtraction
}
__device__ __forceinline__ bool band_ok(int n, int t, int w, int mcol, int Lr) {
    return (unsigned)(n - t) <= (unsigned)(2 * w) && mcol >= 0 && mcol < Lr;
}

// One tape plane's box in a ring slot ([tsw / 4][trows + 1][4] floats), padded so that the second
// plane's TMA destination is 128-byte aligned.
__host__ __device__ inline uint32_t tape_plane_bytes(int trows, int tsw) {
    return ((uint32_t)(trows + 1) * (uint32_t)tsw * 4u + 127u) & ~127u;
}
__host__ __device__ inline int chunk_w(int d, int c) { return d - 256 * c < 256 ? d - 256 * c : 256; }

__host__ __device__ inline uint32_t slot_bytes(int NK) {
    const uint32_t g = ABYTES + (uint32_t)NK * 128u;
    const uint32_t o = 4u * OBOX;
    return g > o ? g : o;
}
// Fixed shared memory besides the slot ring, carved tightly so that one more 40 KB slot
// fits: alignment slack, P / P^T, epilogue staging, per-mode scratch (BWDKV column lse/D,
// FWD row scales), barriers.
constexpr size_t BAR_BYTES = 256;
template <int MODE>
__host__ __device__ inline size_t scratch_bytes(int NK) {
    return MODE == BWDKV ? 2 * (size_t)NK * sizeof(float) : (MODE == FWD ? 3 * 128 * sizeof(float) : 0);
}
template <int MODE>
inline size_t fixed_smem_bytes(int NK) {
    return 1024 + (Cfg<MODE>::PSMEM ? (size_t)NK * 256 : 0) + 4 * NSTG * STG +
           scratch_bytes<MODE>(NK) + BAR_BYTES;
}
template <int MODE>
inline int pick_nst(int NK) {
    const size_t fixed = fixed_smem_bytes<MODE>(NK);
    if (fixed >= SMEM_LIMIT) return 0;
    int n = (int)((SMEM_LIMIT - fixed) / slot_bytes(NK));
    return n < MAX_NST ? n : MAX_NST;
}

using Tile = SchedTile;
using TileCursor = SchedCursor<BM>;

// P / P^T in smem as the K-major SWIZZLE_128B A operand: 64-column atoms of 16 KB, row t at
// t*128, 16-byte granule g at ((g ^ (t & 7)) * 16).  Thread t writes its row's 32-column
// chunk c (16 packed words).
__device__ __forceinline__ void st_p_chunk(uint8_t* P, int t, int c, const uint32_t (&pk)[16]) {
    uint8_t* row = P + (c >> 1) * (BM * 128) + t * 128;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int g = (c & 1) * 4 + q;
        *reinterpret_cast<uint4*>(row + ((g ^ (t & 7)) * 16)) =
            make_uint4(pk[4 * q], pk[4 * q + 1], pk[4 * q + 2], pk[4 * q + 3]);
    }
}

// Masked max of one 32-column score chunk (columns n0 .. n0+31 of the halo).
__device__ __forceinline__ float chunk_max(const uint32_t (&rr)[32], int n0, int t, int w, int kb,
                                           int Lr, float mx) {
#pragma unroll
    for (int e = 0; e < 32; ++e)
        if (band_ok(n0 + e, t, w, kb + n0 + e, Lr)) mx = fmaxf(mx, __uint_as_float(rr[e]));
    return mx;
}
// P = exp2(S*log2e - mxs) on one chunk (masked), packed to bf16 into the smem P operand;
// returns the chunk's contribution to the row sum.
__device__ __forceinline__ float chunk_exp_store(uint8_t* sP, const uint32_t (&rr)[32], int c,
                                                 int t, int w, int kb, int Lr, float mxs) {
    uint32_t pk[16];
    float s0 = 0.f, s1 = 0.f;   // two partial sums, packed f32x2 pairs
#pragma unroll
    for (int e = 0; e < 32; e += 2) {
        const int n = c * 32 + e;
        float a0, a1;
        ffma2_bc(__uint_as_float(rr[e]), __uint_as_float(rr[e + 1]), LOG2E, -mxs, a0, a1);
        const float p0 = band_ok(n, t, w, kb + n, Lr) ? fast_exp2(a0) : 0.f;
        const float p1 = band_ok(n + 1, t, w, kb + n + 1, Lr) ? fast_exp2(a1) : 0.f;
        fadd2_acc(s0, s1, p0, p1);
        pk[e / 2] = pack_bf16x2(p0, p1);
    }
    st_p_chunk(sP, t, c, pk);
    return s0 + s1;
}

// TAPE: score tape read (BWDQ / BWDKV) or written (FWD) -- a separate instantiation, so the plain
// kernels carry no tape code in their softmax loops
template <int MODE, bool TAPE>
__global__ void __launch_bounds__(NTHREADS, 1) tc_band_kernel(const __grid_constant__ Params p) {
    using C = Cfg<MODE>;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int NK = p.NK, nsl = p.nsl, w = p.w, NST = p.nst, d = p.d;
    // backward with a P tape: only the dP GEMM runs in the score phase (one slot per slice)
    constexpr bool tp = TAPE && MODE != FWD;
    // Programmatic dependent launch (BWDQ -> BWDKV, launch_pdl): BWDKV CTAs may take the SMs
    // BWDQ CTAs leave (its persistent CTAs finish 4 or 5 tiles apart) and stream their first
    // tiles' q/k/v/dout -- inputs of the whole backward call, complete before BWDQ started --
    // while BWDQ drains; only BWDKV's softmax warps, which read BWDQ's D, wait for it.
    if (MODE == BWDQ && p.xt) {   // clear this CTA's tile flags before BWDKV may launch
        TileCursor cr(p.sc);
        Tile T;
        while (cr.next(p.sc, T))
            if (threadIdx.x == 0) p.flags[(int64_t)T.u * p.L + T.r + (int64_t)T.m0 * p.dil] = 0u;
        __threadfence();
        __syncthreads();
    } else if (MODE == BWDQ && p.dpoll) {
        // mark this CTA's D rows unset before BWDKV may launch (ld_D_ready); the CTA stores
        // the real values of the same rows later, ordered after this by the barrier
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
    if (MODE == FWD && p.lsepoll) {
        // lse hand-off to a following BWDQ launched with PDL: same scheme as D (ld_lse_ready)
        TileCursor cr(p.sc);
        Tile T;
        while (cr.next(p.sc, T)) {
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;
            for (int i = threadIdx.x; i < BM && T.m0 + i < T.Lr; i += NTHREADS)
                reinterpret_cast<uint32_t*>(p.lse)[rowbase + (int64_t)(T.m0 + i) * p.dil] = D_UNSET;
        }
        __threadfence();
        __syncthreads();
    }
    if (MODE == BWDQ || (MODE == FWD && p.lsepoll))
        asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int nkb = NK / KB;
    const int ncw = (d + 255) / 256;            // output chunks
    // BWDKV with d <= 128: dV and dK accumulate side by side ([256, 256+d) and
    // [256+d, 256+2d)) with interleaved MMAs; otherwise one output per accumulation.
    const bool dual = MODE == BWDKV && 2 * d <= 256;
    // BWDQ with NK + d <= 256 (d = 64, w <= 32): the dQ accumulator fits beside both score
    // regions at [256 + NK, 256 + NK + d), so dS can be handed to the MMA per 64-key block
    // while the softmax is still reading dP, and the next tile's score GEMMs need not wait
    // for the epilogue drain.
    const bool early = MODE == BWDQ && NK + d <= 256;
    const uint32_t acc0 = early ? 256u + (uint32_t)NK : 256u;   // accumulator base column
    const int nacc = dual ? ncw : ncw * C::NOUT;   // accumulations per tile
    const uint32_t SLOT = slot_bytes(NK);
    const uint32_t HB = (uint32_t)NK * 128u;

    uint8_t* sslots = smem;                                          // NST slots
    uint8_t* sP = smem + (size_t)NST * SLOT;                         // P / P^T (PSMEM)
    uint8_t* ostg = sP + (C::PSMEM ? (size_t)NK * 256 : 0);          // [4 warps][NSTG]
    float* scratch = reinterpret_cast<float*>(ostg + 4 * NSTG * STG);
    float* colLse = scratch;                                         // BWDKV [NK]
    float* colD = scratch + NK;                                      // BWDKV [NK]
    float* rowScale = scratch;                                       // FWD [3][128]
    uint64_t* bars = reinterpret_cast<uint64_t*>(reinterpret_cast<uint8_t*>(scratch) +
                                                 scratch_bytes<MODE>(NK));
    uint64_t* full = bars;
    uint64_t* empty = bars + MAX_NST;
    uint64_t* s_full = bars + 2 * MAX_NST;
    uint64_t* p_full = s_full + 1;
    uint64_t* o_full = s_full + 2;
    uint64_t* o_empty = s_full + 3;
    uint64_t* p_free = s_full + 4;   // P smem consumed by the tile's output MMAs
    uint64_t* p_blk = s_full + 5;    // [4] BWD: dS of 64-key block b written (per-block handoff)
    uint64_t* a_free = s_full + 9;   // xt: the tile's dK MMAs are done with dS^T in TMEM
    uint64_t* tape_done = s_full + 10;   // xt3: BWDQ pass 3 read the tile's dS / P from TMEM
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(s_full + 11);
    const bool xt = MODE == BWDKV && p.xt;
    // BWDQ with the dS tape and free TMEM columns [XT3_COL, 256) beside S (NK <= 192): pass 3
    constexpr uint32_t XT3_COL = 192;
    const bool xt3 = !TAPE && MODE == BWDQ && p.xt && NK <= (int)XT3_COL && !early;
    const int ntape = xt ? NK / p.trows : 0;   // tape slots per tile

    if (warp == 8) {
        if (lane == 0) {
            // Arrival counts: both MMA issuers pass every slot; s_full / o_full are committed
            // by the issuers owning a chain of that GEMM (see the MMA issuers below).
            for (int i = 0; i < NST; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], p.two ? 2 : 1); }
            mbar_init(s_full, MODE != FWD && p.two ? 2 : 1);
            mbar_init(p_full, 128);
            mbar_init(o_full, dual && p.two ? 2 : 1);
            mbar_init(o_empty, 128);
            mbar_init(p_free, 1);
            for (int i = 0; i < 4; ++i) mbar_init(&p_blk[i], 128);
            mbar_init(a_free, 1);
            mbar_init(tape_done, 128);
            fence_barrier_init();
            for (int i = 0; i < p.sc.nr; ++i) {
                const Maps& mp = p.maps[i];
                tma_prefetch(&mp.a1); tma_prefetch(&mp.b1); tma_prefetch(&mp.ob1); tma_prefetch(&mp.o1);
                if (C::NA == 2) { tma_prefetch(&mp.a2); tma_prefetch(&mp.b2); }
                if (C::NOUT == 2) { tma_prefetch(&mp.ob2); tma_prefetch(&mp.o2); }
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
        if (lane == 0) {   // ------------------------------------------------ TMA producer
            // Slot order = MMA consumption order.  FWD: G(0), then per tile j:
            // O_0(j), G(j+1), O_1(j) .. O_last(j).  BWD: per tile: G(j), O_0(j) .. O_last(j).
            int st = 0;
            uint32_t ph = 0;
            auto take = [&]() -> uint8_t* {
                mbar_wait(&empty[st], ph ^ 1u);
                return sslots + (size_t)st * SLOT;
            };
            auto adv = [&]() { if (++st == NST) { st = 0; ph ^= 1u; } };
            auto load_g_slice = [&](const Tile& T, int j, int s) {
                const Maps& mp = p.maps[T.rl];
                uint8_t* sp;
                if (!tp) {
                    sp = take();
                    if (s == 0) trace_ev(p, j, 0);
                    mbar_arrive_expect_tx(&full[st], ABYTES + HB);
                    tma_load_3d(sp, &mp.a1, &full[st], s * 64, T.m0, T.u);
                    tma_load_3d(sp + ABYTES, &mp.b1, &full[st], s * 64, T.m0 - w, T.u);
                    adv();
                }
                if (C::NA == 2) {
                    sp = take();
                    mbar_arrive_expect_tx(&full[st], ABYTES + HB);
                    tma_load_3d(sp, &mp.a2, &full[st], s * 64, T.m0, T.u);
                    tma_load_3d(sp + ABYTES, &mp.b2, &full[st], s * 64, T.m0 - w, T.u);
                    adv();
                }
            };
            auto load_o_block = [&](const Tile& T, int a, int kb) {   // key block kb of accumulation a
                const Maps& mp = p.maps[T.rl];
                const int c = dual ? a : a / C::NOUT;
                const CUtensorMap* m = (C::NOUT == 2 && !dual && (a & 1)) ? &mp.ob2 : &mp.ob1;
                const int nbox = chunk_w(d, c) / 64;
                uint8_t* sp = take();
                mbar_arrive_expect_tx(&full[st], (dual ? 2 : 1) * nbox * OBOX);
                for (int b = 0; b < nbox; ++b) {
                    tma_load_3d(sp + b * OBOX, m, &full[st], 256 * c + 64 * b, T.m0 - w + kb * KB, T.u);
                    if (dual)
                        tma_load_3d(sp + (nbox + b) * OBOX, &mp.ob2, &full[st], 256 * c + 64 * b,
                                    T.m0 - w + kb * KB, T.u);
                }
                adv();
            };
            TileCursor cg(p.sc), co(p.sc);
            Tile Tg, To;
            bool hg = cg.next(p.sc, Tg);
            int jg = 0, jo = 0;
            if (MODE == FWD && hg) {
                for (int s = 0; s < nsl; ++s) load_g_slice(Tg, jg, s);
                ++jg;
                hg = cg.next(p.sc, Tg);
            }
            while (co.next(p.sc, To)) {
                if (MODE == FWD) {
                    // G(j+1) slices and O(j) key blocks alternate, the order in which the
                    // two issuers consume them concurrently (one issuer: G(j+1) first).
                    const int nG = hg ? nsl : 0, nO = nacc * nkb;
                    for (int gi = 0, oi = 0; gi < nG || oi < nO;) {
                        if (gi < nG) load_g_slice(Tg, jg, gi++);
                        if (oi < nO && (p.two || gi == nG)) { load_o_block(To, oi / nkb, oi % nkb); ++oi; }
                    }
                    if (hg) { ++jg; hg = cg.next(p.sc, Tg); }
                } else {   // BWD: G(j) then O(j) (dS lives in the S columns)
                    if (xt) {   // dS tape: trows query rows of both planes per slot
                        const Maps& mp = p.maps[To.rl];
                        if (p.dpoll) {   // BWDQ may still run: wait for the tiles of the halo rows
                            const int64_t rowbase = (int64_t)To.u * p.L + To.r;
                            const int lo = max(0, To.m0 - w) / BM, hi = min(To.Lr - 1, To.m0 + BM - 1 + w) / BM;
                            for (int tq = lo; tq <= hi; ++tq) wait_flag(p.flags + rowbase + (int64_t)tq * BM * p.dil);
                            asm volatile("fence.proxy.async.global;" ::: "memory");
                        }
                        const uint32_t pl = tape_plane_bytes(p.trows, p.tsw);
                        for (int b = 0; b < ntape; ++b) {
                            uint8_t* sp = take();
                            if (b == 0) trace_ev(p, jo, 0);
                            mbar_arrive_expect_tx(&full[st], 2u * (uint32_t)(p.trows + 1) * (uint32_t)p.tsw * 4u);
                            tma_load_4d(sp, &mp.tp, &full[st], 0, To.m0 - w + p.trows * b, To.u, 0);
                            tma_load_4d(sp + pl, &mp.ts, &full[st], 0, To.m0 - w + p.trows * b, To.u, 0);
                            adv();
                        }
                    }
                    if (!xt)
                        for (int s = 0; s < nsl; ++s) load_g_slice(To, jo, s);
                    for (int a = 0; a < nacc; ++a)
                        for (int kb = 0; kb < nkb; ++kb) load_o_block(To, a, kb);
                }
                trace_ev(p, jo, 1);
                ++jo;
            }
        }
    } else if (warp == 9 || warp == 10) {
        if (lane == 0 && (warp == 9 || p.two)) {   // ------------------------------ MMA issuers
            // A dependent tcgen05.mma chain advances one instruction per ~350 cycles
            // whatever its N, and one issuing thread sustains ~115-150 cycles per
            // instruction (tools/mma_microbench.cu): independent chains go to different
            // issuers.  Issuer 0: S / S^T, and the BWD outputs (BWDKV dual: dV); issuer 1:
            // dP / dP^T, the FWD outputs O(j) (concurrent with issuer 0's G(j+1)), and
            // BWDKV dual dK.  Both walk every ring slot in order (full wait, then commit or
            // plain arrive on empty, count 2), so slot phases stay consistent.
            // With p.two == 0 warp 9 owns every chain.
            const int h = warp - 9;
            const bool one = !p.two;
            const uint32_t idS = idesc_bf16(128, NK, false, false);
            const bool ownS = one || h == 0, ownDP = one || h == 1;
            const bool ownSmemA = one || (MODE == FWD ? h == 1 : h == 0);   // P / P^T operand
            const bool ownTmemA = one || (dual ? h == 1 : h == 0);           // dS / dS^T operand
            const int otr = MODE == FWD && !one ? 1 : 0;                     // issuer tracing outputs
            int st = 0, ga = 0;   // ga: global accumulation counter (o_full / o_empty phase)
            int jo_cur = 0;       // local index of the tile whose outputs are being issued
            uint32_t ph = 0;
            auto wait_full = [&]() -> uint32_t {
                mbar_wait(&full[st], ph);
                tc_fence_after();
                return smem_u32(sslots + (size_t)st * SLOT);
            };
            auto release = [&](bool used) {
                if (used) mma_commit(&empty[st]);
                else mbar_arrive(&empty[st]);
                if (++st == NST) { st = 0; ph ^= 1u; }
            };
            auto g_slice = [&](int j, int s) {
                if (!tp) {
                    const uint32_t a1 = wait_full();
                    if (s == 0 && h == 0) trace_ev(p, j, 2);
                    if (ownS) {
                        const uint32_t b1 = a1 + ABYTES;
#pragma unroll
                        for (int kk = 0; kk < 4; ++kk)
                            mma_ss(tbase, sdesc_sw128(a1 + kk * 32, 16, 1024),
                                   sdesc_sw128(b1 + kk * 32, 16, 1024), idS, (s | kk) != 0);
                    }
                    release(ownS);
                }
                if (C::NA == 2) {
                    const uint32_t a2 = wait_full();
                    if (ownDP) {
                        const uint32_t b2 = a2 + ABYTES;
#pragma unroll
                        for (int kk = 0; kk < 4; ++kk)
                            mma_ss(tbase + 256, sdesc_sw128(a2 + kk * 32, 16, 1024),
                                   sdesc_sw128(b2 + kk * 32, 16, 1024), idS, (s | kk) != 0);
                    }
                    release(ownDP);
                }
                if (s == nsl - 1) {
                    if ((MODE != FWD && !one) || ownS) mma_commit(s_full);
                    if (h == 0) trace_ev(p, j, 3);
                    if (h == 0 && MODE == FWD && j > 0) trace_ev(p, j - 1, 14);   // G(j) issued during tile j-1
                }
            };
            auto o_block = [&](int a, int kb) {   // key block kb of accumulation a -> [acc0, acc0+cw)
                const int c = dual ? a : a / C::NOUT;
                const int cw = chunk_w(d, c);
                const uint32_t idO = idesc_bf16(128, cw, false, true);
                const bool smemA = ownSmemA && C::PSMEM && (C::NOUT == 1 || dual || (a & 1) == 0);
                const bool tmemA = ownTmemA && (MODE == BWDQ || (MODE == BWDKV && (dual || (a & 1) == 1)));
                const bool own = smemA || tmemA;
                const uint32_t sPa = smem_u32(sP);
                const uint32_t tD0 = tbase + acc0, tD1 = tbase + acc0 + (dual ? cw : 0);
                const uint32_t boff = dual ? (uint32_t)(cw / 64) * OBOX : 0u;   // dK's B boxes
                // the epilogue drained the accumulator.  In BWD the other issuer waits too:
                // it waits on o_empty again before the next score GEMMs, and a parity wait
                // is only unambiguous while the waiter is at most one phase ahead.
                if ((own || MODE != FWD) && kb == 0 && ga > 0) {
                    mbar_wait(o_empty, (ga - 1) & 1);
                    tc_fence_after();
                }
                if (own && a == 0 && kb == 0) trace_ev(p, jo_cur, 12);
                if (own && early && a == 0) {   // dS of this 64-key block written?
                    mbar_wait(&p_blk[kb], jo_cur & 1);
                    tc_fence_after();
                }
                const uint32_t bb = wait_full();
                if (own && a == 0 && kb == 0) trace_ev(p, jo_cur, 13);
#pragma unroll
                for (int k4 = 0; k4 < 4; ++k4) {
                    const int kk = kb * 4 + k4;   // 16-key step over the halo
                    const uint32_t acc = (kk != 0);
                    if (smemA) {   // P (FWD) or P^T (BWDKV dV) from smem
                        const uint64_t bd = sdesc_sw128(bb + k4 * 2048, OBOX, 1024);
                        const uint64_t ad = sdesc_sw128(sPa + (kk >> 2) * (BM * 128) + (kk & 3) * 32, 16, 1024);
                        mma_ss(tD0, ad, bd, idO, acc);
                    }
                    if (tmemA) {   // dS (BWDQ) or dS^T (BWDKV dK), hi/lo in TMEM over S
                        const uint64_t bd = sdesc_sw128(bb + boff + k4 * 2048, OBOX, 1024);
                        const uint32_t tA = tbase + 32u * (kk >> 1) + 8u * (kk & 1);
                        mma_ts(tD1, tA, bd, idO, acc);
                        mma_ts(tD1, tA + 16, bd, idO, 1);
                    }
                }
                release(own);
                if (kb == nkb - 1) {
                    if (own) mma_commit(o_full);
                    ++ga;
                }
            };
            TileCursor cg(p.sc), co(p.sc);
            Tile Tg, To;
            bool hg = cg.next(p.sc, Tg);
            int jg = 0, jo = 0;
            if (MODE == FWD && hg) {   // G(0)
                for (int s = 0; s < nsl; ++s) g_slice(jg, s);
                ++jg;
                hg = cg.next(p.sc, Tg);
            }
            while (co.next(p.sc, To)) {
                jo_cur = jo;
                if (xt) {   // tape slots: wait (phase order), the softmax warps release them
                    for (int b = 0; b < ntape; ++b) {
                        mbar_wait(&full[st], ph);
                        if (b == 0 && h == 0) trace_ev(p, jo, 2);
                        if (++st == NST) { st = 0; ph ^= 1u; }
                    }
                    if (h == 0) trace_ev(p, jo, 3);
                } else if (MODE != FWD) {
                    // the score GEMMs write dP into the accumulator columns (unless early):
                    // the epilogue must have drained the previous tile's last accumulation
                    if (!early && ga > 0) {
                        mbar_wait(o_empty, (ga - 1) & 1);
                        tc_fence_after();
                    }
                    if (xt3 && ownS && jo > 0) {   // pass 3 of the previous tile read its dS
                        mbar_wait(tape_done, (jo - 1) & 1);
                        tc_fence_after();
                    }
                    for (int s = 0; s < nsl; ++s) g_slice(jo, s);
                }
                // FWD: S(j) consumed (G(j+1) may overwrite it) and P(j) in smem.  BWD: dS
                // written; early BWDQ hands dS to issuer 0 per key block instead, and issuer
                // 1 waits here so that dP(j+1) does not overwrite dP(j) under the softmax.
                if (!(early && h == 0)) {
                    mbar_wait(p_full, jo & 1);
                    tc_fence_after();
                }
                if (h == otr) trace_ev(p, jo, 4);
                if (MODE == FWD) {
                    const int nG = hg ? nsl : 0, nO = nacc * nkb;
                    for (int gi = 0, oi = 0; gi < nG || oi < nO;) {
                        if (gi < nG) g_slice(jg, gi++);
                        if (oi < nO && (p.two || gi == nG)) { o_block(oi / nkb, oi % nkb); ++oi; }
                    }
                    if (hg) { ++jg; hg = cg.next(p.sc, Tg); }
                } else {
                    for (int a = 0; a < nacc; ++a)
                        for (int kb = 0; kb < nkb; ++kb) o_block(a, kb);
                }
                if (C::PSMEM && ownSmemA) mma_commit(p_free);
                if (xt && ownTmemA) mma_commit(a_free);
                if (h == otr) trace_ev(p, jo, 5);
                ++jo;
            }
        }
    } else if (warp < 4) {   // ------------------------------------------- softmax warps
        const int t = warp * 32 + lane;
        const uint32_t trow = tbase + ((uint32_t)(warp * 32) << 16);
        const int nch = NK / 32;
        // chunks holding any band column of this warp's rows (warp-uniform):
        // rows 32*warp .. 32*warp+31 need columns [32*warp, 32*warp + 31 + 2w]
        const int c_lo = warp, c_hi = min(nch - 1, (32 * warp + 31 + 2 * w) / 32);
        TileCursor cur(p.sc);
        Tile T;
        int j = 0;
        uint32_t zero16[16];
#pragma unroll
        for (int e = 0; e < 16; ++e) zero16[e] = 0u;
        // D of BWDQ: either wait for the whole BWDQ grid, or (dpoll) read each D row as soon
        // as its BWDQ tile has stored it, so BWDKV's first tiles overlap BWDQ's last ones
        if (MODE == BWDKV && !p.dpoll) asm volatile("griddepcontrol.wait;" ::: "memory");
        bool lse_settled = false;   // ld_lse_ready fell back to griddepcontrol.wait
        while (cur.next(p.sc, T)) {
            const int Lr = T.Lr, m0 = T.m0;
            const int mrow = m0 + t;
            const int kb = m0 - w;   // residue index of halo column 0
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;

            if (MODE == BWDKV && !xt) {
                named_bar_sync(1, 128);   // everyone is done with the previous tile's columns
                for (int n = t; n < NK; n += 128) {
                    const int mc = kb + n;
                    const bool ok = mc >= 0 && mc < Lr;
                    colLse[n] = !ok ? 0.f
                                : p.lsepoll ? ld_D_first(p.lse + rowbase + (int64_t)mc * p.dil)
                                            : p.lse[rowbase + (int64_t)mc * p.dil];
                    colD[n] = !ok ? 0.f
                              : p.dpoll ? ld_D_first(p.D + rowbase + (int64_t)mc * p.dil)
                                        : p.D[rowbase + (int64_t)mc * p.dil];
                }
                if (p.dpoll)   // rows whose BWDQ tile had not stored D yet
                    for (int n = t; n < NK; n += 128)
                        if (__float_as_uint(colD[n]) == D_UNSET)
                            colD[n] = ld_D_ready(p.D + rowbase + (int64_t)(kb + n) * p.dil);
                for (int n = t; n < NK; n += 128) {   // lse rows FWD had not stored yet
                    if (p.lsepoll && __float_as_uint(colLse[n]) == D_UNSET)
                        colLse[n] = ld_lse_ready(p.lse + rowbase + (int64_t)(kb + n) * p.dil, lse_settled);
                    colLse[n] *= LOG2E;
                }
                named_bar_sync(1, 128);
            }
            if (!xt) {
                mbar_wait(s_full, j & 1);
                tc_fence_after();
            }
            if (t == 0) trace_ev(p, j, 6);

            if (MODE == FWD) {
                // Band-empty chunks of P never change: zero them once per CTA.
                if (j == 0)
                    for (int c = 0; c < nch; ++c)
                        if (c < c_lo || c > c_hi) st_p_chunk(sP, t, c, zero16);
                float mx = -INFINITY;
                // score tape: this row's band scores, entry n - t = k + w
                float* ts = TAPE && mrow < Lr ? p.tape + (rowbase + (int64_t)mrow * p.dil) * p.tstride : nullptr;
                for (int c = c_lo; c <= c_hi; ++c) {
                    uint32_t rr[32];
                    tmem_ld32(trow + c * 32, rr);
                    tmem_wait_ld();
                    mx = chunk_max(rr, c * 32, t, w, kb, Lr, mx);
                    if (ts) {
#pragma unroll
                        for (int e = 0; e < 32; ++e)
                            if (band_ok(c * 32 + e, t, w, kb + c * 32 + e, Lr)) ts[c * 32 + e - t] = __uint_as_float(rr[e]);
                    }
                }
                if (mx == -INFINITY) mx = 0.f;   // only rows beyond the sequence (never stored)
                const float mxs = mx * LOG2E;
                if (t == 0) trace_ev(p, j, 10);
                if (j > 0) mbar_wait(p_free, (j - 1) & 1);   // P smem of the previous tile consumed
                if (t == 0) trace_ev(p, j, 11);
                float sum = 0.f;
                for (int c = c_lo; c <= c_hi; ++c) {
                    uint32_t rr[32];
                    tmem_ld32(trow + c * 32, rr);
                    tmem_wait_ld();
                    sum += chunk_exp_store(sP, rr, c, t, w, kb, Lr, mxs);
                }
                rowScale[(j % 3) * 128 + t] = 1.f / sum;
                fence_proxy_async_smem();   // P (generic-proxy stores) -> tensor core (async proxy)
                tc_fence_before();
                mbar_arrive(p_full);
                if (mrow < Lr) p.lse[rowbase + (int64_t)mrow * p.dil] = (mxs + log2f(sum)) * LN2;
            } else if (MODE == BWDQ) {
                const float lse2 = mrow >= Lr ? 0.f
                                   : (p.lsepoll ? ld_lse_ready(p.lse + rowbase + (int64_t)mrow * p.dil, lse_settled)
                                                : p.lse[rowbase + (int64_t)mrow * p.dil]) * LOG2E;
                float D = 0.f;
                // tape: this row's band scores read back (entry n - t); rows beyond the sequence get P = 0
                const float* tq = tp && mrow < Lr ? p.tape + (rowbase + (int64_t)mrow * p.dil) * p.tstride : nullptr;
                auto tape_p = [&](int n) -> float { return fast_exp2(fmaf(__ldg(tq + (n - t)), LOG2E, -lse2)); };
                for (int c = c_lo; c <= c_hi; ++c) {   // pass 1: D = sum_j P_ij dP_ij
                    uint32_t rs[32], rd[32];
                    if (!tp) tmem_ld32(trow + c * 32, rs);
                    tmem_ld32(trow + 256 + c * 32, rd);
                    tmem_wait_ld();
                    if constexpr (tp) {
#pragma unroll
                        for (int e = 0; e < 32; ++e) {
                            const int n = c * 32 + e;
                            const bool ok = band_ok(n, t, w, kb + n, Lr);
                            const float pv = ok && tq ? tape_p(n) : 0.f;
                            D = fmaf(pv, __uint_as_float(rd[e]), D);
                        }
                    } else {   // packed f32x2 pairs, four partial sums
                        float Dp[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                        for (int e = 0; e < 32; e += 2) {
                            const int n = c * 32 + e, q = e & 2;
                            float a0, a1;
                            ffma2_bc(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, -lse2, a0, a1);
                            const float p0 = band_ok(n, t, w, kb + n, Lr) ? fast_exp2(a0) : 0.f;
                            const float p1 = band_ok(n + 1, t, w, kb + n + 1, Lr) ? fast_exp2(a1) : 0.f;
                            ffma2(p0, p1, __uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), Dp[q], Dp[q + 1], Dp[q], Dp[q + 1]);
                        }
                        D += (Dp[0] + Dp[1]) + (Dp[2] + Dp[3]);
                    }
                }
                auto block_done = [&](int c) {   // early: hand block c/2 to the MMA
                    if (early && (c & 1)) {
                        tmem_wait_st();
                        tc_fence_before();
                        mbar_arrive(&p_blk[c >> 1]);
                    }
                };
                for (int c = 0; c < nch; ++c) {   // pass 2: dS = P (dP - D) -> TMEM (bf16 hi/lo)
                    if (c < c_lo || c > c_hi) {
                        tmem_st16(trow + c * 32, zero16);
                        tmem_st16(trow + c * 32 + 16, zero16);
                        block_done(c);
                        continue;
                    }
                    uint32_t rs[32], rd[32], pk[16], pl[16], pp[16];
                    if (!tp) tmem_ld32(trow + c * 32, rs);
                    tmem_ld32(trow + 256 + c * 32, rd);
                    tmem_wait_ld();
                    // dS tape (xt): entry e = n - t of row mrow at float (mrow & 3) + e = ob + (n - 32 c),
                    // four entries per 16-byte store ((mrow & 3) == (t & 3), m0 % 128 == 0).  With
                    // free TMEM columns (xt3) P goes there as bf16 and pass 3 stores the tape after
                    // p_full, off the MMAs' critical path; else the stores are issued here.
                    const int ob = (t & 3) + c * 32 - t;
#pragma unroll
                    for (int g4 = 0; g4 < 8; ++g4) {
                        float pv[4], dv[4];
                        if constexpr (tp) {
#pragma unroll
                            for (int x = 0; x < 4; ++x) {
                                const int n = c * 32 + 4 * g4 + x;
                                const bool ok = band_ok(n, t, w, kb + n, Lr);
                                pv[x] = ok && tq ? tape_p(n) : 0.f;
                                dv[x] = pv[x] * (__uint_as_float(rd[4 * g4 + x]) - D);
                            }
                        } else {   // packed f32x2 pairs
#pragma unroll
                            for (int x = 0; x < 4; x += 2) {
                                const int n = c * 32 + 4 * g4 + x, i = 4 * g4 + x;
                                float a0, a1, q0, q1;
                                ffma2_bc(__uint_as_float(rs[i]), __uint_as_float(rs[i + 1]), LOG2E, -lse2, a0, a1);
                                pv[x] = band_ok(n, t, w, kb + n, Lr) ? fast_exp2(a0) : 0.f;
                                pv[x + 1] = band_ok(n + 1, t, w, kb + n + 1, Lr) ? fast_exp2(a1) : 0.f;
                                ffma2_bc(__uint_as_float(rd[i]), __uint_as_float(rd[i + 1]), 1.f, -D, q0, q1);
                                fmul2(pv[x], pv[x + 1], q0, q1, dv[x], dv[x + 1]);
                            }
                        }
                        split_bf16x2(dv[0], dv[1], pk[2 * g4], pl[2 * g4]);
                        split_bf16x2(dv[2], dv[3], pk[2 * g4 + 1], pl[2 * g4 + 1]);
                        pp[2 * g4] = pack_bf16x2(pv[0], pv[1]);
                        pp[2 * g4 + 1] = pack_bf16x2(pv[2], pv[3]);
                        const int o = ob + 4 * g4;
                        if (!TAPE && p.xt && !xt3 && mrow < Lr && o >= 0 && o < p.tsw) {
                            const size_t ro = ((size_t)(o >> 2) * p.grows + rowbase + (int64_t)mrow * p.dil) * 4;
                            *reinterpret_cast<float4*>(p.tP + ro) = make_float4(pv[0], pv[1], pv[2], pv[3]);
                            *reinterpret_cast<float4*>(p.tS + ro) = make_float4(dv[0], dv[1], dv[2], dv[3]);
                        }
                    }
                    tmem_st16(trow + c * 32, pk);
                    tmem_st16(trow + c * 32 + 16, pl);
                    if (xt3) tmem_st16(trow + XT3_COL + 16 * (c - c_lo), pp);
                    block_done(c);
                }
                tmem_wait_st();
                tc_fence_before();
                mbar_arrive(p_full);
                if (mrow < Lr) p.D[rowbase + (int64_t)mrow * p.dil] = D;
                if (xt3) {   // pass 3: the tape from dS hi / lo and P (bf16) in TMEM
                    for (int c = c_lo; c <= c_hi; ++c) {
                        uint32_t hi[16], lo[16], pb[16];
                        tmem_ld16(trow + c * 32, hi);
                        tmem_ld16(trow + c * 32 + 16, lo);
                        tmem_ld16(trow + XT3_COL + 16 * (c - c_lo), pb);
                        tmem_wait_ld();
                        if (c == c_hi) {   // the S columns may take the next tile's scores
                            tc_fence_before();
                            mbar_arrive(tape_done);
                        }
                        const int ob = (t & 3) + c * 32 - t;
#pragma unroll
                        for (int g4 = 0; g4 < 8; ++g4) {
                            const int o = ob + 4 * g4;
                            if (mrow < Lr && o >= 0 && o < p.tsw) {
                                auto f0 = [](uint32_t x) { return __uint_as_float(x << 16); };
                                auto f1 = [](uint32_t x) { return __uint_as_float(x & 0xFFFF0000u); };
                                const uint32_t h0 = hi[2 * g4], h1 = hi[2 * g4 + 1];
                                const uint32_t l0 = lo[2 * g4], l1 = lo[2 * g4 + 1];
                                const uint32_t b0 = pb[2 * g4], b1 = pb[2 * g4 + 1];
                                const size_t ro = ((size_t)(o >> 2) * p.grows + rowbase + (int64_t)mrow * p.dil) * 4;
                                *reinterpret_cast<float4*>(p.tP + ro) = make_float4(f0(b0), f1(b0), f0(b1), f1(b1));
                                *reinterpret_cast<float4*>(p.tS + ro) =
                                    make_float4(f0(h0) + f0(l0), f1(h0) + f1(l0), f0(h1) + f0(l1), f1(h1) + f1(l1));
                            }
                        }
                    }
                }
                if (!TAPE && p.xt) {   // publish the tile's tape rows to BWDKV
                    __threadfence();
                    named_bar_sync(2, 128);
                    if (t == 0) st_release_gpu(p.flags + rowbase + (int64_t)m0 * p.dil, 1u);
                }
            } else if (xt) {   // BWDKV from the dS tape: P^T -> smem (bf16), dS^T -> TMEM (hi / lo)
                if (j > 0) {   // the previous tile's dV / dK MMAs are done with P^T / dS^T
                    mbar_wait(p_free, (j - 1) & 1);
                    mbar_wait(a_free, (j - 1) & 1);
                    tc_fence_after();
                }
                if (t == 0) trace_ev(p, j, 10);
                const int per = ntape + nacc * nkb, cps = p.trows / 32;
                for (int b = 0; b < ntape; ++b) {
                    const int k = j * per + b, st = k % NST;
                    mbar_wait(&full[st], (uint32_t)(k / NST) & 1u);
                    if (t == 0) trace_ev(p, j, b == 0 ? 11 : 15);
                    const float* sv = reinterpret_cast<const float*>(sslots + (size_t)st * SLOT);
                    const float* sS = sv + tape_plane_bytes(p.trows, p.tsw) / 4;
                    const int gstr = 4 * (p.trows + 1);   // floats between granule rows of a plane
                    for (int c = b * cps; c < (b + 1) * cps; ++c) {
                        if (c < c_lo || c > c_hi) {
                            if (j == 0) st_p_chunk(sP, t, c, zero16);   // P^T zeros persist
                            tmem_st16(trow + c * 32, zero16);
                            tmem_st16(trow + c * 32 + 16, zero16);
                            continue;
                        }
                        uint32_t pk[16], dk[16], dl[16];
#pragma unroll
                        for (int e = 0; e < 32; e += 2) {
                            float pv[2], dv[2];
#pragma unroll
                            for (int h = 0; h < 2; ++h) {
                                // query column n (tape row kb + n), key t: entry t - n + 2w
                                const int n = c * 32 + e + h, mq = kb + n;
                                // branch-free (all loads of a chunk issue back to back): an entry
                                // outside the band reads offset 0 of the slot and is zeroed
                                const bool ok = band_ok(n, t, w, mq, Lr);
                                const int oo = (mq & 3) + t - n + 2 * w;
                                const int o = ok ? (oo >> 2) * gstr + (n - b * p.trows) * 4 + (oo & 3) : 0;
                                const float xp = sv[o], xs = sS[o];
                                pv[h] = ok ? xp : 0.f;
                                dv[h] = ok ? xs : 0.f;
                            }
                            pk[e / 2] = pack_bf16x2(pv[0], pv[1]);
                            split_bf16x2(dv[0], dv[1], dk[e / 2], dl[e / 2]);
                        }
                        st_p_chunk(sP, t, c, pk);
                        tmem_st16(trow + c * 32, dk);
                        tmem_st16(trow + c * 32 + 16, dl);
                    }
                    named_bar_sync(1, 128);   // all four warps are done with this slot
                    if (t == 0) {
                        mbar_arrive(&empty[st]);
                        if (p.two) mbar_arrive(&empty[st]);
                    }
                }
                fence_proxy_async_smem();
                tmem_wait_st();
                tc_fence_before();
                mbar_arrive(p_full);
            } else {   // BWDKV: rows are keys, columns are halo queries
                if (j > 0) mbar_wait(p_free, (j - 1) & 1);
                for (int c = 0; c < nch; ++c) {
                    if (c < c_lo || c > c_hi) {
                        if (j == 0) st_p_chunk(sP, t, c, zero16);   // P^T zeros persist
                        tmem_st16(trow + c * 32, zero16);
                        tmem_st16(trow + c * 32 + 16, zero16);
                        continue;
                    }
                    uint32_t rs[32], rd[32], pk[16], dk[16], dl[16];
                    if (!tp) tmem_ld32(trow + c * 32, rs);
                    tmem_ld32(trow + 256 + c * 32, rd);
                    tmem_wait_ld();
#pragma unroll
                    for (int e = 0; e < 32; e += 2) {
                        float pv[2], dv[2];
                        if constexpr (tp) {
#pragma unroll
                            for (int h = 0; h < 2; ++h) {
                                const int n = c * 32 + e + h;
                                // tape: S^T[key t][query n] = tape[query kb + n][t - n + 2w] (offset of
                                // key m0 + t from query kb + n is t - n + w); one 128-byte line per warp
                                const bool ok = band_ok(n, t, w, kb + n, Lr) && mrow < Lr;
                                pv[h] = !ok ? 0.f
                                        : fast_exp2(fmaf(__ldg(p.tape + (rowbase + (int64_t)(kb + n) * p.dil) * p.tstride + (t - n + 2 * w)),
                                                         LOG2E, -colLse[n]));
                                dv[h] = pv[h] * (__uint_as_float(rd[e + h]) - colD[n]);
                            }
                        } else {   // packed f32x2 pairs
                            const int n = c * 32 + e;
                            float a0, a1, q0, q1;
                            ffma2(__uint_as_float(rs[e]), __uint_as_float(rs[e + 1]), LOG2E, LOG2E, -colLse[n], -colLse[n + 1], a0, a1);
                            pv[0] = band_ok(n, t, w, kb + n, Lr) ? fast_exp2(a0) : 0.f;
                            pv[1] = band_ok(n + 1, t, w, kb + n + 1, Lr) ? fast_exp2(a1) : 0.f;
                            ffma2(__uint_as_float(rd[e]), __uint_as_float(rd[e + 1]), 1.f, 1.f, -colD[n], -colD[n + 1], q0, q1);
                            fmul2(pv[0], pv[1], q0, q1, dv[0], dv[1]);
                        }
                        pk[e / 2] = pack_bf16x2(pv[0], pv[1]);
                        split_bf16x2(dv[0], dv[1], dk[e / 2], dl[e / 2]);
                    }
                    st_p_chunk(sP, t, c, pk);
                    tmem_st16(trow + c * 32, dk);
                    tmem_st16(trow + c * 32 + 16, dl);
                }
                fence_proxy_async_smem();
                tmem_wait_st();
                tc_fence_before();
                mbar_arrive(p_full);
            }
            if (t == 0) trace_ev(p, j, 7);
            ++j;
        }
    } else if (warp < 8) {   // ------------------------------------------ epilogue warps
        const int ew = warp - 4;   // TMEM lanes 32*ew .. 32*ew+31  (warp % 4 == ew)
        const uint32_t trow = tbase + ((uint32_t)(ew * 32) << 16);
        uint8_t* mystg = ostg + ew * NSTG * STG;
        TileCursor cur(p.sc);
        Tile T;
        int j = 0, ga = 0, sidx = 0;
        while (cur.next(p.sc, T)) {
            const Maps& mp = p.maps[T.rl];
            float scale = 1.f;
            if (MODE == FWD) {   // 1/l of this row, published before p_full
                mbar_wait(p_full, j & 1);
                scale = rowScale[(j % 3) * 128 + ew * 32 + lane];
            }
            for (int a = 0; a < nacc; ++a, ++ga) {
                const int c = dual ? a : a / C::NOUT;
                const int cw = chunk_w(d, c);
                // dual: slices 0..cw/64-1 are dV (o1), the next cw/64 are dK (o2)
                const int nsl_c = (dual ? 2 : 1) * cw / 64;
                mbar_wait(o_full, ga & 1);
                tc_fence_after();
                // BWDQ launched early (lse hand-off): its first global store waits for the
                // preceding grid, so stream order holds for every buffer it writes
                if (MODE == BWDQ && p.lsepoll && ga == 0) asm volatile("griddepcontrol.wait;" ::: "memory");
                if (lane == 0 && ew == 0 && a == 0) trace_ev(p, j, 8);
                // Drain the accumulator 128 columns at a time: both 64-column halves are
                // loaded before the wait, and o_empty is released as soon as every column is
                // in registers, so the next accumulation's MMAs start before the stores.
                for (int s0 = 0; s0 < nsl_c; s0 += 2) {
                    const int ns = min(2, nsl_c - s0);
                    uint32_t ov[2][64];
#pragma unroll
                    for (int h = 0; h < 2; ++h) {
                        if (h < ns) {
                            const uint32_t tcol = acc0 + 64u * (s0 + h);
                            tmem_ld32(trow + tcol, *reinterpret_cast<uint32_t(*)[32]>(&ov[h][0]));
                            tmem_ld32(trow + tcol + 32, *reinterpret_cast<uint32_t(*)[32]>(&ov[h][32]));
                        }
                    }
                    tmem_wait_ld();
                    if (s0 + ns == nsl_c) {
                        tc_fence_before();
                        mbar_arrive(o_empty);
                    }
#pragma unroll
                    for (int h = 0; h < 2; ++h) {
                        if (h >= ns) break;
                        const int s = s0 + h;
                        uint8_t* stg = mystg + (sidx % NSTG) * STG;
                        if (lane == 0 && sidx >= NSTG) tma_store_wait_read<NSTG - 1>();
                        __syncwarp();
#pragma unroll
                        for (int q = 0; q < 8; ++q) {
                            uint4 val;
                            val.x = pack_bf16x2(__uint_as_float(ov[h][8 * q + 0]) * scale, __uint_as_float(ov[h][8 * q + 1]) * scale);
                            val.y = pack_bf16x2(__uint_as_float(ov[h][8 * q + 2]) * scale, __uint_as_float(ov[h][8 * q + 3]) * scale);
                            val.z = pack_bf16x2(__uint_as_float(ov[h][8 * q + 4]) * scale, __uint_as_float(ov[h][8 * q + 5]) * scale);
                            val.w = pack_bf16x2(__uint_as_float(ov[h][8 * q + 6]) * scale, __uint_as_float(ov[h][8 * q + 7]) * scale);
                            *reinterpret_cast<uint4*>(stg + lane * 128 + ((q ^ (lane & 7)) * 16)) = val;
                        }
                        fence_proxy_async_smem();
                        __syncwarp();
                        const bool second = dual ? (64 * s >= cw) : (C::NOUT == 2 && (a & 1));
                        const CUtensorMap* om = second ? &mp.o2 : &mp.o1;
                        const int col = 256 * c + (dual && second ? 64 * s - cw : 64 * s);
                        if (lane == 0) {
                            tma_store_3d(om, stg, col, T.m0 + 32 * ew, T.u);
                            tma_store_commit();
                        }
                        ++sidx;
                    }
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
        tmem_dealloc(tbase, 512);
    }
}

int tape_stride(int64_t wc);

template <int MODE, bool TAPE>
void set_attr_once() {
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_band_kernel<MODE, TAPE>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             227 * 1024);
    });
}

bool pdl_enabled() { return knob(K_PDL) != 0; }

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
    return (int)(((BM + 2 * wc) + 63) / 64 * 64);
}

// Tensors per mode: a1, b1 (score GEMM 1), a2, b2 (score GEMM 2), ob1, ob2 (output-GEMM
// B operands), o1, o2 (outputs).
template <int MODE>
cudaError_t launch(const void* a1, const void* b1, const void* a2, const void* b2, const void* ob1,
                   const void* ob2, void* o1, void* o2, float* lse, float* D, int64_t B, int64_t H,
                   int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st, int* launches,
                   float* tape = nullptr, const DsTape* ds = nullptr) {
    const int64_t wc = w < L ? w : L;
    const int NK = halo_rows(L, w);
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    const int nst = pick_nst<MODE>(NK);
    if (nst < 2) return cudaErrorInvalidConfiguration;
    set_attr_once<MODE, false>();
    set_attr_once<MODE, true>();
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
                      make_residue_map(&m.ob1, ob1, L, d, units, dil, r, KB) &&
                      make_residue_map(&m.o1, o1, L, d, units, dil, r, 32);
            if (ok && a2) ok = make_residue_map(&m.a2, a2, L, d, units, dil, r, BM);
            if (ok && b2) ok = make_residue_map(&m.b2, b2, L, d, units, dil, r, NK);
            if (ok && ob2) ok = make_residue_map(&m.ob2, ob2, L, d, units, dil, r, KB);
            if (ok && o2) ok = make_residue_map(&m.o2, o2, L, d, units, dil, r, 32);
            if (ok && ds && !tape && MODE == BWDKV) {
                const int trows = 2 * tape_plane_bytes(64, ds->tsw) <= slot_bytes(NK) ? 64 : 32;
                ok = make_residue_map_tape(&m.tp, ds->P, L, ds->tsw, units, dil, r, trows + 1, ds->grows) &&
                     make_residue_map_tape(&m.ts, ds->S, L, ds->tsw, units, dil, r, trows + 1, ds->grows);
            }
            if (!ok) return cudaErrorInvalidValue;
        }
        p.lse = lse;
        p.D = D;
        p.L = L;
        p.d = (int)d;
        p.w = (int)wc;
        p.dil = (int)dil;
        p.NK = NK;
        p.nsl = (int)(d / 64);
        p.nst = nst;
        const int64_t Lr0 = ceil_div(L - r0, dil);   // longest residue of this group
        p.trace = (unsigned long long*)trace_buffer(MODE);
        p.two = 1;   // two MMA issuers (measured faster for every mode and d, profiles/README.md)
        p.dpoll = MODE != FWD && dpoll_enabled();
        const int tiles = (int)ceil_div(Lr0, BM);
        const int64_t total = units * nr * tiles;
        p.lsepoll = lsepoll_enabled() && r0 == 0 && lsepoll_worth(total, num_sms()) && tape == nullptr;
        p.tape = tape;
        p.tstride = tape_stride(wc);
        if (ds && !tape && MODE != FWD) {
            p.xt = 1;
            p.tsw = ds->tsw;
            p.trows = 2 * tape_plane_bytes(64, ds->tsw) <= slot_bytes(NK) ? 64 : 32;
            p.grows = ds->grows;
            p.flags = ds->flags;
            p.tP = ds->P;
            p.tS = ds->S;
        }
        dim3 grid((unsigned)(total < num_sms() ? total : num_sms()));
        sched_init(p.sc, L, dil, r0, nr, units, tiles, (int)grid.x);
        const size_t smem = fixed_smem_bytes<MODE>(NK) + (size_t)nst * slot_bytes(NK);
        if (MODE != FWD && r0 == 0 && pdl_enabled() && (MODE == BWDKV || p.lsepoll)) {
            // BWDKV directly follows this call's last BWDQ launch on the stream; BWDQ
            // (lse hand-off) typically follows the forward's band launch
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
            cudaLaunchKernelEx(&cfg, tape ? tc_band_kernel<MODE, true> : tc_band_kernel<MODE, false>, p);
        } else {
            if (tape) tc_band_kernel<MODE, true><<<grid, NTHREADS, smem, st>>>(p);
            else tc_band_kernel<MODE, false><<<grid, NTHREADS, smem, st>>>(p);
        }
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
    const int NK = halo_rows(L, w);
    return d % 64 == 0 && d <= 512 && wc <= 64 && dil <= 256 &&
           units * ((L + 127) / 128) < (1 << 30) && pick_nst<BWDKV>(NK) >= 2 &&
           pick_nst<FWD>(NK) >= 2 && pick_nst<BWDQ>(NK) >= 2;
}

int tape_stride(int64_t wc) { return (int)(2 * wc + 1); }

int band_launches(int64_t L, int64_t dil) {
    const int64_t nres = dil < L ? dil : L;
    return (int)ceil_div(nres, RES_PER_LAUNCH);
}

}  // namespace

// Wide windows (halo > 256 rows): the one-pass wide kernels (d in {64, 128}), else the chunked
// fallback kernels where their shared-memory plan fits.
static bool wide_fwd_ok(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    return knob(K_WIDE) && tc_wide_supported(units, L, d, w, dil);
}
static bool wide_bwd_ok(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    return knob(K_WIDE) && tc_wide_bwd_supported(units, L, d, w, dil);
}
bool tc_fwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    return halo_rows(L, w) <= 256 ? band_supported(units, L, d, w, dil)
                                  : (wide_fwd_ok(units, L, d, w, dil) || tc_chunk_supported(units, L, d, w, dil));
}
bool tc_bwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    return halo_rows(L, w) <= 256 ? band_supported(units, L, d, w, dil)
                                  : (wide_bwd_ok(units, L, d, w, dil) || tc_chunk_supported(units, L, d, w, dil));
}
int tc_fwd_launches(int64_t L, int64_t d, int64_t w, int64_t dil) {
    if (tc_narrow_supported(1, L, d, w, dil)) return tc_narrow_launches(L, dil);
    return halo_rows(L, w) <= 256 ? band_launches(L, dil) : tc_chunk_launches(L, dil);
}
int tc_bwd_launches(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    if (tc_narrow_bwd_supported(1, L, d, w, dil)) return 2 * tc_narrow_launches(L, dil);
    if (halo_rows(L, w) <= 256) return 2 * band_launches(L, dil);
    return 2 * tc_chunk_launches(L, dil);
}

cudaError_t tc_fwd(const void* q, const void* k, const void* v, void* out, float* lse, int64_t B,
                   int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st,
                   int* launches) {
    if (launches) *launches = 0;
    if (halo_rows(L, w) > 256) {
        if (!wide_fwd_ok(B * H, L, d, w, dil))
            return tc_chunk_fwd(q, k, v, out, lse, B, H, L, d, w, dil, st, launches);
        return tc_wide_fwd(q, k, v, out, lse, B, H, L, d, w, dil, st, launches);
    }
    if (tc_narrow_supported(B * H, L, d, w, dil))
        return tc_narrow_fwd(q, k, v, out, lse, B, H, L, d, w, dil, st, launches);
    return launch<FWD>(q, k, nullptr, nullptr, v, nullptr, out, nullptr, lse, nullptr, B, H, L,
                       d, w, dil, st, launches);
}

bool tc_band_dstape_ok(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    return halo_rows(L, w) <= 256 && !tc_narrow_bwd_supported(units, L, d, w, dil) &&
           band_supported(units, L, d, w, dil);
}

cudaError_t tc_bwd(const void* q, const void* k, const void* v, const void* out,
                   const float* lse, const void* dout, void* dq, void* dk, void* dv, float* Dws,
                   int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                   cudaStream_t st, int* launches, const DsTape* ds) {
    // band kernels: D_i is recomputed exactly as sum_j P_ij dP_ij by BWDQ (reading R1); the
    // wide kernels also compute it exactly, and read out only for the first-guess D~
    if (launches) *launches = 0;
    if (halo_rows(L, w) > 256) {
        if (!wide_bwd_ok(B * H, L, d, w, dil))
            return tc_chunk_bwd(q, k, v, lse, dout, dq, dk, dv, Dws, B, H, L, d, w, dil, st, launches);
        return tc_wide_bwd(q, k, v, out, lse, dout, dq, dk, dv, Dws, B, H, L, d, w, dil, st, launches);
    }
    if (tc_narrow_bwd_supported(B * H, L, d, w, dil))
        return tc_narrow_bwd(q, k, v, lse, dout, dq, dk, dv, Dws, B, H, L, d, w, dil, st, launches);
    cudaError_t e = launch<BWDQ>(q, k, dout, v, k, nullptr, dq, nullptr, const_cast<float*>(lse),
                                 Dws, B, H, L, d, w, dil, st, launches, nullptr, ds);
    if (e != cudaSuccess) return e;
    // BWDKV accumulation order per chunk: dV (P^T dO, ob1 = dout) then dK (dS^T Q, ob2 = q)
    return launch<BWDKV>(k, q, v, dout, dout, q, dv, dk, const_cast<float*>(lse), Dws, B, H, L,
                         d, w, dil, st, launches, nullptr, ds);
}

bool tc_tape_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    return halo_rows(L, w) <= 256 && band_supported(units, L, d, w, dil);
}

cudaError_t tc_tape_fwd(const void* q, const void* k, const void* v, void* out, float* lse, void* tape,
                        int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st,
                        int* launches) {
    if (launches) *launches = 0;
    return launch<FWD>(q, k, nullptr, nullptr, v, nullptr, out, nullptr, lse, nullptr, B, H, L, d, w, dil, st,
                       launches, static_cast<float*>(tape));
}

cudaError_t tc_tape_bwd(const void* q, const void* k, const void* v, const float* lse, const void* tape,
                        const void* dout, void* dq, void* dk, void* dv, float* Dws, int64_t B, int64_t H,
                        int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st, int* launches) {
    if (launches) *launches = 0;
    float* t = const_cast<float*>(static_cast<const float*>(tape));
    cudaError_t e = launch<BWDQ>(q, k, dout, v, k, nullptr, dq, nullptr, const_cast<float*>(lse), Dws, B, H, L, d,
                                 w, dil, st, launches, t);
    if (e != cudaSuccess) return e;
    return launch<BWDKV>(k, q, v, dout, dout, q, dv, dk, const_cast<float*>(lse), Dws, B, H, L, d, w, dil, st,
                         launches, t);
}

}  // namespace ftw
