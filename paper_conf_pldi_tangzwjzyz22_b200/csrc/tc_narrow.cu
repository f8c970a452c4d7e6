// tc_narrow.cu -- forward of banded window attention for head dim d = 64 and w <= 32 on
// sm_100a: the HBM-bound shape of the C5 sweep (w = 32 rows).
//
// At d = 64 one 128-row tile moves only 64 KB (q, k, v in; o out), ~1.5 us of the SM's
// share of HBM bandwidth, while its row softmax (96 band columns per row, PAPER.md
// Fig. 8/10, lines 215-231 and 306-321) takes longer than that on one warpgroup.  So two
// softmax warpgroups work on alternate tiles (ping-pong): everything a tile owns in TMEM is
// double-buffered, and a 3-stage TMA ring keeps the next tiles' operands in flight.
//
//   S(j)  = Q_j K_h^T      tcgen05.mma SS, M=128, N=NK=192, K=64      -> TMEM S[j&1]
//   P(j)  = exp(S - max), row sums, lse -> HBM; P packed to bf16 over S[j&1] in place
//   O(j)  = P(j) V_h       tcgen05.mma TS (A = P from TMEM), N=64, K=192 -> TMEM O[j&1]
//   out   = O / l  -> bf16 -> smem -> TMA store (by the tile's softmax warpgroup)
//
// The K/V halo rows m0-w .. m0-w+191 of the tile's (unit, residue) problem are staged by TMA
// from the strided residue view (tmap.h), the cached window of PAPER.md Fig. 14 (lines
// 402-423); no padded or as_strided copy of K is made.
//
// Roles (320 threads): warps 0-3 softmax group 0 (even local tiles), warps 4-7 group 1 (odd
// tiles) -- warp w reads TMEM lanes 32*(w%4)..+31, thread <-> query row; warp 8 TMA producer
// and TMEM allocator; warp 9 MMA issuer.
// TMEM (512 columns): S[0] = [0,192), S[1] = [192,384), O[0] = [384,448), O[1] = [448,512).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>

#include "internal.h"
#ifndef FT_MBAR_SUSPEND_NS
#define FT_MBAR_SUSPEND_NS 0   // latency-critical handoffs: no suspend-time hint
#endif
#include "tc_common.cuh"
#include "tile_sched.cuh"
#include "tmap.h"

namespace ftw {
namespace {

using namespace tc;

constexpr int BM = 128;                      // query rows per tile
constexpr int D = 64;                        // head dim
constexpr int NK = 192;                      // halo rows (keys m0-w .. m0-w+191), w <= 32
constexpr int NSTAGE = 3;
constexpr int NTHREADS = 320;
constexpr int RES_PER_LAUNCH = 8;
static_assert(RES_PER_LAUNCH <= SCHED_MAX_RES, "residue table of the tile cursor");
constexpr uint32_t QBYTES = BM * D * 2;      // 16 KB
constexpr uint32_t HBYTES = NK * D * 2;      // 24 KB
constexpr uint32_t STAGE = QBYTES + 2 * HBYTES;
constexpr uint32_t STG = 32 * 128;           // one warp's 32-row output staging slice
constexpr size_t SMEM_BYTES = 1024 + (size_t)NSTAGE * STAGE + 8 * STG + 256;
constexpr float LOG2E = 1.4426950408889634f;
constexpr float LN2 = 0.6931471805599453f;
constexpr uint32_t TS0 = 0, TO0 = 384;       // TMEM column bases

struct NMaps {
    CUtensorMap q, k, v, o;
};
struct NParams {
    NMaps maps[RES_PER_LAUNCH];
    float* lse;
    int64_t L;
    int w, dil;
    SchedParams sc;
    int lsepoll;   // lse hand-off to the narrow dQ kernel (tc_common.cuh ld_lse_ready)
};

using Tile = SchedTile;
using TileCursor = SchedCursor<BM>;

__device__ __forceinline__ float fast_exp2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

__global__ void __launch_bounds__(NTHREADS, 1) tc_narrow_fwd_kernel(const __grid_constant__ NParams p) {
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);
    uint8_t* stages = smem;                                   // [NSTAGE] {Q, K_h, V_h}
    uint8_t* ostg = smem + (size_t)NSTAGE * STAGE;            // [8 warps] 4 KB
    uint64_t* bars = reinterpret_cast<uint64_t*>(ostg + 8 * STG);
    uint64_t* qk_full = bars;                 // [NSTAGE]
    uint64_t* v_full = bars + NSTAGE;         // [NSTAGE]
    uint64_t* empty = bars + 2 * NSTAGE;      // [NSTAGE]
    uint64_t* s_full = bars + 3 * NSTAGE;     // [2]
    uint64_t* p_full = s_full + 2;            // [2]
    uint64_t* o_full = s_full + 4;            // [2]
    uint64_t* o_free = s_full + 6;            // [2]
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(s_full + 8);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int w = p.w;

    if (p.lsepoll) {   // lse rows unset, then let the dQ kernel (PDL) launch
        TileCursor cr(p.sc);
        Tile T;
        while (cr.next(p.sc, T)) {
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;
            for (int i = threadIdx.x; i < BM && T.m0 + i < T.Lr; i += NTHREADS)
                reinterpret_cast<uint32_t*>(p.lse)[rowbase + (int64_t)(T.m0 + i) * p.dil] = D_UNSET;
        }
        __threadfence();
        __syncthreads();
        asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    }
    if (warp == 8) {
        if (lane == 0) {
            for (int i = 0; i < NSTAGE; ++i) {
                mbar_init(&qk_full[i], 1);
                mbar_init(&v_full[i], 1);
                mbar_init(&empty[i], 1);
            }
            for (int b = 0; b < 2; ++b) {
                mbar_init(&s_full[b], 1);
                mbar_init(&p_full[b], 4);
                mbar_init(&o_full[b], 1);
                mbar_init(&o_free[b], 4);
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

    if (warp == 8) {
        if (lane == 0) {   // ---------------------------------------------------- TMA producer
            TileCursor cur(p.sc);
            Tile T;
            for (int j = 0; cur.next(p.sc, T); ++j) {
                const int s = j % NSTAGE;
                if (j >= NSTAGE) mbar_wait(&empty[s], ((j / NSTAGE) - 1) & 1);
                uint8_t* st = stages + (size_t)s * STAGE;
                const NMaps& mp = p.maps[T.rl];
                mbar_arrive_expect_tx(&qk_full[s], QBYTES + HBYTES);
                tma_load_3d(st, &mp.q, &qk_full[s], 0, T.m0, T.u);
                tma_load_3d(st + QBYTES, &mp.k, &qk_full[s], 0, T.m0 - w, T.u);
                mbar_arrive_expect_tx(&v_full[s], HBYTES);
                tma_load_3d(st + QBYTES + HBYTES, &mp.v, &v_full[s], 0, T.m0 - w, T.u);
            }
        }
    } else if (warp == 9) {
        if (lane == 0) {   // ------------------------------------------------------ MMA issuer
            constexpr uint32_t idS = idesc_bf16(BM, NK, false, false);
            constexpr uint32_t idO = idesc_bf16(BM, D, false, true);
            // O(i) = P(i) V_h: 12 K-steps of 16 keys; A = packed P (8 TMEM columns per step),
            // B = V_h rows 16kk.. (MN-major SW128: 2048 B per step, LBO unused for N = 64)
            auto pv = [&](int i) {
                const int b = i & 1, s = i % NSTAGE;
                mbar_wait(&p_full[b], (i >> 1) & 1);
                if (i >= 2) mbar_wait(&o_free[b], ((i - 2) >> 1) & 1);
                mbar_wait(&v_full[s], (i / NSTAGE) & 1);
                tc_fence_after();
                const uint32_t sv = smem_u32(stages + (size_t)s * STAGE + QBYTES + HBYTES);
                const uint32_t tA = tbase + TS0 + 192u * b, tD = tbase + TO0 + 64u * b;
#pragma unroll
                for (int g = 0; g < 3; ++g)
                    mma_ts_x4<8, 128>(tD, tA + 32u * g, sdesc_sw128(sv + 8192u * g, 8192, 1024), idO, g);
                mma_commit(&o_full[b]);
                mma_commit(&empty[s]);
            };
            TileCursor cur(p.sc);
            Tile T;
            int j = 0;
            for (; cur.next(p.sc, T); ++j) {
                const int b = j & 1, s = j % NSTAGE;
                mbar_wait(&qk_full[s], (j / NSTAGE) & 1);
                // S[b] held P(j-2), read by O(j-2): wait for it to complete
                if (j >= 2) mbar_wait(&o_full[b], ((j - 2) >> 1) & 1);
                tc_fence_after();
                const uint32_t sq = smem_u32(stages + (size_t)s * STAGE);
                mma_ss_x4<2, 2>(tbase + TS0 + 192u * b, sdesc_sw128(sq, 16, 1024),
                                sdesc_sw128(sq + QBYTES, 16, 1024), idS, 0);
                mma_commit(&s_full[b]);
                if (j >= 1) pv(j - 1);
            }
            if (j >= 1) pv(j - 1);
        }
    } else {   // ---------------------------------------------------------- softmax groups
        const int g = warp >> 2, wq = warp & 3;
        const int t = wq * 32 + lane;
        const uint32_t lane_off = (uint32_t)(wq * 32) << 16;
        const uint32_t tS = tbase + lane_off + TS0 + 192u * g;
        const uint32_t tO = tbase + lane_off + TO0 + 64u * g;
        uint8_t* mystg = ostg + warp * STG;
        uint32_t zero16[16];
#pragma unroll
        for (int e = 0; e < 16; ++e) zero16[e] = 0u;
        TileCursor cur(p.sc);
        Tile T;
        int jl = 0;   // local tile index
        int k = 0;    // this group's tile count
        for (; cur.next(p.sc, T); ++jl) {
            if ((jl & 1) != g) continue;
            const int ph = k & 1;
            ++k;
            const int Lr = T.Lr, m0 = T.m0, kb = m0 - w;
            mbar_wait(&s_full[g], ph);
            tc_fence_after();
            // this row's band columns n in [t, t+2w] (and inside the sequence) lie in the
            // 32-column chunks wq, wq+1, wq+2
            uint32_t rr[3][32];
#pragma unroll
            for (int i = 0; i < 3; ++i) tmem_ld32(tS + 32u * (wq + i), rr[i]);
            tmem_wait_ld();
            const int lo = max(t, -kb) - 32 * wq, hi = min(t + 2 * w, Lr - 1 - kb) - 32 * wq;
            float m4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
            for (int i = 0; i < 3; ++i) {
                const int l0 = max(lo - 32 * i, 0), h0 = min(hi - 32 * i, 31);
                const uint32_t bits = h0 < l0 ? 0u : ((0xffffffffu >> (31 - h0)) & (0xffffffffu << l0));
#pragma unroll
                for (int e = 0; e < 32; ++e) {
                    if (!((bits >> e) & 1u)) rr[i][e] = 0xff800000u;   // -inf
                    m4[e & 3] = fmaxf(m4[e & 3], __uint_as_float(rr[i][e]));
                }
            }
            float mx = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3]));
            if (mx == -INFINITY) mx = 0.f;   // no key in range (rows beyond the sequence only)
            const float mxs = mx * LOG2E;
            float l4[4] = {0.f, 0.f, 0.f, 0.f};
            // P packed to bf16 over S in place: keys 2c, 2c+1 -> column c.  Chunks outside
            // this warp's band range are zero.
#pragma unroll
            for (int c = 0; c < NK / 32; ++c)
                if (c < wq || c > wq + 2) tmem_st16(tS + 16u * c, zero16);
#pragma unroll
            for (int i = 0; i < 3; ++i) {
                uint32_t pk[16];
#pragma unroll
                for (int e = 0; e < 32; e += 2) {
                    const float p0 = fast_exp2(fmaf(__uint_as_float(rr[i][e]), LOG2E, -mxs));
                    const float p1 = fast_exp2(fmaf(__uint_as_float(rr[i][e + 1]), LOG2E, -mxs));
                    l4[e & 3] += p0;
                    l4[(e & 3) + 1] += p1;
                    pk[e / 2] = pack_bf16x2(p0, p1);
                }
                tmem_st16(tS + 16u * (wq + i), pk);
            }
            tmem_wait_st();
            tc_fence_before();
            warp_arrive(&p_full[g]);
            const float l = (l4[0] + l4[1]) + (l4[2] + l4[3]);
            const int mrow = m0 + t;
            if (mrow < Lr)
                p.lse[((int64_t)T.u * p.L + T.r) + (int64_t)mrow * p.dil] = (mxs + log2f(l)) * LN2;
            const float inv = 1.f / l;

            // epilogue: O / l -> bf16 -> smem -> TMA store (rows 32*wq .. +31)
            mbar_wait(&o_full[g], ph);
            tc_fence_after();
            uint32_t ov[2][32];
            tmem_ld32(tO, ov[0]);
            tmem_ld32(tO + 32, ov[1]);
            tmem_wait_ld();
            tc_fence_before();
            warp_arrive(&o_free[g]);
            if (lane == 0) tma_store_wait_read<0>();
            __syncwarp();
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const uint32_t* src = &ov[q >> 2][(q & 3) * 8];
                uint4 val;
                val.x = pack_bf16x2(__uint_as_float(src[0]) * inv, __uint_as_float(src[1]) * inv);
                val.y = pack_bf16x2(__uint_as_float(src[2]) * inv, __uint_as_float(src[3]) * inv);
                val.z = pack_bf16x2(__uint_as_float(src[4]) * inv, __uint_as_float(src[5]) * inv);
                val.w = pack_bf16x2(__uint_as_float(src[6]) * inv, __uint_as_float(src[7]) * inv);
                *reinterpret_cast<uint4*>(mystg + lane * 128 + ((q ^ (lane & 7)) * 16)) = val;
            }
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) {
                tma_store_3d(&p.maps[T.rl].o, mystg, 0, m0 + 32 * wq, T.u);
                tma_store_commit();
            }
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

int num_sms_n() {
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

bool tc_narrow_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    const int64_t wc = w < L ? w : L;
    if (!knob(K_NARROW)) return false;   // A/B: the band kernels
    return d == D && wc <= 32 && dil <= 256 && units * ((L + BM - 1) / BM) < (1 << 30);
}

bool tc_narrow_bwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    return tc_narrow_supported(units, L, d, w, dil);
}

int tc_narrow_launches(int64_t L, int64_t dil) {
    const int64_t nres = dil < L ? dil : L;
    return (int)ceil_div(nres, RES_PER_LAUNCH);
}

cudaError_t tc_narrow_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                          int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                          cudaStream_t st, int* launches) {
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_narrow_fwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)SMEM_BYTES);
    });
    const int64_t wc = w < L ? w : L;
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    int n = 0;
    for (int64_t r0 = 0; r0 < nres; r0 += RES_PER_LAUNCH) {
        NParams p;
        memset(&p, 0, sizeof(p));
        const int nr = (int)(nres - r0 < RES_PER_LAUNCH ? nres - r0 : RES_PER_LAUNCH);
        for (int i = 0; i < nr; ++i) {
            const int64_t r = r0 + i;
            NMaps& m = p.maps[i];
            if (!(make_residue_map(&m.q, q, L, d, units, dil, r, BM) &&
                  make_residue_map(&m.k, k, L, d, units, dil, r, NK) &&
                  make_residue_map(&m.v, v, L, d, units, dil, r, NK) &&
                  make_residue_map(&m.o, out, L, d, units, dil, r, 32)))
                return cudaErrorInvalidValue;
        }
        p.lse = lse;
        p.L = L;
        p.w = (int)wc;
        p.dil = (int)dil;

        const int64_t Lr0 = ceil_div(L - r0, dil);
        const int tiles = (int)ceil_div(Lr0, BM);
        const int64_t total = units * nr * tiles;
        // only inside ft_winattn_fwd_bwd, where the dQ kernel (NQ, PDL-launched) follows
        p.lsepoll = r0 == 0 && lsepoll_enabled() && lsepoll_worth(total, num_sms_n());
        dim3 grid((unsigned)(total < num_sms_n() ? total : num_sms_n()));
        sched_init(p.sc, L, dil, r0, nr, units, tiles, (int)grid.x);
        tc_narrow_fwd_kernel<<<grid, NTHREADS, SMEM_BYTES, st>>>(p);
        prof_mark(st);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        ++n;
    }
    if (launches) *launches += n;
    return cudaSuccess;
}

}  // namespace ftw
