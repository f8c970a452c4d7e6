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
// dS enters the output MMAs as a bf16 hi + lo pair (reading A10): a single bf16 dS put dq
// 1.1e-2 off at one element of 8.4M in the 16 x 8192 parity case.  TMEM: NQ writes dS_hi |
// dS_lo over S; NKV writes P^T | dS^T_hi over S^T and dS^T_lo over the first 96 columns of
// dP^T, so its output MMAs are issued before the next tile's S^T (which reuses that region).
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
#include "tmap.h"

namespace ftw {
namespace {

using namespace tc;

enum { NQ = 0, NKV = 1 };

constexpr int BM = 128;
constexpr int D = 64;
constexpr int NK = 192;
constexpr int NSTAGE = 2;
constexpr int NTHREADS = 320;
constexpr int RES_PER_LAUNCH = 3;
constexpr uint32_t ABYTES = BM * D * 2;      // 16 KB: a 128-row tile
constexpr uint32_t HBYTES = NK * D * 2;      // 24 KB: a 192-row halo
constexpr uint32_t STAGE = 2 * ABYTES + 2 * HBYTES;   // {A1, A2, B1, B2}
constexpr uint32_t STG = 32 * 128;
constexpr size_t SMEM_BYTES = 1024 + (size_t)NSTAGE * STAGE + 8 * STG + 2 * 2 * NK * 4 + 2 * 2 * BM * 4 + 256;
constexpr float LOG2E = 1.4426950408889634f;
constexpr uint32_t TACC = 384;

// a1/b1: first score GEMM (A: 128 rows at m0, B: halo at m0-w); a2/b2: second; o1/o2: outputs.
struct BMaps {
    CUtensorMap a1, a2, b1, b2, o1, o2;
};
struct BParams {
    BMaps maps[RES_PER_LAUNCH];
    const float* lse;
    float* D;   // NQ: written; NKV: read
    int64_t L;
    int w, dil, r0, nr, units, tiles;
};

struct Tile {
    int u, rl, r, Lr, m0;
};
__device__ __forceinline__ bool decode_tile(const BParams& p, int tau, Tile& T) {
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
    __device__ bool next(const BParams& p, int total, Tile& T) {
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
    __nv_bfloat162 hb = __floats2bfloat162_rn(x0, x1);
    const float2 hf = __bfloat1622float2(hb);
    hi = *reinterpret_cast<uint32_t*>(&hb);
    lo = pack_bf16x2(x0 - hf.x, x1 - hf.y);
}

// rows 32*wq .. +31 of a 64-column accumulator -> bf16 -> this warp's staging -> TMA store
// (the accumulator is released on `freed` as soon as it is in registers)
__device__ __forceinline__ void drain_store(uint32_t tacc, uint8_t* stg, const CUtensorMap* m, int row0,
                                           int u, int lane, uint64_t* freed) {
    uint32_t ov[2][32];
    tmem_ld32(tacc, ov[0]);
    tmem_ld32(tacc + 32, ov[1]);
    tmem_wait_ld();
    tc_fence_before();
    mbar_arrive(freed);
    if (lane == 0) tma_store_wait_read<0>();
    __syncwarp();
#pragma unroll
    for (int q = 0; q < 8; ++q) {
        const uint32_t* src = &ov[q >> 2][(q & 3) * 8];
        uint4 val;
        val.x = pack_bf16x2(__uint_as_float(src[0]), __uint_as_float(src[1]));
        val.y = pack_bf16x2(__uint_as_float(src[2]), __uint_as_float(src[3]));
        val.z = pack_bf16x2(__uint_as_float(src[4]), __uint_as_float(src[5]));
        val.w = pack_bf16x2(__uint_as_float(src[6]), __uint_as_float(src[7]));
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
    uint8_t* stages = smem;                                        // [NSTAGE] {A1, A2, B1, B2}
    uint8_t* ostg = smem + (size_t)NSTAGE * STAGE;                 // [8 warps] 4 KB
    float* colv = reinterpret_cast<float*>(ostg + 8 * STG);        // NKV [2][2][NK]: lse*log2e, D
    float* dx = colv + 2 * 2 * NK;                                 // NQ [2][2][BM]: D halves
    uint64_t* bars = reinterpret_cast<uint64_t*>(dx + 2 * 2 * BM);
    uint64_t* full1 = bars;                 // [NSTAGE] A1 + B1
    uint64_t* full2 = bars + NSTAGE;        // [NSTAGE] A2 + B2
    uint64_t* empty = bars + 2 * NSTAGE;    // [NSTAGE]
    uint64_t* s_full = bars + 3 * NSTAGE;   // S and dP of the tile done
    uint64_t* p_done = s_full + 1;          // softmax read dP and wrote the operand
    uint64_t* acc_full = s_full + 2;
    uint64_t* acc_free = s_full + 3;
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(s_full + 4);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int w = p.w;
    const int total = p.units * p.nr * p.tiles;
    constexpr int NDRAIN = MODE == NQ ? 128 : 256;

    if (warp == 8) {
        if (lane == 0) {
            for (int i = 0; i < NSTAGE; ++i) {
                mbar_init(&full1[i], 1);
                mbar_init(&full2[i], 1);
                mbar_init(&empty[i], 1);
            }
            mbar_init(s_full, 1);
            mbar_init(p_done, 256);
            mbar_init(acc_full, 1);
            mbar_init(acc_free, NDRAIN);
            fence_barrier_init();
            for (int i = 0; i < p.nr; ++i) {
                const BMaps& m = p.maps[i];
                tma_prefetch(&m.a1); tma_prefetch(&m.a2); tma_prefetch(&m.b1); tma_prefetch(&m.b2);
                tma_prefetch(&m.o1);
                if (MODE == NKV) tma_prefetch(&m.o2);
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
            TileCursor cur(blockIdx.x);
            Tile T;
            for (int j = 0; cur.next(p, total, T); ++j) {
                const int s = j % NSTAGE;
                if (j >= NSTAGE) mbar_wait(&empty[s], ((j / NSTAGE) - 1) & 1);
                uint8_t* st = stages + (size_t)s * STAGE;
                const BMaps& mp = p.maps[T.rl];
                mbar_arrive_expect_tx(&full1[s], ABYTES + HBYTES);
                tma_load_3d(st, &mp.a1, &full1[s], 0, T.m0, T.u);
                tma_load_3d(st + 2 * ABYTES, &mp.b1, &full1[s], 0, T.m0 - w, T.u);
                mbar_arrive_expect_tx(&full2[s], ABYTES + HBYTES);
                tma_load_3d(st + ABYTES, &mp.a2, &full2[s], 0, T.m0, T.u);
                tma_load_3d(st + 2 * ABYTES + HBYTES, &mp.b2, &full2[s], 0, T.m0 - w, T.u);
            }
        }
    } else if (warp == 9) {
        if (lane == 0) {   // ------------------------------------------------------ MMA issuer
            constexpr uint32_t idS = idesc_bf16(BM, NK, false, false);
            constexpr uint32_t idO = idesc_bf16(BM, D, false, true);
            // output MMAs of tile i: A = bf16 operand packed in region i&1 (8 columns per
            // 16-key step), B = a halo as MN-major SW128 (2048 B per step)
            auto out = [&](int i) {
                const int s = i % NSTAGE;
                const uint32_t st = smem_u32(stages + (size_t)s * STAGE);
                const uint32_t tR = tbase + 192u * (i & 1), tR2 = tbase + 192u * ((i + 1) & 1);
                if (i >= 1) mbar_wait(acc_free, (i - 1) & 1);
                tc_fence_after();
                if (MODE == NQ) {   // dQ = (dS_hi + dS_lo) K_h
                    const uint32_t sb = st + 2 * ABYTES;
#pragma unroll
                    for (int g = 0; g < 3; ++g) {
                        const uint64_t bd = sdesc_sw128(sb + 8192u * g, 8192, 1024);
                        mma_ts_x4<8, 128>(tbase + TACC, tR + 32u * g, bd, idO, g);
                        mma_ts_x4<8, 128>(tbase + TACC, tR + 96u + 32u * g, bd, idO, 1);
                    }
                } else {            // dV = P^T dO_h, dK = (dS^T_hi + dS^T_lo) Q_h
                    const uint32_t sq = st + 2 * ABYTES, sdo = sq + HBYTES;
#pragma unroll
                    for (int g = 0; g < 3; ++g) {
                        const uint64_t bq = sdesc_sw128(sq + 8192u * g, 8192, 1024);
                        mma_ts_x4<8, 128>(tbase + TACC, tR + 32u * g, sdesc_sw128(sdo + 8192u * g, 8192, 1024), idO, g);
                        mma_ts_x4<8, 128>(tbase + TACC + 64, tR + 96u + 32u * g, bq, idO, g);
                        mma_ts_x4<8, 128>(tbase + TACC + 64, tR2 + 32u * g, bq, idO, 1);
                    }
                }
                mma_commit(acc_full);
                mma_commit(&empty[s]);
            };
            TileCursor cur(blockIdx.x);
            Tile T;
            int j = 0;
            for (; cur.next(p, total, T); ++j) {
                const int s = j % NSTAGE, ph = (j / NSTAGE) & 1;
                const uint32_t st = smem_u32(stages + (size_t)s * STAGE);
                const uint32_t rS = tbase + 192u * (j & 1), rP = tbase + 192u * ((j + 1) & 1);
                // region j&1 held dP(j-1) (NKV: and dS^T_lo(j-1)); region (j+1)&1 the operands
                // of j-1.  out(j-1) is issued first; the MMAs below run after it in issue order.
                if (j >= 1) {
                    mbar_wait(p_done, (j - 1) & 1);
                    out(j - 1);
                }
                mbar_wait(&full1[s], ph);
                tc_fence_after();
                mma_ss_x4<2, 2>(rS, sdesc_sw128(st, 16, 1024), sdesc_sw128(st + 2 * ABYTES, 16, 1024), idS, 0);
                mbar_wait(&full2[s], ph);
                tc_fence_after();
                mma_ss_x4<2, 2>(rP, sdesc_sw128(st + ABYTES, 16, 1024),
                                sdesc_sw128(st + 2 * ABYTES + HBYTES, 16, 1024), idS, 0);
                mma_commit(s_full);
            }
            if (j >= 1) {
                mbar_wait(p_done, (j - 1) & 1);
                out(j - 1);
            }
        }
    } else {   // ------------------------------------------------------------ softmax warps
        const int wq = warp & 3, h = warp >> 2;
        const int t = wq * 32 + lane;
        const uint32_t lane_off = (uint32_t)(wq * 32) << 16;
        const int c0 = 32 * wq + 48 * h;         // first of this warp's 48 score columns
        const uint32_t pc = 16u * wq + 24u * h;  // its packed bf16 operand columns
        uint8_t* mystg = ostg + warp * STG;
        uint32_t zero16[16];
#pragma unroll
        for (int e = 0; e < 16; ++e) zero16[e] = 0u;
        // 48 packed columns of an operand at base (+ zeros on the columns outside every band
        // column of this row: h = 0 writes the ones before, h = 1 the ones after)
        auto st_operand = [&](uint32_t base, const uint32_t (&pk)[24]) {
            tmem_st16(base + pc, *reinterpret_cast<const uint32_t(*)[16]>(&pk[0]));
            tmem_st8(base + pc + 16, &pk[16]);
            if (h == 0) {
                for (int c = 0; c < wq; ++c) tmem_st16(base + 16u * c, zero16);
            } else {
                for (int c = wq + 3; c < NK / 32; ++c) tmem_st16(base + 16u * c, zero16);
            }
        };
        // per-tile values from HBM are loaded one tile ahead (NQ: this row's lse; NKV: lse and
        // D of halo column threadIdx.x), so their latency hides behind the previous tile
        TileCursor cur(blockIdx.x), nxt(blockIdx.x);
        Tile T, Tn;
        bool hn = nxt.next(p, total, Tn);
        float pre_l = 0.f, pre_d = 0.f;
        auto prefetch = [&](const Tile& X) {
            const int64_t rb = (int64_t)X.u * p.L + X.r;
            if (MODE == NKV) {
                const int mc = X.m0 - w + (int)threadIdx.x;
                const bool ok = threadIdx.x < NK && mc >= 0 && mc < X.Lr;
                pre_l = ok ? p.lse[rb + (int64_t)mc * p.dil] : 0.f;
                pre_d = ok ? p.D[rb + (int64_t)mc * p.dil] : 0.f;
            } else {
                const int mrow = X.m0 + t;
                pre_l = mrow < X.Lr ? p.lse[rb + (int64_t)mrow * p.dil] : 0.f;
            }
        };
        if (hn) prefetch(Tn);
        for (int j = 0; cur.next(p, total, T); ++j) {
            const int Lr = T.Lr, m0 = T.m0, kb = m0 - w;
            const int64_t rowbase = (int64_t)T.u * p.L + T.r;
            const uint32_t tS = tbase + lane_off + 192u * (j & 1);
            const uint32_t tP = tbase + lane_off + 192u * ((j + 1) & 1);
            float* cl = colv + (j & 1) * 2 * NK;   // NKV: this tile's column lse*log2e and D
            float lse2 = 0.f;
            if (MODE == NKV) {
                if (threadIdx.x < NK) {
                    cl[threadIdx.x] = pre_l * LOG2E;
                    cl[NK + threadIdx.x] = pre_d;
                }
            } else {
                lse2 = pre_l * LOG2E;
            }
            hn = nxt.next(p, total, Tn);
            if (hn) prefetch(Tn);
            if (MODE == NKV) named_bar_sync(5, 256);
            // band columns of this row: n in [t, t+2w] within the sequence
            const int lo = max(t, -kb) - c0, hi = min(t + 2 * w, Lr - 1 - kb) - c0;
            const int l0 = max(lo, 0), h0 = min(hi, 47);
            const uint64_t bits = h0 < l0 ? 0ull : ((~0ull >> (63 - h0)) & (~0ull << l0));

            mbar_wait(s_full, j & 1);
            tc_fence_after();
            uint32_t rs[48], rd[48];
            tmem_ld16(tS + c0, *reinterpret_cast<uint32_t(*)[16]>(&rs[0]));
            tmem_ld16(tS + c0 + 16, *reinterpret_cast<uint32_t(*)[16]>(&rs[16]));
            tmem_ld16(tS + c0 + 32, *reinterpret_cast<uint32_t(*)[16]>(&rs[32]));
            tmem_ld16(tP + c0, *reinterpret_cast<uint32_t(*)[16]>(&rd[0]));
            tmem_ld16(tP + c0 + 16, *reinterpret_cast<uint32_t(*)[16]>(&rd[16]));
            tmem_ld16(tP + c0 + 32, *reinterpret_cast<uint32_t(*)[16]>(&rd[32]));
            tmem_wait_ld();
            uint32_t pk[24], pk2[24], pk3[24];
            if (MODE == NQ) {
                float dpart[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                for (int e = 0; e < 48; ++e) {
                    const float pv = ((bits >> e) & 1ull) ? fast_exp2(fmaf(__uint_as_float(rs[e]), LOG2E, -lse2)) : 0.f;
                    rs[e] = __float_as_uint(pv);
                    dpart[e & 3] = fmaf(pv, __uint_as_float(rd[e]), dpart[e & 3]);
                }
                float* dxb = dx + (j & 1) * 2 * BM;
                dxb[h * BM + t] = (dpart[0] + dpart[1]) + (dpart[2] + dpart[3]);
                named_bar_sync(1 + wq, 64);   // both halves read S/dP and posted their D part
                const float Dv = dxb[t] + dxb[BM + t];
#pragma unroll
                for (int e = 0; e < 48; e += 2) {
                    const float d0 = __uint_as_float(rs[e]) * (__uint_as_float(rd[e]) - Dv);
                    const float d1 = __uint_as_float(rs[e + 1]) * (__uint_as_float(rd[e + 1]) - Dv);
                    split_bf16x2(d0, d1, pk[e / 2], pk2[e / 2]);
                }
                // dS_hi | dS_lo packed over S (keys 2c, 2c+1 -> column c of each half)
                st_operand(tS, pk);
                st_operand(tS + 96, pk2);
                const int mrow = m0 + t;
                if (h == 0 && mrow < Lr) p.D[rowbase + (int64_t)mrow * p.dil] = Dv;
            } else {
                const float* cL = cl + c0;
                const float* cD = cl + NK + c0;
#pragma unroll
                for (int e = 0; e < 48; e += 2) {
                    float pv[2], dv[2];
#pragma unroll
                    for (int x = 0; x < 2; ++x) {
                        pv[x] = ((bits >> (e + x)) & 1ull) ? fast_exp2(fmaf(__uint_as_float(rs[e + x]), LOG2E, -cL[e + x])) : 0.f;
                        dv[x] = pv[x] * (__uint_as_float(rd[e + x]) - cD[e + x]);
                    }
                    pk[e / 2] = pack_bf16x2(pv[0], pv[1]);
                    split_bf16x2(dv[0], dv[1], pk2[e / 2], pk3[e / 2]);
                }
                named_bar_sync(1 + wq, 64);   // both halves read S^T / dP^T
                // P^T | dS^T_hi over S^T, dS^T_lo over dP^T
                st_operand(tS, pk);
                st_operand(tS + 96, pk2);
                st_operand(tP, pk3);
            }
            tmem_wait_st();
            tc_fence_before();
            mbar_arrive(p_done);

            // epilogue: drain the accumulator of this tile (NQ: dQ by the h = 0 warps; NKV: dV
            // by h = 0, dK by h = 1) once its output MMAs completed
            if (MODE == NKV || h == 0) {
                mbar_wait(acc_full, j & 1);
                tc_fence_after();
                const BMaps& mp = p.maps[T.rl];
                drain_store(tbase + lane_off + TACC + 64u * h, mystg, h == 0 ? &mp.o1 : &mp.o2,
                            m0 + 32 * wq, T.u, lane, acc_free);
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
        p.L = L;
        p.w = (int)wc;
        p.dil = (int)dil;
        p.r0 = (int)r0;
        p.nr = nr;
        p.units = (int)units;
        const int64_t Lr0 = ceil_div(L - r0, dil);
        p.tiles = (int)ceil_div(Lr0, BM);
        const int64_t total = (int64_t)p.units * p.nr * p.tiles;
        dim3 grid((unsigned)(total < num_sms_nb() ? total : num_sms_nb()));
        tc_narrow_bwd_kernel<MODE><<<grid, NTHREADS, SMEM_BYTES, st>>>(p);
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
