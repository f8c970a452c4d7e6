// tc_fwd.cu -- tcgen05/TMEM tensor-core forward of banded window attention (bf16 storage,
// fp32 scores, softmax statistics and accumulation), sm_100a.
//
// One CTA owns BM = 128 query rows m0..m0+127 of one (unit, residue) band problem and the
// key halo m0-w .. m0+127+w (NK = round_up(128 + 2w, 32) <= 256 rows): the cached
// a[i:i+m] window of PAPER.md Fig. 14 (lines 402-423), staged by TMA instead of the
// (2w+1)-fold as_strided copy of Q that the operator baseline makes.
//
//   warp 4  TMA producer  : Q / K d-slices (64 cols, SWIZZLE_128B), then V d-slices
//   warp 5  MMA issuer    : S[128 x NK] = Q K^T  (tcgen05.mma kind::f16, SS, fp32 in TMEM)
//                           O_n[128 x 64] = P V_n (TS: P read from TMEM, V from smem)
//   warps 0-3 softmax/epi : thread t owns query row m0+t (TMEM lane t): band mask, row max,
//                           exp2, row sum (the fused dot/max of PAPER.md Fig. 10 and the
//                           dot_norm/softmax of Fig. 8), P -> TMEM as bf16,
//                           lse -> HBM; then O_n * (1/l) -> bf16 -> smem -> TMA store.
//
// TMEM (256 columns): S fp32 in [0, NK); P bf16 overwrites [0, NK/2) as S is consumed;
// two O slice buffers at [128, 192) and [192, 256) (used only after all of S is read).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <mutex>

#include "internal.h"
#include "tc_common.cuh"
#include "tmap.h"

namespace ftw {
namespace {

using namespace tc;

constexpr int BM = 128;
constexpr int NST = 2;          // smem pipeline stages
constexpr int NTHREADS = 192;   // 4 softmax/epilogue warps + producer + MMA
constexpr int RES_PER_LAUNCH = 4;
constexpr uint32_t QBYTES = BM * 128;   // one 128-row x 64-col bf16 slice
constexpr uint32_t OSTG = BM * 128;     // one output staging slice
constexpr float LOG2E = 1.4426950408889634f;
constexpr float LN2 = 0.6931471805599453f;

struct FwdMaps {
    CUtensorMap q, k, v, o;
};
struct FwdParams {
    FwdMaps maps[RES_PER_LAUNCH];
    float* lse;
    int64_t L;
    int d, w, dil, r0, NK, nsl;
};

__host__ __device__ inline uint32_t fwd_stage_bytes(int NK) { return QBYTES + (uint32_t)NK * 128u; }
inline size_t fwd_smem_bytes(int NK) {
    return 1024 + NST * (size_t)fwd_stage_bytes(NK) + 2 * OSTG + 256;
}

__global__ void __launch_bounds__(NTHREADS, 1) tc_fwd_band_kernel(const __grid_constant__ FwdParams p) {
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_u32 = smem_u32(smem_raw);
    uint8_t* smem = smem_raw + (((raw_u32 + 1023u) & ~1023u) - raw_u32);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int rl = blockIdx.y, u = blockIdx.z;
    const int r = p.r0 + rl;
    const int Lr = (int)((p.L - r + p.dil - 1) / p.dil);
    const int m0 = blockIdx.x * BM;
    if (m0 >= Lr) return;
    const FwdMaps& mp = p.maps[rl];
    const int NK = p.NK, nsl = p.nsl, w = p.w;
    const uint32_t SB = fwd_stage_bytes(NK);

    uint8_t* ostg = smem + NST * SB;
    uint64_t* bars = reinterpret_cast<uint64_t*>(ostg + 2 * OSTG);
    uint64_t* full = bars;
    uint64_t* empty = bars + NST;
    uint64_t* s_full = bars + 2 * NST;
    uint64_t* p_full = s_full + 1;
    uint64_t* o_full = s_full + 2;    // [2]
    uint64_t* o_empty = s_full + 4;   // [2]
    uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(s_full + 6);

    if (warp == 4) {
        if (lane == 0) {
            for (int i = 0; i < NST; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
            mbar_init(s_full, 1);
            mbar_init(p_full, 128);
            for (int i = 0; i < 2; ++i) { mbar_init(&o_full[i], 1); mbar_init(&o_empty[i], 128); }
            fence_barrier_init();
            tma_prefetch(&mp.q); tma_prefetch(&mp.k); tma_prefetch(&mp.v); tma_prefetch(&mp.o);
        }
        __syncwarp();
        tmem_alloc(tmem_holder, 256);
        tmem_relinquish();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tbase = *tmem_holder;

    if (warp == 4) {
        if (lane == 0) {   // ------------------------------------------------ TMA producer
            int st = 0;
            uint32_t ph = 0;
            const uint32_t kbytes = (uint32_t)NK * 128u;
            for (int s = 0; s < nsl; ++s) {
                mbar_wait(&empty[st], ph ^ 1u);
                uint8_t* sq = smem + st * SB;
                mbar_arrive_expect_tx(&full[st], QBYTES + kbytes);
                tma_load_3d(sq, &mp.q, &full[st], s * 64, m0, u);
                tma_load_3d(sq + QBYTES, &mp.k, &full[st], s * 64, m0 - w, u);
                if (++st == NST) { st = 0; ph ^= 1u; }
            }
            for (int n = 0; n < nsl; ++n) {
                mbar_wait(&empty[st], ph ^ 1u);
                uint8_t* sv = smem + st * SB + QBYTES;
                mbar_arrive_expect_tx(&full[st], kbytes);
                tma_load_3d(sv, &mp.v, &full[st], n * 64, m0 - w, u);
                if (++st == NST) { st = 0; ph ^= 1u; }
            }
        }
    } else if (warp == 5) {
        if (lane == 0) {   // ------------------------------------------------ MMA issuer
            const uint32_t idS = idesc_bf16(128, NK, false, false);
            const uint32_t idO = idesc_bf16(128, 64, false, true);
            int st = 0;
            uint32_t ph = 0;
            for (int s = 0; s < nsl; ++s) {
                mbar_wait(&full[st], ph);
                tc_fence_after();
                const uint32_t qa = smem_u32(smem + st * SB), ka = qa + QBYTES;
#pragma unroll
                for (int kk = 0; kk < 4; ++kk)
                    mma_ss(tbase, sdesc_sw128(qa + kk * 32, 16, 1024),
                           sdesc_sw128(ka + kk * 32, 16, 1024), idS, (s | kk) != 0);
                mma_commit(&empty[st]);
                if (++st == NST) { st = 0; ph ^= 1u; }
            }
            mma_commit(s_full);
            mbar_wait(p_full, 0);
            tc_fence_after();
            for (int n = 0; n < nsl; ++n) {
                const int buf = n & 1;
                if (n >= 2) {
                    mbar_wait(&o_empty[buf], ((n >> 1) - 1) & 1);
                    tc_fence_after();
                }
                mbar_wait(&full[st], ph);
                tc_fence_after();
                const uint32_t va = smem_u32(smem + st * SB + QBYTES);
                const uint32_t tO = tbase + 128 + 64 * buf;
                for (int kk = 0; kk < NK / 16; ++kk)
                    mma_ts(tO, tbase + kk * 8, sdesc_sw128(va + kk * 2048, NK * 128, 1024), idO,
                           kk != 0);
                mma_commit(&empty[st]);
                mma_commit(&o_full[buf]);
                if (++st == NST) { st = 0; ph ^= 1u; }
            }
        }
    } else {   // --------------------------------------------------------- softmax + epilogue
        const int t = warp * 32 + lane;
        const uint32_t trow = tbase + ((uint32_t)(warp * 32) << 16);
        const int mq = m0 + t;
        const int kb = m0 - w;   // residue index of key column 0
        const int nch = NK / 32;

        mbar_wait(s_full, 0);
        tc_fence_after();
        float mx = -INFINITY;
        for (int c = 0; c < nch; ++c) {
            uint32_t rr[32];
            tmem_ld32(trow + c * 32, rr);
            tmem_wait_ld();
#pragma unroll
            for (int e = 0; e < 32; ++e) {
                const int n = c * 32 + e, mk = kb + n;
                const bool ok = (unsigned)(n - t) <= (unsigned)(2 * w) && mk >= 0 && mk < Lr;
                if (ok) mx = fmaxf(mx, __uint_as_float(rr[e]));
            }
        }
        if (mx == -INFINITY) mx = 0.f;   // only rows beyond the sequence (never stored)
        const float mxs = mx * LOG2E;
        float sum = 0.f;
        for (int c = 0; c < nch; ++c) {
            uint32_t rr[32], pk[16];
            tmem_ld32(trow + c * 32, rr);
            tmem_wait_ld();
#pragma unroll
            for (int e = 0; e < 32; e += 2) {
                float pv[2];
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int n = c * 32 + e + h, mk = kb + n;
                    const bool ok = (unsigned)(n - t) <= (unsigned)(2 * w) && mk >= 0 && mk < Lr;
                    pv[h] = ok ? exp2f(fmaf(__uint_as_float(rr[e + h]), LOG2E, -mxs)) : 0.f;
                    sum += pv[h];
                }
                pk[e / 2] = pack_bf16x2(pv[0], pv[1]);
            }
            tmem_st16(trow + c * 16, pk);
        }
        tmem_wait_st();
        tc_fence_before();
        mbar_arrive(p_full);
        if (mq < Lr) p.lse[(int64_t)u * p.L + r + (int64_t)mq * p.dil] = (mxs + log2f(sum)) * LN2;
        const float inv = 1.f / sum;

        for (int n = 0; n < nsl; ++n) {
            const int buf = n & 1;
            mbar_wait(&o_full[buf], (n >> 1) & 1);
            tc_fence_after();
            uint32_t o[64];
            tmem_ld32(trow + 128 + 64 * buf, *reinterpret_cast<uint32_t(*)[32]>(&o[0]));
            tmem_ld32(trow + 128 + 64 * buf + 32, *reinterpret_cast<uint32_t(*)[32]>(&o[32]));
            tmem_wait_ld();
            tc_fence_before();
            mbar_arrive(&o_empty[buf]);

            uint8_t* stg = ostg + buf * OSTG;
            if (t == 0 && n >= 2) tma_store_wait_read<1>();
            named_bar_sync(1, 128);
#pragma unroll
            for (int c = 0; c < 8; ++c) {
                uint4 val;
                val.x = pack_bf16x2(__uint_as_float(o[8 * c + 0]) * inv, __uint_as_float(o[8 * c + 1]) * inv);
                val.y = pack_bf16x2(__uint_as_float(o[8 * c + 2]) * inv, __uint_as_float(o[8 * c + 3]) * inv);
                val.z = pack_bf16x2(__uint_as_float(o[8 * c + 4]) * inv, __uint_as_float(o[8 * c + 5]) * inv);
                val.w = pack_bf16x2(__uint_as_float(o[8 * c + 6]) * inv, __uint_as_float(o[8 * c + 7]) * inv);
                *reinterpret_cast<uint4*>(stg + t * 128 + ((c ^ (t & 7)) * 16)) = val;
            }
            fence_proxy_async_smem();
            named_bar_sync(1, 128);
            if (t == 0) {
                tma_store_3d(&mp.o, stg, n * 64, m0, u);
                tma_store_commit();
            }
        }
        if (t == 0) tma_store_wait_all<0>();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 4) {
        tc_fence_after();
        tmem_dealloc(tbase, 256);
    }
}

}  // namespace

bool tc_fwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    const int64_t wc = w < L ? w : L;
    return d % 64 == 0 && d <= 512 && wc <= 64 && dil <= 256 && units <= 65535;
}

int tc_fwd_launches(int64_t L, int64_t d, int64_t w, int64_t dil) {
    (void)d; (void)w;
    const int64_t nres = dil < L ? dil : L;
    return (int)ceil_div(nres, RES_PER_LAUNCH);
}

cudaError_t tc_fwd(const void* q, const void* k, const void* v, void* out, float* lse, int64_t B,
                   int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st,
                   int* launches) {
    const int64_t wc = w < L ? w : L;
    const int NK = (int)(((BM + 2 * wc) + 31) / 32 * 32);
    const int64_t units = B * H;
    const int64_t nres = dil < L ? dil : L;
    const size_t smem = fwd_smem_bytes(NK);
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(tc_fwd_band_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             227 * 1024);
    });
    int n = 0;
    for (int64_t r0 = 0; r0 < nres; r0 += RES_PER_LAUNCH) {
        FwdParams p;
        memset(&p, 0, sizeof(p));
        const int nr = (int)(nres - r0 < RES_PER_LAUNCH ? nres - r0 : RES_PER_LAUNCH);
        for (int i = 0; i < nr; ++i) {
            const int64_t r = r0 + i;
            if (!make_residue_map(&p.maps[i].q, q, L, d, units, dil, r, BM) ||
                !make_residue_map(&p.maps[i].k, k, L, d, units, dil, r, NK) ||
                !make_residue_map(&p.maps[i].v, v, L, d, units, dil, r, NK) ||
                !make_residue_map(&p.maps[i].o, out, L, d, units, dil, r, BM))
                return cudaErrorInvalidValue;
        }
        p.lse = lse;
        p.L = L;
        p.d = (int)d;
        p.w = (int)wc;
        p.dil = (int)dil;
        p.r0 = (int)r0;
        p.NK = NK;
        p.nsl = (int)(d / 64);
        const int64_t Lr0 = ceil_div(L - r0, dil);   // longest residue of this group
        dim3 grid((unsigned)ceil_div(Lr0, BM), (unsigned)nr, (unsigned)units);
        tc_fwd_band_kernel<<<grid, NTHREADS, smem, st>>>(p);
        prof_mark(st);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        ++n;
    }
    if (launches) *launches = n;
    return cudaSuccess;
}

}  // namespace ftw
