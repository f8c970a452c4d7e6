// simt.cu -- CUDA-core (FMA) window-attention kernels for sm_100a: fp32 math for fp32 or
// bf16 storage, any d (multiple of 16, <= 512), any w, any dilation.
//
// Tiling follows the paper's redundancy-free formulation (keys are
// indexed directly as j+k, never copied (2w+1)-fold).  A CTA owns a tile of T rows of one
// (unit, residue) band problem and streams only the key chunks that intersect its band
// [m0 - w, m0 + T - 1 + w]: the "cache a[i:i+m]" of PAPER.md Fig. 14 (lines 402-423) is the
// per-chunk K/V staging in shared memory.  Scores and the running row max are produced in
// one pass (the dot/max fusion of Fig. 10); the normalisation uses the
// online-softmax rewrite so the dot_max dependence does not force a second
// sweep.  The backward recomputes P from the saved lse (selective materialization,
// PAPER.md:489-497) and writes dq (query-major kernel) and dk/dv (key-major kernel) each
// from exactly one CTA: no atomics, deterministic (the Fig. 13(d) parallel-reduction
// choice rather than Fig. 13(e) atomics).
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include <mutex>

#include "internal.h"

namespace ftw {
namespace {

constexpr int NT = 256;      // threads per CTA (16 x 16 thread grid)
constexpr int C = 64;        // key (or query) chunk per step
constexpr int DS = 32;       // d-slice staged per step
constexpr int SP = DS + 1;   // padded slice row (bank-conflict free column reads)
constexpr float LOG2E = 1.4426950408889634f;
constexpr float LN2 = 0.6931471805599453f;

template <typename T> struct Vec;
template <> struct Vec<float> {
    static constexpr int N = 4;
    __device__ static void load(const float* p, float* o) {
        float4 x = __ldg(reinterpret_cast<const float4*>(p));
        o[0] = x.x; o[1] = x.y; o[2] = x.z; o[3] = x.w;
    }
    __device__ static void store1(float* p, float x) { *p = x; }
    __device__ static float to_f(float x) { return x; }
};
template <> struct Vec<__nv_bfloat16> {
    static constexpr int N = 8;
    __device__ static void load(const __nv_bfloat16* p, float* o) {
        uint4 x = __ldg(reinterpret_cast<const uint4*>(p));
        const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&x);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
            float2 f = __bfloat1622float2(h[e]);
            o[2 * e] = f.x; o[2 * e + 1] = f.y;
        }
    }
    __device__ static void store1(__nv_bfloat16* p, float x) { *p = __float2bfloat16_rn(x); }
    __device__ static float to_f(__nv_bfloat16 x) { return __bfloat162float(x); }
};


struct TileCoord {
    int64_t u, r;
    int Lr, m0;
    int64_t off;       // element offset of row m=0 of this (unit, residue)
    int64_t rstride;   // element stride between consecutive m
    int64_t row0;      // flat row id (u*L + r) of m=0; flat(m) = row0 + m*dil
};

__device__ __forceinline__ bool decode(const Geo& g, TileCoord& c) {
    int64_t b = blockIdx.x;
    const int64_t t = b % g.tiles;
    b /= g.tiles;
    c.r = b % g.nres;
    c.u = b / g.nres;
    c.Lr = (int)((g.L - c.r + g.dil - 1) / g.dil);
    c.m0 = (int)t * g.T;
    c.off = (c.u * g.L + c.r) * g.d;
    c.rstride = g.dil * g.d;
    c.row0 = c.u * g.L + c.r;
    return c.m0 < c.Lr;
}

__device__ __forceinline__ float hmax16(float x) {
#pragma unroll
    for (int o = 8; o >= 1; o >>= 1) x = fmaxf(x, __shfl_xor_sync(0xffffffffu, x, o));
    return x;
}
__device__ __forceinline__ float hsum16(float x) {
#pragma unroll
    for (int o = 8; o >= 1; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    return x;
}

// ------------------------------------------------------------------------------ forward
// tape (nullable): the raw band scores s_ij, fp32 [B*H*L][2w+1] indexed by the query's flat
// row and k + w (residue-space offset k = m_j - m_i) -- the materialized `dot` of Fig. 8 that
// the tape-based backward reads instead of recomputing it.
// ------------------------------------------------------------------------------ forward
// A CTA owns 64 rows of one (unit, residue) problem and streams the 64-key chunks of its band:
// S = Q K^T over d-slices, online row max / sum, O += P V.  The shared-memory traffic of the two
// micro-GEMMs is cut four-fold: Q and K slices are staged TRANSPOSED ([d column][row], rows padded to 68 floats) so
// a thread's four rows (4ty..4ty+3) and four keys (4tx..4tx+3) are one 16-byte load each per
// d column, and P is staged transposed ([key][row]) so the P.V loop reads a thread's four rows
// of P with one 16-byte load and two V columns (2tx, 2tx+1) with one 8-byte load.  The scalar
// version issued eight 4-byte loads per 16 FMAs and was bound by shared-memory instructions
// (ncu: 34 % issue utilisation at one 8-warp CTA per SM).
constexpr int TP = 64 + 4;     // padded row count of a transposed slice (16-byte aligned rows)
constexpr int VSP = DS + 4;    // padded V slice row (16-byte aligned)

// Register-staged slice loads for software pipelining: a thread fetches its share of slice
// i+1 from HBM into registers while the CTA computes on slice i in shared memory, then stores it
// after the barrier -- the global latency is hidden behind the micro-GEMM instead of being paid
// by every slice (one 8-warp CTA per SM cannot hide it by occupancy).
template <typename Tin, int R>
struct SliceRegs {
    static constexpr int V = Vec<Tin>::N, NV = DS / V, PER = (R * NV + NT - 1) / NT;
    float vals[PER][V];
    __device__ void fetch(const Tin* __restrict__ base, int64_t rstride, int mbase, int Lr, int col0, int d) {
#pragma unroll
        for (int it = 0; it < PER; ++it) {
            const int idx = threadIdx.x + it * NT;
            const int row = idx / NV, cv = idx % NV;
            const int m = mbase + row, c = col0 + cv * V;
            if (idx < R * NV && m >= 0 && m < Lr && c < d) {
                Vec<Tin>::load(base + (int64_t)m * rstride + c, vals[it]);
            } else {
#pragma unroll
                for (int e = 0; e < V; ++e) vals[it][e] = 0.f;
            }
        }
    }
    template <int RP = TP>
    __device__ void store_t(float* dst) const {   // transposed: [col][row], rows padded to RP
#pragma unroll
        for (int it = 0; it < PER; ++it) {
            const int idx = threadIdx.x + it * NT;
            if (idx >= R * NV) break;
            const int row = idx / NV, cv = idx % NV;
#pragma unroll
            for (int e = 0; e < V; ++e) dst[(cv * V + e) * RP + row] = vals[it][e];
        }
    }
    __device__ void store_p(float (*dst)[SP]) const {   // row-major, rows padded to SP
#pragma unroll
        for (int it = 0; it < PER; ++it) {
            const int idx = threadIdx.x + it * NT;
            if (idx >= R * NV) break;
            const int row = idx / NV, cv = idx % NV;
#pragma unroll
            for (int e = 0; e < V; ++e) dst[row][cv * V + e] = vals[it][e];
        }
    }
    __device__ void store_v(float* dst) const {   // row-major, rows padded to VSP
#pragma unroll
        for (int it = 0; it < PER; ++it) {
            const int idx = threadIdx.x + it * NT;
            if (idx >= R * NV) break;
            const int row = idx / NV, cv = idx % NV;
#pragma unroll
            for (int e = 0; e < V; e += 4)
                *reinterpret_cast<float4*>(&dst[row * VSP + cv * V + e]) =
                    make_float4(vals[it][e], vals[it][e + 1], vals[it][e + 2], vals[it][e + 3]);
        }
    }
};

template <typename Tin>
__global__ void __launch_bounds__(NT) simt_fwd_v2_kernel(const Tin* __restrict__ q,
                                                         const Tin* __restrict__ k,
                                                         const Tin* __restrict__ v,
                                                         Tin* __restrict__ out, float* __restrict__ lse,
                                                         float* __restrict__ tape, Geo g) {
    constexpr int T = 64;
    extern __shared__ float smem[];
    float* Qt = smem;                 // [DS][TP]
    float* Kt = Qt + DS * TP;         // [DS][TP]
    float* Vs = Kt + DS * TP;         // [C][VSP]
    float* Pt = Vs + C * VSP;         // [C][TP]   P transposed: key-major
    float* Os = Pt + C * TP;          // [T][d]
    float* rowM = Os + T * g.d;
    float* rowL = rowM + T;

    TileCoord tc;
    if (!decode(g, tc)) return;
    const int d = (int)g.d, w = (int)g.w, Lr = tc.Lr, m0 = tc.m0;
    const Tin* Qb = q + tc.off;
    const Tin* Kb = k + tc.off;
    const Tin* Vb = v + tc.off;
    const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;

    for (int i = threadIdx.x; i < T * d; i += NT) Os[i] = 0.f;
    float mrow[4], lrow[4];
#pragma unroll
    for (int a = 0; a < 4; ++a) { mrow[a] = -INFINITY; lrow[a] = 0.f; }

    const int kbeg = max(0, m0 - w);
    const int kend = min(Lr, m0 + T + w);
    for (int c0 = kbeg; c0 < kend; c0 += C) {
        float s[4][4];
#pragma unroll
        for (int a = 0; a < 4; ++a)
#pragma unroll
            for (int b = 0; b < 4; ++b) s[a][b] = 0.f;
        SliceRegs<Tin, T> rq;
        SliceRegs<Tin, C> rk;
        rq.fetch(Qb, tc.rstride, m0, Lr, 0, d);
        rk.fetch(Kb, tc.rstride, c0, kend, 0, d);
        for (int col0 = 0; col0 < d; col0 += DS) {
            __syncthreads();
            rq.store_t(Qt);
            rk.store_t(Kt);
            __syncthreads();
            if (col0 + DS < d) {   // next slice in flight during this one's micro-GEMM
                rq.fetch(Qb, tc.rstride, m0, Lr, col0 + DS, d);
                rk.fetch(Kb, tc.rstride, c0, kend, col0 + DS, d);
            }
#pragma unroll 8
            for (int p = 0; p < DS; ++p) {
                const float4 qa = *reinterpret_cast<const float4*>(&Qt[p * TP + 4 * ty]);
                const float4 kb = *reinterpret_cast<const float4*>(&Kt[p * TP + 4 * tx]);
                const float qv[4] = {qa.x, qa.y, qa.z, qa.w}, kv[4] = {kb.x, kb.y, kb.z, kb.w};
#pragma unroll
                for (int a = 0; a < 4; ++a)
#pragma unroll
                    for (int b = 0; b < 4; ++b) s[a][b] = fmaf(qv[a], kv[b], s[a][b]);
            }
        }
        // band mask + online softmax (log2 domain); rows 4ty+a are shared by the 16 tx lanes
        float alpha[4];
        __syncthreads();   // the previous chunk's P.V reads of Pt are done
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const int mq = m0 + 4 * ty + a;
            float cmax = -INFINITY;
#pragma unroll
            for (int b = 0; b < 4; ++b) {
                const int mk = c0 + 4 * tx + b;
                const bool ok = (mk < kend) && (abs(mk - mq) <= w);
                if (tape && ok && mq < Lr)
                    tape[(tc.row0 + (int64_t)mq * g.dil) * (2 * w + 1) + (mk - mq + w)] = s[a][b];
                s[a][b] = ok ? s[a][b] * LOG2E : -INFINITY;
                cmax = fmaxf(cmax, s[a][b]);
            }
            cmax = hmax16(cmax);
            const float mnew = fmaxf(mrow[a], cmax);
            alpha[a] = (mnew == -INFINITY) ? 1.f : exp2f(mrow[a] - mnew);
            float sum = 0.f;
#pragma unroll
            for (int b = 0; b < 4; ++b) {
                const float pv = (s[a][b] == -INFINITY) ? 0.f : exp2f(s[a][b] - mnew);
                Pt[(4 * tx + b) * TP + 4 * ty + a] = pv;
                sum += pv;
            }
            sum = hsum16(sum);
            lrow[a] = lrow[a] * alpha[a] + sum;
            mrow[a] = mnew;
        }
        // O = alpha * O + P V, 32 output columns per staged V slice
        SliceRegs<Tin, C> rv;
        rv.fetch(Vb, tc.rstride, c0, kend, 0, d);
        for (int col0 = 0; col0 < d; col0 += DS) {
            __syncthreads();
            rv.store_v(Vs);
            __syncthreads();
            if (col0 + DS < d) rv.fetch(Vb, tc.rstride, c0, kend, col0 + DS, d);
            float acc[4][2];
#pragma unroll
            for (int a = 0; a < 4; ++a) { acc[a][0] = 0.f; acc[a][1] = 0.f; }
#pragma unroll 8
            for (int kk = 0; kk < C; ++kk) {
                const float4 pv = *reinterpret_cast<const float4*>(&Pt[kk * TP + 4 * ty]);
                const float2 vv = *reinterpret_cast<const float2*>(&Vs[kk * VSP + 2 * tx]);
                const float pa[4] = {pv.x, pv.y, pv.z, pv.w};
#pragma unroll
                for (int a = 0; a < 4; ++a) {
                    acc[a][0] = fmaf(pa[a], vv.x, acc[a][0]);
                    acc[a][1] = fmaf(pa[a], vv.y, acc[a][1]);
                }
            }
#pragma unroll
            for (int a = 0; a < 4; ++a)
#pragma unroll
                for (int b = 0; b < 2; ++b) {
                    const int col = col0 + 2 * tx + b;
                    if (col < d) {
                        float* o = &Os[(4 * ty + a) * d + col];
                        *o = *o * alpha[a] + acc[a][b];
                    }
                }
        }
    }
    if (tx == 0) {
#pragma unroll
        for (int a = 0; a < 4; ++a) { rowM[4 * ty + a] = mrow[a]; rowL[4 * ty + a] = lrow[a]; }
    }
    __syncthreads();
    const int nrows = min(T, Lr - m0);
    for (int i = threadIdx.x; i < nrows * d; i += NT) {
        const int row = i / d, col = i % d;
        Vec<Tin>::store1(out + tc.off + (int64_t)(m0 + row) * tc.rstride + col, Os[i] / rowL[row]);
    }
    for (int row = threadIdx.x; row < nrows; row += NT)
        lse[tc.row0 + (int64_t)(m0 + row) * g.dil] = (rowM[row] + log2f(rowL[row])) * LN2;
}

// ------------------------------------------------------------------------------ backward: dq
// Query-major: for owned query rows i,
//     D_i  = sum_j P_ij dP_ij                 (= dout_i . o_i exactly, without reading the
//                                              stored, possibly bf16-rounded, out)
//     dq_i = sum_j P_ij (dP_ij - D_i) k_j  =  sum_j (P_ij dP_ij) k_j  -  D_i sum_j P_ij k_j
// so one sweep over the band accumulates A_i = sum (P dP) k, B_i = sum P k and D_i, and
// dq_i = A_i - D_i B_i at the end.  D is also written to the workspace for the key-major
// kernel.
// TAPE: s_ij is read from the forward's tape instead of being recomputed as q_i . k_j, so the
// score loop stages only dout and V (half its FMAs and shared-memory traffic).
// dq, v2: the same sweep with the vectorised staging of simt_fwd_v2_kernel -- a thread owns the
// RA consecutive rows RA*ty.. and the four consecutive keys 4tx.., Q / dO / K / V slices are
// staged transposed ([d column][row]) and P, P*dP transposed ([key][row]), so every operand of
// both micro-GEMMs is one 8- or 16-byte shared load.
template <int RA>
__device__ __forceinline__ void ldrows(const float* p, float (&o)[RA]) {
    if (RA == 4) {
        const float4 x = *reinterpret_cast<const float4*>(p);
        o[0] = x.x; o[1] = x.y; o[RA > 2 ? 2 : 0] = x.z; o[RA > 3 ? 3 : 0] = x.w;
    } else {
        const float2 x = *reinterpret_cast<const float2*>(p);
        o[0] = x.x; o[1] = x.y;
    }
}

template <typename Tin, int T, bool TAPE>
__global__ void __launch_bounds__(NT, T == 32 ? 1 : 0) simt_dq_v2_kernel(const Tin* __restrict__ q,
                                                        const Tin* __restrict__ k,
                                                        const Tin* __restrict__ v,
                                                        const Tin* __restrict__ dout,
                                                        const float* __restrict__ lse,
                                                        const float* __restrict__ tape,
                                                        float* __restrict__ Dws,
                                                        Tin* __restrict__ dq, Geo g) {
    constexpr int RA = T / 16;
    constexpr int RP = T + 4;                 // padded row count of a transposed T-row slice
    extern __shared__ float smem[];
    float* Qt = smem;                         // [DS][RP]
    float* Gt = Qt + DS * RP;                 // [DS][RP]
    float* Kt = Gt + DS * RP;                 // [DS][TP]
    float* Vt = Kt + DS * TP;                 // [DS][TP]
    float* PDt = Vt + DS * TP;                // [C][RP]  (P * dP) transposed
    float* Pt = PDt + C * RP;                 // [C][RP]
    float* Ko = Qt;                           // [C][VSP] output-loop K slices (reuses Qt / Gt)
    float* rowD = Pt + C * RP;
    float* OsA = rowD + T;
    float* OsB = OsA + T * g.d;
    static_assert(C * VSP <= 2 * DS * RP, "output K slice fits in the Q / dO staging");

    TileCoord tc;
    if (!decode(g, tc)) return;
    const int d = (int)g.d, w = (int)g.w, Lr = tc.Lr, m0 = tc.m0;
    const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
    for (int i = threadIdx.x; i < T * d; i += NT) { OsA[i] = 0.f; OsB[i] = 0.f; }

    float lse2[RA], Dacc[RA];
#pragma unroll
    for (int a = 0; a < RA; ++a) {
        const int mq = m0 + RA * ty + a;
        lse2[a] = mq < Lr ? lse[tc.row0 + (int64_t)mq * g.dil] * LOG2E : 0.f;
        Dacc[a] = 0.f;
    }
    const int kbeg = max(0, m0 - w);
    const int kend = min(Lr, m0 + T + w);
    for (int c0 = kbeg; c0 < kend; c0 += C) {
        float s[RA][4], dp[RA][4];
#pragma unroll
        for (int a = 0; a < RA; ++a)
#pragma unroll
            for (int b = 0; b < 4; ++b) { s[a][b] = 0.f; dp[a][b] = 0.f; }
        SliceRegs<Tin, T> rq, rg;
        SliceRegs<Tin, C> rk, rv;
        auto fetch = [&](int col0) {
            if (!TAPE) rq.fetch(q + tc.off, tc.rstride, m0, Lr, col0, d);
            rg.fetch(dout + tc.off, tc.rstride, m0, Lr, col0, d);
            if (!TAPE) rk.fetch(k + tc.off, tc.rstride, c0, kend, col0, d);
            rv.fetch(v + tc.off, tc.rstride, c0, kend, col0, d);
        };
        fetch(0);
        for (int col0 = 0; col0 < d; col0 += DS) {
            __syncthreads();
            if (!TAPE) rq.template store_t<RP>(Qt);
            rg.template store_t<RP>(Gt);
            if (!TAPE) rk.template store_t<TP>(Kt);
            rv.template store_t<TP>(Vt);
            __syncthreads();
            if (col0 + DS < d) fetch(col0 + DS);
#pragma unroll 4
            for (int p = 0; p < DS; ++p) {
                float qa[RA], ga[RA];
                if (!TAPE) ldrows<RA>(&Qt[p * RP + RA * ty], qa);
                ldrows<RA>(&Gt[p * RP + RA * ty], ga);
                float4 kb4 = make_float4(0.f, 0.f, 0.f, 0.f);
                if (!TAPE) kb4 = *reinterpret_cast<const float4*>(&Kt[p * TP + 4 * tx]);
                const float4 vb4 = *reinterpret_cast<const float4*>(&Vt[p * TP + 4 * tx]);
                const float kb[4] = {kb4.x, kb4.y, kb4.z, kb4.w}, vb[4] = {vb4.x, vb4.y, vb4.z, vb4.w};
#pragma unroll
                for (int a = 0; a < RA; ++a)
#pragma unroll
                    for (int b = 0; b < 4; ++b) {
                        if (!TAPE) s[a][b] = fmaf(qa[a], kb[b], s[a][b]);
                        dp[a][b] = fmaf(ga[a], vb[b], dp[a][b]);
                    }
            }
        }
#pragma unroll
        for (int a = 0; a < RA; ++a) {
            const int mq = m0 + RA * ty + a;
#pragma unroll
            for (int b = 0; b < 4; ++b) {
                const int mk = c0 + 4 * tx + b;
                const bool ok = (mk < kend) && (abs(mk - mq) <= w) && mq < Lr;
                if (TAPE && ok) s[a][b] = tape[(tc.row0 + (int64_t)mq * g.dil) * (2 * w + 1) + (mk - mq + w)];
                const float pv = ok ? exp2f(s[a][b] * LOG2E - lse2[a]) : 0.f;
                const float pd = pv * dp[a][b];
                Dacc[a] += pd;
                PDt[(4 * tx + b) * RP + RA * ty + a] = pd;
                Pt[(4 * tx + b) * RP + RA * ty + a] = pv;
            }
        }
        SliceRegs<Tin, C> rk2;
        rk2.fetch(k + tc.off, tc.rstride, c0, kend, 0, d);
        for (int col0 = 0; col0 < d; col0 += DS) {
            __syncthreads();
            rk2.store_v(Ko);
            __syncthreads();
            if (col0 + DS < d) rk2.fetch(k + tc.off, tc.rstride, c0, kend, col0 + DS, d);
            float aA[RA][2], aB[RA][2];
#pragma unroll
            for (int a = 0; a < RA; ++a) { aA[a][0] = aA[a][1] = aB[a][0] = aB[a][1] = 0.f; }
#pragma unroll 4
            for (int kk = 0; kk < C; ++kk) {
                const float2 kv = *reinterpret_cast<const float2*>(&Ko[kk * VSP + 2 * tx]);
                float pd[RA], pv[RA];
                ldrows<RA>(&PDt[kk * RP + RA * ty], pd);
                ldrows<RA>(&Pt[kk * RP + RA * ty], pv);
#pragma unroll
                for (int a = 0; a < RA; ++a) {
                    aA[a][0] = fmaf(pd[a], kv.x, aA[a][0]);
                    aA[a][1] = fmaf(pd[a], kv.y, aA[a][1]);
                    aB[a][0] = fmaf(pv[a], kv.x, aB[a][0]);
                    aB[a][1] = fmaf(pv[a], kv.y, aB[a][1]);
                }
            }
#pragma unroll
            for (int a = 0; a < RA; ++a)
#pragma unroll
                for (int b = 0; b < 2; ++b) {
                    const int col = col0 + 2 * tx + b;
                    if (col < d) {
                        OsA[(RA * ty + a) * d + col] += aA[a][b];
                        OsB[(RA * ty + a) * d + col] += aB[a][b];
                    }
                }
        }
    }
#pragma unroll
    for (int a = 0; a < RA; ++a) {
        const float D = hsum16(Dacc[a]);
        if (tx == 0) rowD[RA * ty + a] = D;
    }
    __syncthreads();
    const int nrows = min(T, Lr - m0);
    for (int i = threadIdx.x; i < nrows * d; i += NT) {
        const int row = i / d, col = i % d;
        Vec<Tin>::store1(dq + tc.off + (int64_t)(m0 + row) * tc.rstride + col,
                         OsA[i] - rowD[row] * OsB[i]);
    }
    for (int row = threadIdx.x; row < nrows; row += NT)
        Dws[tc.row0 + (int64_t)(m0 + row) * g.dil] = rowD[row];
}

// ------------------------------------------------------------------------------ backward: dk, dv
// Key-major: for owned key rows j, dk_j = sum_i dS_ij q_i and dv_j = sum_i P_ij dout_i over
// the queries i whose window contains j (the band is symmetric: |m_i - m_j| <= w).
// dk / dv: key-major, with the staging of simt_dq_v2_kernel -- a thread owns key
// rows RA*ty.. and the four consecutive queries 4tx..; K / V / Q / dO slices transposed, P and
// dS transposed ([query][key row]), the output loop's Q / dO slices row-major (float2 loads).
template <typename Tin, int T, bool TAPE>
__global__ void __launch_bounds__(NT) simt_dkdv_v2_kernel(const Tin* __restrict__ q,
                                                          const Tin* __restrict__ k,
                                                          const Tin* __restrict__ v,
                                                          const Tin* __restrict__ dout,
                                                          const float* __restrict__ lse,
                                                          const float* __restrict__ tape,
                                                          const float* __restrict__ Dws,
                                                          Tin* __restrict__ dk, Tin* __restrict__ dv,
                                                          Geo g) {
    constexpr int RA = T / 16;
    constexpr int RP = T + 4;
    extern __shared__ float smem[];
    float* Kt = smem;                 // [DS][RP]
    float* Vt = Kt + DS * RP;         // [DS][RP]
    float* Qt = Vt + DS * RP;         // [DS][TP]
    float* Gt = Qt + DS * TP;         // [DS][TP]
    float* Pt = Gt + DS * TP;         // [C][RP]
    float* DSt = Pt + C * RP;         // [C][RP]
    float* Qo = smem;                 // [C][VSP] output-loop slices (reuse Kt .. Gt)
    float* Go = Qo + C * VSP;
    float* qlse = DSt + C * RP;
    float* qD = qlse + C;
    float* OsK = qD + C;
    float* OsV = OsK + T * g.d;
    static_assert(2 * C * VSP <= 2 * DS * RP + 2 * DS * TP, "output slices fit in the staging");

    TileCoord tc;
    if (!decode(g, tc)) return;
    const int d = (int)g.d, w = (int)g.w, Lr = tc.Lr, m0 = tc.m0;
    const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
    for (int i = threadIdx.x; i < T * d; i += NT) { OsK[i] = 0.f; OsV[i] = 0.f; }

    const int qbeg = max(0, m0 - w);
    const int qend = min(Lr, m0 + T + w);
    for (int c0 = qbeg; c0 < qend; c0 += C) {
        float s[RA][4], dp[RA][4];
#pragma unroll
        for (int a = 0; a < RA; ++a)
#pragma unroll
            for (int b = 0; b < 4; ++b) { s[a][b] = 0.f; dp[a][b] = 0.f; }
        __syncthreads();
        for (int i = threadIdx.x; i < C; i += NT) {
            const int mq = c0 + i;
            const int64_t fr = tc.row0 + (int64_t)mq * g.dil;
            qlse[i] = mq < qend ? lse[fr] * LOG2E : 0.f;
            qD[i] = mq < qend ? Dws[fr] : 0.f;
        }
        SliceRegs<Tin, T> rk, rv;
        SliceRegs<Tin, C> rq, rg;
        auto fetch = [&](int col0) {
            if (!TAPE) rk.fetch(k + tc.off, tc.rstride, m0, Lr, col0, d);
            rv.fetch(v + tc.off, tc.rstride, m0, Lr, col0, d);
            if (!TAPE) rq.fetch(q + tc.off, tc.rstride, c0, qend, col0, d);
            rg.fetch(dout + tc.off, tc.rstride, c0, qend, col0, d);
        };
        fetch(0);
        for (int col0 = 0; col0 < d; col0 += DS) {
            __syncthreads();
            if (!TAPE) rk.template store_t<RP>(Kt);
            rv.template store_t<RP>(Vt);
            if (!TAPE) rq.template store_t<TP>(Qt);
            rg.template store_t<TP>(Gt);
            __syncthreads();
            if (col0 + DS < d) fetch(col0 + DS);
#pragma unroll 4
            for (int p = 0; p < DS; ++p) {
                float ka[RA], va[RA];
                if (!TAPE) ldrows<RA>(&Kt[p * RP + RA * ty], ka);
                ldrows<RA>(&Vt[p * RP + RA * ty], va);
                float4 qb4 = make_float4(0.f, 0.f, 0.f, 0.f);
                if (!TAPE) qb4 = *reinterpret_cast<const float4*>(&Qt[p * TP + 4 * tx]);
                const float4 gb4 = *reinterpret_cast<const float4*>(&Gt[p * TP + 4 * tx]);
                const float qb[4] = {qb4.x, qb4.y, qb4.z, qb4.w}, gb[4] = {gb4.x, gb4.y, gb4.z, gb4.w};
#pragma unroll
                for (int a = 0; a < RA; ++a)
#pragma unroll
                    for (int b = 0; b < 4; ++b) {
                        if (!TAPE) s[a][b] = fmaf(ka[a], qb[b], s[a][b]);
                        dp[a][b] = fmaf(va[a], gb[b], dp[a][b]);
                    }
            }
        }
#pragma unroll
        for (int a = 0; a < RA; ++a) {
            const int mk = m0 + RA * ty + a;
#pragma unroll
            for (int b = 0; b < 4; ++b) {
                const int qi = 4 * tx + b;
                const int mq = c0 + qi;
                const bool ok = (mq < qend) && (abs(mq - mk) <= w) && mk < Lr;
                if (TAPE && ok) s[a][b] = tape[(tc.row0 + (int64_t)mq * g.dil) * (2 * w + 1) + (mk - mq + w)];
                const float p = ok ? exp2f(s[a][b] * LOG2E - qlse[qi]) : 0.f;
                Pt[qi * RP + RA * ty + a] = p;
                DSt[qi * RP + RA * ty + a] = p * (dp[a][b] - qD[qi]);
            }
        }
        SliceRegs<Tin, C> rq2, rg2;
        rq2.fetch(q + tc.off, tc.rstride, c0, qend, 0, d);
        rg2.fetch(dout + tc.off, tc.rstride, c0, qend, 0, d);
        for (int col0 = 0; col0 < d; col0 += DS) {
            __syncthreads();
            rq2.store_v(Qo);
            rg2.store_v(Go);
            __syncthreads();
            if (col0 + DS < d) {
                rq2.fetch(q + tc.off, tc.rstride, c0, qend, col0 + DS, d);
                rg2.fetch(dout + tc.off, tc.rstride, c0, qend, col0 + DS, d);
            }
            float ak[RA][2], av[RA][2];
#pragma unroll
            for (int a = 0; a < RA; ++a) { ak[a][0] = ak[a][1] = av[a][0] = av[a][1] = 0.f; }
#pragma unroll 4
            for (int qi = 0; qi < C; ++qi) {
                const float2 qv = *reinterpret_cast<const float2*>(&Qo[qi * VSP + 2 * tx]);
                const float2 gv = *reinterpret_cast<const float2*>(&Go[qi * VSP + 2 * tx]);
                float ds[RA], pv[RA];
                ldrows<RA>(&DSt[qi * RP + RA * ty], ds);
                ldrows<RA>(&Pt[qi * RP + RA * ty], pv);
#pragma unroll
                for (int a = 0; a < RA; ++a) {
                    ak[a][0] = fmaf(ds[a], qv.x, ak[a][0]);
                    ak[a][1] = fmaf(ds[a], qv.y, ak[a][1]);
                    av[a][0] = fmaf(pv[a], gv.x, av[a][0]);
                    av[a][1] = fmaf(pv[a], gv.y, av[a][1]);
                }
            }
#pragma unroll
            for (int a = 0; a < RA; ++a)
#pragma unroll
                for (int b = 0; b < 2; ++b) {
                    const int col = col0 + 2 * tx + b;
                    if (col < d) {
                        OsK[(RA * ty + a) * d + col] += ak[a][b];
                        OsV[(RA * ty + a) * d + col] += av[a][b];
                    }
                }
        }
    }
    __syncthreads();
    const int nrows = min(T, Lr - m0);
    for (int i = threadIdx.x; i < nrows * d; i += NT) {
        const int row = i / d, col = i % d;
        const int64_t o = tc.off + (int64_t)(m0 + row) * tc.rstride + col;
        Vec<Tin>::store1(dk + o, OsK[i]);
        Vec<Tin>::store1(dv + o, OsV[i]);
    }
}

size_t dkdv_v2_smem(int T, int64_t d) {
    return sizeof(float) * (2 * DS * (T + 4) + 2 * DS * TP + 2 * C * (T + 4) + 2 * C + 2 * T * d);
}
size_t fwd_v2_smem(int64_t d) { return sizeof(float) * (2 * DS * TP + C * VSP + C * TP + 64 * d + 128); }
size_t dq_v2_smem(int T, int64_t d) {
    return sizeof(float) * (2 * DS * (T + 4) + 2 * DS * TP + 2 * C * (T + 4) + T + 2 * T * d);
}

template <typename F>
void set_smem_once(F* f, size_t bytes, std::once_flag& flag) {
    std::call_once(flag, [&] {
        cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(227 * 1024));
    });
    (void)bytes;
}

template <typename Tin>
cudaError_t fwd_impl(const void* q, const void* k, const void* v, void* out, float* lse, float* tape,
                     int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                     cudaStream_t st) {
    static std::once_flag once;
    Geo g = make_geo(B, H, L, d, w, dil, 64);
    set_smem_once(simt_fwd_v2_kernel<Tin>, fwd_v2_smem(d), once);
    simt_fwd_v2_kernel<Tin><<<(unsigned)geo_blocks(g), NT, fwd_v2_smem(d), st>>>(
        (const Tin*)q, (const Tin*)k, (const Tin*)v, (Tin*)out, lse, tape, g);
    prof_mark(st);
    return cudaGetLastError();
}

template <typename Tin, int T, bool TAPE>
cudaError_t bwd_launch(const void* q, const void* k, const void* v, const float* lse, const float* tape,
                       const void* dout, void* dq, void* dk, void* dv, float* Dws, const Geo& g,
                       cudaStream_t st) {
    static std::once_flag o1, o2;
    const int64_t d = g.d;
    set_smem_once(simt_dq_v2_kernel<Tin, T, TAPE>, dq_v2_smem(T, d), o1);
    simt_dq_v2_kernel<Tin, T, TAPE><<<(unsigned)geo_blocks(g), NT, dq_v2_smem(T, d), st>>>(
        (const Tin*)q, (const Tin*)k, (const Tin*)v, (const Tin*)dout, lse, tape, Dws, (Tin*)dq, g);
    prof_mark(st);
    cudaError_t e;
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    set_smem_once(simt_dkdv_v2_kernel<Tin, T, TAPE>, dkdv_v2_smem(T, d), o2);
    simt_dkdv_v2_kernel<Tin, T, TAPE><<<(unsigned)geo_blocks(g), NT, dkdv_v2_smem(T, d), st>>>(
        (const Tin*)q, (const Tin*)k, (const Tin*)v, (const Tin*)dout, lse, tape, Dws, (Tin*)dk,
        (Tin*)dv, g);
    prof_mark(st);
    return cudaGetLastError();
}

template <typename Tin>
cudaError_t bwd_impl(const void* q, const void* k, const void* v, const void* out,
                     const float* lse, const float* tape, const void* dout, void* dq, void* dk, void* dv,
                     float* Dws, int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                     cudaStream_t st) {
    (void)out;   // D_i is recomputed exactly as sum_j P_ij dP_ij (see simt_dq_v2_kernel)
    const int T = d <= 256 ? 64 : 32;
    Geo g = make_geo(B, H, L, d, w, dil, T);
    if (tape) {
        return T == 64 ? bwd_launch<Tin, 64, true>(q, k, v, lse, tape, dout, dq, dk, dv, Dws, g, st)
                       : bwd_launch<Tin, 32, true>(q, k, v, lse, tape, dout, dq, dk, dv, Dws, g, st);
    }
    return T == 64 ? bwd_launch<Tin, 64, false>(q, k, v, lse, nullptr, dout, dq, dk, dv, Dws, g, st)
                   : bwd_launch<Tin, 32, false>(q, k, v, lse, nullptr, dout, dq, dk, dv, Dws, g, st);
}

}  // namespace

cudaError_t simt_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                     int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                     ft_dtype dt, cudaStream_t st, float* tape) {
    if (dt == FT_F32) return fwd_impl<float>(q, k, v, out, lse, tape, B, H, L, d, w, dil, st);
    return fwd_impl<__nv_bfloat16>(q, k, v, out, lse, tape, B, H, L, d, w, dil, st);
}

cudaError_t simt_bwd(const void* q, const void* k, const void* v, const void* out,
                     const float* lse, const void* dout, void* dq, void* dk, void* dv,
                     float* Dws, int64_t B, int64_t H, int64_t L, int64_t d, int64_t w,
                     int64_t dil, ft_dtype dt, cudaStream_t st, const float* tape) {
    if (dt == FT_F32)
        return bwd_impl<float>(q, k, v, out, lse, tape, dout, dq, dk, dv, Dws, B, H, L, d, w, dil, st);
    return bwd_impl<__nv_bfloat16>(q, k, v, out, lse, tape, dout, dq, dk, dv, Dws, B, H, L, d, w, dil, st);
}

int simt_fwd_launches() { return 1; }
int simt_bwd_launches() { return 2; }

}  // namespace ftw
