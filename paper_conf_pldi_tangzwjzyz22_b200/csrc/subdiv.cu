// subdiv.cu -- SubdivNet's circular difference (Section 2.2, Fig. 2) on sm_100a:
// forward and backward kernels and their extern "C" boundary (include/ft_subdiv.h).
//
// The work is a gather: face i reads the three rows e[adj[i][0..2]] and writes one row, so it
// is HBM-bound (a few flops per byte).  One kernel per direction, no intermediates:
//   * thread <-> (face, 16-byte chunk of the feature row): consecutive threads read consecutive
//     chunks of the same neighbour rows, so every gathered row is read with full 16-byte,
//     coalesced transactions; the three neighbours of a face are fetched independently
//     (memory-level parallelism), the adjacency row once per chunk thread (L1 broadcast);
//   * grid = a multiple of the SM count, grid-stride loop;
//   * the backward scatters +-sign(e_a - e_b) * dy_i into de with vector fp32 reductions
//     (red.global.add.v4.f32 -- a face is referenced by ~3 others, so contention is low), into
//     de itself for fp32 or an fp32 workspace converted to bf16 afterwards.
// Every row is read from HBM about once: the ~3 references to a face's row come from faces
// near it in a well-ordered mesh and hit L2.
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <mutex>

#include "ft_subdiv.h"
#include "internal.h"

namespace ftw {
namespace {

template <typename T> struct V8;   // 16 bytes of T as fp32
template <> struct V8<float> {
    static constexpr int N = 4;
    __device__ static void load(const float* p, float* o) {
        const float4 x = __ldg(reinterpret_cast<const float4*>(p));
        o[0] = x.x; o[1] = x.y; o[2] = x.z; o[3] = x.w;
    }
    __device__ static void store(float* p, const float* o) {
        *reinterpret_cast<float4*>(p) = make_float4(o[0], o[1], o[2], o[3]);
    }
};
template <> struct V8<__nv_bfloat16> {
    static constexpr int N = 8;
    __device__ static void load(const __nv_bfloat16* p, float* o) {
        const uint4 x = __ldg(reinterpret_cast<const uint4*>(p));
        const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&x);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const float2 f = __bfloat1622float2(h[i]);
            o[2 * i] = f.x; o[2 * i + 1] = f.y;
        }
    }
    __device__ static void store(__nv_bfloat16* p, const float* o) {
        uint4 x;
        __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&x);
#pragma unroll
        for (int i = 0; i < 4; ++i) h[i] = __floats2bfloat162_rn(o[2 * i], o[2 * i + 1]);
        *reinterpret_cast<uint4*>(p) = x;
    }
};

__device__ __forceinline__ float sgnf(float x) { return x > 0.f ? 1.f : (x < 0.f ? -1.f : 0.f); }

__device__ __forceinline__ void red_add4(float* p, float a, float b, float c, float d) {
    asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(a), "f"(b), "f"(c), "f"(d)
                 : "memory");
}

// Vector path: n_feats % N == 0.
template <typename T>
__global__ void __launch_bounds__(256) circdiff_fwd_vec(const T* __restrict__ e, const int32_t* __restrict__ adj,
                                                        T* __restrict__ y, int64_t n_faces, int64_t n_feats) {
    constexpr int N = V8<T>::N;
    const int64_t nch = n_feats / N, total = n_faces * nch;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = idx / nch, c = (idx - i * nch) * N;
        const int32_t a0 = __ldg(adj + 3 * i), a1 = __ldg(adj + 3 * i + 1), a2 = __ldg(adj + 3 * i + 2);
        float x0[N], x1[N], x2[N], o[N];
        V8<T>::load(e + a0 * n_feats + c, x0);
        V8<T>::load(e + a1 * n_feats + c, x1);
        V8<T>::load(e + a2 * n_feats + c, x2);
#pragma unroll
        for (int t = 0; t < N; ++t) o[t] = fabsf(x0[t] - x1[t]) + fabsf(x1[t] - x2[t]) + fabsf(x2[t] - x0[t]);
        V8<T>::store(y + i * n_feats + c, o);
    }
}

// Scalar path (any n_feats).
template <typename T>
__device__ __forceinline__ float ld1(const T* p) { return (float)p[0]; }
template <>
__device__ __forceinline__ float ld1<__nv_bfloat16>(const __nv_bfloat16* p) { return __bfloat162float(p[0]); }
template <typename T>
__device__ __forceinline__ void st1(T* p, float x) { p[0] = x; }
template <>
__device__ __forceinline__ void st1<__nv_bfloat16>(__nv_bfloat16* p, float x) { p[0] = __float2bfloat16_rn(x); }

template <typename T>
__global__ void __launch_bounds__(256) circdiff_fwd_scalar(const T* __restrict__ e, const int32_t* __restrict__ adj,
                                                           T* __restrict__ y, int64_t n_faces, int64_t n_feats) {
    const int64_t total = n_faces * n_feats;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = idx / n_feats, k = idx - i * n_feats;
        const float x0 = ld1(e + adj[3 * i] * n_feats + k), x1 = ld1(e + adj[3 * i + 1] * n_feats + k),
                    x2 = ld1(e + adj[3 * i + 2] * n_feats + k);
        st1(y + idx, fabsf(x0 - x1) + fabsf(x1 - x2) + fabsf(x2 - x0));
    }
}

// Backward: dy/de_a0 = sign(x0-x1) - sign(x2-x0), de_a1 = sign(x1-x2) - sign(x0-x1),
// de_a2 = sign(x2-x0) - sign(x1-x2) (each pair (a, b) adds +s to a and -s to b).
template <typename T>
__global__ void __launch_bounds__(256) circdiff_bwd_vec(const T* __restrict__ e, const int32_t* __restrict__ adj,
                                                        const T* __restrict__ dy, float* __restrict__ acc,
                                                        int64_t n_faces, int64_t n_feats) {
    constexpr int N = V8<T>::N;
    const int64_t nch = n_feats / N, total = n_faces * nch;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = idx / nch, c = (idx - i * nch) * N;
        const int32_t a[3] = {__ldg(adj + 3 * i), __ldg(adj + 3 * i + 1), __ldg(adj + 3 * i + 2)};
        float x0[N], x1[N], x2[N], g[N];
        V8<T>::load(e + a[0] * n_feats + c, x0);
        V8<T>::load(e + a[1] * n_feats + c, x1);
        V8<T>::load(e + a[2] * n_feats + c, x2);
        V8<T>::load(dy + i * n_feats + c, g);
        float d0[N], d1[N], d2[N];
#pragma unroll
        for (int t = 0; t < N; ++t) {
            const float s01 = sgnf(x0[t] - x1[t]) * g[t], s12 = sgnf(x1[t] - x2[t]) * g[t],
                        s20 = sgnf(x2[t] - x0[t]) * g[t];
            d0[t] = s01 - s20;
            d1[t] = s12 - s01;
            d2[t] = s20 - s12;
        }
        const float* ds[3] = {d0, d1, d2};
#pragma unroll
        for (int j = 0; j < 3; ++j) {
            float* p = acc + a[j] * n_feats + c;
#pragma unroll
            for (int t = 0; t < N; t += 4) red_add4(p + t, ds[j][t], ds[j][t + 1], ds[j][t + 2], ds[j][t + 3]);
        }
    }
}

template <typename T>
__global__ void __launch_bounds__(256) circdiff_bwd_scalar(const T* __restrict__ e, const int32_t* __restrict__ adj,
                                                           const T* __restrict__ dy, float* __restrict__ acc,
                                                           int64_t n_faces, int64_t n_feats) {
    const int64_t total = n_faces * n_feats;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = idx / n_feats, k = idx - i * n_feats;
        const int64_t a0 = adj[3 * i], a1 = adj[3 * i + 1], a2 = adj[3 * i + 2];
        const float x0 = ld1(e + a0 * n_feats + k), x1 = ld1(e + a1 * n_feats + k), x2 = ld1(e + a2 * n_feats + k);
        const float g = ld1(dy + idx);
        const float s01 = sgnf(x0 - x1) * g, s12 = sgnf(x1 - x2) * g, s20 = sgnf(x2 - x0) * g;
        atomicAdd(acc + a0 * n_feats + k, s01 - s20);
        atomicAdd(acc + a1 * n_feats + k, s12 - s01);
        atomicAdd(acc + a2 * n_feats + k, s20 - s12);
    }
}

// Gather backward for edge adjacencies of closed manifold meshes (f in adj[g] <=> g in adj[f],
// once each): the faces whose circular difference involves e[f] are exactly f's neighbours g,
// and f's terms in y[g] are the pairs (f, next) and (prev, f) of g's cyclic list, so
//     de[f] = sum_{g in adj[f]} dy[g] * (sign(e[f] - e[next_g(f)]) + sign(e[f] - e[prev_g(f)]))
// -- every de row has one writer: no atomics, no zeroing pass, deterministic.  The extra reads
// (the neighbours' adjacency rows and second-ring features) are L2 hits on a well-ordered mesh.
template <typename T>
__global__ void __launch_bounds__(256) circdiff_bwd_gather(const T* __restrict__ e, const int32_t* __restrict__ adj,
                                                           const T* __restrict__ dy, T* __restrict__ de,
                                                           int64_t n_faces, int64_t n_feats) {
    constexpr int N = V8<T>::N;
    const int64_t nch = n_feats / N, total = n_faces * nch;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t f = idx / nch, c = (idx - f * nch) * N;
        // three dependent phases, each with all its loads in flight: the neighbour ids, their
        // adjacency rows, then the nine feature chunks (plus e[f])
        int32_t g[3], b[3][3];
#pragma unroll
        for (int j = 0; j < 3; ++j) g[j] = __ldg(adj + 3 * f + j);
#pragma unroll
        for (int j = 0; j < 3; ++j)
#pragma unroll
            for (int r = 0; r < 3; ++r) b[j][r] = __ldg(adj + 3 * (int64_t)g[j] + r);
        float xf[N], xn[3][N], xp[3][N], gg[3][N];
        V8<T>::load(e + f * n_feats + c, xf);
#pragma unroll
        for (int j = 0; j < 3; ++j) {
            const int32_t nxt = b[j][0] == f ? b[j][1] : (b[j][1] == f ? b[j][2] : b[j][0]);
            const int32_t prv = b[j][0] == f ? b[j][2] : (b[j][1] == f ? b[j][0] : b[j][1]);
            V8<T>::load(e + nxt * n_feats + c, xn[j]);
            V8<T>::load(e + prv * n_feats + c, xp[j]);
            V8<T>::load(dy + (int64_t)g[j] * n_feats + c, gg[j]);
        }
        float acc[N];
#pragma unroll
        for (int t = 0; t < N; ++t) {
            float a = 0.f;
#pragma unroll
            for (int j = 0; j < 3; ++j) a = fmaf(gg[j][t], sgnf(xf[t] - xn[j][t]) + sgnf(xf[t] - xp[j][t]), a);
            acc[t] = a;
        }
        V8<T>::store(de + f * n_feats + c, acc);
    }
}

__global__ void __launch_bounds__(256) zero_f32(float4* __restrict__ p, int64_t n4, float* __restrict__ tail, int ntail) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    if (blockIdx.x == 0 && (int)threadIdx.x < ntail) tail[threadIdx.x] = 0.f;
}

__global__ void __launch_bounds__(256) f32_to_bf16(const float* __restrict__ a, __nv_bfloat16* __restrict__ o, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        o[i] = __float2bfloat16_rn(a[i]);
}

int sms() {
    static int n = 0;
    static std::once_flag once;
    std::call_once(once, [] {
        int dev = 0;
        cudaGetDevice(&dev);
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
    });
    return n;
}

unsigned grid_for(int64_t work) {
    const int64_t per = 256, cap = (int64_t)sms() * 8;   // 8 x 256 threads resident per SM
    const int64_t g = (work + per - 1) / per;
    return (unsigned)(g < cap ? (g < 1 ? 1 : g) : cap);
}

template <typename T>
cudaError_t fwd_t(const void* e, const int32_t* adj, void* y, int64_t nf, int64_t F, cudaStream_t st) {
    if (F % V8<T>::N == 0) {
        circdiff_fwd_vec<T><<<grid_for(nf * (F / V8<T>::N)), 256, 0, st>>>((const T*)e, adj, (T*)y, nf, F);
    } else {
        circdiff_fwd_scalar<T><<<grid_for(nf * F), 256, 0, st>>>((const T*)e, adj, (T*)y, nf, F);
    }
    prof_mark(st);
    return cudaGetLastError();
}

template <typename T>
cudaError_t bwd_t(const void* e, const int32_t* adj, const void* dy, float* acc, int64_t nf, int64_t F,
                  cudaStream_t st) {
    const int64_t n = nf * F;
    zero_f32<<<grid_for(n / 4), 256, 0, st>>>((float4*)acc, n / 4, acc + (n / 4) * 4, (int)(n % 4));
    prof_mark(st);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) return err;
    if (F % V8<T>::N == 0) {
        circdiff_bwd_vec<T><<<grid_for(nf * (F / V8<T>::N)), 256, 0, st>>>((const T*)e, adj, (const T*)dy, acc, nf, F);
    } else {
        circdiff_bwd_scalar<T><<<grid_for(n), 256, 0, st>>>((const T*)e, adj, (const T*)dy, acc, nf, F);
    }
    prof_mark(st);
    return cudaGetLastError();
}

bool al16(const void* p) { return ((uintptr_t)p & 15u) == 0; }
struct Sp {
    uintptr_t lo, hi;
};
bool ovl(Sp a, Sp b) { return a.lo < b.hi && b.lo < a.hi; }

}  // namespace
}  // namespace ftw

using namespace ftw;

extern "C" {

size_t ft_subdiv_circdiff_bwd_workspace_bytes(int64_t n_faces, int64_t n_feats, ft_dtype dtype) {
    if (n_faces < 1 || n_feats < 1 || dtype != FT_BF16) return 0;
    return ((size_t)(n_faces * n_feats) * 4 + 255) / 256 * 256;
}

ft_status ft_subdiv_circdiff_fwd(const void* e, const int32_t* adj, void* y, int64_t n_faces, int64_t n_feats,
                                 ft_dtype dtype, void* stream) {
    if (!e || !adj || !y || n_faces < 1 || n_feats < 1) return FT_ERR_INVALID_VALUE;
    if (dtype != FT_F32 && dtype != FT_BF16) return FT_ERR_NOT_SUPPORTED;
    if ((double)n_faces * (double)n_feats >= 1099511627776.0) return FT_ERR_NOT_SUPPORTED;
    if (!al16(e) || !al16(y) || ((uintptr_t)adj & 3u)) return FT_ERR_MISALIGNED;
    const size_t eb = dtype == FT_F32 ? 4 : 2, nb = (size_t)(n_faces * n_feats) * eb;
    const Sp se = {(uintptr_t)e, (uintptr_t)e + nb}, sa = {(uintptr_t)adj, (uintptr_t)adj + (size_t)n_faces * 12},
             sy = {(uintptr_t)y, (uintptr_t)y + nb};
    if (ovl(sy, se) || ovl(sy, sa)) return FT_ERR_INVALID_VALUE;
    prof_reset();
    cudaStream_t st = (cudaStream_t)stream;
    const cudaError_t err = dtype == FT_F32 ? fwd_t<float>(e, adj, y, n_faces, n_feats, st)
                                            : fwd_t<__nv_bfloat16>(e, adj, y, n_faces, n_feats, st);
    return err == cudaSuccess ? FT_OK : cuda_error(err);
}

ft_status ft_subdiv_circdiff_bwd(const void* e, const int32_t* adj, const void* dy, void* de, int64_t n_faces,
                                 int64_t n_feats, ft_dtype dtype, int symmetric, void* workspace,
                                 size_t workspace_bytes, void* stream) {
    if (!e || !adj || !dy || !de || n_faces < 1 || n_feats < 1) return FT_ERR_INVALID_VALUE;
    if (dtype != FT_F32 && dtype != FT_BF16) return FT_ERR_NOT_SUPPORTED;
    if ((double)n_faces * (double)n_feats >= 1099511627776.0) return FT_ERR_NOT_SUPPORTED;
    const size_t need = ft_subdiv_circdiff_bwd_workspace_bytes(n_faces, n_feats, dtype);
    if (workspace_bytes < need || (need > 0 && !workspace)) return FT_ERR_INVALID_VALUE;
    if (!al16(e) || !al16(dy) || !al16(de) || (need > 0 && !al16(workspace)) || ((uintptr_t)adj & 3u))
        return FT_ERR_MISALIGNED;
    const size_t eb = dtype == FT_F32 ? 4 : 2, nb = (size_t)(n_faces * n_feats) * eb;
    const Sp ins[3] = {{(uintptr_t)e, (uintptr_t)e + nb},
                       {(uintptr_t)adj, (uintptr_t)adj + (size_t)n_faces * 12},
                       {(uintptr_t)dy, (uintptr_t)dy + nb}};
    const Sp sd = {(uintptr_t)de, (uintptr_t)de + nb}, sw = {(uintptr_t)workspace, (uintptr_t)workspace + need};
    for (const Sp& x : ins) {
        if (ovl(sd, x)) return FT_ERR_INVALID_VALUE;
        if (need > 0 && ovl(sw, x)) return FT_ERR_INVALID_VALUE;
    }
    if (need > 0 && ovl(sw, sd)) return FT_ERR_INVALID_VALUE;
    prof_reset();
    cudaStream_t st = (cudaStream_t)stream;
    cudaError_t err;
    const int vec = dtype == FT_F32 ? 4 : 8;
    if (symmetric && n_feats % vec == 0) {
        if (dtype == FT_F32)
            circdiff_bwd_gather<float><<<grid_for(n_faces * (n_feats / 4)), 256, 0, st>>>(
                (const float*)e, adj, (const float*)dy, (float*)de, n_faces, n_feats);
        else
            circdiff_bwd_gather<__nv_bfloat16><<<grid_for(n_faces * (n_feats / 8)), 256, 0, st>>>(
                (const __nv_bfloat16*)e, adj, (const __nv_bfloat16*)dy, (__nv_bfloat16*)de, n_faces, n_feats);
        prof_mark(st);
        err = cudaGetLastError();
        return err == cudaSuccess ? FT_OK : cuda_error(err);
    }
    if (dtype == FT_F32) {
        err = bwd_t<float>(e, adj, dy, (float*)de, n_faces, n_feats, st);
    } else {
        err = bwd_t<__nv_bfloat16>(e, adj, dy, (float*)workspace, n_faces, n_feats, st);
        if (err == cudaSuccess) {
            const int64_t n = n_faces * n_feats;
            f32_to_bf16<<<grid_for(n), 256, 0, st>>>((const float*)workspace, (__nv_bfloat16*)de, n);
            prof_mark(st);
            err = cudaGetLastError();
        }
    }
    return err == cudaSuccess ? FT_OK : cuda_error(err);
}

}  // extern "C"
