// api.cu -- the extern "C" boundary of ft_winattn (declared and documented in
// include/ft_winattn.h): argument validation, kernel-family selection, dispatch.
//
// The library is stateless: it never allocates, frees, synchronises or copies between
// host and device.  Every check runs before the first launch, so a failing call leaves
// the outputs untouched.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "ft_winattn.h"
#include <atomic>
#include <mutex>
#include "internal.h"

namespace {

thread_local char g_cuda_msg[256] = "CUDA error";
thread_local void* const* g_prof_events = nullptr;
thread_local int g_prof_n = 0;
thread_local int g_prof_i = 0;
thread_local void* g_trace[3] = {nullptr, nullptr, nullptr};

ft_status cuda_fail(cudaError_t e) {
    snprintf(g_cuda_msg, sizeof(g_cuda_msg), "FT_ERR_CUDA: %s (%s)", cudaGetErrorName(e),
             cudaGetErrorString(e));
    return FT_ERR_CUDA;
}

size_t elt_size(ft_dtype dt) { return dt == FT_F32 ? 4 : 2; }

ft_status check_scalars(int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                        ft_dtype dt) {
    if (B < 1 || H < 1 || L < 1 || d < 1 || w < 0 || dil < 1) return FT_ERR_INVALID_VALUE;
    if (dt != FT_F32 && dt != FT_BF16) return FT_ERR_NOT_SUPPORTED;
    if (d % 16 != 0 || d > 512) return FT_ERR_NOT_SUPPORTED;
    // Tiling uses 31-bit row indices inside a (unit, residue) and a 1-D grid of CTAs.
    if (L > (int64_t)1 << 30 || B * H > (int64_t)1 << 30) return FT_ERR_NOT_SUPPORTED;
    const int64_t nres = dil < L ? dil : L;
    const int64_t tiles = ftw::ceil_div(ftw::ceil_div(L, dil), 32);
    if ((double)B * H * nres * tiles > 2147483647.0) return FT_ERR_NOT_SUPPORTED;
    return FT_OK;
}

bool aligned16(const void* p) { return ((uintptr_t)p & 15u) == 0; }

struct Span {
    uintptr_t lo, hi;
};
bool overlap(Span a, Span b) { return a.lo < b.hi && b.lo < a.hi; }

// Debug / A-B knobs (ft_winattn_debug_set), initialised once from the environment.
std::atomic<int> g_knob[ftw::K_NUM];
std::once_flag g_knob_once;
int env_int(const char* name, int dflt) {
    const char* s = getenv(name);
    return (s && *s) ? atoi(s) : dflt;
}
void knob_init() {
    std::call_once(g_knob_once, [] {
        const char* s = getenv("FT_WINATTN_PATH");
        g_knob[ftw::K_PATH] = (s && !strcmp(s, "simt")) ? 1 : (s && !strcmp(s, "tc")) ? 2 : 0;
        g_knob[ftw::K_PDL] = env_int("FT_WINATTN_PDL", 1) != 0;
        g_knob[ftw::K_NARROW] = env_int("FT_WINATTN_NARROW", 1) != 0;
        g_knob[ftw::K_WIDE] = env_int("FT_WINATTN_WIDE", 1) != 0;
        g_knob[ftw::K_SIDE] = env_int("FT_WINATTN_MIXED_SERIAL", 0) != 1;
        g_knob[ftw::K_DSTAPE] = env_int("FT_WINATTN_DSTAPE", 1) < 0 ? 0 : (env_int("FT_WINATTN_DSTAPE", 1) > 2 ? 2 : env_int("FT_WINATTN_DSTAPE", 1));
    });
}
thread_local bool g_handoff = false;   // inside ft_winattn_fwd_bwd

int forced_path() { return ftw::knob(ftw::K_PATH); }

ft_status choose_path(int is_bwd, int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil, ft_dtype dt,
                      int* path) {
    const bool tc_ok = dt == FT_BF16 ? (is_bwd ? ftw::tc_bwd_supported(units, L, d, w, dil)
                                               : ftw::tc_fwd_supported(units, L, d, w, dil))
                                     : ftw::tc32_supported(units, L, d, w, dil);
    const int f = forced_path();
    if (f == 1) { *path = FT_PATH_SIMT; return FT_OK; }
    if (f == 2) {
        if (!tc_ok) return FT_ERR_NOT_SUPPORTED;
        *path = FT_PATH_TC;
        return FT_OK;
    }
    *path = tc_ok ? FT_PATH_TC : FT_PATH_SIMT;
    return FT_OK;
}

// Backward workspace: D_i = dout_i . out_i per row (fp32), and -- for shapes the fp32 tensor-core
// kernels serve -- the dS tape between the dQ and dK/dV kernels (ftw::DsTape): one flag word per
// row and two fp32 planes of tsw floats per row.  Each region is 256-byte aligned; a slice of rows
// [row0, ...) (per-head-dilation calls) uses the same offsets into every region.
struct WsLayout {
    size_t dB = 0, fB = 0, pB = 0;
    int tsw = 0;
    int64_t rows = 0;
    bool tape = false;
    size_t total() const { return dB + fB + 2 * pB; }
};
size_t round256(size_t x) { return (x + 255) / 256 * 256; }
WsLayout ws_layout(int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, ft_dtype dt) {
    WsLayout l;
    const size_t rows = (size_t)(B * H * L);
    l.rows = (int64_t)rows;
    l.dB = round256(rows * sizeof(float));
    l.tape = (ftw::dstape_pays(d, dt) || ftw::knob(ftw::K_DSTAPE) == 2) && (dt == FT_F32 ? (w < L ? w : L) <= 32 && ftw::tc32_supported(B * H, L, d, w, dil)
                                                   : ftw::tc_band_dstape_ok(B * H, L, d, w, dil));
    if (l.tape) {
        l.tsw = ftw::dstape_tsw(w < L ? w : L);
        l.fB = round256(rows * sizeof(uint32_t));
        l.pB = round256(rows * (size_t)l.tsw * sizeof(float));
    }
    return l;
}

}  // namespace

namespace ftw {
int knob(Knob k) {
    knob_init();
    return g_knob[k].load(std::memory_order_relaxed);
}
bool call_handoff() { return g_handoff; }
ft_status cuda_error(cudaError_t e) { return cuda_fail(e); }
void prof_reset() { g_prof_i = 0; }
void* trace_buffer(int mode) { return (mode >= 0 && mode < 3) ? g_trace[mode] : nullptr; }
void prof_mark(cudaStream_t st) {
    if (g_prof_events && g_prof_i < g_prof_n)
        cudaEventRecord(static_cast<cudaEvent_t>(g_prof_events[g_prof_i]), st);
    ++g_prof_i;
}
}  // namespace ftw

extern "C" {

ft_status ft_winattn_debug_trace(int kernel_mode, void* device_buffer) {
    if (kernel_mode < 0 || kernel_mode > 2) return FT_ERR_INVALID_VALUE;
    g_trace[kernel_mode] = device_buffer;
    return FT_OK;
}

ft_status ft_winattn_profile_events(void* const* events, int n) {
    g_prof_events = n > 0 ? events : nullptr;
    g_prof_n = n > 0 ? n : 0;
    g_prof_i = 0;
    return FT_OK;
}

int ft_winattn_abi_version(void) { return FT_WINATTN_ABI_VERSION; }

ft_status ft_winattn_debug_set(int which, int value) {
    if (which < 0 || which >= ftw::K_NUM) return FT_ERR_INVALID_VALUE;
    const int vmax = (which == ftw::K_PATH || which == ftw::K_DSTAPE) ? 2 : 1;
    if (value < 0 || value > vmax) return FT_ERR_INVALID_VALUE;
    knob_init();
    g_knob[which].store(value, std::memory_order_relaxed);
    return FT_OK;
}

int ft_winattn_debug_get(int which) {
    if (which < 0 || which >= ftw::K_NUM) return -1;
    return ftw::knob((ftw::Knob)which);
}

const char* ft_status_str(ft_status s) {
    switch (s) {
        case FT_OK: return "FT_OK";
        case FT_ERR_INVALID_VALUE: return "FT_ERR_INVALID_VALUE: invalid argument";
        case FT_ERR_NOT_SUPPORTED: return "FT_ERR_NOT_SUPPORTED: unsupported dtype / head dim / size";
        case FT_ERR_MISALIGNED: return "FT_ERR_MISALIGNED: tensor pointer not 16-byte aligned";
        case FT_ERR_CUDA: return g_cuda_msg;
    }
    return "unknown ft_status";
}

size_t ft_winattn_bwd_workspace_bytes(int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                                      int64_t w, int64_t dilation, ft_dtype dtype) {
    if (check_scalars(batch, heads, seq_len, d, w, dilation, dtype) != FT_OK) return 0;
    return ws_layout(batch, heads, seq_len, d, w, dilation, dtype).total();
}

ft_status ft_winattn_plan(int is_bwd, int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                          int64_t w, int64_t dilation, ft_dtype dtype, int* path,
                          int* num_launches) {
    ft_status s = check_scalars(batch, heads, seq_len, d, w, dilation, dtype);
    if (s != FT_OK) return s;
    int p = 0;
    s = choose_path(is_bwd, batch * heads, seq_len, d, w, dilation, dtype, &p);
    if (s != FT_OK) return s;
    int n;
    if (p == FT_PATH_TC && dtype == FT_F32)
        n = is_bwd ? ftw::tc32_bwd_launches(seq_len, w, dilation) : ftw::tc32_fwd_launches(seq_len, w, dilation);
    else if (p == FT_PATH_TC)
        n = is_bwd ? ftw::tc_bwd_launches(batch * heads, seq_len, d, w, dilation)
                   : ftw::tc_fwd_launches(seq_len, d, w, dilation);
    else
        n = is_bwd ? ftw::simt_bwd_launches() : ftw::simt_fwd_launches();
    if (path) *path = p;
    if (num_launches) *num_launches = n;
    return FT_OK;
}

}  // extern "C"

namespace {

// Argument checks of the forward (before any launch).
ft_status check_fwd(const void* q, const void* k, const void* v, void* out, float* lse, int64_t batch,
                    int64_t heads, int64_t seq_len, int64_t d, int64_t w, int64_t dilation, ft_dtype dtype) {
    if (!q || !k || !v || !out || !lse) return FT_ERR_INVALID_VALUE;
    ft_status s = check_scalars(batch, heads, seq_len, d, w, dilation, dtype);
    if (s != FT_OK) return s;
    if (!aligned16(q) || !aligned16(k) || !aligned16(v) || !aligned16(out) || !aligned16(lse))
        return FT_ERR_MISALIGNED;
    const size_t nb = (size_t)(batch * heads * seq_len * d) * elt_size(dtype);
    const size_t lb = (size_t)(batch * heads * seq_len) * sizeof(float);
    const Span in[3] = {{(uintptr_t)q, (uintptr_t)q + nb}, {(uintptr_t)k, (uintptr_t)k + nb},
                        {(uintptr_t)v, (uintptr_t)v + nb}};
    const Span so = {(uintptr_t)out, (uintptr_t)out + nb}, sl = {(uintptr_t)lse, (uintptr_t)lse + lb};
    if (overlap(so, sl)) return FT_ERR_INVALID_VALUE;
    for (const Span& x : in)
        if (overlap(x, so) || overlap(x, sl)) return FT_ERR_INVALID_VALUE;
    int path = 0;
    return choose_path(0, batch * heads, seq_len, d, w, dilation, dtype, &path);
}

// Errors this call's launches report must be this call's: a non-sticky error another library
// left pending on the calling thread (e.g. on PyTorch's autograd worker thread) would otherwise be
// returned by the cudaGetLastError after our first launch.  Sticky errors persist and are reported.
void clear_stale_error() { (void)cudaGetLastError(); }

// The TMA descriptors are encoded with the driver API (cuTensorMapEncodeTiled), which needs the
// device's context current on the calling thread.  A thread whose runtime calls so far did not
// bind it -- PyTorch's autograd worker thread running a backward -- would get every encode
// rejected; cudaSetDevice binds the primary context of the caller's current device.
void bind_context() {
    thread_local int bound = -1;
    int dev = 0;
    if (cudaGetDevice(&dev) == cudaSuccess && dev != bound) {
        cudaSetDevice(dev);
        bound = dev;
    }
}

// Enqueue a validated forward.
ft_status run_fwd(const void* q, const void* k, const void* v, void* out, float* lse, int64_t batch,
                  int64_t heads, int64_t seq_len, int64_t d, int64_t w, int64_t dilation, ft_dtype dtype,
                  void* stream) {
    int path = 0;
    ft_status s = choose_path(0, batch * heads, seq_len, d, w, dilation, dtype, &path);
    if (s != FT_OK) return s;
    cudaStream_t st = (cudaStream_t)stream;
    cudaError_t e;
    bind_context();
    clear_stale_error();
    if (path == FT_PATH_TC && dtype == FT_F32) {
        int n = 0;
        e = ftw::tc32_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, st, &n);
    } else if (path == FT_PATH_TC) {
        int n = 0;
        e = ftw::tc_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, st, &n);
    } else {
        e = ftw::simt_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, dtype, st);
    }
    return e == cudaSuccess ? FT_OK : cuda_fail(e);
}

ft_status check_bwd(const void* q, const void* k, const void* v, const void* out, const float* lse,
                    const void* dout, void* dq, void* dk, void* dv, int64_t batch, int64_t heads,
                    int64_t seq_len, int64_t d, int64_t w, int64_t dilation, ft_dtype dtype,
                    void* workspace, size_t workspace_bytes) {
    if (!q || !k || !v || !out || !lse || !dout || !dq || !dk || !dv) return FT_ERR_INVALID_VALUE;
    ft_status s = check_scalars(batch, heads, seq_len, d, w, dilation, dtype);
    if (s != FT_OK) return s;
    const size_t need = ft_winattn_bwd_workspace_bytes(batch, heads, seq_len, d, w, dilation, dtype);
    if (workspace_bytes < need || (need > 0 && !workspace)) return FT_ERR_INVALID_VALUE;
    const void* ptrs[] = {q, k, v, out, lse, dout, dq, dk, dv, workspace};
    for (const void* p : ptrs)
        if (p && !aligned16(p)) return FT_ERR_MISALIGNED;
    const size_t nb = (size_t)(batch * heads * seq_len * d) * elt_size(dtype);
    const size_t lb = (size_t)(batch * heads * seq_len) * sizeof(float);
    const Span ins[6] = {{(uintptr_t)q, (uintptr_t)q + nb},     {(uintptr_t)k, (uintptr_t)k + nb},
                         {(uintptr_t)v, (uintptr_t)v + nb},     {(uintptr_t)out, (uintptr_t)out + nb},
                         {(uintptr_t)lse, (uintptr_t)lse + lb}, {(uintptr_t)dout, (uintptr_t)dout + nb}};
    const Span outs[4] = {{(uintptr_t)dq, (uintptr_t)dq + nb},
                          {(uintptr_t)dk, (uintptr_t)dk + nb},
                          {(uintptr_t)dv, (uintptr_t)dv + nb},
                          {(uintptr_t)workspace, (uintptr_t)workspace + need}};
    for (int a = 0; a < 4; ++a) {
        if (outs[a].hi == outs[a].lo) continue;
        for (const Span& x : ins)
            if (overlap(outs[a], x)) return FT_ERR_INVALID_VALUE;
        for (int b = a + 1; b < 4; ++b)
            if (outs[b].hi != outs[b].lo && overlap(outs[a], outs[b])) return FT_ERR_INVALID_VALUE;
    }
    int path = 0;
    return choose_path(1, batch * heads, seq_len, d, w, dilation, dtype, &path);
}

// Enqueue a validated backward.  ws: the workspace of a call whose layout is `lay`; this backward
// covers its rows [row0, row0 + batch * heads * seq_len).
ft_status run_bwd(const void* q, const void* k, const void* v, const void* out, const float* lse,
                  const void* dout, void* dq, void* dk, void* dv, int64_t batch, int64_t heads,
                  int64_t seq_len, int64_t d, int64_t w, int64_t dilation, ft_dtype dtype,
                  void* ws, const WsLayout& lay, int64_t row0, void* stream) {
    int path = 0;
    ft_status s = choose_path(1, batch * heads, seq_len, d, w, dilation, dtype, &path);
    if (s != FT_OK) return s;
    cudaStream_t st = (cudaStream_t)stream;
    char* base = static_cast<char*>(ws);
    float* Dws = base ? (float*)(base + row0 * 4) : nullptr;
    // the dS tape regions of these rows (tensor-core families check that they can use it)
    ftw::DsTape tape;
    const bool use_tape = lay.tape && base && ftw::knob(ftw::K_DSTAPE);
    if (use_tape) {
        tape.flags = (uint32_t*)(base + lay.dB + row0 * 4);
        tape.P = (float*)(base + lay.dB + lay.fB + (size_t)row0 * 16);   // granule-major planes
        tape.S = (float*)(base + lay.dB + lay.fB + lay.pB + (size_t)row0 * 16);
        tape.tsw = lay.tsw;
        tape.grows = lay.rows;
    }
    cudaError_t e;
    bind_context();
    clear_stale_error();
    if (path == FT_PATH_TC && dtype == FT_F32) {
        int n = 0;
        const bool ok = ftw::tc32_supported(batch * heads, seq_len, d, w, dilation);
        e = ftw::tc32_bwd(q, k, v, out, lse, dout, dq, dk, dv, Dws, use_tape && ok ? &tape : nullptr, batch, heads,
                          seq_len, d, w, dilation, st, &n);
    } else if (path == FT_PATH_TC) {
        int n = 0;
        const bool ok = ftw::tc_band_dstape_ok(batch * heads, seq_len, d, w, dilation);
        e = ftw::tc_bwd(q, k, v, out, lse, dout, dq, dk, dv, Dws, batch, heads, seq_len, d, w,
                        dilation, st, &n, use_tape && ok ? &tape : nullptr);
    } else {
        e = ftw::simt_bwd(q, k, v, out, lse, dout, dq, dk, dv, Dws, batch, heads, seq_len, d, w,
                          dilation, dtype, st);
    }
    return e == cudaSuccess ? FT_OK : cuda_fail(e);
}

// Head groups of a per-head-dilation call: (first head, head count, dilation) per group, and
// whether the groups are contiguous over the whole batch (batch == 1 or a single group).
struct Group {
    int64_t h0, nh, dil;
};
int mixed_groups(int64_t heads, int64_t dilation, int64_t hd, Group (&g)[2]) {
    int n = 0;
    if (hd > 0) g[n++] = {0, hd, dilation};
    if (hd < heads) g[n++] = {hd, heads - hd, 1};
    return n;
}

// The slices of a mixed call are independent: they alternate between the caller's stream and
// one library-owned side stream per device (fork / join through events, so the call stays
// asynchronous and capturable in a CUDA graph). Each slice's persistent kernels then take the
// SMs the other slice's last CTAs leave, instead of running their own partial last waves one
// after the other. FT_WINATTN_MIXED_SERIAL=1 keeps every slice on the caller's stream.
struct Side {
    cudaStream_t s = nullptr;
    cudaEvent_t fork = nullptr, join = nullptr;
    bool ok = false;
};
// One side stream and fork / join event pair per host thread and device: two threads calling
// concurrently never share the events (a record on one thread's stream could otherwise be
// overwritten by the other's before the wait is enqueued).  They live for the thread.
Side* side_stream() {
    if (!ftw::knob(ftw::K_SIDE)) return nullptr;
    constexpr int MAXDEV = 64;
    struct PerThread {
        Side sides[MAXDEV];
        bool tried[MAXDEV] = {};
        ~PerThread() {
            for (Side& x : sides) {
                if (x.fork) cudaEventDestroy(x.fork);
                if (x.join) cudaEventDestroy(x.join);
                if (x.s) cudaStreamDestroy(x.s);
            }
        }
    };
    thread_local PerThread pt;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= MAXDEV) return nullptr;
    Side& x = pt.sides[dev];
    if (!pt.tried[dev]) {
        pt.tried[dev] = true;
        x.ok = cudaStreamCreateWithFlags(&x.s, cudaStreamNonBlocking) == cudaSuccess &&
               cudaEventCreateWithFlags(&x.fork, cudaEventDisableTiming) == cudaSuccess &&
               cudaEventCreateWithFlags(&x.join, cudaEventDisableTiming) == cudaSuccess;
    }
    return x.ok ? &x : nullptr;
}
// stream of slice i (fork before the first slice, join after the last)
struct ForkJoin {
    Side* side;
    cudaStream_t main;
    bool forked = false;
    ForkJoin(cudaStream_t st, int nslices) : side(nslices > 1 ? side_stream() : nullptr), main(st) {
        stream_of(1);   // fork now, before any slice is enqueued on the caller's stream
    }
    cudaStream_t stream_of(int i) {
        if (!side || i % 2 == 0) return main;
        if (!forked) {   // called before slice 0 is enqueued: the side stream must not wait for it
            cudaEventRecord(side->fork, main);
            cudaStreamWaitEvent(side->s, side->fork, 0);
            forked = true;
        }
        return side->s;
    }
    ft_status finish(ft_status s) {
        if (forked) {
            cudaEventRecord(side->join, side->s);
            cudaStreamWaitEvent(main, side->join, 0);
            const cudaError_t e = cudaGetLastError();
            if (s == FT_OK && e != cudaSuccess) return cuda_fail(e);
        }
        return s;
    }
};

}  // namespace

extern "C" {

ft_status ft_winattn_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                         int64_t batch, int64_t heads, int64_t seq_len, int64_t d, int64_t w,
                         int64_t dilation, ft_dtype dtype, void* stream) {
    ft_status s = check_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, dtype);
    if (s != FT_OK) return s;
    ftw::prof_reset();
    return run_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, dtype, stream);
}

ft_status ft_winattn_bwd(const void* q, const void* k, const void* v, const void* out,
                         const float* lse, const void* dout, void* dq, void* dk, void* dv,
                         int64_t batch, int64_t heads, int64_t seq_len, int64_t d, int64_t w,
                         int64_t dilation, ft_dtype dtype, void* workspace,
                         size_t workspace_bytes, void* stream) {
    ft_status s = check_bwd(q, k, v, out, lse, dout, dq, dk, dv, batch, heads, seq_len, d, w, dilation,
                            dtype, workspace, workspace_bytes);
    if (s != FT_OK) return s;
    ftw::prof_reset();
    return run_bwd(q, k, v, out, lse, dout, dq, dk, dv, batch, heads, seq_len, d, w, dilation, dtype,
                   workspace, ws_layout(batch, heads, seq_len, d, w, dilation, dtype), 0, stream);
}

ft_status ft_winattn_fwd_mixed(const void* q, const void* k, const void* v, void* out, float* lse,
                               int64_t batch, int64_t heads, int64_t seq_len, int64_t d, int64_t w,
                               int64_t dilation, int64_t dilated_heads, ft_dtype dtype, void* stream) {
    if (dilated_heads < 0 || heads < 1 || dilated_heads > heads) return FT_ERR_INVALID_VALUE;
    // every group's configuration is validated before anything is enqueued
    ft_status s = check_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, dtype);
    if (s != FT_OK) return s;
    s = check_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, 1, dtype);
    if (s != FT_OK) return s;
    Group g[2];
    const int ng = mixed_groups(heads, dilation, dilated_heads, g);
    const size_t e = elt_size(dtype);
    const int64_t nb = ng == 1 ? 1 : batch;   // one group spans the whole batch contiguously
    ftw::prof_reset();
    ForkJoin fj((cudaStream_t)stream, (int)(nb * ng));
    for (int64_t b = 0; b < nb; ++b) {
        for (int i = 0; i < ng; ++i) {
            const int64_t B1 = ng == 1 ? batch : 1, H1 = ng == 1 ? heads : g[i].nh;
            const int64_t row0 = (b * heads + g[i].h0) * seq_len;   // first (unit, row) of the slice
            const size_t off = (size_t)row0 * d * e;
            s = run_fwd((const char*)q + off, (const char*)k + off, (const char*)v + off, (char*)out + off,
                        lse + row0, B1, H1, seq_len, d, w, g[i].dil, dtype, fj.stream_of((int)(b * ng + i)));
            if (s != FT_OK) return fj.finish(s);
        }
    }
    return fj.finish(FT_OK);
}

ft_status ft_winattn_bwd_mixed(const void* q, const void* k, const void* v, const void* out,
                               const float* lse, const void* dout, void* dq, void* dk, void* dv,
                               int64_t batch, int64_t heads, int64_t seq_len, int64_t d, int64_t w,
                               int64_t dilation, int64_t dilated_heads, ft_dtype dtype, void* workspace,
                               size_t workspace_bytes, void* stream) {
    if (dilated_heads < 0 || heads < 1 || dilated_heads > heads) return FT_ERR_INVALID_VALUE;
    ft_status s = check_bwd(q, k, v, out, lse, dout, dq, dk, dv, batch, heads, seq_len, d, w, dilation,
                            dtype, workspace, workspace_bytes);
    if (s != FT_OK) return s;
    s = check_bwd(q, k, v, out, lse, dout, dq, dk, dv, batch, heads, seq_len, d, w, 1, dtype, workspace,
                  workspace_bytes);
    if (s != FT_OK) return s;
    Group g[2];
    const int ng = mixed_groups(heads, dilation, dilated_heads, g);
    const size_t e = elt_size(dtype);
    const int64_t nb = ng == 1 ? 1 : batch;
    const WsLayout lay = ws_layout(batch, heads, seq_len, d, w, dilation, dtype);
    ftw::prof_reset();
    ForkJoin fj((cudaStream_t)stream, (int)(nb * ng));
    for (int64_t b = 0; b < nb; ++b) {
        for (int i = 0; i < ng; ++i) {
            const int64_t B1 = ng == 1 ? batch : 1, H1 = ng == 1 ? heads : g[i].nh;
            const int64_t row0 = (b * heads + g[i].h0) * seq_len;
            const size_t off = (size_t)row0 * d * e;
            // every workspace region is per row: the slice's rows start at row0
            s = run_bwd((const char*)q + off, (const char*)k + off, (const char*)v + off, (const char*)out + off,
                        lse + row0, (const char*)dout + off, (char*)dq + off, (char*)dk + off, (char*)dv + off,
                        B1, H1, seq_len, d, w, g[i].dil, dtype, workspace, lay, row0,
                        fj.stream_of((int)(b * ng + i)));
            if (s != FT_OK) return fj.finish(s);
        }
    }
    return fj.finish(FT_OK);
}

size_t ft_winattn_tape_bytes(int64_t batch, int64_t heads, int64_t seq_len, int64_t w) {
    if (batch < 1 || heads < 1 || seq_len < 1 || w < 0) return 0;
    const int64_t wc = w < seq_len ? w : seq_len;
    return (size_t)(batch * heads * seq_len) * (size_t)(2 * wc + 1) * sizeof(float);
}

}  // extern "C"

namespace {
// Kernel family of a tape call (the same rule for the forward and the backward): the band
// tensor-core kernels for bf16 where they apply, else the CUDA-core kernels.
ft_status tape_path(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil, ft_dtype dt, int* path) {
    const bool tc_ok = dt == FT_BF16 && ftw::tc_tape_supported(units, L, d, w, dil);
    const int f = forced_path();
    if (f == 2 && !tc_ok) return FT_ERR_NOT_SUPPORTED;
    *path = (f != 1 && tc_ok) ? FT_PATH_TC : FT_PATH_SIMT;
    return FT_OK;
}
}  // namespace

extern "C" {

ft_status ft_winattn_fwd_tape(const void* q, const void* k, const void* v, void* out, float* lse,
                              void* tape, int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                              int64_t w, int64_t dilation, ft_dtype dtype, void* stream) {
    ft_status s = check_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, dtype);
    if (s != FT_OK) return s;
    if (!tape) return FT_ERR_INVALID_VALUE;
    if (!aligned16(tape)) return FT_ERR_MISALIGNED;
    int path = 0;
    s = tape_path(batch * heads, seq_len, d, w, dilation, dtype, &path);
    if (s != FT_OK) return s;
    ftw::prof_reset();
    bind_context();
    clear_stale_error();
    int n = 0;
    const cudaError_t e =
        path == FT_PATH_TC
            ? ftw::tc_tape_fwd(q, k, v, out, lse, tape, batch, heads, seq_len, d, w, dilation, (cudaStream_t)stream, &n)
            : ftw::simt_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, dtype, (cudaStream_t)stream,
                            static_cast<float*>(tape));
    return e == cudaSuccess ? FT_OK : cuda_fail(e);
}

ft_status ft_winattn_bwd_tape(const void* q, const void* k, const void* v, const void* out,
                              const float* lse, const void* tape, const void* dout, void* dq, void* dk,
                              void* dv, int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                              int64_t w, int64_t dilation, ft_dtype dtype, void* workspace,
                              size_t workspace_bytes, void* stream) {
    ft_status s = check_bwd(q, k, v, out, lse, dout, dq, dk, dv, batch, heads, seq_len, d, w, dilation,
                            dtype, workspace, workspace_bytes);
    if (s != FT_OK) return s;
    if (!tape) return FT_ERR_INVALID_VALUE;
    if (!aligned16(tape)) return FT_ERR_MISALIGNED;
    int path = 0;
    s = tape_path(batch * heads, seq_len, d, w, dilation, dtype, &path);
    if (s != FT_OK) return s;
    ftw::prof_reset();
    bind_context();
    clear_stale_error();
    int n = 0;
    const cudaError_t e =
        path == FT_PATH_TC
            ? ftw::tc_tape_bwd(q, k, v, lse, tape, dout, dq, dk, dv, (float*)workspace, batch, heads, seq_len, d, w,
                               dilation, (cudaStream_t)stream, &n)
            : ftw::simt_bwd(q, k, v, out, lse, dout, dq, dk, dv, (float*)workspace, batch, heads, seq_len, d, w,
                            dilation, dtype, (cudaStream_t)stream, static_cast<const float*>(tape));
    return e == cudaSuccess ? FT_OK : cuda_fail(e);
}

ft_status ft_winattn_fwd_bwd(const void* q, const void* k, const void* v, const void* dout, void* out,
                             float* lse, void* dq, void* dk, void* dv, int64_t batch, int64_t heads,
                             int64_t seq_len, int64_t d, int64_t w, int64_t dilation, ft_dtype dtype,
                             void* workspace, size_t workspace_bytes, void* stream) {
    if (!dout || !dq || !dk || !dv) return FT_ERR_INVALID_VALUE;
    ft_status s = check_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, dtype);
    if (s != FT_OK) return s;
    s = check_bwd(q, k, v, out, lse, dout, dq, dk, dv, batch, heads, seq_len, d, w, dilation, dtype,
                  workspace, workspace_bytes);
    if (s != FT_OK) return s;
    // out and lse are outputs here: dout must not overlap them either (check_bwd treats them as
    // inputs, so it allowed dout == out)
    const size_t nb = (size_t)(batch * heads * seq_len * d) * elt_size(dtype);
    const size_t lb = (size_t)(batch * heads * seq_len) * sizeof(float);
    const Span sdo = {(uintptr_t)dout, (uintptr_t)dout + nb};
    if (overlap(sdo, {(uintptr_t)out, (uintptr_t)out + nb}) || overlap(sdo, {(uintptr_t)lse, (uintptr_t)lse + lb}))
        return FT_ERR_INVALID_VALUE;
    ftw::prof_reset();
    g_handoff = true;
    s = run_fwd(q, k, v, out, lse, batch, heads, seq_len, d, w, dilation, dtype, stream);
    if (s == FT_OK)
        s = run_bwd(q, k, v, out, lse, dout, dq, dk, dv, batch, heads, seq_len, d, w, dilation, dtype,
                    workspace, ws_layout(batch, heads, seq_len, d, w, dilation, dtype), 0, stream);
    g_handoff = false;
    return s;
}

}  // extern "C"
