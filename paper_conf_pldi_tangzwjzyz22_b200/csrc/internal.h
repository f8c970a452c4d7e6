// internal.h -- shared launch-side declarations of the ft_winattn library (not part of the ABI).
//
// Geometry: every (batch, head) unit u and dilation residue r (0 <= r < min(dilation, L))
// forms an independent dilation-1 band problem on the strided rows i = r + m*dilation,
// m in [0, Lr), Lr = ceil((L - r) / dilation)  (reading A4; the oracle pins the
// equivalence in tests/test_oracle.py::test_dilation_is_residue_decomposition).
// Kernels tile m ("residue space"), so dilation costs only an address stride.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "ft_winattn.h"

namespace ftw {

struct Geo {
    int64_t L;        // seq_len
    int64_t d;        // head dim
    int64_t w;        // one-sided window, clamped to L (|k| >= L never hits the sequence)
    int64_t dil;      // dilation
    int64_t units;    // batch * heads
    int64_t nres;     // min(dil, L) non-empty residues
    int64_t tiles;    // tiles per residue = ceil(ceil(L / dil) / T)
    int T;            // rows per tile
};

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

inline Geo make_geo(int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, int T) {
    Geo g;
    g.L = L;
    g.d = d;
    g.w = w < L ? w : L;
    g.dil = dil;
    g.units = B * H;
    g.nres = dil < L ? dil : L;
    g.tiles = ceil_div(ceil_div(L, dil), T);
    g.T = T;
    return g;
}

inline int64_t geo_blocks(const Geo& g) { return g.units * g.nres * g.tiles; }

// The dS tape between the two backward kernels (selective materialization),
// fp32 (tc_band32.cu) and bf16 band (tc_band.cu) tensor-core kernels: the dQ kernel stores every
// band entry's P_ij and dS_ij and publishes flags[first row of each 128-row tile] = 1; the dK/dV
// kernel then reads its P^T / dS^T from the tape instead of recomputing S^T and dP^T.
// Plane layout (fp32): entry e = j - i + w of row i sits at offset o = (m & 3) + e of that row
// (m = i's row in its residue, so the dQ kernel's 16-byte stores are aligned), and the row's
// offsets are grouped in 16-byte granules G = o / 4 stored granule-major: float (G grows + i) 4
// + o % 4 -- a warp's stores of one granule index cover consecutive rows.  Workspace: api.cu.
struct DsTape {
    uint32_t* flags;   // one word per row (only tile-first rows used)
    float* P;          // [tsw / 4][grows][4]
    float* S;          // [tsw / 4][grows][4]
    int tsw;           // floats per row, a multiple of 4
    int64_t grows;     // granule stride in rows (the rows of the whole call)
};
inline int dstape_tsw(int64_t wc) { return (int)((2 * wc + 4 + 3) / 4 * 4); }
// The tape costs 2 tsw floats per row written and read; it replaces the dK/dV kernel's score phase
// (K, V, Q, dO slices, two GEMMs; in fp32 also their operand conversion).  Measured
// (tools/tape_ablation.py): fp32 1.14-1.33x faster at d >= 256; bf16 0.91-0.95x at
// d = 128, even at d = 256, 1.05-1.13x at d = 512.
inline bool dstape_pays(int64_t d, ft_dtype dt) { return dt == FT_F32 ? d >= 256 : d > 256; }

// SIMT (CUDA-core) kernels -- simt.cu
// tape (optional): the raw band scores s_ij, fp32 [B*H*L][2w+1] (w clamped to L); the forward
// writes it and the backward reads it instead of recomputing q_i . k_j (ft_winattn_*_tape).
cudaError_t simt_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                     int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                     ft_dtype dt, cudaStream_t st, float* tape = nullptr);
cudaError_t simt_bwd(const void* q, const void* k, const void* v, const void* out,
                     const float* lse, const void* dout, void* dq, void* dk, void* dv,
                     float* Dws, int64_t B, int64_t H, int64_t L, int64_t d, int64_t w,
                     int64_t dil, ft_dtype dt, cudaStream_t st, const float* tape = nullptr);
int simt_fwd_launches();
int simt_bwd_launches();

// tcgen05 / TMEM kernels -- tc_fwd.cu, tc_bwd.cu (bf16 only)
bool tc_fwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
bool tc_bwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
cudaError_t tc_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                   int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                   cudaStream_t st, int* launches);
cudaError_t tc_bwd(const void* q, const void* k, const void* v, const void* out,
                   const float* lse, const void* dout, void* dq, void* dk, void* dv,
                   float* Dws, int64_t B, int64_t H, int64_t L, int64_t d, int64_t w,
                   int64_t dil, cudaStream_t st, int* launches, const DsTape* ds = nullptr);
// the bf16 backward of this shape runs on the band kernels, which can use the dS tape
bool tc_band_dstape_ok(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
int tc_fwd_launches(int64_t L, int64_t d, int64_t w, int64_t dil);
int tc_bwd_launches(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);

// wide-window tensor-core kernels -- tc_chunk.cu (used when 128 + 2w > 256)
bool tc_chunk_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
cudaError_t tc_chunk_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                         int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                         cudaStream_t st, int* launches);
cudaError_t tc_chunk_bwd(const void* q, const void* k, const void* v, const float* lse,
                         const void* dout, void* dq, void* dk, void* dv, float* Dws, int64_t B,
                         int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st,
                         int* launches);
int tc_chunk_launches(int64_t L, int64_t dil);

// wide-window forward, two-pass with partial accumulators -- tc_wide.cu
bool tc_wide_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
cudaError_t tc_wide_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                        int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                        cudaStream_t st, int* launches);
int tc_wide_launches(int64_t L, int64_t dil);
// wide-window backward, TMEM region rotation, three MMA issuers -- tc_wide_bwd.cu
bool tc_wide_bwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
cudaError_t tc_wide_bwd(const void* q, const void* k, const void* v, const void* out,
                        const float* lse, const void* dout, void* dq, void* dk, void* dv, float* Dws,
                        int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                        cudaStream_t st, int* launches);

// d = 64, w <= 32 forward with two ping-pong softmax warpgroups -- tc_narrow.cu
bool tc_narrow_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
cudaError_t tc_narrow_fwd(const void* q, const void* k, const void* v, void* out, float* lse,
                          int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil,
                          cudaStream_t st, int* launches);
int tc_narrow_launches(int64_t L, int64_t dil);
bool tc_narrow_bwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
cudaError_t tc_narrow_bwd(const void* q, const void* k, const void* v, const float* lse,
                          const void* dout, void* dq, void* dk, void* dv, float* Dws, int64_t B,
                          int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st,
                          int* launches);

// fp32 tensor-core kernels (bf16 hi / lo planes, 3 products) for w <= 32, d % 64 == 0 --
// tc_band32.cu
bool tc32_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
int tc32_fwd_launches(int64_t L, int64_t w, int64_t dil);
int tc32_bwd_launches(int64_t L, int64_t w, int64_t dil);
cudaError_t tc32_fwd(const void* q, const void* k, const void* v, void* out, float* lse, int64_t B, int64_t H,
                     int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st, int* launches);
cudaError_t tc32_bwd(const void* q, const void* k, const void* v, const void* out, const float* lse, const void* dout, void* dq,
                     void* dk, void* dv, float* Dws, const DsTape* tape, int64_t B, int64_t H, int64_t L,
                     int64_t d, int64_t w, int64_t dil, cudaStream_t st, int* launches);

// Score tape on the band kernels (bf16, w <= 64, d % 64 == 0): the forward also writes the band
// scores (fp32 [rows][2w + 1], the CUDA-core kernels' format), the backward reads them and skips
// the score GEMM -- tc_band.cu
bool tc_tape_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);
cudaError_t tc_tape_fwd(const void* q, const void* k, const void* v, void* out, float* lse, void* tape,
                        int64_t B, int64_t H, int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st,
                        int* launches);
cudaError_t tc_tape_bwd(const void* q, const void* k, const void* v, const float* lse, const void* tape,
                        const void* dout, void* dq, void* dk, void* dv, float* Dws, int64_t B, int64_t H,
                        int64_t L, int64_t d, int64_t w, int64_t dil, cudaStream_t st, int* launches);

// FT_ERR_CUDA with the CUDA error text recorded for ft_status_str (api.cu)
ft_status cuda_error(cudaError_t e);

// Debug / A-B knobs (ft_winattn_debug_set; initialised once from the environment, see
// include/ft_winattn.h).  They pick among kernels that compute the same result.
enum Knob {
    K_PATH = 0,     // 0 auto, 1 CUDA-core (SIMT) kernels, 2 tensor-core kernels (FT_WINATTN_PATH=simt|tc)
    K_PDL = 1,      // 1: programmatic dependent launch inside a call; 0: plain stream order (FT_WINATTN_PDL=0)
    K_NARROW = 2,   // 1: d = 64, w <= 32 narrow kernels; 0: band kernels (FT_WINATTN_NARROW=0)
    K_WIDE = 3,     // 1: w > 64 wide kernels; 0: the chunked fallback kernels (FT_WINATTN_WIDE=0)
    K_SIDE = 4,     // 1: per-head-dilation calls use a side stream; 0: serial (FT_WINATTN_MIXED_SERIAL=1)
    K_DSTAPE = 5,   // 1: tensor-core backward hands P / dS over on a tape where it pays (d >= 256), 2: wherever
                    // the kernels can, 0: recompute (FT_WINATTN_DSTAPE=0|1|2)
    K_NUM = 6
};
int knob(Knob k);

// True while ft_winattn_fwd_bwd enqueues its forward and backward back to back on one stream
// (the forward -> dQ-kernel lse hand-off is allowed only then).
bool call_handoff();
// The forward marks its lse rows and triggers, and the dQ kernel (PDL) polls them, only inside
// ft_winattn_fwd_bwd; the dQ -> dK/dV kernel D hand-off (always inside one call) needs PDL on.
inline bool lsepoll_enabled() { return call_handoff() && knob(K_PDL) != 0; }
inline bool dpoll_enabled() { return knob(K_PDL) != 0; }

// Profiling hook (ft_winattn_profile_events): record the next caller event after a launch.
void prof_reset();
void* trace_buffer(int kernel_mode);   // ft_winattn_debug_trace target for a kernel mode, or null
void prof_mark(cudaStream_t st);

}  // namespace ftw
