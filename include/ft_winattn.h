/* include/ft_winattn.h -- C ABI of the B200 (sm_100a) banded window-attention library.
 *
 * The operation is the hot path of FreeTensor's Longformer workload (PAPER.md:58
 * "computes correlations for pairs of nearby tokens that have a distance no greater
 * than a threshold"; Fig. 5 caption PAPER.md:172 "The range j-w to j+w marks the
 * sliding window"; the inlined program Fig. 8).  Each query row i
 * of every (batch, head) unit attends to the window
 *
 *     N(i) = { j = i + k*dilation : |k| <= w, 0 <= j < seq_len }
 *
 * (inclusive window, reading A1; out-of-sequence keys excluded, reading A2;
 * dilation as in Longformer [8], reading A4).  No logit scale is applied
 * (Fig. 8 "dot[k+w] += Q[j,p] * K[j+k,p]", reading A3): callers pre-scale q.
 *
 *   forward:
 *     s_ij  = sum_p q_ip k_jp,  lse_i = log sum_{j in N(i)} exp(s_ij),
 *     out_i = sum_{j in N(i)} exp(s_ij - lse_i) v_j
 *   backward  (the gradient program of PAPER.md:447-453, P recomputed from lse as in
 *              PAPER.md:489-497 "selective materialization", reading A6):
 *     P_ij = exp(s_ij - lse_i),  D_i = sum_j P_ij (dout_i . v_j)  (= dout_i . out_i exactly;
 *     the kernels form it from the recomputed band, reading R1),  dS_ij = P_ij (dout_i . v_j - D_i)
 *     dq_i = sum_j dS_ij k_j,  dk_j = sum_i dS_ij q_i,  dv_j = sum_i P_ij dout_i
 *
 * Layout (reading A9): q, k, v, out, dout, dq, dk, dv are contiguous row-major
 * [batch, heads, seq_len, d] in the storage dtype; lse is contiguous fp32
 * [batch, heads, seq_len] (natural log).  All pointers are DEVICE pointers.
 *
 * Ownership: the caller owns every buffer (including the workspace).  The library
 * never allocates, frees, synchronises or copies host<->device.  Outputs are fully
 * overwritten, never accumulated into.
 *
 * Async: work is enqueued on `stream` (a cudaStream_t passed as void*; NULL = legacy
 * default stream) and the call returns immediately.  Stream order is preserved for the
 * caller: every kernel of a call starts after all work enqueued on `stream` before the call
 * has completed, and work enqueued after the call starts after it.  Inside ONE call the
 * library may overlap its own kernels (programmatic dependent launch: ft_winattn_bwd's dK/dV
 * kernel reads D rows as its dQ kernel stores them; ft_winattn_fwd_bwd's dQ kernel reads lse
 * rows as its forward stores them), never across calls.  No kernel of a call reads an input
 * or writes any memory before the previous work on `stream` is complete.
 *
 * Errors: all argument checks run before any launch; on failure nothing is launched
 * and the outputs are untouched.
 *   FT_ERR_INVALID_VALUE  null pointer; batch, heads, seq_len or d < 1; w < 0;
 *                         dilation < 1; an output buffer overlapping an input or
 *                         another output; workspace smaller than required.
 *   FT_ERR_MISALIGNED     a tensor pointer not 16-byte aligned.
 *   FT_ERR_NOT_SUPPORTED  d not a multiple of 16 or d > 512; unknown dtype;
 *                         seq_len * d or batch * heads too large for 31-bit tiling.
 *   FT_ERR_CUDA           a CUDA launch failed (cudaGetLastError after the launch).
 * Domain: any w >= 0 (w >= seq_len is full attention), any dilation >= 1.
 * Thread safety: stateless; safe to call concurrently from several host threads.
 */
#ifndef FT_WINATTN_H
#define FT_WINATTN_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define FT_WINATTN_ABI_VERSION 2

typedef enum {
    FT_OK = 0,
    FT_ERR_INVALID_VALUE = 1,
    FT_ERR_NOT_SUPPORTED = 2,
    FT_ERR_MISALIGNED = 3,
    FT_ERR_CUDA = 4
} ft_status;

typedef enum { FT_F32 = 0, FT_BF16 = 1 } ft_dtype;

/* Kernel family chosen for a call (reported by ft_winattn_plan; tests may force one with
 * ft_winattn_debug_set(FT_KNOB_PATH, ...)). */
typedef enum {
    FT_PATH_SIMT = 0,   /* CUDA-core FMA kernels (fp32 math), any dtype / d / w      */
    FT_PATH_TC = 1      /* tcgen05/TMEM tensor-core kernels: bf16 (any w, d % 64 == 0,
                           d <= 512 for w <= 64; d in {64, 128} above), and fp32 as bf16
                           hi / lo planes with 3 products (w <= 32, d % 64 == 0)        */
} ft_path;

/* Forward.  q, k, v: [B,H,L,d] dtype (inputs).  out: [B,H,L,d] dtype, lse: [B,H,L]
 * fp32 (outputs).  w: one-sided window (keys per side), dilation: key stride. */
ft_status ft_winattn_fwd(const void* q, const void* k, const void* v,
                         void* out, float* lse,
                         int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                         int64_t w, int64_t dilation, ft_dtype dtype, void* stream);

/* Backward.  q, k, v, out (the forward's output), lse (the forward's lse) and dout
 * are inputs; dq, dk, dv ([B,H,L,d] dtype) are overwritten.  workspace must hold at
 * least ft_winattn_bwd_workspace_bytes(...) bytes of device memory (16-byte aligned;
 * may be NULL when that size is 0); its contents on entry are ignored. */
ft_status ft_winattn_bwd(const void* q, const void* k, const void* v,
                         const void* out, const float* lse, const void* dout,
                         void* dq, void* dk, void* dv,
                         int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                         int64_t w, int64_t dilation, ft_dtype dtype,
                         void* workspace, size_t workspace_bytes, void* stream);

/* Forward then backward in one call, for the recompute / activation-checkpointing pattern
 * (the gradient program of PAPER.md:449, 523 as one unit): computes out and lse exactly as
 * ft_winattn_fwd and dq, dk, dv exactly as ft_winattn_bwd with that out and lse.  Inputs q, k,
 * v, dout; outputs out, lse, dq, dk, dv, workspace (ft_winattn_bwd_workspace_bytes).  Because
 * both halves are enqueued by the library, its dQ kernel may start while the forward drains and
 * read each lse row as the forward stores it (the forward marks its lse rows with the bit
 * pattern 0xFFFFFFFF first; DESIGN.md §7 "lse hand-off").  Errors: those of ft_winattn_fwd and
 * ft_winattn_bwd, plus FT_ERR_INVALID_VALUE when dout overlaps out or lse. */
ft_status ft_winattn_fwd_bwd(const void* q, const void* k, const void* v, const void* dout,
                             void* out, float* lse, void* dq, void* dk, void* dv,
                             int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                             int64_t w, int64_t dilation, ft_dtype dtype,
                             void* workspace, size_t workspace_bytes, void* stream);

/* Per-head dilation (Longformer [8] and the FreeTensor artefact's mixed heads, PAPER.md:625;
 * SURVEY.md §8(f) item 1, reading A4): heads [0, dilated_heads) of every batch element attend
 * with `dilation`, heads [dilated_heads, heads) with dilation 1.  Arguments, layout, ownership
 * and errors are those of ft_winattn_fwd / ft_winattn_bwd, plus FT_ERR_INVALID_VALUE when
 * dilated_heads is outside [0, heads].  The workspace size is ft_winattn_bwd_workspace_bytes
 * of the same shape.  One launch set per head group when batch == 1 or one group is empty,
 * else one per group and batch element.  The slices are independent and alternate between
 * `stream` and a side stream the library creates per host thread and device (with two events): the side
 * stream waits on an event recorded on `stream` before the first slice, and `stream` waits
 * on the side stream's last slice, so the call stays asynchronous, ordered with respect to
 * `stream` and capturable in a CUDA graph.  The side stream and events belong to the calling
 * host thread (one set per thread and device).  FT_KNOB_SIDE = 0 keeps every slice on
 * `stream`. */
ft_status ft_winattn_fwd_mixed(const void* q, const void* k, const void* v,
                               void* out, float* lse,
                               int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                               int64_t w, int64_t dilation, int64_t dilated_heads, ft_dtype dtype,
                               void* stream);
ft_status ft_winattn_bwd_mixed(const void* q, const void* k, const void* v,
                               const void* out, const float* lse, const void* dout,
                               void* dq, void* dk, void* dv,
                               int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                               int64_t w, int64_t dilation, int64_t dilated_heads, ft_dtype dtype,
                               void* workspace, size_t workspace_bytes, void* stream);

/* Tape vs recompute (the selective-materialization trade-off of PAPER.md:489-497 / Fig. 18,
 * SURVEY.md §8(f) item 2).  The plain entry points save only lse and RECOMPUTE the band
 * scores in the backward.  The _tape variants MATERIALIZE them instead (Fig. 8's `dot`): the
 * forward also writes tape, fp32 [batch*heads*seq_len][2*min(w, seq_len)+1] -- entry (row i, k + w)
 * holds s_ij for key j = i + k*dilation (entries of keys outside the sequence are left unwritten)
 * -- and the backward reads it instead of running the score GEMM q_i . k_j, computing
 * P = exp(s - lse) from it.  bf16 calls the band tensor-core kernels can serve (w <= 64,
 * d % 64 == 0, d <= 512) run on them; the rest on the CUDA-core kernels; forward and backward
 * pick the same family for the same arguments (and FT_KNOB_PATH).  tape must hold
 * ft_winattn_tape_bytes(...) bytes of device memory, 16-byte aligned, not overlapping any other
 * argument (not checked).  Errors: those of ft_winattn_fwd / ft_winattn_bwd, plus
 * FT_ERR_INVALID_VALUE for a NULL tape and FT_ERR_MISALIGNED for a misaligned one. */
size_t    ft_winattn_tape_bytes(int64_t batch, int64_t heads, int64_t seq_len, int64_t w);
ft_status ft_winattn_fwd_tape(const void* q, const void* k, const void* v,
                              void* out, float* lse, void* tape,
                              int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                              int64_t w, int64_t dilation, ft_dtype dtype, void* stream);
ft_status ft_winattn_bwd_tape(const void* q, const void* k, const void* v,
                              const void* out, const float* lse, const void* tape, const void* dout,
                              void* dq, void* dk, void* dv,
                              int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                              int64_t w, int64_t dilation, ft_dtype dtype,
                              void* workspace, size_t workspace_bytes, void* stream);

/* Device workspace the backward needs: the per-row D_i (fp32), and, for shapes the tensor-core
 * kernels serve with the dS tape (fp32 with d >= 256; bf16 band kernels with d > 256; or any they
 * can serve while FT_KNOB_DSTAPE = 2), one flag word per row and two fp32 planes of
 * 4 ceil((2w + 4) / 4) floats per row (P and dS of every band entry, written by the dQ kernel and
 * read by the dK/dV kernel of the same call: selective materialization).  The
 * size depends on FT_KNOB_DSTAPE; query it with the knobs the call will run under. */
size_t ft_winattn_bwd_workspace_bytes(int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                                      int64_t w, int64_t dilation, ft_dtype dtype);

/* Describe what a call would launch, without launching: the kernel family and the
 * number of kernel launches of the forward (is_bwd = 0) or backward (is_bwd = 1).
 * Returns the same validation status the real call would for its scalar arguments. */
ft_status ft_winattn_plan(int is_bwd, int64_t batch, int64_t heads, int64_t seq_len, int64_t d,
                          int64_t w, int64_t dilation, ft_dtype dtype,
                          int* path, int* num_launches);

/* Profiling hook (off by default).  After ft_winattn_profile_events(evs, n) with n > 0,
 * every subsequent fwd/bwd call on the calling host thread records evs[i] (cudaEvent_t
 * handles passed as void*, created by the caller) on its stream right after its i-th
 * kernel launch, for i < n, so a caller can time each kernel on the launching stream.
 * ft_winattn_profile_events(NULL, 0) turns it off.  Always returns FT_OK. */
ft_status ft_winattn_profile_events(void* const* events, int n);

/* Debug trace (off by default): while device_buffer is non-NULL, tensor-core kernels of
 * the given mode (0 = forward, 1 = backward dq, 2 = backward dk/dv) launched from the
 * calling host thread write globaltimer stamps of their pipeline phases into it:
 * uint64 [gridDim.x][8 tiles][48 slots] (slot meanings documented in csrc/tc_band.cu and
 * csrc/tc_wide.cu).  The buffer must hold 148*8*48*8 bytes per SM-sized grid.  Profiling
 * only. */
ft_status ft_winattn_debug_trace(int kernel_mode, void* device_buffer);

/* Debug / A-B knobs (tests and profiling only; process-wide, initialised once from the
 * environment variable named in brackets).  Every setting computes the same result; they select
 * among kernel families or launch schedules:
 *   0 FT_KNOB_PATH    0 auto, 1 CUDA-core kernels, 2 tensor-core kernels (FT_ERR_NOT_SUPPORTED
 *                     from calls they cannot serve)              [FT_WINATTN_PATH=simt|tc]
 *   1 FT_KNOB_PDL     1 programmatic dependent launch inside a call, 0 plain stream order
 *                                                                [FT_WINATTN_PDL=0]
 *   2 FT_KNOB_NARROW  1 the d = 64, w <= 32 kernels, 0 the band kernels  [FT_WINATTN_NARROW=0]
 *   3 FT_KNOB_WIDE    1 the w > 64 wide kernels, 0 the chunked fallback  [FT_WINATTN_WIDE=0]
 *   4 FT_KNOB_SIDE    1 per-head-dilation calls use a side stream, 0 serial
 *                                                                [FT_WINATTN_MIXED_SERIAL=1]
 *   5 FT_KNOB_DSTAPE  1 the tensor-core dK/dV kernel (fp32; bf16 band kernels) reads P and dS
 *                     from the dQ kernel's tape in the workspace where that pays (d >= 256),
 *                     2 wherever the kernels can, 0 it recomputes them  [FT_WINATTN_DSTAPE]
 * ft_winattn_debug_set returns FT_ERR_INVALID_VALUE for an unknown knob or value;
 * ft_winattn_debug_get returns the current value (-1 for an unknown knob). */
enum { FT_KNOB_PATH = 0, FT_KNOB_PDL = 1, FT_KNOB_NARROW = 2, FT_KNOB_WIDE = 3, FT_KNOB_SIDE = 4,
       FT_KNOB_DSTAPE = 5 };
ft_status ft_winattn_debug_set(int knob, int value);
int       ft_winattn_debug_get(int knob);

/* Human-readable text for a status (static storage, never NULL).  For FT_ERR_CUDA it
 * includes the CUDA error string of the last failure on the calling thread. */
const char* ft_status_str(ft_status s);

/* ABI version of the loaded library (FT_WINATTN_ABI_VERSION it was built with). */
int ft_winattn_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* FT_WINATTN_H */
