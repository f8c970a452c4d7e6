/* oracle/winattn_ref.h -- fp64 CPU reference for banded (dilated) window attention.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header or constant with the CUDA path (paper_conf_pldi_tangzwjzyz22_b200/csrc).
 *
 * Semantics (Fig. 8, Fig. 10):
 *   N(i) = { j = i + k*dil : |k| <= w, 0 <= j < L }           (readings A1, A2, A4)
 *   S_ij = sum_p q_ip k_jp          (no scale, reading A3; Fig. 8 line "dot[k+w] += Q[j,p]*K[j+k,p]")
 *   m_i = max_j S_ij, l_i = sum_j exp(S_ij - m_i), lse_i = m_i + ln l_i  (Fig. 8 dot_max / dot_norm)
 *   o_i = sum_{j in N(i)} exp(S_ij - lse_i) v_j                 ("attn = softmax(dot)")
 * Backward (PAPER.md:447-453 gradient program; reading A6: P recomputed from lse):
 *   D_i = sum_p g_ip o_ip ; dP_ij = g_i . v_j ; dS_ij = P_ij (dP_ij - D_i)
 *   dq_i = sum_j dS_ij k_j ; dk_j = sum_{i: j in N(i)} dS_ij q_i ; dv_j = sum_i P_ij g_i
 *
 * Layout: every tensor is contiguous [units, L, d] fp64 (units = batch*heads);
 * lse is [units, L].  Computation is fp64, no fast-math, OpenMP over rows.
 */
#ifndef WINATTN_REF_H
#define WINATTN_REF_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Number of threads OpenMP will use (for the cpu_baseline "cores" field). */
int ref_num_threads(void);
void ref_set_num_threads(int n);

/* Forward over all rows.  out [units,L,d], lse [units,L]. */
void ref_winattn_fwd(const double* q, const double* k, const double* v,
                     double* out, double* lse,
                     int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);

/* Backward over all rows, given the forward's out and lse. */
void ref_winattn_bwd(const double* q, const double* k, const double* v,
                     const double* out, const double* lse, const double* dout,
                     double* dq, double* dk, double* dv,
                     int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil);

/* Sampled forward: rows[n] are flat row ids (u*L + i).  Writes out_rows [n,d], lse_rows [n]. */
void ref_winattn_fwd_rows(const double* q, const double* k, const double* v,
                          int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil,
                          const int64_t* rows, int64_t n, double* out_rows, double* lse_rows);

/* Sampled backward: dq/dk/dv of the listed rows, everything (lse, o, D of every
 * neighbour) recomputed from q,k,v,dout in fp64.  Outputs [n,d] each. */
void ref_winattn_bwd_rows(const double* q, const double* k, const double* v, const double* dout,
                          int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil,
                          const int64_t* rows, int64_t n,
                          double* dq_rows, double* dk_rows, double* dv_rows);

#ifdef __cplusplus
}
#endif
#endif
