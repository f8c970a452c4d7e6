/* include/ft_subdiv.h -- C ABI of SubdivNet's circular difference on B200 (sm_100a), the second
 * workload of SURVEY.md §8(f) item 4.
 *
 * Operation (Section 2.2, Figure 2, lines 89-119): for each central face i of a
 * triangle mesh with edge-adjacent faces adj[i][0..2] (an adjacency array) and per-face feature
 * vectors e[f][0..n_feats),
 *
 *     y[i][k] = sum_{j=0..2} | e[adj[i][j]][k] - e[adj[i][(j+1) % 3]][k] |
 *
 * computed in one kernel that gathers the three neighbour rows on demand -- no adj_feat
 * [n_faces, 3, n_feats] intermediate, the redundancy of the operator-based Fig. 2(b)/(c).
 * Backward (for the loss sum(y * dy); subgradient sign(0) = 0, reading S1 of DESIGN.md):
 *
 *     de[a][k] += s,  de[b][k] -= s,  s = sign(e[a][k] - e[b][k]) * dy[i][k]
 *     for every face i and pair (a, b) = (adj[i][j], adj[i][(j+1) % 3]).
 *
 * Layout: e, y, dy, de are contiguous row-major [n_faces, n_feats] in the storage dtype
 * (FT_F32 or FT_BF16; arithmetic in fp32); adj is contiguous int32 [n_faces, 3] with values in
 * [0, n_faces) (not checked; out-of-range indices are undefined behaviour).  All pointers are
 * DEVICE pointers.  Ownership, async and threading rules are those of ft_winattn.h: the caller
 * owns every buffer (including the workspace), work is enqueued on `stream`, and outputs are
 * fully overwritten.
 *
 * Backward, two algorithms:
 *   symmetric = 1: adj is the edge adjacency of a closed manifold triangle mesh (f is in adj[g]
 *     exactly when g is in adj[f], once each; not checked).  Then the faces whose y involves
 *     e[f] are f's own neighbours, and de[f] is GATHERED from them: one writer per row, no
 *     atomics, deterministic, no workspace (requires n_feats % 4 == 0 for FT_F32, % 8 for
 *     FT_BF16; otherwise the scatter below runs).
 *   symmetric = 0: any adjacency array.  Contributions are SCATTERED into an fp32 accumulator
 *     (de itself for FT_F32, the workspace for FT_BF16) with atomic adds, so the summation order,
 *     and for fp32 the last bit, may vary between runs.
 *
 * Errors (checked before any launch; on failure nothing is launched):
 *   FT_ERR_INVALID_VALUE  null pointer, n_faces or n_feats < 1, an output overlapping an input,
 *                         workspace smaller than required.
 *   FT_ERR_MISALIGNED     e, y, dy, de or the workspace not 16-byte aligned, adj not 4-byte aligned.
 *   FT_ERR_NOT_SUPPORTED  unknown dtype, or n_faces * n_feats >= 2^40.
 *   FT_ERR_CUDA           a launch failed.
 */
#ifndef FT_SUBDIV_H
#define FT_SUBDIV_H

#include <stddef.h>
#include <stdint.h>

#include "ft_winattn.h"

#ifdef __cplusplus
extern "C" {
#endif

ft_status ft_subdiv_circdiff_fwd(const void* e, const int32_t* adj, void* y, int64_t n_faces,
                                 int64_t n_feats, ft_dtype dtype, void* stream);

/* fp32 accumulation buffer the backward needs: n_faces * n_feats * 4 bytes for FT_BF16, 0 for
 * FT_F32 (de itself accumulates). */
size_t ft_subdiv_circdiff_bwd_workspace_bytes(int64_t n_faces, int64_t n_feats, ft_dtype dtype);

ft_status ft_subdiv_circdiff_bwd(const void* e, const int32_t* adj, const void* dy, void* de,
                                 int64_t n_faces, int64_t n_feats, ft_dtype dtype, int symmetric,
                                 void* workspace, size_t workspace_bytes, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* FT_SUBDIV_H */
