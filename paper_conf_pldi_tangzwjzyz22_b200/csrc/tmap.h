// tmap.h -- host-side TMA tensor-map encoding for strided residue views.
//
// A (unit, residue r) band problem reads rows i = r + m*dilation of a [units, L, d] bf16
// tensor.  Its TMA view is 3-D: dim0 = d (contiguous), dim1 = m in [0, Lr) with byte
// stride dilation*d*2, dim2 = unit with byte stride L*d*2, based at element r*d.  Rows
// outside [0, Lr) (including negative coordinates for the left halo) are zero-filled on
// load and clipped on store, so the residue view never touches memory outside the tensor
// (SURVEY.md §7 hard part 6).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdint.h>

#include <mutex>

namespace ftw {

inline PFN_cuTensorMapEncodeTiled_v12000 tmap_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q;
        void* p = nullptr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) ==
                cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    });
    return fn;
}

// bf16 residue view with a {64 x box_rows} SWIZZLE_128B box.  Returns false on failure.
inline bool make_residue_map(CUtensorMap* m, const void* tensor, int64_t L, int64_t d,
                             int64_t units, int64_t dil, int64_t r, int box_rows) {
    auto enc = tmap_encoder();
    if (!enc) return false;
    const int64_t Lr = (L - r + dil - 1) / dil;
    const char* base = static_cast<const char*>(tensor) + r * d * 2;
    cuuint64_t dims[3] = {(cuuint64_t)d, (cuuint64_t)Lr, (cuuint64_t)units};
    cuuint64_t strides[2] = {(cuuint64_t)(dil * d * 2), (cuuint64_t)(L * d * 2)};
    cuuint32_t box[3] = {64u, (cuuint32_t)box_rows, 1u};
    cuuint32_t estr[3] = {1u, 1u, 1u};
    CUresult res = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<char*>(base), dims,
                       strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                       CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return res == CUDA_SUCCESS;
}

// fp32 residue view with a {box_cols x box_rows} box, for tc_band32.cu: 32 columns (128-byte rows,
// SWIZZLE_128B) or 16 columns (64-byte rows, SWIZZLE_64B).
inline bool make_residue_map_f32(CUtensorMap* m, const void* tensor, int64_t L, int64_t d,
                                 int64_t units, int64_t dil, int64_t r, int box_rows, int box_cols = 32) {
    auto enc = tmap_encoder();
    if (!enc) return false;
    const int64_t Lr = (L - r + dil - 1) / dil;
    const char* base = static_cast<const char*>(tensor) + r * d * 4;
    cuuint64_t dims[3] = {(cuuint64_t)d, (cuuint64_t)Lr, (cuuint64_t)units};
    cuuint64_t strides[2] = {(cuuint64_t)(dil * d * 4), (cuuint64_t)(L * d * 4)};
    cuuint32_t box[3] = {(cuuint32_t)box_cols, (cuuint32_t)box_rows, 1u};
    cuuint32_t estr[3] = {1u, 1u, 1u};
    CUresult res = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<char*>(base), dims,
                       strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                       box_cols == 16 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B,
                       CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return res == CUDA_SUCCESS;
}

// Residue view of a dS-tape plane (ftw::DsTape): 16-byte granules, element (row R, granule G) at
// float (G grows + R) 4 of the plane.  4-D: {4 floats, residue row m (stride dil granules), unit
// (stride L granules), G (stride grows granules)}; a {4, box_rows, 1, tsw / 4} box lands in shared
// memory as [G][box_rows][4] (box_rows odd multiple of 1 beyond a power of two, so that a warp
// reading one entry per key row hits distinct banks).
inline bool make_residue_map_tape(CUtensorMap* m, const void* plane, int64_t L, int64_t tsw,
                                  int64_t units, int64_t dil, int64_t r, int box_rows, int64_t grows) {
    auto enc = tmap_encoder();
    if (!enc) return false;
    const int64_t Lr = (L - r + dil - 1) / dil;
    const char* base = static_cast<const char*>(plane) + r * 16;
    cuuint64_t dims[4] = {4, (cuuint64_t)Lr, (cuuint64_t)units, (cuuint64_t)(tsw / 4)};
    cuuint64_t strides[3] = {(cuuint64_t)(dil * 16), (cuuint64_t)(L * 16), (cuuint64_t)(grows * 16)};
    cuuint32_t box[4] = {4u, (cuuint32_t)box_rows, 1u, (cuuint32_t)(tsw / 4)};
    cuuint32_t estr[4] = {1u, 1u, 1u, 1u};
    CUresult res = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, const_cast<char*>(base), dims,
                       strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                       CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return res == CUDA_SUCCESS;
}

}  // namespace ftw
