// tc_bwd.cu -- tcgen05/TMEM tensor-core backward (placeholder until the kernel lands: the
// backward is routed to the SIMT kernels, which tc_bwd_supported() makes explicit).
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace ftw {

bool tc_bwd_supported(int64_t units, int64_t L, int64_t d, int64_t w, int64_t dil) {
    (void)units; (void)L; (void)d; (void)w; (void)dil;
    return false;
}

int tc_bwd_launches(int64_t L, int64_t d, int64_t w, int64_t dil) {
    (void)L; (void)d; (void)w; (void)dil;
    return 0;
}

cudaError_t tc_bwd(const void*, const void*, const void*, const void*, const float*, const void*,
                   void*, void*, void*, float*, int64_t, int64_t, int64_t, int64_t, int64_t,
                   int64_t, cudaStream_t, int*) {
    return cudaErrorNotSupported;
}

}  // namespace ftw
