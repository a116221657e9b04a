// gemm_tc.cu -- placeholder until the tcgen05 limb GEMM lands: every entry reports
// PSML_ERR_UNSUPPORTED so callers take the CUDA-core path.
#include "engine.h"

namespace psml {

bool tc_available() { return false; }
size_t tc_ring_gemm_ws_bytes(int, int64_t, int64_t, int64_t) { return 0; }
psml_status tc_ring_gemm_plain(int, const void *, const void *, int64_t, int64_t, int64_t, void *, void *, size_t,
                               cudaStream_t) {
    return PSML_ERR_UNSUPPORTED;
}
template <typename T>
psml_status tc_beaver_matmul(Ctx *, const T *const[2], const T *const[2], const T *const[2], const T *const[2],
                             const T *const[2], int64_t, int64_t, int64_t, int, int, T *const[2], cudaStream_t) {
    return PSML_ERR_UNSUPPORTED;
}
template psml_status tc_beaver_matmul<uint64_t>(Ctx *, const uint64_t *const[2], const uint64_t *const[2],
                                                const uint64_t *const[2], const uint64_t *const[2],
                                                const uint64_t *const[2], int64_t, int64_t, int64_t, int, int,
                                                uint64_t *const[2], cudaStream_t);
template psml_status tc_beaver_matmul<uint32_t>(Ctx *, const uint32_t *const[2], const uint32_t *const[2],
                                                const uint32_t *const[2], const uint32_t *const[2],
                                                const uint32_t *const[2], int64_t, int64_t, int64_t, int, int,
                                                uint32_t *const[2], cudaStream_t);
}  // namespace psml
