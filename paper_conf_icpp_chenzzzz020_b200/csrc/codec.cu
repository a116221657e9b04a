// codec.cu -- compressed transmission of PAPER.md Sec. 4.4 (Eqs. 10-12): the delta of a
// party's masked message against its previous opening, sent as CSR when >= 75% of it is zero.
//   pass 1  one warp per row counts nonzero deltas (ballot + popc)
//   pass 2  CUB inclusive scan of the counts -> row_ptr
//   pass 3  one warp per row compacts (col, delta) pairs in column order, or writes dense delta
#include <cub/cub.cuh>

#include "engine.h"

namespace psml {

template <typename T>
__global__ void delta_count_kernel(const T *__restrict__ cur, const T *__restrict__ prev, int64_t rows, int64_t cols,
                                   int32_t *__restrict__ cnt) {
    const int lane = threadIdx.x & 31;
    for (int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < rows;
         r += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        int c = 0;
        for (int64_t j = lane; j < cols; j += 32) c += (cur[r * cols + j] - prev[r * cols + j]) != 0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
        if (lane == 0) cnt[r] = c;
    }
}

template <typename T>
__global__ void delta_compact_kernel(const T *__restrict__ cur, const T *__restrict__ prev, int64_t rows, int64_t cols,
                                     const int32_t *__restrict__ row_ptr, int32_t *__restrict__ col_idx,
                                     T *__restrict__ vals) {
    const int lane = threadIdx.x & 31;
    for (int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < rows;
         r += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        int32_t base = row_ptr[r];
        for (int64_t j0 = 0; j0 < cols; j0 += 32) {
            const int64_t j = j0 + lane;
            T d = j < cols ? (T)(cur[r * cols + j] - prev[r * cols + j]) : (T)0;
            unsigned bal = __ballot_sync(0xffffffffu, d != 0);
            if (d != 0) {
                int pos = base + __popc(bal & ((1u << lane) - 1u));
                col_idx[pos] = (int32_t)j;
                vals[pos] = d;
            }
            base += __popc(bal);
        }
    }
}

template <typename T>
__global__ void delta_dense_kernel(const T *__restrict__ cur, const T *__restrict__ prev, int64_t n, T *__restrict__ d) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        d[i] = cur[i] - prev[i];
}

template <typename T>
__global__ void delta_apply_csr_kernel(int64_t rows, int64_t cols, const int32_t *__restrict__ row_ptr,
                                       const int32_t *__restrict__ col_idx, const T *__restrict__ vals,
                                       T *__restrict__ target) {
    const int lane = threadIdx.x & 31;
    for (int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < rows;
         r += ((int64_t)gridDim.x * blockDim.x) >> 5)
        for (int32_t k = row_ptr[r] + lane; k < row_ptr[r + 1]; k += 32) target[r * cols + col_idx[k]] += vals[k];
}

template <typename T>
static psml_status encode_t(Ctx *c, const void *cur, const void *prev, int64_t rows, int64_t cols, int32_t *row_ptr,
                            int32_t *col_idx, void *vals, void *dense, int64_t *nnz_host, int32_t *is_csr_host,
                            cudaStream_t s) {
    size_t temp = 0;
    cub::DeviceScan::InclusiveSum(nullptr, temp, (int32_t *)nullptr, (int32_t *)nullptr, (int)rows, s);
    const size_t cnt_bytes = ((sizeof(int32_t) * rows + 255) / 256) * 256;
    PSML_TRY(c->ensure_ws(cnt_bytes + temp + 256));
    int32_t *cnt = (int32_t *)c->ws;
    void *tmp = (char *)c->ws + cnt_bytes;
    const int blocks = grid_for(rows * 32, 256);
    delta_count_kernel<T><<<blocks, 256, 0, s>>>((const T *)cur, (const T *)prev, rows, cols, cnt);
    PSML_LAUNCH_CHECK();
    PSML_CUDA_TRY(cudaMemsetAsync(row_ptr, 0, sizeof(int32_t), s));
    PSML_CUDA_TRY(cub::DeviceScan::InclusiveSum(tmp, temp, cnt, row_ptr + 1, (int)rows, s));
    int32_t nnz = 0;
    PSML_CUDA_TRY(cudaMemcpyAsync(&nnz, row_ptr + rows, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    PSML_CUDA_TRY(cudaStreamSynchronize(s));
    const int32_t is_csr = (int64_t)4 * nnz <= rows * cols;
    if (is_csr) {
        delta_compact_kernel<T><<<blocks, 256, 0, s>>>((const T *)cur, (const T *)prev, rows, cols, row_ptr, col_idx,
                                                       (T *)vals);
    } else {
        delta_dense_kernel<T><<<grid_for(rows * cols, 256), 256, 0, s>>>((const T *)cur, (const T *)prev, rows * cols,
                                                                         (T *)dense);
    }
    PSML_LAUNCH_CHECK();
    if (nnz_host) *nnz_host = nnz;
    if (is_csr_host) *is_csr_host = is_csr;
    return PSML_OK;
}

}  // namespace psml

using namespace psml;

// ABI definitions: C linkage and default visibility come from include/psml.h.

psml_status psml_delta_encode(psml_ctx ctx, const void *cur, const void *prev, int64_t rows, int64_t cols,
                              int32_t *row_ptr, int32_t *col_idx, void *vals, void *dense, int64_t *nnz_host,
                              int32_t *is_csr_host, psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (rows <= 0 || cols <= 0 || rows * cols >= ((int64_t)1 << 31)) return fail(PSML_ERR_SHAPE, "bad rows/cols");
    PSML_TRY(check_ptrs({cur, prev, row_ptr, col_idx, vals, dense}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64)
        return encode_t<uint64_t>(c, cur, prev, rows, cols, row_ptr, col_idx, vals, dense, nnz_host, is_csr_host, s);
    return encode_t<uint32_t>(c, cur, prev, rows, cols, row_ptr, col_idx, vals, dense, nnz_host, is_csr_host, s);
}

psml_status psml_delta_apply(psml_ctx ctx, int64_t rows, int64_t cols, int32_t is_csr, const int32_t *row_ptr,
                             const int32_t *col_idx, const void *vals, const void *dense, void *target,
                             psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (rows <= 0 || cols <= 0) return fail(PSML_ERR_SHAPE, "bad rows/cols");
    cudaStream_t s = (cudaStream_t)stream;
    if (is_csr) {
        PSML_TRY(check_ptrs({row_ptr, target}));
        const int blocks = grid_for(rows * 32, 256);
        if (c->ring.l == 64)
            delta_apply_csr_kernel<uint64_t><<<blocks, 256, 0, s>>>(rows, cols, row_ptr, col_idx, (const uint64_t *)vals,
                                                                    (uint64_t *)target);
        else
            delta_apply_csr_kernel<uint32_t><<<blocks, 256, 0, s>>>(rows, cols, row_ptr, col_idx, (const uint32_t *)vals,
                                                                    (uint32_t *)target);
    } else {
        PSML_TRY(check_ptrs({dense, target}));
        const int64_t n = rows * cols;
        if (c->ring.l == 64)
            add_kernel<uint64_t><<<grid_for(n, 256), 256, 0, s>>>((const uint64_t *)target, (const uint64_t *)dense, n,
                                                                  (uint64_t *)target);
        else
            add_kernel<uint32_t><<<grid_for(n, 256), 256, 0, s>>>((const uint32_t *)target, (const uint32_t *)dense, n,
                                                                  (uint32_t *)target);
    }
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

