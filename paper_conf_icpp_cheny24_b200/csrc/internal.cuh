// internal.cuh -- shared declarations of the libspaden.so implementation.
// Product code only: nothing here is shared with oracle/.
#pragma once

#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <stdint.h>
#include <string>

#include "spaden.h"

// ------------------------------------------------------------------ handle
struct spaden_matrix_s {
    int64_t m = 0, n = 0, nnz = 0;
    int64_t Bnrow = 0, Bnnz = 0;
    spaden_dtype_t storage = SPADEN_R_32F;
    int device = 0;

    // bitBSR (§4.2): owned device arrays (each padded to a 16-byte multiple + 16)
    int32_t *blk_rowptr = nullptr;   // [Bnrow+1]
    int32_t *blk_col = nullptr;      // [Bnnz]
    uint64_t *bitmap = nullptr;      // [Bnnz]
    int32_t *blk_offset = nullptr;   // [Bnnz+1]
    void *values = nullptr;          // [nnz]

    // SpMV schedule (aux)
    int64_t aux_bytes = 0;
    int64_t n_tiles = 0;

    // host-API staging buffers (lazily allocated)
    float *stage_x = nullptr;
    float *stage_y = nullptr;
};

namespace spaden {

// ---------------------------------------------------------------- errors
void set_error(const std::string &msg);
spaden_status_t cuda_status(cudaError_t e, const char *what);

#define SPADEN_CUDA_TRY(expr)                                          \
    do {                                                               \
        cudaError_t e_ = (expr);                                       \
        if (e_ != cudaSuccess) return ::spaden::cuda_status(e_, #expr); \
    } while (0)

// ------------------------------------------------- device error flag bits
enum : uint32_t {
    ERRF_ROWPTR = 1u,     // rowptr not monotone / out of [0, nnz] / ends wrong
    ERRF_RANGE = 2u,      // colidx outside [0, n)
    ERRF_UNSORTED = 4u,   // colidx not strictly ascending in a row
};

// ------------------------------------------------------------ SpMV schedule
// A tile is a run of whole block-rows [br_begin, br_end) processed by one warp
// group, or (long block-rows) one chunk [b_begin, b_end) of a single block-row
// whose partial row sums go to a carry slot and are combined by a fix-up pass.
struct Tile {
    int32_t br_begin;
    int32_t br_end;
};

using Matrix = ::spaden_matrix_s;

// converter (convert.cu)
spaden_status_t convert_csr(int64_t m, int64_t n, int64_t nnz, const int32_t *rowptr,
                            const int32_t *colidx, const void *values, spaden_dtype_t vdt,
                            spaden_dtype_t sdt, cudaStream_t stream, Matrix *A);

// SpMV (spmv.cu)
spaden_status_t spmv_launch(const Matrix &A, float alpha, const float *x, float beta, float *y,
                            cudaStream_t stream);

// exclusive scan of int32 (scan.cu): out[i] = sum_{j<i} in[j], out[count] = total.
// `in` and `out` may alias.  tmp must hold scan_tmp_ints(count) int32.
size_t scan_tmp_ints(int64_t count);
cudaError_t exclusive_scan_i32(const int32_t *in, int32_t *out, int64_t count, int32_t *tmp,
                               cudaStream_t stream);

// device helpers
__device__ __forceinline__ int warp_min_i32(int v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

__device__ __forceinline__ int warp_excl_scan_i32(int v, int lane, int *total) {
    int s = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int t = __shfl_up_sync(0xffffffffu, s, o);
        if (lane >= o) s += t;
    }
    *total = __shfl_sync(0xffffffffu, s, 31);
    return s - v;
}

inline size_t pad16(size_t bytes) { return ((bytes + 15) / 16) * 16 + 16; }

}  // namespace spaden
