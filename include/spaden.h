/*
 * spaden.h -- C ABI of the B200-native bitBSR SpMV library (libspaden.so).
 *
 * Method: Y. Chen, J. X. Yu, "Bitmap-Based Sparse Matrix-Vector Multiplication
 * with Tensor Cores" (Spaden), ICPP '24.  Passages are cited as P:L<n> =
 * line n of PAPER.md, with the section / algorithm they fall in.
 *
 * The library computes y = alpha * A x + beta * y for a sparse A that it first
 * converts from CSR (§2.1) into bitBSR (§4.2, Fig. 4):
 *   - A is cut into 8x8 blocks; Bnrow = ceil(m/8) block-rows.
 *   - The non-empty blocks of a block-row are listed CSR-style
 *     in ascending block column:            blk_rowptr int32[Bnrow+1],
 *                                           blk_col    int32[Bnnz].
 *   - Each block is one 64-bit occupancy bitmap, bit 8*(r%8)+(c%8),
 *     LSB = top-left, MSB = bottom-right, row 0 in the low byte:
 *                                           bitmap     uint64[Bnnz].
 *   - Per-block nonzero counts, exclusive-scanned:
 *                                           blk_offset int32[Bnnz+1] (last = nnz).
 *   - The nonzeros, "stored consecutively" block after block and in
 *     ascending bit order inside a block:   values     fp32|fp16[nnz].
 *   The value of set bit `bit` of block b is values[blk_offset[b] +
 *   popcount(bitmap[b] & ((1<<bit)-1))] (reading R1 of Alg. 2).
 *
 * Conventions for every entry point:
 *   - Pointers named d_* are DEVICE pointers on the device that is current
 *     when the call is made; h_* are HOST pointers (pinned recommended).
 *     Inputs are borrowed: the caller keeps them alive until the stream work
 *     that uses them has completed.  No entry point takes ownership of caller
 *     memory.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *     All device work is stream-ordered on it.
 *   - Every call returns a spaden_status_t; nothing aborts or throws across the
 *     ABI.  On failure a thread-local message is available from
 *     spaden_last_error_message() and output handles are set to NULL.
 *   - Indices are int32 (nnz < 2^31, m, n < 2^31).
 */
#ifndef SPADEN_H_
#define SPADEN_H_

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define SPADEN_API __attribute__((visibility("default")))
#else
#define SPADEN_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    SPADEN_OK = 0,
    SPADEN_ERR_INVALID_ARGUMENT = 1,     /* bad sizes, NULL pointers, host pointer where device expected,
                                            rowptr[0] != 0, rowptr[m] != nnz, non-monotone rowptr */
    SPADEN_ERR_INDEX_OUT_OF_RANGE = 2,   /* some colidx outside [0, n)                          */
    SPADEN_ERR_UNSORTED_OR_DUPLICATE = 3,/* colidx not strictly ascending within a row           */
    SPADEN_ERR_UNSUPPORTED = 4,          /* dtype combination / size limit not supported         */
    SPADEN_ERR_OUT_OF_MEMORY = 5,        /* device allocation failed                             */
    SPADEN_ERR_CUDA = 6                  /* any other CUDA runtime error                         */
} spaden_status_t;

typedef enum {
    SPADEN_R_32F = 0,   /* IEEE binary32 */
    SPADEN_R_16F = 1    /* IEEE binary16 */
} spaden_dtype_t;

/* Opaque handle: owns the device bitBSR arrays of one matrix on one device. */
typedef struct spaden_matrix_s *spaden_matrix_t;

typedef struct {
    int64_t m, n, nnz;          /* matrix shape and stored entries                        */
    int64_t Bnrow, Bnnz;        /* block-rows ceil(m/8), non-empty 8x8 blocks              */
    int32_t storage_dtype;      /* spaden_dtype_t of values[]                              */
    int32_t device;             /* CUDA device ordinal the arrays live on                 */
    int64_t format_bytes;       /* 4(Bnrow+1) + 4Bnnz + 8Bnnz + 4(Bnnz+1) + s_v*nnz: the
                                   bitBSR footprint (2.85 B/nnz with fp16 values) */
    int64_t aux_bytes;          /* extra device bytes (SpMV work schedule, padding)       */
    int64_t n_tiles;            /* SpMV work tiles in the schedule                         */
    int64_t n_long;             /* block-rows too large for a tile (processed in chunks)  */
    int64_t residual_nnz;       /* entries held in the CSR residual (hybrid mode, else 0);
                                   format_bytes then also counts 4(m+1) + (4+s_v)*residual_nnz */
    int32_t residual_max_popc;  /* hybrid threshold t in effect (0 = pure bitBSR; the value the
                                   automatic choice took when opts asked for -1)              */
    int32_t residual_parts;     /* column parts of the residual (x > 64 MB), 0 when pure      */
} spaden_info_t;

typedef struct {                /* borrowed device views; valid until spaden_free         */
    const int32_t  *blk_rowptr; /* [Bnrow+1] */
    const int32_t  *blk_col;    /* [Bnnz]    */
    const uint64_t *bitmap;     /* [Bnnz]    */
    const int32_t  *blk_offset; /* [Bnnz+1]  */
    const void     *values;     /* [nnz - residual_nnz] of storage_dtype */
    const int32_t  *res_rowptr; /* [m+1] hybrid residual CSR (NULL when residual_nnz == 0, or when
                                   the residual is split into column parts because 4n > 64 MB) */
    const int32_t  *res_colidx; /* [residual_nnz] */
    const void     *res_values; /* [residual_nnz] of storage_dtype */
} spaden_arrays_t;

/* Conversion options (spaden_convert_csr_to_bitmap_ex).  Zero-initialise. */
typedef struct {
    int32_t struct_size;        /* sizeof(spaden_convert_opts_t)                          */
    int32_t residual_max_popc;  /* hybrid format: blocks holding at
                                   most this many entries are stored as a CSR residual
                                   instead of bitBSR blocks (0 = pure bitBSR, max 64;
                                   -1 = automatic: 4 when the mean block fill nnz/Bnnz
                                   is below 8, else 0)                                     */
    float   auto_mean_fill;     /* > 0: the mean block fill nnz/Bnnz the automatic choice
                                   (residual_max_popc = -1) uses instead of this matrix's
                                   own.  A row-partitioned caller passes the WHOLE matrix's
                                   fill (spaden_count_blocks + a sum over ranks) so every
                                   slice takes the same t (partition invariance).  0 = own. */
    int32_t reserved[5];
} spaden_convert_opts_t;

/*
 * spaden_convert_csr_to_bitmap -- CSR -> bitBSR on the GPU (§4.2).
 *
 *   m, n            matrix shape, 0 <= m, n < 2^31.
 *   nnz             number of stored entries, 0 <= nnz < 2^31.
 *   d_rowptr        int32[m+1], rowptr[0] == 0, non-decreasing, rowptr[m] == nnz.
 *   d_colidx        int32[nnz], each row's columns strictly ascending, in [0, n).
 *   d_values        [nnz] of values_dtype.
 *   values_dtype    dtype of d_values.
 *   storage_dtype   dtype of the stored bitBSR values: 32F->32F and 16F->16F move
 *                   raw bits; 32F->16F rounds to nearest even; 16F->32F is exact.
 *   stream          cudaStream_t (void*).
 *   out             receives the new handle (NULL on error).
 *
 * Stream-ordered.  The host synchronises `stream` a few times, each to read a
 * size before allocating: the block count Bnnz and the validation result, the
 * SpMV schedule's tile / long-row counts, the long-row chunk count (only when
 * long block-rows exist); the hybrid split (_ex, t > 0) adds its own (kept
 * counts, residual column parts).  Other streams and the device are never
 * synchronised.  Row rotations for the decode's shared-memory banks are chosen
 * here as well (a schedule pass; they never change y).  A stored 0.0 keeps
 * its bit (the round trip bitBSR -> CSR is the identity).  Invalid CSR is
 * reported as INVALID_ARGUMENT / INDEX_OUT_OF_RANGE / UNSORTED_OR_DUPLICATE;
 * nothing is leaked on error.  m == 0, n == 0 or nnz == 0 give a valid handle.
 * The handle's arrays are stream-ordered allocations (on `stream`) from a
 * library-private memory pool per device that keeps up to 4 GiB of freed
 * memory mapped, so converting again after spaden_free reuses it.
 */
SPADEN_API spaden_status_t spaden_convert_csr_to_bitmap(int64_t m, int64_t n, int64_t nnz,
                                             const int32_t *d_rowptr, const int32_t *d_colidx,
                                             const void *d_values, spaden_dtype_t values_dtype,
                                             spaden_dtype_t storage_dtype, void *stream,
                                             spaden_matrix_t *out);

/*
 * spaden_count_blocks -- the converter's validation + block-count pass only
 * (C1 of the conversion): *Bnnz receives the number of non-empty
 * 8x8 blocks of the CSR matrix, without building the format.  Same argument
 * rules and error codes as spaden_convert_csr_to_bitmap; one host
 * synchronisation; allocates only stream-ordered temporaries.  Bnnz is additive
 * over 8-row-aligned row slices, so ranks of a row partition sum it to get the
 * whole matrix's mean fill (spaden_convert_opts_t.auto_mean_fill).
 */
SPADEN_API spaden_status_t spaden_count_blocks(int64_t m, int64_t n, int64_t nnz, const int32_t *d_rowptr,
                                               const int32_t *d_colidx, void *stream, int64_t *Bnnz);

/*
 * Reordering before conversion (second half).  The
 * paper names reordering (degree-based, Gorder, Rabbit) as the usual remedy
 * for irregular, low-degree matrices (§6) -- the regime where
 * bitmaps cost more than they save.  Placing high-degree
 * rows/columns first raises the fill of the 8x8 blocks they share and puts the
 * hub entries of x on common cache lines.
 *
 * spaden_degree_order -- d_perm[k] = the row placed k-th: rows by descending
 * degree (rowptr[i+1] - rowptr[i]), equal degrees in ascending row order.
 *   m         rows, 0 <= m < 2^31.
 *   d_rowptr  int32[m+1] device CSR row pointers (non-decreasing).
 *   d_perm    int32[m] device output (caller-owned).
 * Stream-ordered, no host synchronisation; temporaries from the library pool.
 * Deterministic (a stable radix sort).
 *
 * spaden_permute_csr -- the symmetric permutation B = P A P^T of a square CSR
 * matrix A (m x m): row k of B is row perm[k] of A with every column j renamed
 * iperm[j] (iperm[perm[k]] = k) and the row's entries sorted by the new column.
 * Hence B (P x) = P (A x) with (P x)[k] = x[perm[k]]: an iteration on B runs
 * in the permuted space (PageRank keeps x permuted; only its start and end are
 * mapped).
 *   m, nnz            shape (square) and entries; A must be a valid CSR with
 *                     columns in [0, m) (as spaden_convert_csr_to_bitmap checks;
 *                     violations return INDEX_OUT_OF_RANGE).
 *   d_rowptr, d_colidx, d_values  A on the device, values of dtype (16F or 32F,
 *                     moved as raw bits).
 *   d_perm            int32[m], a permutation of [0, m) (e.g. spaden_degree_order);
 *                     anything else returns INVALID_ARGUMENT (checked first).
 *   d_out_rowptr, d_out_colidx, d_out_values  B, caller-owned device arrays of
 *                     m+1, nnz and nnz elements (must not alias the inputs).
 * Stream-ordered; two host synchronisations (the column range and the
 * permutation checks).
 */
SPADEN_API spaden_status_t spaden_degree_order(int64_t m, const int32_t *d_rowptr, int32_t *d_perm, void *stream);
SPADEN_API spaden_status_t spaden_permute_csr(int64_t m, int64_t nnz, const int32_t *d_rowptr,
                                              const int32_t *d_colidx, const void *d_values,
                                              spaden_dtype_t dtype, const int32_t *d_perm,
                                              int32_t *d_out_rowptr, int32_t *d_out_colidx,
                                              void *d_out_values, void *stream);

/*
 * spaden_convert_csr_to_bitmap_ex -- as spaden_convert_csr_to_bitmap, with options
 * (opts may be NULL = defaults).  With residual_max_popc = t > 0 the matrix is
 * split by block: 8x8 blocks with <= t entries go to a CSR residual (row-sorted,
 * global columns), the others stay bitBSR; spaden_spmv then computes
 * y = alpha*(A_bit + A_res) x + beta*y.  Useful for low-degree matrices whose
 * blocks hold ~1 entry (bitmaps are a burden there).  One more
 * host synchronisation than the pure conversion.
 */
SPADEN_API spaden_status_t spaden_convert_csr_to_bitmap_ex(int64_t m, int64_t n, int64_t nnz,
                                             const int32_t *d_rowptr, const int32_t *d_colidx,
                                             const void *d_values, spaden_dtype_t values_dtype,
                                             spaden_dtype_t storage_dtype,
                                             const spaden_convert_opts_t *opts, void *stream,
                                             spaden_matrix_t *out);

/*
 * spaden_spmv -- y = alpha * A x + beta * y on the GPU (§4.3: "takes bitBSR
 * and a dense vector x as input and produces a dense vector y").
 *
 *   A         handle from spaden_convert_csr_to_bitmap.  The bitBSR arrays are
 *             immutable; block-rows too large for a pipeline stage use one of 4
 *             per-handle scratch sets, taken round robin per call, so up to 4
 *             calls on one handle may run concurrently on different streams.
 *   d_x       float32[n] (read-only; only entries referenced by a set bit are read,
 *             structural zeros are never multiplied).
 *   d_y       float32[m]; with beta == 0 it is write-only (its old contents, even
 *             NaN, are ignored).  d_x and d_y must not overlap.
 *   stream    cudaStream_t (void*).
 *
 * Accumulation is fp32 in a fixed order that depends only on each block-row's own
 * blocks: deterministic, and bitwise identical for any row partition aligned to
 * 8 rows (whether a block-row takes the tile path or the long-row path is a
 * constant cost threshold, kLongRowBytes; the hybrid's automatic threshold is
 * the same on every slice when spaden_convert_opts_t.auto_mean_fill carries the
 * whole matrix's fill).  Never allocates and never synchronises: CUDA-graph
 * capturable.
 */
SPADEN_API spaden_status_t spaden_spmv(spaden_matrix_t A, float alpha, const float *d_x, float beta,
                            float *d_y, void *stream);

/*
 * spaden_spmv_scatter -- fused SpMV + all-gather epilogue
 * for row-partitioned iterated SpMV: computes this rank's slice
 * y = alpha * A x + beta * y (A = the rank's row slice, global columns) and stores
 * every y value straight into each destination buffer:
 *   h_out_ptrs[p][out_offset + i] = y_i   for p < npeers, i < m
 * from the SpMV epilogue (plain stores; on a multi-GPU node the pointers are the
 * NVLink-mapped next-x buffers of every rank, e.g. torch symmetric memory peer
 * pointers, including this rank's own), so the exchange overlaps the compute
 * tile by tile instead of following it as a separate collective.  The caller
 * adds the cross-GPU barrier before the buffers are read.  Values are bitwise
 * identical to spaden_spmv.
 *   h_out_ptrs  HOST array of npeers device pointers (1 <= npeers <= 8).
 *   d_y         local y (read if beta != 0, also written if non-NULL; may be NULL).
 * Requires a pure bitBSR handle (converted with residual_max_popc = 0, or an
 * automatic choice that took t = 0); a hybrid handle returns
 * SPADEN_ERR_UNSUPPORTED.
 */
SPADEN_API spaden_status_t spaden_spmv_scatter(spaden_matrix_t A, float alpha, const float *d_x, float beta,
                                               float *d_y, float *const *h_out_ptrs, int32_t npeers,
                                               int64_t out_offset, void *stream);

/*
 * spaden_spmm -- k products at once (SURVEY.md §8(f) NEXT-4, P:L336 future work):
 * Y[:, j] = alpha * A X[:, j] + beta * Y[:, j] for j < k, with column-major device
 * matrices: vector j of X at d_X + j*ldx (ldx >= n), of Y at d_Y + j*ldy (ldy >= m).
 * Each block is decoded once for up to 4 vectors (its values are loaded once
 * from shared memory and multiplied into every vector), so throughput per
 * vector rises with k.  Column j is bitwise identical to spaden_spmv on
 * vector j.  The first call for a given group size (2 or 4) builds a small
 * schedule and synchronises `stream` once; if a block-row cannot fit a
 * pipeline stage with that many vectors the call falls back to k SpMVs.
 * X and Y must not overlap.  Calls on one handle must be ordered.
 */
SPADEN_API spaden_status_t spaden_spmm(spaden_matrix_t A, float alpha, const float *d_X, int64_t ldx,
                                       int32_t k, float beta, float *d_Y, int64_t ldy, void *stream);

/*
 * spaden_spmm_tc_pack_x -- x slabs for spaden_spmm_tc, in groups of 128
 * vectors: d_Xb[g][bc][jj][c] = fp16(d_X[j*ldx + 8*bc + c]) with j = 128g + jj,
 * for groups g < ceil(k/128), block columns bc < ceil(n/8), jj < 128, c < 8
 * (round to nearest even; entries past n and vectors j >= k are 0).  The slabs
 * of one group are contiguous across block columns, so the kernel fetches a
 * run of consecutive block columns with one bulk copy.  d_X: float32,
 * column-major (vector j at d_X + j*ldx, ldx >= n).  d_Xb: DEVICE buffer of
 * 2048 * ceil(n/8) * ceil(k/128) bytes (spaden_spmm_tc_xb_bytes), 16-byte
 * aligned, owned by the caller.  Stream-ordered.
 */
SPADEN_API spaden_status_t spaden_spmm_tc_pack_x(int64_t n, int32_t k, const float *d_X, int64_t ldx, void *d_Xb,
                                                 void *stream);

/* Bytes of the slab buffer spaden_spmm_tc_pack_x fills for n columns and k vectors. */
SPADEN_API int64_t spaden_spmm_tc_xb_bytes(int64_t n, int32_t k);

/*
 * spaden_spmm_tc -- Y[:, j] = alpha * A X[:, j] + beta * Y[:, j], j < k, on the
 * tcgen05 tensor cores (the paper's SpMM future work,
 * P:L336).  X enters as fp16 slabs from spaden_spmm_tc_pack_x (fp16 inputs and
 * fp32 accumulation: the paper's tensor-core precision); Y is float32,
 * column-major (ldy >= m).  Per block-row, every pair of consecutive blocks is
 * one tcgen05.mma (M = 128 vectors, N = 8 rows, K = 16) accumulating in TMEM
 * in block order: deterministic.  Unlike the CUDA-core paths, structural zeros
 * of a stored block are multiplied (as in the paper's MMA), so X must be finite.
 *   A       pure bitBSR handle with fp16 storage (else SPADEN_ERR_UNSUPPORTED).
 *   d_Xb    slabs of the k vectors (see above); d_Y must not overlap it.
 * Never allocates or synchronises.
 */
SPADEN_API spaden_status_t spaden_spmm_tc(spaden_matrix_t A, float alpha, const void *d_Xb, int32_t k, float beta,
                                          float *d_Y, int64_t ldy, void *stream);

/*
 * spaden_spmv_host -- the same operation with HOST vectors: copies h_x (and h_y if
 * beta != 0) to device staging buffers owned by the handle, runs spaden_spmv,
 * copies y back to h_y and synchronises `stream`.  Not thread-safe per handle.
 */
SPADEN_API spaden_status_t spaden_spmv_host(spaden_matrix_t A, float alpha, const float *h_x, float beta,
                                 float *h_y, void *stream);

/*
 * spaden_spmv_host_batched -- nvec independent products y_k = alpha*A*x_k + beta*y_k
 * with HOST vectors, pipelined: the host->device copy of x_{k+1} and the
 * device->host copy of y_{k-1} overlap the SpMV of vector k (two internal copy
 * streams owned by the handle, device staging in 3 slots by default;
 * SPADEN_PIPE_SLOTS=2..8, read when the handle first builds its pipeline).
 *
 *   h_x     host float32, vector k at h_x + k*ldx (ldx >= n); pinned memory
 *           is required for the copies to overlap.
 *   h_y     host float32, vector k at h_y + k*ldy (ldy >= m); read when beta != 0.
 *   nvec    number of vectors (>= 0).
 *   stream  cudaStream_t (void*) on which the SpMVs run; the call returns after
 *           every y_k is back on the host.  Not thread-safe per handle.
 */
SPADEN_API spaden_status_t spaden_spmv_host_batched(spaden_matrix_t A, float alpha, const float *h_x,
                                                    int64_t ldx, float beta, float *h_y, int64_t ldy,
                                                    int64_t nvec, void *stream);

/* spaden_free -- synchronises the handle's device, then returns all device
 * arrays owned by A to the library's pool (up to 4 GiB stays mapped for later
 * conversions, the rest goes back to the driver).  spaden_free(NULL) returns
 * SPADEN_OK. */
SPADEN_API spaden_status_t spaden_free(spaden_matrix_t A);

/* Introspection (tests, bench, the bytes-per-nnz metric). */
SPADEN_API spaden_status_t spaden_get_info(spaden_matrix_t A, spaden_info_t *info);
SPADEN_API spaden_status_t spaden_get_arrays(spaden_matrix_t A, spaden_arrays_t *arrays);

/*
 * spaden_spmv_launch_count -- number of kernel launches (and memsets) one
 * spaden_spmv(A, ..., beta, ...) call issues on its stream with the current
 * environment (decode / ablation overrides): the tiled kernel, long-row chunk
 * and fix-up kernels, the hybrid residual pass.  For the bench's launch
 * accounting; no device work, no synchronisation.  *count must be non-NULL.
 */
SPADEN_API spaden_status_t spaden_spmv_launch_count(spaden_matrix_t A, float beta, int32_t *count);

/* Static strings; never NULL. */
SPADEN_API const char *spaden_status_string(spaden_status_t s);
SPADEN_API const char *spaden_last_error_message(void);
SPADEN_API const char *spaden_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SPADEN_H_ */
