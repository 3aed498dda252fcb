/*
 * oracle.c -- plain, slow, obviously-correct CPU reference for the Spaden hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant with the CUDA path
 * (paper_conf_icpp_cheny24_b200/csrc), and nothing here is ever called by
 * the product path.
 *
 * Paper: Y. Chen, J. X. Yu, "Bitmap-Based Sparse Matrix-Vector Multiplication
 * with Tensor Cores", ICPP '24 (/root/reference/PAPER.md, cited as P:L<n>).
 *
 * Functions and the passage each follows:
 *   oracle_csr_spmv_f64      Algorithm 1, standard CSR SpMV (§2.1), fp64.
 *   oracle_csr_spmv_f64_omp  The same Algorithm 1 with the row loop split over OpenMP
 *                            threads (schedule(static)); every row is still one
 *                            sequential-k sum, so y and s are bitwise equal to the
 *                            serial function (bench.py's all-cores cpu_baseline).
 *   oracle_bitbsr_count      §4.2 bitBSR, block positions "encoded as CSR".
 *   oracle_csr_to_bitbsr     §4.2 / Fig. 4 bitBSR conversion: 8x8 blocks
 *                            (P:L132), bit = 8*(r%8)+(c%8) with LSB = top-left,
 *                            MSB = bottom-right and row0 in the low byte,
 *                            nonzeros "stored consecutively" in bit order, per-block
 *                            counts exclusive-scanned into offsets.
 *   oracle_bitbsr_to_csr     The inverse: bitBSR decoding (§4.3.1) with the
 *                            value index read as the popcount rank of the bit
 *                            (reading R1 of Alg. 2 line 5-6).
 *   oracle_f32_to_f16_rne    IEEE binary16 round-to-nearest-even (fp16 storage,
 *                            DESIGN.md reading R10; paper's TC inputs are half).
 *   oracle_pagerank_f64      Iterated SpMV x <- d*A*x + (1-d)/n (rmat25 workload,
 *                            SURVEY.md §8(c)), each step = oracle_csr_spmv_f64.
 *
 * Pins (tests/test_oracle.py): hand-worked H1/H2 (tests/golden), dense
 * brute force (numpy A@x), identity/permutation/diagonal closed forms, closed-form
 * bitmaps, Table 1 footprint, numpy float16 rounding,
 * PageRank fixed point by a dense linear solve.  Parity-unpinned: none.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <omp.h>

/* status codes of the oracle's own input checks (independent of include/spaden.h) */
enum { ORC_OK = 0, ORC_BAD_ROWPTR = 1, ORC_COL_RANGE = 2, ORC_UNSORTED = 3, ORC_NOMEM = 4 };

/* ---------------------------------------------------------------- Alg. 1 */
/* y_i = sum_{k=rp[i]}^{rp[i+1]-1} val[k] * x[col[k]], sequential k.
 * s_i = sum |val[k]| * |x[col[k]]|   (condition number denominator for the
 * componentwise error test). s may be NULL.          */
void oracle_csr_spmv_f64(int64_t m, const int64_t *rowptr, const int32_t *colidx,
                         const double *val, const double *x, double *y, double *s)
{
    for (int64_t i = 0; i < m; ++i) {
        double acc = 0.0, abs_acc = 0.0;
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
            double p = val[k] * x[colidx[k]];
            acc += p;
            abs_acc += fabs(p);
        }
        y[i] = acc;
        if (s) s[i] = abs_acc;
    }
}

/* Alg. 1 over all host cores: rows split statically over OpenMP threads, each
 * row the same sequential sum as above.  Returns the number of threads used. */
int oracle_csr_spmv_f64_omp(int64_t m, const int64_t *rowptr, const int32_t *colidx,
                            const double *val, const double *x, double *y, double *s)
{
    int threads = 1;
#pragma omp parallel
    {
#pragma omp single
        threads = omp_get_num_threads();
#pragma omp for schedule(static)
        for (int64_t i = 0; i < m; ++i) {
            double acc = 0.0, abs_acc = 0.0;
            for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
                double p = val[k] * x[colidx[k]];
                acc += p;
                abs_acc += fabs(p);
            }
            y[i] = acc;
            if (s) s[i] = abs_acc;
        }
    }
    return threads;
}

/* ---------------------------------------------------------- input checks */
static int check_csr(int64_t m, int64_t n, int64_t nnz, const int64_t *rowptr,
                     const int32_t *colidx)
{
    if (m < 0 || n < 0 || nnz < 0) return ORC_BAD_ROWPTR;
    if (rowptr[0] != 0 || rowptr[m] != nnz) return ORC_BAD_ROWPTR;
    for (int64_t i = 0; i < m; ++i)
        if (rowptr[i + 1] < rowptr[i]) return ORC_BAD_ROWPTR;
    for (int64_t i = 0; i < m; ++i) {
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
            if (colidx[k] < 0 || colidx[k] >= n) return ORC_COL_RANGE;
        }
    }
    for (int64_t i = 0; i < m; ++i)
        for (int64_t k = rowptr[i] + 1; k < rowptr[i + 1]; ++k)
            if (colidx[k] <= colidx[k - 1]) return ORC_UNSORTED;
    return ORC_OK;
}

/* one entry of a block-row, keyed by (block column, bit position) */
typedef struct { int64_t bc; int bit; int64_t k; } entry_t;

static int cmp_entry(const void *pa, const void *pb)
{
    const entry_t *a = (const entry_t *)pa, *b = (const entry_t *)pb;
    if (a->bc != b->bc) return a->bc < b->bc ? -1 : 1;
    return (a->bit > b->bit) - (a->bit < b->bit);
}

/* Collect the entries of block-row br (rows 8br .. min(8br+8, m)-1), sorted by
 * (block column bc = col/8, bit = 8*(row%8) + col%8).  Returns the count.     */
static int64_t gather_block_row(int64_t br, int64_t m, const int64_t *rowptr,
                                const int32_t *colidx, entry_t *buf)
{
    int64_t cnt = 0;
    for (int64_t i = 8 * br; i < 8 * br + 8 && i < m; ++i) {
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
            buf[cnt].bc = colidx[k] / 8;
            buf[cnt].bit = (int)(8 * (i % 8) + colidx[k] % 8);
            buf[cnt].k = k;
            ++cnt;
        }
    }
    qsort(buf, (size_t)cnt, sizeof(entry_t), cmp_entry);
    return cnt;
}

static int64_t max_block_row_nnz(int64_t m, const int64_t *rowptr)
{
    int64_t mx = 0;
    for (int64_t br = 0; 8 * br < m; ++br) {
        int64_t hi = 8 * br + 8 < m ? 8 * br + 8 : m;
        int64_t c = rowptr[hi] - rowptr[8 * br];
        if (c > mx) mx = c;
    }
    return mx;
}

/* Number of non-empty 8x8 blocks (Bnnz).  P:L128: "These non-empty blocks'
 * positions are encoded in CSR".  Returns an ORC_* status.                    */
int oracle_bitbsr_count(int64_t m, int64_t n, int64_t nnz, const int64_t *rowptr,
                        const int32_t *colidx, int64_t *bnnz_out)
{
    int st = check_csr(m, n, nnz, rowptr, colidx);
    if (st != ORC_OK) return st;
    entry_t *buf = (entry_t *)malloc(sizeof(entry_t) * (size_t)(max_block_row_nnz(m, rowptr) + 1));
    if (!buf) return ORC_NOMEM;
    int64_t bnnz = 0;
    for (int64_t br = 0; 8 * br < m; ++br) {
        int64_t cnt = gather_block_row(br, m, rowptr, colidx, buf);
        for (int64_t e = 0; e < cnt; ++e)
            if (e == 0 || buf[e].bc != buf[e - 1].bc) ++bnnz;
    }
    free(buf);
    *bnnz_out = bnnz;
    return ORC_OK;
}

/* bitBSR conversion (Fig. 4).
 * Outputs (caller-allocated):
 *   blk_rowptr[Bnrow+1]  CSR over block-rows, Bnrow = ceil(m/8)
 *   blk_col[Bnnz]        block column, ascending within a block-row (reading R5)
 *   bitmap[Bnnz]         bit 8*(r%8)+(c%8) set for every stored entry;
 *                        a stored 0.0 keeps its bit (reading R7)
 *   blk_offset[Bnnz+1]   exclusive scan of per-block counts; last = nnz
 *   vals_out[nnz]        raw value bits (val_bytes = 2 or 4) in block order, and
 *                        in ascending bit order within a block (reading R4).      */
int oracle_csr_to_bitbsr(int64_t m, int64_t n, int64_t nnz, const int64_t *rowptr,
                         const int32_t *colidx, const void *vals, int val_bytes,
                         int64_t *blk_rowptr, int32_t *blk_col, uint64_t *bitmap,
                         int64_t *blk_offset, void *vals_out)
{
    int st = check_csr(m, n, nnz, rowptr, colidx);
    if (st != ORC_OK) return st;
    entry_t *buf = (entry_t *)malloc(sizeof(entry_t) * (size_t)(max_block_row_nnz(m, rowptr) + 1));
    if (!buf) return ORC_NOMEM;
    const unsigned char *vin = (const unsigned char *)vals;
    unsigned char *vout = (unsigned char *)vals_out;
    int64_t b = -1;            /* current block index */
    int64_t pos = 0;           /* next value slot     */
    int64_t Bnrow = (m + 7) / 8;
    blk_rowptr[0] = 0;
    for (int64_t br = 0; br < Bnrow; ++br) {
        int64_t cnt = gather_block_row(br, m, rowptr, colidx, buf);
        for (int64_t e = 0; e < cnt; ++e) {
            if (e == 0 || buf[e].bc != buf[e - 1].bc) {
                ++b;
                blk_col[b] = (int32_t)buf[e].bc;
                bitmap[b] = 0;
                blk_offset[b] = pos;     /* exclusive scan of counts */
            }
            bitmap[b] |= (uint64_t)1 << buf[e].bit;
            memcpy(vout + (size_t)pos * val_bytes, vin + (size_t)buf[e].k * val_bytes, (size_t)val_bytes);
            ++pos;
        }
        blk_rowptr[br + 1] = b + 1;
    }
    blk_offset[b + 1] = pos;
    free(buf);
    return ORC_OK;
}

static int popcount64(uint64_t v)
{
    int c = 0;
    for (int i = 0; i < 64; ++i) c += (int)((v >> i) & 1u);
    return c;
}

/* Decode bitBSR back to CSR.  For each block b of block-row br and each set bit
 * (r, c) of bitmap[b], the entry is (8br + r, 8*blk_col[b] + c) with value
 * vals[blk_offset[b] + popcount(bitmap[b] & ((1 << bit) - 1))]  (reading R1).
 * Entries are emitted row by row, blocks in stored order, bits ascending, which
 * is CSR order when blk_col ascends within the block-row.  rowptr_out[m+1],
 * colidx_out[nnz], vals_out[nnz] caller-allocated.                           */
void oracle_bitbsr_to_csr(int64_t m, const int64_t *blk_rowptr, const int32_t *blk_col,
                          const uint64_t *bitmap, const int64_t *blk_offset,
                          const void *vals, int val_bytes,
                          int64_t *rowptr_out, int32_t *colidx_out, void *vals_out)
{
    const unsigned char *vin = (const unsigned char *)vals;
    unsigned char *vout = (unsigned char *)vals_out;
    int64_t Bnrow = (m + 7) / 8;
    int64_t k = 0;
    rowptr_out[0] = 0;
    for (int64_t br = 0; br < Bnrow; ++br) {
        for (int r = 0; r < 8 && 8 * br + r < m; ++r) {
            for (int64_t b = blk_rowptr[br]; b < blk_rowptr[br + 1]; ++b) {
                for (int c = 0; c < 8; ++c) {
                    int bit = 8 * r + c;
                    if (!((bitmap[b] >> bit) & 1u)) continue;
                    uint64_t below = bit == 0 ? 0 : (bitmap[b] & (((uint64_t)1 << bit) - 1));
                    int64_t idx = blk_offset[b] + popcount64(below);
                    colidx_out[k] = (int32_t)(8 * (int64_t)blk_col[b] + c);
                    memcpy(vout + (size_t)k * val_bytes, vin + (size_t)idx * val_bytes, (size_t)val_bytes);
                    ++k;
                }
            }
            rowptr_out[8 * br + r + 1] = k;
        }
    }
}

/* IEEE binary16 with round-to-nearest-even, via the C23/GCC _Float16 type
 * (conversion from float follows the current rounding mode, RN by default). */
void oracle_f32_to_f16_rne(int64_t count, const float *in, uint16_t *out)
{
    for (int64_t i = 0; i < count; ++i) {
        _Float16 h = (_Float16)in[i];
        memcpy(&out[i], &h, sizeof(h));
    }
}

/* x_{k+1} = d * A x_k + (1 - d)/n, x_0 = x0, in fp64 (rmat25 iteration). */
void oracle_pagerank_f64(int64_t n, const int64_t *rowptr, const int32_t *colidx,
                         const double *val, double d, int iters, const double *x0,
                         double *x_out)
{
    double *cur = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
    double *nxt = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
    memcpy(cur, x0, sizeof(double) * (size_t)n);
    for (int it = 0; it < iters; ++it) {
        oracle_csr_spmv_f64(n, rowptr, colidx, val, cur, nxt, NULL);
        for (int64_t i = 0; i < n; ++i) nxt[i] = d * nxt[i] + (1.0 - d) / (double)n;
        double *t = cur; cur = nxt; nxt = t;
    }
    memcpy(x_out, cur, sizeof(double) * (size_t)n);
    free(cur);
    free(nxt);
}
