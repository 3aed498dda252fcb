// hybrid.cu -- fill-adaptive hybrid format.
//
// "bitBSR is expected to be effective for high-degree
// matrices.  As for low-degree matrices, the utilization of bitmaps may become
// burdensome, e.g., if one block only contains a single nonzero element."  In
// hybrid mode the converted bitBSR is split: blocks holding at most t entries
// become a row-sorted CSR residual (global columns), the rest stay bitBSR.
// spaden_spmv then runs the residual pass first (y = beta*y + alpha*A_res*x;
// rows binned by length, 2^c lanes per row of class c, fixed per-lane order and
// xor tree: deterministic and independent of the row partition), followed by
// the bitBSR kernels accumulating with beta = 1 (programmatic dependent launch
// along the chain).
//
// Split = count kernel (per block-row: kept blocks / values, residual entries
// per row) -> exclusive scans -> one host sync (sizes) -> fill kernel (compacts
// the kept blocks, appends residual entries row by row in ascending column) ->
// column parts when x > kXSegBytes (segment_residual) -> per part: long-row
// chunk lists and the length-class row permutation (residual_schedule).
#include <algorithm>
#include <cstdlib>

#include "internal.cuh"

namespace spaden {
namespace {

constexpr unsigned kFull = 0xffffffffu;

__device__ __forceinline__ int warp_sum(int v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    return v;
}

// one warp per block-row
__global__ void k_split_count(int64_t m, int64_t Bnrow, int t, const int32_t *__restrict__ brp,
                              const uint64_t *__restrict__ bitmap, int32_t *__restrict__ res_rowcnt,
                              int32_t *__restrict__ kept_blk, int32_t *__restrict__ kept_val) {
    const int64_t br = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (br >= Bnrow) return;
    const int b0 = brp[br], b1 = brp[br + 1];
    int cnt[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    int kb = 0, kv = 0;
    for (int base = b0; base < b1; base += 32) {
        const int b = base + lane;
        const uint64_t bm = b < b1 ? bitmap[b] : 0ull;
        const int pc = __popcll(bm);
        const bool res = b < b1 && pc <= t;
        const bool keep = b < b1 && !res;
        kb += __popc(__ballot_sync(kFull, keep));
        kv += warp_sum(keep ? pc : 0);
#pragma unroll
        for (int r = 0; r < 8; ++r) cnt[r] += warp_sum(res ? __popc((uint32_t)(bm >> (8 * r)) & 0xffu) : 0);
    }
#pragma unroll
    for (int r = 0; r < 8; ++r)
        if (lane == r && 8 * br + r < m) res_rowcnt[8 * br + r] = cnt[r];
    if (lane == 0) {
        kept_blk[br] = kb;
        kept_val[br] = kv;
    }
}

template <typename V>
__global__ void k_split_fill(int64_t m, int64_t Bnrow, int t, const int32_t *__restrict__ brp,
                             const int32_t *__restrict__ bcol, const uint64_t *__restrict__ bitmap,
                             const int32_t *__restrict__ boff, const V *__restrict__ vals,
                             const int32_t *__restrict__ new_brp, const int32_t *__restrict__ new_vstart,
                             int32_t *__restrict__ n_col, uint64_t *__restrict__ n_bmp, int32_t *__restrict__ n_off,
                             V *__restrict__ n_vals, const int32_t *__restrict__ res_rowptr,
                             int32_t *__restrict__ res_col, V *__restrict__ res_val) {
    const int64_t br = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (br >= Bnrow) return;
    const int b0 = brp[br], b1 = brp[br + 1];
    int nb = new_brp[br], nv = new_vstart[br];
    int rpos = (lane < 8 && 8 * br + lane < m) ? res_rowptr[8 * br + lane] : 0;  // lane r: next slot of row r
    for (int base = b0; base < b1; base += 32) {
        const int b = base + lane;
        const uint64_t bm = b < b1 ? bitmap[b] : 0ull;
        const int pc = __popcll(bm);
        const bool res = b < b1 && pc <= t;
        const bool keep = b < b1 && !res;
        const int col = b < b1 ? bcol[b] : 0;
        const int off = b < b1 ? boff[b] : 0;
        // kept blocks, compacted in order
        const unsigned km = __ballot_sync(kFull, keep);
        int vtot;
        const int vex = warp_excl_scan_i32(keep ? pc : 0, lane, &vtot);
        if (keep) {
            const int idx = nb + __popc(km & ((1u << lane) - 1u));
            n_col[idx] = col;
            n_bmp[idx] = bm;
            n_off[idx] = nv + vex;
            for (int j = 0; j < pc; ++j) n_vals[nv + vex + j] = vals[off + j];
        }
        nb += __popc(km);
        nv += vtot;
        // residual entries, row by row: lanes (blocks) in ascending column order
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            uint32_t byte = res ? ((uint32_t)(bm >> (8 * r)) & 0xffu) : 0u;
            int rtot;
            const int rex = warp_excl_scan_i32(__popc(byte), lane, &rtot);
            const int start = __shfl_sync(kFull, rpos, r) + rex;
            int q = off + __popcll(bm & ((1ull << (8 * r)) - 1ull));
            int j = 0;
            while (byte) {
                const int c = __ffs(byte) - 1;
                byte &= byte - 1;
                res_col[start + j] = 8 * col + c;
                res_val[start + j] = vals[q + j];
                ++j;
            }
            if (lane == r) rpos += rtot;
        }
    }
    if (br == Bnrow - 1 && lane == 0) n_off[nb] = nv;  // blk_offset[Bnnz'] = kept nnz
}

__global__ void k_split_summary(const int32_t *a, const int32_t *b, const int32_t *c, int32_t *out) {
    out[0] = *a;
    out[1] = *b;
    out[2] = *c;
}

// Load hints of the binned pass (SPADEN_RES_HINT, experiment hook): 0 none;
// 1 colidx/values streamed with L1::no_allocate; 2 = 1 + L2 evict_first policy
// on the stream; 3 = 2 + L2 evict_last policy on the x gathers.
#ifndef SPADEN_RES_HINT
#define SPADEN_RES_HINT 3
#endif
__device__ __forceinline__ uint64_t res_policy(bool last) {
    uint64_t p;
    if (last) asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    else asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint32_t ld_stream_b32(const void *ptr, uint64_t pol) {
    uint32_t v;
    if constexpr (SPADEN_RES_HINT >= 2)
        asm("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(ptr), "l"(pol));
    else if constexpr (SPADEN_RES_HINT == 1)
        asm("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(v) : "l"(ptr));
    else
        v = __ldg((const unsigned int *)ptr);
    return v;
}
__device__ __forceinline__ float ld_x(const float *ptr, uint64_t pol) {
    float v;
    if constexpr (SPADEN_RES_HINT >= 3)
        asm("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(ptr), "l"(pol));
    else
        v = __ldg(ptr);
    return v;
}

// One lane's share of entries [kb, k1) at stride L: entries kb, kb+L, ... summed
// sequentially in ascending order, four colidx/value loads and then four x
// gathers in flight per round.
template <typename V, int L>
__device__ __forceinline__ float res_lane_sum(int kb, int k1, const int32_t *__restrict__ col,
                                              const V *__restrict__ val, const float *__restrict__ x) {
    const uint64_t pol_s = SPADEN_RES_HINT >= 2 ? res_policy(false) : 0ull;
    const uint64_t pol_x = SPADEN_RES_HINT >= 3 ? res_policy(true) : 0ull;
    float a = 0.f;
    for (int base = kb; base < k1; base += 4 * L) {
        int c[4];
        float v[4], xv[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int k = base + u * L;
            c[u] = 0;
            v[u] = 0.f;
            if (k < k1) {
                c[u] = (int)ld_stream_b32(col + k, pol_s);
                if constexpr (sizeof(V) == 2) v[u] = __half2float(val[k]);
                else v[u] = __uint_as_float(ld_stream_b32(val + k, pol_s));
            }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) xv[u] = base + u * L < k1 ? ld_x(x + c[u], pol_x) : 0.f;
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (base + u * L < k1) a = fmaf(v[u], xv[u], a);
    }
    return a;
}

// residual CSR: L lanes per row (32/L rows per warp).  Fixed per-row order:
// the row is cut into kResChunk-entry chunks; in a chunk lane l sums entries l,
// l+L, ... sequentially, a log2(L)-level xor tree combines the lanes, and chunk
// sums are added in order -- a function of the row alone (partition
// invariant).  This fixed-L kernel is the SPADEN_RES=fixed ablation of the
// binned pass below.  Rows longer than kResLongRow are skipped by both: their
// kResChunk-entry chunks run in parallel (k_res_chunks, one warp per chunk, lane
// l summing entries l, l+32, ... of the chunk, xor tree) and the warp finishing
// a row's last chunk adds the chunk sums in chunk order (res_fixup_row).
template <typename V, int L>
__device__ __forceinline__ float res_chunk_sum(int c0, int c1, int sub, unsigned gmask,
                                               const int32_t *__restrict__ col, const V *__restrict__ val,
                                               const float *__restrict__ x) {
    float a = 0.f;
#pragma unroll 4
    for (int k = c0 + sub; k < c1; k += L) {
        float v;
        if constexpr (sizeof(V) == 2) v = __half2float(val[k]);
        else v = __ldg(val + k);
        a = fmaf(v, __ldg(x + __ldg(col + k)), a);
    }
#pragma unroll
    for (int o = L / 2; o > 0; o >>= 1) a += __shfl_xor_sync(gmask, a, o);
    return a;
}

// one L-lane group per row, no grid-stride loop (the block scheduler keeps the
// SM full of rows, so the rowptr -> colidx -> x gather chains of many rows
// overlap); the old y is fetched before the gathers so its latency hides too
template <typename V, int L>
__global__ void __launch_bounds__(256)
k_residual(int64_t m, const int32_t *__restrict__ rp, const int32_t *__restrict__ col, const V *__restrict__ val,
           const float *__restrict__ x, float alpha, float *__restrict__ y) {
    const int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / L;
    const int sub = threadIdx.x & (L - 1);
    const unsigned gmask = (L == 32 ? 0xffffffffu : ((1u << (L & 31)) - 1u)) << (threadIdx.x & (32 - L));  // this row's L lanes
    if (row >= m) return;  // uniform within the group
    const int k0 = __ldg(rp + row), k1 = __ldg(rp + row + 1);
    if (k0 == k1 || k1 - k0 > kResLongRow) return;
    const float yold = sub == 0 ? y[row] : 0.f;
    float sum = 0.f;
    for (int c0 = k0; c0 < k1; c0 += kResChunk) sum += res_chunk_sum<V, L>(c0, min(k1, c0 + kResChunk), sub, gmask, col, val, x);
    if (sub == 0) y[row] = fmaf(alpha, sum, yold);
}

// fix-up of long residual row j by one warp: lane l adds the chunk sums l,
// l+32, ... in order, then a fixed xor tree (a function of the row's chunk count)
__device__ __forceinline__ void res_fixup_row(int j, int lane, const int32_t *__restrict__ long_rows,
                                              const int32_t *__restrict__ chunk_start, const float *carry,
                                              float alpha, float *__restrict__ y) {
    float sum = 0.f;
    for (int c = chunk_start[j] + lane; c < chunk_start[j + 1]; c += 32) sum += __ldcg(carry + c);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(kFull, sum, o);
    if (lane == 0) {
        const int row = long_rows[j];
        y[row] = fmaf(alpha, sum, y[row]);
    }
}

__global__ void __launch_bounds__(256)
k_res_fixup(int64_t nlong, const int32_t *__restrict__ long_rows, const int32_t *__restrict__ chunk_start,
            const float *carry, float alpha, float *__restrict__ y) {
    const int64_t j = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    pdl_wait();
    if (j < nlong) res_fixup_row((int)j, threadIdx.x & 31, long_rows, chunk_start, carry, alpha, y);
}

// long residual rows: one warp per kResChunk-entry chunk (lane l sums entries
// l, l+32, ... of the chunk, xor tree); FUSED (few chunks): the
// warp finishing a row's last chunk runs the fix-up (threadfence + completion
// counter, reset for the next call), else k_res_fixup does after the launch
template <typename V, bool FUSED>
__global__ void __launch_bounds__(256)
k_res_chunks(int64_t nchunks, const int32_t *__restrict__ long_rows, const int32_t *__restrict__ chunk_start,
             const int32_t *__restrict__ chunk_row, const int32_t *__restrict__ rp, const int32_t *__restrict__ col,
             const V *__restrict__ val, const float *__restrict__ x, float *carry, int32_t *__restrict__ done,
             float alpha, float *__restrict__ y) {
    pdl_trigger();
    const int64_t g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;  // one warp per chunk
    const int lane = threadIdx.x & 31;
    if (g >= nchunks) return;  // uniform per warp
    const int j = chunk_row[g];
    const int row = long_rows[j];
    const int k1 = rp[row + 1];
    const int c0 = rp[row] + (int)(g - chunk_start[j]) * kResChunk;
    float a = res_lane_sum<V, 32>(c0 + lane, min(k1, c0 + kResChunk), col, val, x);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(kFull, a, o);
    int last = 0;
    if (lane == 0) {
        __stcg(carry + g, a);
        if constexpr (FUSED) {
            __threadfence();
            last = atomicAdd(done + j, 1) == chunk_start[j + 1] - chunk_start[j] - 1;
        }
    }
    pdl_wait();  // fix-up below reads y; unfused: still complete only after the predecessor
    if (FUSED && __shfl_sync(kFull, last, 0)) {
        __threadfence();
        res_fixup_row(j, lane, long_rows, chunk_start, carry, alpha, y);
        if (lane == 0) done[j] = 0;
    }
}

// Length-binned residual rows (default residual pass).  Rows of 1..kResLongRow
// entries are grouped by res_class(len) into a row permutation built at convert
// time; class c runs L = 2^c lanes per row, lane l summing entries l, l+L, ...
// in ascending order (four gathers in flight per lane per round), then a
// log2(L)-level xor tree.  L is a function of the row length, so the order is a
// function of the row alone (deterministic, partition invariant), and a
// warp's rows have similar lengths: no lane idles on a short row while a long
// row of the same warp runs, and short rows get one lane each (32 rows, and 32
// independent gather chains, per warp) instead of a 16-lane group.
template <typename V, int L>
__device__ __forceinline__ void res_binned_row(int64_t g, int64_t nrows, const int32_t *__restrict__ perm,
                                               const int32_t *__restrict__ rp, const int32_t *__restrict__ col,
                                               const V *__restrict__ val, const float *__restrict__ x, float alpha,
                                               float beta, float *__restrict__ y) {
    const int sub = threadIdx.x & (L - 1);
    if (g >= nrows) return;  // uniform within the group
    const int row = __ldg(perm + g);
    const int k0 = __ldg(rp + row), k1 = __ldg(rp + row + 1);
    const float yold = (sub == 0 && beta != 0.f) ? y[row] : 0.f;  // fetched before the gathers
    float a = res_lane_sum<V, L>(k0 + sub, k1, col, val, x);
    if constexpr (L > 1) {
        const unsigned gmask = (L == 32 ? kFull : ((1u << (L & 31)) - 1u)) << (threadIdx.x & (32 - L));
#pragma unroll
        for (int o = L / 2; o > 0; o >>= 1) a += __shfl_xor_sync(gmask, a, o);
    }
    if (sub == 0) y[row] = fmaf(alpha, a, beta != 0.f ? beta * yold : 0.f);
}

// rows without binned entries (empty, or long: their chunks accumulate later):
// y = beta*y only (y not read when beta = 0, untouched when beta = 1)
__device__ __forceinline__ void res_scale_row(int64_t g, int64_t nrows, const int32_t *__restrict__ perm, float beta,
                                              float *__restrict__ y) {
    if (g >= nrows || beta == 1.f) return;
    const int row = __ldg(perm + g);
    y[row] = beta != 0.f ? beta * y[row] : 0.f;
}

template <typename V>
__global__ void __launch_bounds__(256)
k_residual_binned(ResBins bins, const int32_t *__restrict__ perm, const int32_t *__restrict__ rp,
                  const int32_t *__restrict__ col, const V *__restrict__ val, const float *__restrict__ x,
                  float alpha, float beta, float *__restrict__ y) {
    pdl_trigger();
    // class of this CTA; static indices only (a dynamic index into the kernel
    // parameter struct would copy it to local memory in every thread)
    int c = 0;
    int64_t cs = bins.cta_start[0], r0 = bins.row_start[0], r1 = bins.row_start[1];
#pragma unroll
    for (int k = 1; k <= kResClasses; ++k)
        if ((int64_t)blockIdx.x >= bins.cta_start[k]) {
            c = k;
            cs = bins.cta_start[k];
            r0 = bins.row_start[k];
            r1 = bins.row_start[k + 1];
        }
    const int64_t cta = (int64_t)blockIdx.x - cs, nrows = r1 - r0;
    const int32_t *p = perm + r0;
    switch (c) {  // block-uniform
    case 0: res_binned_row<V, 1>(cta * 256 + threadIdx.x, nrows, p, rp, col, val, x, alpha, beta, y); break;
    case 1: res_binned_row<V, 2>(cta * 128 + threadIdx.x / 2, nrows, p, rp, col, val, x, alpha, beta, y); break;
    case 2: res_binned_row<V, 4>(cta * 64 + threadIdx.x / 4, nrows, p, rp, col, val, x, alpha, beta, y); break;
    case 3: res_binned_row<V, 8>(cta * 32 + threadIdx.x / 8, nrows, p, rp, col, val, x, alpha, beta, y); break;
    case 4: res_binned_row<V, 16>(cta * 16 + threadIdx.x / 16, nrows, p, rp, col, val, x, alpha, beta, y); break;
    case 5: res_binned_row<V, 32>(cta * 8 + threadIdx.x / 32, nrows, p, rp, col, val, x, alpha, beta, y); break;
    default: res_scale_row(cta * 256 + threadIdx.x, nrows, p, beta, y);  // class kResClasses
    }
}

// row binning: class flag -> scan -> scatter, one class at a time (ascending
// row order inside a class)
__global__ void k_res_class_flag(int64_t m, const int32_t *__restrict__ rp, int c, int32_t *__restrict__ flag) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < m) {
        const int len = rp[i + 1] - rp[i];
        const bool binned = len > 0 && len <= kResLongRow;
        flag[i] = (c == kResClasses ? !binned : (binned && res_class(len) == c)) ? 1 : 0;
    }
}
__global__ void k_res_class_scatter(int64_t m, const int32_t *__restrict__ pos, int32_t *__restrict__ perm) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < m && pos[i + 1] != pos[i]) perm[pos[i]] = (int32_t)i;
}

// long residual rows: flag -> scan -> list; chunk counts -> scan -> chunk owners
__global__ void k_res_long_flag(int64_t m, const int32_t *__restrict__ rp, int32_t *__restrict__ flag) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < m) flag[i] = (rp[i + 1] - rp[i]) > kResLongRow ? 1 : 0;
}
__global__ void k_res_long_list(int64_t m, const int32_t *__restrict__ rp, const int32_t *__restrict__ pos,
                                int32_t *__restrict__ long_rows, int32_t *__restrict__ nch) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < m && pos[i + 1] != pos[i]) {
        long_rows[pos[i]] = (int32_t)i;
        nch[pos[i]] = (rp[i + 1] - rp[i] + kResChunk - 1) / kResChunk;
    }
}
__global__ void k_res_chunk_rows(int64_t nlong, const int32_t *__restrict__ cs, int32_t *__restrict__ crow) {
    const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < nlong)
        for (int c = cs[j]; c < cs[j + 1]; ++c) crow[c] = (int32_t)j;
}

// long-row chunk lists and the length-class row permutation of one residual part
spaden_status_t residual_schedule(Matrix *A, ResPart &P, cudaStream_t st) {
    const int64_t m = A->m;
    const size_t nt = scan_tmp_ints(m + 1);
    int32_t *tmp = nullptr;
    SPADEN_CUDA_TRY(cudaMallocAsync(&tmp, ((size_t)m + 1 + nt + 4) * sizeof(int32_t), st));
    int32_t *flag = tmp, *scan_tmp = tmp + (m + 1);
    const unsigned g = (unsigned)((m + 255) / 256);
    k_res_long_flag<<<g, 256, 0, st>>>(m, P.rowptr, flag);
    cudaError_t e = exclusive_scan_i32(flag, flag, m, scan_tmp, st);
    int32_t nl = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(&nl, flag + m, 4, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e == cudaSuccess && nl > 0) {
        P.n_long = nl;
        e = dmalloc(&P.long_rows, 4 * (size_t)nl, st);
        if (e == cudaSuccess) e = dmalloc(&P.chunk_start, 4 * ((size_t)nl + 1), st);
        if (e == cudaSuccess) {
            k_res_long_list<<<g, 256, 0, st>>>(m, P.rowptr, flag, P.long_rows, P.chunk_start);
            e = exclusive_scan_i32(P.chunk_start, P.chunk_start, nl, scan_tmp, st);
        }
        int32_t nc = 0;
        if (e == cudaSuccess) e = cudaMemcpyAsync(&nc, P.chunk_start + nl, 4, cudaMemcpyDeviceToHost, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
        if (e == cudaSuccess) {
            P.n_chunks = nc;
            e = dmalloc(&P.chunk_row, 4 * (size_t)std::max(1, nc), st);
        }
        constexpr int SL = Matrix::kScratchSlots;
        if (e == cudaSuccess) e = dmalloc(&P.carry, 4 * (size_t)std::max(1, nc) * SL, st);
        if (e == cudaSuccess) e = dmalloc(&P.done, 4 * (size_t)nl * SL, st);
        if (e == cudaSuccess) e = cudaMemsetAsync(P.done, 0, 4 * (size_t)nl * SL, st);
        if (e == cudaSuccess) {
            k_res_chunk_rows<<<(unsigned)((nl + 255) / 256), 256, 0, st>>>(nl, P.chunk_start, P.chunk_row);
            e = cudaGetLastError();
        }
    }
    // every row in one class: length bins of the rows with 1..kResLongRow
    // entries, then class kResClasses (empty or long rows: beta only)
    int32_t *perm_pos = nullptr;
    ResBins bins{};
    int64_t total = 0;
    if (e == cudaSuccess) e = dmalloc(&perm_pos, 4 * (size_t)std::max<int64_t>(1, m), st);
    for (int c = 0; c <= kResClasses && e == cudaSuccess; ++c) {
        bins.row_start[c] = total;
        k_res_class_flag<<<g, 256, 0, st>>>(m, P.rowptr, c, flag);
        e = exclusive_scan_i32(flag, flag, m, scan_tmp, st);
        int32_t cnt = 0;
        if (e == cudaSuccess) e = cudaMemcpyAsync(&cnt, flag + m, 4, cudaMemcpyDeviceToHost, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
        if (e == cudaSuccess && cnt > 0) {
            k_res_class_scatter<<<g, 256, 0, st>>>(m, flag, perm_pos + total);
            e = cudaGetLastError();
        }
        total += cnt;
    }
    bins.row_start[kResClasses + 1] = total;
    int64_t ctas = 0;
    for (int c = 0; c <= kResClasses; ++c) {
        bins.cta_start[c] = ctas;
        const int lpr = c < kResClasses ? (1 << c) : 1;  // lanes per row
        const int64_t lanes = (bins.row_start[c + 1] - bins.row_start[c]) * lpr;
        ctas += (lanes + 255) / 256;
    }
    bins.cta_start[kResClasses + 1] = ctas;
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    cudaFreeAsync(tmp, st);
    if (e != cudaSuccess) {
        if (perm_pos) dev_free(perm_pos, st);
        return cuda_status(e, "hybrid residual schedule");
    }
    P.perm = perm_pos;
    P.bins = bins;
    A->res_aux_bytes += 4 * total + 4 * (2 * P.n_long + 1 + P.n_chunks) + 4 * P.n_chunks;
    return SPADEN_OK;
}

// Column segmentation of the residual (rows keep ascending columns): part s
// holds columns [c_s, c_{s+1}).  One warp per row: lane s < S finds the row's
// first entry with column >= c_s by binary search; counts per (part, row) ->
// per-part scans -> the warp copies each part's slice of the row.
__global__ void k_seg_count(int64_t m, int S, int64_t seg_cols, const int32_t *__restrict__ rp,
                            const int32_t *__restrict__ col, int32_t *__restrict__ cnt /* [S][m+1] */) {
    const int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (row >= m) return;
    const int k0 = rp[row], k1 = rp[row + 1];
    int lo = k1;  // lane s: first entry of part s
    if (lane <= S) {
        const int64_t c = (int64_t)lane * seg_cols;
        int a = k0, b = k1;
        while (a < b) {
            const int mid = (a + b) >> 1;
            if ((int64_t)col[mid] < c) a = mid + 1;
            else b = mid;
        }
        lo = lane == S ? k1 : a;
    }
    const int hi = __shfl_down_sync(0xffffffffu, lo, 1);
    if (lane < S) cnt[(int64_t)lane * (m + 1) + row] = hi - lo;
}
template <typename V>
__global__ void k_seg_fill(int64_t m, int S, int64_t seg_cols, const int32_t *__restrict__ rp,
                           const int32_t *__restrict__ col, const V *__restrict__ val,
                           const int32_t *__restrict__ pos /* [S][m+1] scanned */, int32_t *const *dst_col,
                           V *const *dst_val) {
    const int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (row >= m) return;
    const int k0 = rp[row];
    for (int s = 0; s < S; ++s) {
        const int o = pos[(int64_t)s * (m + 1) + row], n = pos[(int64_t)s * (m + 1) + row + 1] - o;
        // this part's slice starts after the row's slices of parts < s
        int skip = 0;
        for (int q = 0; q < s; ++q) skip += pos[(int64_t)q * (m + 1) + row + 1] - pos[(int64_t)q * (m + 1) + row];
        for (int j = lane; j < n; j += 32) {
            dst_col[s][o + j] = col[k0 + skip + j];
            dst_val[s][o + j] = val[k0 + skip + j];
        }
    }
}

}  // namespace

// x larger than kXSegBytes: split the residual into S column parts (each a CSR
// over all rows) so that every part's x gathers stay L2-resident; part q covers
// columns [q*seg_cols, (q+1)*seg_cols).  Conversion-time only.
static spaden_status_t segment_residual(Matrix *A, cudaStream_t st) {
    const int64_t m = A->m, n = A->n;
    int64_t seg_cols = kXSegBytes / 4;
    if (const char *e = getenv("SPADEN_XSEG_COLS")) seg_cols = std::max<int64_t>(8, atoll(e));
    const int S = (int)std::min<int64_t>(Matrix::kMaxResParts, (n + seg_cols - 1) / std::max<int64_t>(1, seg_cols));
    if (S <= 1 || A->res_nnz == 0) return SPADEN_OK;
    seg_cols = (n + S - 1) / S;  // balanced parts
    const size_t sv = A->storage == SPADEN_R_16F ? 2 : 4;
    ResPart full = A->res[0];
    const size_t nt = scan_tmp_ints(m + 1);
    int32_t *cnt = nullptr, *scan_tmp = nullptr;
    int32_t **d_cols = nullptr;
    void **d_vals = nullptr;
    cudaError_t e = dmalloc(&cnt, 4 * (size_t)S * (m + 1), st);
    if (e == cudaSuccess) e = dmalloc(&scan_tmp, 4 * (nt + 4), st);
    if (e == cudaSuccess) e = dmalloc(&d_cols, sizeof(void *) * 2 * S, st);
    d_vals = (void **)(d_cols + S);
    const unsigned g = (unsigned)((32 * m + 255) / 256);
    if (e == cudaSuccess) {
        k_seg_count<<<g, 256, 0, st>>>(m, S, seg_cols, full.rowptr, full.colidx, cnt);
        e = cudaGetLastError();
    }
    int32_t *h_cols[Matrix::kMaxResParts] = {};
    void *h_vals[Matrix::kMaxResParts] = {};
    for (int q = 0; q < S && e == cudaSuccess; ++q) {
        ResPart &P = A->res[q];
        P = ResPart{};
        P.col0 = q * seg_cols;
        P.col1 = std::min<int64_t>(n, (q + 1) * seg_cols);
        int32_t *c = cnt + (size_t)q * (m + 1);
        e = exclusive_scan_i32(c, c, m, scan_tmp, st);
        int32_t tot = 0;
        if (e == cudaSuccess) e = cudaMemcpyAsync(&tot, c + m, 4, cudaMemcpyDeviceToHost, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
        P.nnz = tot;
        if (e == cudaSuccess) e = dmalloc(&P.rowptr, pad16(4 * (m + 1)), st);
        if (e == cudaSuccess) e = dmalloc(&P.colidx, pad16(4 * (size_t)tot), st);
        if (e == cudaSuccess) e = dmalloc(&P.values, pad16(sv * (size_t)tot), st);
        if (e == cudaSuccess) e = cudaMemcpyAsync(P.rowptr, c, 4 * (m + 1), cudaMemcpyDeviceToDevice, st);
        h_cols[q] = P.colidx;
        h_vals[q] = P.values;
    }
    A->n_res_parts = S;
    if (e == cudaSuccess) e = cudaMemcpyAsync(d_cols, h_cols, sizeof(void *) * S, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaMemcpyAsync(d_vals, h_vals, sizeof(void *) * S, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) {
        if (A->storage == SPADEN_R_16F)
            k_seg_fill<__half><<<g, 256, 0, st>>>(m, S, seg_cols, full.rowptr, full.colidx,
                                                  (const __half *)full.values, cnt, d_cols, (__half *const *)d_vals);
        else
            k_seg_fill<float><<<g, 256, 0, st>>>(m, S, seg_cols, full.rowptr, full.colidx,
                                                 (const float *)full.values, cnt, d_cols, (float *const *)d_vals);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    dev_free(full.rowptr, st);
    dev_free(full.colidx, st);
    dev_free(full.values, st);
    if (cnt) dev_free(cnt, st);
    if (scan_tmp) dev_free(scan_tmp, st);
    if (d_cols) dev_free(d_cols, st);
    if (e != cudaSuccess) return cuda_status(e, "hybrid residual column segmentation");
    A->res_aux_bytes += 4 * (int64_t)(S - 1) * (m + 1);  // rowptrs beyond the first
    return SPADEN_OK;
}

spaden_status_t split_residual(Matrix *A, int t, cudaStream_t st) {
    A->res_max_popc = t;
    const int64_t m = A->m, Bnrow = A->Bnrow;
    if (t <= 0 || m == 0) return SPADEN_OK;
    const size_t sv = A->storage == SPADEN_R_16F ? 2 : 4;
    const size_t nt = scan_tmp_ints(std::max<int64_t>(m, Bnrow) + 1);
    int32_t *tmp = nullptr;
    const size_t ints = (size_t)(m + 1) + 2 * (size_t)(Bnrow + 1) + nt + 4;
    SPADEN_CUDA_TRY(cudaMallocAsync(&tmp, ints * sizeof(int32_t), st));
    int32_t *res_cnt = tmp, *kept_blk = tmp + (m + 1), *kept_val = kept_blk + (Bnrow + 1);
    int32_t *scan_tmp = kept_val + (Bnrow + 1), *summary = scan_tmp + nt;
    auto fail = [&](cudaError_t e, const char *what) {
        cudaFreeAsync(tmp, st);
        return cuda_status(e, what);
    };
    const unsigned grid = (unsigned)((32 * Bnrow + 255) / 256);
    k_split_count<<<grid, 256, 0, st>>>(m, Bnrow, t, A->blk_rowptr, A->bitmap, res_cnt, kept_blk, kept_val);
    cudaError_t e = exclusive_scan_i32(res_cnt, res_cnt, m, scan_tmp, st);
    if (e == cudaSuccess) e = exclusive_scan_i32(kept_blk, kept_blk, Bnrow, scan_tmp, st);
    if (e == cudaSuccess) e = exclusive_scan_i32(kept_val, kept_val, Bnrow, scan_tmp, st);
    int32_t h[3] = {0, 0, 0};
    if (e == cudaSuccess) {
        k_split_summary<<<1, 1, 0, st>>>(res_cnt + m, kept_blk + Bnrow, kept_val + Bnrow, summary);
        e = cudaMemcpyAsync(h, summary, sizeof(h), cudaMemcpyDeviceToHost, st);
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return fail(e, "hybrid split (count)");
    const int64_t res_nnz = h[0], nB = h[1], nV = h[2];
    int32_t *n_col = nullptr, *n_off = nullptr, *r_col = nullptr;
    uint64_t *n_bmp = nullptr;
    void *n_vals = nullptr, *r_vals = nullptr;
    e = dmalloc(&n_col, pad16(4 * nB), st);
    if (e == cudaSuccess) e = dmalloc(&n_bmp, pad16(8 * nB), st);
    if (e == cudaSuccess) e = dmalloc(&n_off, pad16(4 * (nB + 1)), st);
    if (e == cudaSuccess) e = dmalloc(&n_vals, pad16(sv * nV), st);
    ResPart &P0 = A->res[0];
    if (e == cudaSuccess) e = dmalloc(&P0.rowptr, pad16(4 * (m + 1)), st);
    if (e == cudaSuccess) e = dmalloc(&r_col, pad16(4 * res_nnz), st);
    if (e == cudaSuccess) e = dmalloc(&r_vals, pad16(sv * res_nnz), st);
    if (e != cudaSuccess) {
        for (void *p : {(void *)n_col, (void *)n_bmp, (void *)n_off, n_vals, (void *)r_col, r_vals})
            if (p) dev_free(p, st);
        return fail(e, "hybrid split (allocation)");
    }
    cudaMemsetAsync(n_off, 0, pad16(4 * (nB + 1)), st);
    e = cudaMemcpyAsync(P0.rowptr, res_cnt, 4 * (m + 1), cudaMemcpyDeviceToDevice, st);
    if (A->storage == SPADEN_R_16F)
        k_split_fill<__half><<<grid, 256, 0, st>>>(m, Bnrow, t, A->blk_rowptr, A->blk_col, A->bitmap, A->blk_offset,
                                                   (const __half *)A->values, kept_blk, kept_val, n_col, n_bmp, n_off,
                                                   (__half *)n_vals, P0.rowptr, r_col, (__half *)r_vals);
    else
        k_split_fill<float><<<grid, 256, 0, st>>>(m, Bnrow, t, A->blk_rowptr, A->blk_col, A->bitmap, A->blk_offset,
                                                  (const float *)A->values, kept_blk, kept_val, n_col, n_bmp, n_off,
                                                  (float *)n_vals, P0.rowptr, r_col, (float *)r_vals);
    if (e == cudaSuccess) e = cudaMemcpyAsync(A->blk_rowptr, kept_blk, 4 * (Bnrow + 1), cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess) e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    cudaFreeAsync(tmp, st);
    // install the compacted bitBSR (free the old arrays) and the residual
    dev_free(A->blk_col, st);
    dev_free(A->bitmap, st);
    dev_free(A->blk_offset, st);
    dev_free(A->values, st);
    A->blk_col = n_col;
    A->bitmap = n_bmp;
    A->blk_offset = n_off;
    A->values = n_vals;
    P0.colidx = r_col;
    P0.values = r_vals;
    P0.col0 = 0;
    P0.col1 = A->n;
    P0.nnz = res_nnz;
    A->n_res_parts = 1;
    A->Bnnz = nB;
    A->res_nnz = res_nnz;
    if (e != cudaSuccess) return cuda_status(e, "hybrid split (fill)");
    spaden_status_t ss = segment_residual(A, st);
    for (int q = 0; q < A->n_res_parts && ss == SPADEN_OK; ++q) ss = residual_schedule(A, A->res[q], st);
    return ss;
}

namespace {
__global__ void k_scale(int64_t m, float beta, float *__restrict__ y) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x)
        y[i] *= beta;
}
}  // namespace

// Hybrid SpMV, first part: y = beta*y + alpha*A_res*x on every row.  Per
// residual part (column segment) the binned kernel (a normal launch: it follows
// whatever produced x, or the previous part) applies beta itself -- part 0 with
// the caller's beta, later parts with 1 -- rows of the last class only get
// y = beta*y, so y is fetched before the gathers; long residual rows then
// accumulate their chunks (PDL launches).  Per row the parts are added in
// column order (a function of the row and of n: partition invariant).
// SPADEN_RES=fixed: beta pass (memset / scale) + the 16-lane kernel (ablation).
// `any`: whether a kernel of this SpMV call has been launched already; a
// kernel may use programmatic dependent launch only after one (the first
// kernel of a call must wait for everything before it on the stream).
static cudaError_t residual_part(const Matrix &A, const ResPart &P, bool binned, float alpha, const float *x,
                                 float beta, float *y, cudaStream_t st, int slot, bool &any) {
    cudaError_t e = cudaSuccess;
    if (binned) {
        // the last class (empty / long rows) only scales y: skipped when beta = 1
        const int64_t nc = P.bins.cta_start[beta == 1.f ? kResClasses : kResClasses + 1];
        if (nc > 0) {
            any = true;
            if (A.storage == SPADEN_R_16F)
                e = launch_k(false, k_residual_binned<__half>, dim3((unsigned)nc), dim3(256), 0, st, P.bins,
                             (const int32_t *)P.perm, (const int32_t *)P.rowptr, (const int32_t *)P.colidx,
                             (const __half *)P.values, x, alpha, beta, y);
            else
                e = launch_k(false, k_residual_binned<float>, dim3((unsigned)nc), dim3(256), 0, st, P.bins,
                             (const int32_t *)P.perm, (const int32_t *)P.rowptr, (const int32_t *)P.colidx,
                             (const float *)P.values, x, alpha, beta, y);
        }
    } else {
        any = any || beta != 1.f || P.nnz > 0;
        if (beta == 0.f) e = cudaMemsetAsync(y, 0, sizeof(float) * (size_t)A.m, st);
        else if (beta != 1.f)
            k_scale<<<(unsigned)std::min<int64_t>((A.m + 255) / 256, 148 * 16), 256, 0, st>>>(A.m, beta, y);
        const unsigned grid = (unsigned)((kResLanes * A.m + 255) / 256);  // one lane group per row
        if (e == cudaSuccess && P.nnz > 0) {
            if (A.storage == SPADEN_R_16F)
                k_residual<__half, kResLanes><<<grid, 256, 0, st>>>(A.m, P.rowptr, P.colidx,
                                                                    (const __half *)P.values, x, alpha, y);
            else
                k_residual<float, kResLanes><<<grid, 256, 0, st>>>(A.m, P.rowptr, P.colidx,
                                                                   (const float *)P.values, x, alpha, y);
        }
    }
    if (e == cudaSuccess && P.n_long > 0) {
        const unsigned gc = (unsigned)((32 * P.n_chunks + 255) / 256);
        const bool fused = P.n_chunks <= fused_fixup_max();
        const bool dep = any;  // PDL only behind a kernel of this call
        any = true;
        float *carry = P.carry + (size_t)slot * (size_t)std::max<int64_t>(1, P.n_chunks);
        int32_t *done = P.done + (size_t)slot * (size_t)P.n_long;
        if (A.storage == SPADEN_R_16F)
            e = launch_k(dep, fused ? k_res_chunks<__half, true> : k_res_chunks<__half, false>, dim3(gc), dim3(256),
                         0, st, (int64_t)P.n_chunks, (const int32_t *)P.long_rows, (const int32_t *)P.chunk_start,
                         (const int32_t *)P.chunk_row, (const int32_t *)P.rowptr, (const int32_t *)P.colidx,
                         (const __half *)P.values, x, carry, done, alpha, y);
        else
            e = launch_k(dep, fused ? k_res_chunks<float, true> : k_res_chunks<float, false>, dim3(gc), dim3(256),
                         0, st, (int64_t)P.n_chunks, (const int32_t *)P.long_rows, (const int32_t *)P.chunk_start,
                         (const int32_t *)P.chunk_row, (const int32_t *)P.rowptr, (const int32_t *)P.colidx,
                         (const float *)P.values, x, carry, done, alpha, y);
        if (e == cudaSuccess && !fused)
            e = launch_k(true, k_res_fixup, dim3((unsigned)((32 * P.n_long + 255) / 256)), dim3(256), 0, st,
                         (int64_t)P.n_long, (const int32_t *)P.long_rows, (const int32_t *)P.chunk_start,
                         (const float *)carry, alpha, y);
    }
    return e;
}

bool residual_binned_enabled(const Matrix &A) {
    const char *env = getenv("SPADEN_RES");  // "fixed": the 16-lane kernel (ablation), read per call
    return A.n_res_parts > 0 && A.res[0].perm && !(env && env[0] == 'f');
}

cudaError_t residual_first(const Matrix &A, float alpha, const float *x, float beta, float *y, cudaStream_t st,
                           int slot, bool *launched) {
    *launched = false;
    if (A.m == 0 || A.n_res_parts == 0) return cudaSuccess;
    const bool binned = residual_binned_enabled(A);
    cudaError_t e = cudaSuccess;
    bool any = false;
    for (int q = 0; q < A.n_res_parts && e == cudaSuccess; ++q)
        e = residual_part(A, A.res[q], binned, alpha, x, q == 0 ? beta : 1.f, y, st, slot, any);
    *launched = any;
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

}  // namespace spaden
