// reorder.cu -- optional reordering before conversion (SURVEY.md §8(f) NEXT-1,
// second half): a degree ordering of the rows and the symmetric permutation
// B = P A P^T of a square CSR matrix.  PAPER.md §6 lists reordering
// (degree-based, Gorder, Rabbit) as the standard remedy for low-degree,
// irregular matrices, the regime where bitmaps are a burden (P:L142,
// P:L236): hubs placed first share 8x8 blocks (higher fill) and their x
// entries share cache lines.
//
// Both sorts are CUB device radix sorts (library primitives, stable and
// deterministic); every other step is a kernel of this file.
#include <cub/device/device_radix_sort.cuh>

#include "internal.cuh"

namespace spaden {
namespace {

// key = ~degree (ascending key = descending degree; the radix sort is stable,
// so equal degrees keep ascending row index), value = row
__global__ void k_degree_keys(int64_t m, const int32_t *__restrict__ rowptr, uint32_t *__restrict__ key,
                              int32_t *__restrict__ idx) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
        key[i] = ~(uint32_t)(rowptr[i + 1] - rowptr[i]);
        idx[i] = (int32_t)i;
    }
}

// iperm[perm[k]] = k (iperm pre-filled with -1); entries outside [0, m) set *bad
__global__ void k_inverse(int64_t m, const int32_t *__restrict__ perm, int32_t *__restrict__ iperm, uint32_t *bad) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t p = perm[k];
        if (p < 0 || p >= m) atomicOr(bad, 1u);
        else iperm[p] = (int32_t)k;
    }
}

// a permutation leaves no -1 in iperm (a repeated entry leaves a hole)
__global__ void k_check_inverse(int64_t m, const int32_t *__restrict__ iperm, uint32_t *bad) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x)
        if (iperm[i] < 0) atomicOr(bad, 1u);
}

// entry e of row i -> key (iperm[i] << cb) | iperm[col], value e (one warp per row)
__global__ void k_entry_keys(int64_t m, int cb, const int32_t *__restrict__ rowptr,
                             const int32_t *__restrict__ colidx, const int32_t *__restrict__ iperm,
                             uint64_t *__restrict__ key, int32_t *__restrict__ idx) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < m; i += warps) {
        const uint64_t hi = (uint64_t)(uint32_t)iperm[i] << cb;
        for (int64_t e = (int64_t)rowptr[i] + lane; e < rowptr[i + 1]; e += 32) {  // int64: nnz may reach 2^31 - 2
            key[e] = hi | (uint32_t)iperm[colidx[e]];
            idx[e] = (int32_t)e;
        }
    }
}

// new rowptr counts: row k of B is row perm[k] of A
__global__ void k_perm_counts(int64_t m, const int32_t *__restrict__ rowptr, const int32_t *__restrict__ perm,
                              int32_t *__restrict__ cnt) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t i = perm[k];
        cnt[k] = rowptr[i + 1] - rowptr[i];
    }
}

template <typename T>
__global__ void k_gather_entries(int64_t nnz, uint64_t cmask, const uint64_t *__restrict__ key,
                                 const int32_t *__restrict__ idx, const T *__restrict__ vin,
                                 int32_t *__restrict__ cout, T *__restrict__ vout) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nnz; k += (int64_t)gridDim.x * blockDim.x) {
        cout[k] = (int32_t)(key[k] & cmask);
        vout[k] = vin[idx[k]];
    }
}

unsigned grid_for(int64_t n, int threads) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>((n + threads - 1) / threads, 148ll * 64));
}

}  // namespace

spaden_status_t degree_order(int64_t m, const int32_t *rowptr, int32_t *perm, cudaStream_t st) {
    if (m == 0) return SPADEN_OK;
    uint32_t *key = nullptr;
    int32_t *idx = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    cudaError_t e = cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, (const uint32_t *)nullptr,
                                                    (uint32_t *)nullptr, (const int32_t *)nullptr,
                                                    (int32_t *)nullptr, (int)m, 0, 32, st);
    if (e == cudaSuccess) e = dmalloc(&key, 2 * sizeof(uint32_t) * (size_t)m, st);
    if (e == cudaSuccess) e = dmalloc(&idx, sizeof(int32_t) * (size_t)m, st);
    if (e == cudaSuccess) e = dmalloc(&tmp, std::max<size_t>(16, tmp_bytes), st);
    if (e == cudaSuccess) {
        k_degree_keys<<<grid_for(m, 256), 256, 0, st>>>(m, rowptr, key, idx);
        e = cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, key, key + m, idx, perm, (int)m, 0, 32, st);
    }
    dev_free(key, st);
    dev_free(idx, st);
    dev_free(tmp, st);
    if (e == cudaSuccess) e = cudaGetLastError();
    return e == cudaSuccess ? SPADEN_OK : cuda_status(e, "degree ordering");
}

spaden_status_t permute_csr(int64_t m, int64_t nnz, const int32_t *rowptr, const int32_t *colidx, const void *values,
                            int value_bytes, const int32_t *perm, int32_t *out_rowptr, int32_t *out_colidx,
                            void *out_values, cudaStream_t st) {
    if (m == 0) {
        return cudaMemsetAsync(out_rowptr, 0, sizeof(int32_t), st) == cudaSuccess
                   ? SPADEN_OK
                   : cuda_status(cudaGetLastError(), "permuting CSR");
    }
    int cb = 1;
    while ((1ll << cb) < m) ++cb;  // bits of a column (and of a row) index
    int32_t *iperm = nullptr, *cnt = nullptr, *idx = nullptr, *scan_tmp = nullptr;
    uint64_t *key = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    const size_t nz = (size_t)std::max<int64_t>(1, nnz);
    cudaError_t e = cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, (const uint64_t *)nullptr,
                                                    (uint64_t *)nullptr, (const int32_t *)nullptr,
                                                    (int32_t *)nullptr, (int)nz, 0, 2 * cb, st);
    uint32_t *bad = nullptr, hbad = 0;
    if (e == cudaSuccess) e = dmalloc(&iperm, sizeof(int32_t) * (size_t)m, st);
    if (e == cudaSuccess) e = dmalloc(&bad, sizeof(uint32_t), st);
    if (e == cudaSuccess) e = dmalloc(&cnt, sizeof(int32_t) * (size_t)(m + 1), st);
    if (e == cudaSuccess) e = dmalloc(&scan_tmp, sizeof(int32_t) * scan_tmp_ints(m + 1), st);
    if (e == cudaSuccess) e = dmalloc(&key, 2 * sizeof(uint64_t) * nz, st);
    if (e == cudaSuccess) e = dmalloc(&idx, 2 * sizeof(int32_t) * nz, st);
    if (e == cudaSuccess) e = dmalloc(&tmp, std::max<size_t>(16, tmp_bytes), st);
    if (e == cudaSuccess) e = cudaMemsetAsync(iperm, 0xff, sizeof(int32_t) * (size_t)m, st);
    if (e == cudaSuccess) e = cudaMemsetAsync(bad, 0, sizeof(uint32_t), st);
    if (e == cudaSuccess) {  // the permutation is checked before it indexes anything
        k_inverse<<<grid_for(m, 256), 256, 0, st>>>(m, perm, iperm, bad);
        k_check_inverse<<<grid_for(m, 256), 256, 0, st>>>(m, iperm, bad);
        e = cudaMemcpyAsync(&hbad, bad, sizeof(hbad), cudaMemcpyDeviceToHost, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    }
    if (e == cudaSuccess && hbad) {
        for (void *p : {(void *)iperm, (void *)cnt, (void *)scan_tmp, (void *)key, (void *)idx, tmp, (void *)bad})
            dev_free(p, st);
        set_error("perm is not a permutation of [0, m)");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (e == cudaSuccess) {
        k_perm_counts<<<grid_for(m, 256), 256, 0, st>>>(m, rowptr, perm, cnt);
        e = exclusive_scan_i32(cnt, out_rowptr, m, scan_tmp, st);
    }
    if (e == cudaSuccess && nnz > 0) {
        k_entry_keys<<<grid_for(32 * m, 256), 256, 0, st>>>(m, cb, rowptr, colidx, iperm, key, idx);
        e = cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, key, key + nz, idx, idx + nz, (int)nnz, 0, 2 * cb, st);
        const uint64_t cmask = (1ull << cb) - 1ull;
        if (e == cudaSuccess) {
            if (value_bytes == 2)
                k_gather_entries<<<grid_for(nnz, 256), 256, 0, st>>>(nnz, cmask, key + nz, idx + nz,
                                                                     (const uint16_t *)values, out_colidx,
                                                                     (uint16_t *)out_values);
            else
                k_gather_entries<<<grid_for(nnz, 256), 256, 0, st>>>(nnz, cmask, key + nz, idx + nz,
                                                                     (const uint32_t *)values, out_colidx,
                                                                     (uint32_t *)out_values);
            e = cudaGetLastError();
        }
    }
    for (void *p : {(void *)iperm, (void *)cnt, (void *)scan_tmp, (void *)key, (void *)idx, tmp, (void *)bad})
        dev_free(p, st);
    return e == cudaSuccess ? SPADEN_OK : cuda_status(e, "permuting CSR");
}

}  // namespace spaden
