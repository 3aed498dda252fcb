// capi.cu -- the extern "C" boundary declared in include/spaden.h: argument
// validation, handle lifetime, error strings.  All compute is in convert.cu /
// spmv.cu kernels.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <new>
#include <string>

#include <nvtx3/nvToolsExt.h>

#include "internal.cuh"


// NVTX range over a C-ABI call (named after the entry point): profilers (ncu
// --nvtx, nsys) can attribute the call's kernels; near free without a tool
namespace {
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};
}  // namespace
#define SPADEN_NVTX(name) NvtxRange nvtx_range_(name)

namespace spaden {

static thread_local std::string g_last_error;

void set_error(const std::string &msg) { g_last_error = msg; }

spaden_status_t cuda_status(cudaError_t e, const char *what) {
    set_error(std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")");
    cudaGetLastError();  // clear sticky-free errors
    if (e == cudaErrorMemoryAllocation) return SPADEN_ERR_OUT_OF_MEMORY;
    return SPADEN_ERR_CUDA;
}

// device pointer on the current device (or managed), else INVALID_ARGUMENT
static spaden_status_t check_device_ptr(const void *p, const char *name, int dev) {
    cudaPointerAttributes at;
    cudaError_t e = cudaPointerGetAttributes(&at, p);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error(std::string(name) + " is not a CUDA device pointer");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (at.type != cudaMemoryTypeDevice && at.type != cudaMemoryTypeManaged) {
        set_error(std::string(name) + " must be device memory");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (at.type == cudaMemoryTypeDevice && at.device != dev) {
        set_error(std::string(name) + " lives on another device");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    return SPADEN_OK;
}

// ---------------------------------------------------------- memory pool
namespace {
std::mutex g_pool_mu;
cudaMemPool_t g_pool[64] = {};
}  // namespace

cudaError_t dev_alloc(void **ptr, size_t bytes, cudaStream_t st) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
    cudaMemPool_t pool;
    {
        std::lock_guard<std::mutex> lock(g_pool_mu);
        if (!g_pool[dev]) {
            cudaMemPoolProps props = {};
            props.allocType = cudaMemAllocationTypePinned;
            props.location.type = cudaMemLocationTypeDevice;
            props.location.id = dev;
            e = cudaMemPoolCreate(&g_pool[dev], &props);
            if (e != cudaSuccess) {
                g_pool[dev] = nullptr;
                return e;
            }
            uint64_t keep = kPoolKeepBytes;
            cudaMemPoolSetAttribute(g_pool[dev], cudaMemPoolAttrReleaseThreshold, &keep);
        }
        pool = g_pool[dev];
    }
    return cudaMallocFromPoolAsync(ptr, bytes, pool, st);
}

void dev_free(void *ptr, cudaStream_t st) {
    if (ptr) cudaFreeAsync(ptr, st);
}

static void release(Matrix *A) {
    if (!A) return;
    // the handle's arrays may still be read by work on any stream the caller
    // used (spaden_free's contract says none is in flight; cudaFree used to
    // synchronise the device implicitly): keep that behaviour
    cudaDeviceSynchronize();
    void *ptrs[] = {A->blk_rowptr, A->blk_col, A->bitmap,   A->blk_offset, A->values,
                    A->stage_x,     A->stage_y,  A->tiles, A->rot,
                    A->long_rows,   A->chunk_start, A->chunk_row, A->carry, A->chunk_done,
                    A->spmm_tiles[0], A->spmm_tiles[1], A->spmm_tiles[2], A->tc_chunks, A->tc_cta_start};
    for (void *p : ptrs) dev_free(p, 0);
    for (int j = 0; j < Matrix::kMaxPipe; ++j) {
        dev_free(A->pipe_x[j], 0);
        dev_free(A->pipe_y[j], 0);
    }
    for (int q = 0; q < A->n_res_parts; ++q) {
        const spaden::ResPart &P = A->res[q];
        void *rp[] = {P.rowptr, P.colidx, P.values, P.long_rows, P.chunk_start, P.chunk_row, P.carry, P.done, P.perm};
        for (void *p : rp) dev_free(p, 0);
    }
    for (cudaEvent_t e : A->ev)
        if (e) cudaEventDestroy(e);
    if (A->s_h2d) cudaStreamDestroy(A->s_h2d);
    if (A->s_d2h) cudaStreamDestroy(A->s_d2h);
    delete A;
}

// slots of the batched host pipeline (SPADEN_PIPE_SLOTS overrides, 2..kMaxPipe)
constexpr int kDefaultPipe = 3;

// lazily create the batched host pipeline resources
static spaden_status_t ensure_pipeline(Matrix *A) {
    if (A->s_h2d) return SPADEN_OK;
    int slots = kDefaultPipe;
    if (const char *e = getenv("SPADEN_PIPE_SLOTS")) slots = atoi(e);
    A->pipe_slots = slots < 2 ? 2 : (slots > Matrix::kMaxPipe ? Matrix::kMaxPipe : slots);
    for (int j = 0; j < A->pipe_slots; ++j) {
        if (A->n > 0) SPADEN_CUDA_TRY(dmalloc(&A->pipe_x[j], pad16(4 * A->n), 0));
        if (A->m > 0) SPADEN_CUDA_TRY(dmalloc(&A->pipe_y[j], pad16(4 * A->m), 0));
    }
    SPADEN_CUDA_TRY(cudaStreamSynchronize(0));  // pool allocations visible to the non-blocking copy streams
    for (cudaEvent_t &e : A->ev) SPADEN_CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    SPADEN_CUDA_TRY(cudaStreamCreateWithFlags(&A->s_d2h, cudaStreamNonBlocking));
    SPADEN_CUDA_TRY(cudaStreamCreateWithFlags(&A->s_h2d, cudaStreamNonBlocking));
    return SPADEN_OK;
}

}  // namespace spaden

using namespace spaden;

extern "C" {

const char *spaden_version(void) { return "spaden-b200 0.1 (sm_100a)"; }

const char *spaden_status_string(spaden_status_t s) {
    switch (s) {
    case SPADEN_OK: return "SPADEN_OK";
    case SPADEN_ERR_INVALID_ARGUMENT: return "SPADEN_ERR_INVALID_ARGUMENT";
    case SPADEN_ERR_INDEX_OUT_OF_RANGE: return "SPADEN_ERR_INDEX_OUT_OF_RANGE";
    case SPADEN_ERR_UNSORTED_OR_DUPLICATE: return "SPADEN_ERR_UNSORTED_OR_DUPLICATE";
    case SPADEN_ERR_UNSUPPORTED: return "SPADEN_ERR_UNSUPPORTED";
    case SPADEN_ERR_OUT_OF_MEMORY: return "SPADEN_ERR_OUT_OF_MEMORY";
    case SPADEN_ERR_CUDA: return "SPADEN_ERR_CUDA";
    }
    return "SPADEN_ERR_UNKNOWN";
}

const char *spaden_last_error_message(void) { return g_last_error.c_str(); }

spaden_status_t spaden_convert_csr_to_bitmap(int64_t m, int64_t n, int64_t nnz, const int32_t *d_rowptr,
                                             const int32_t *d_colidx, const void *d_values,
                                             spaden_dtype_t values_dtype, spaden_dtype_t storage_dtype,
                                             void *stream, spaden_matrix_t *out) {
    return spaden_convert_csr_to_bitmap_ex(m, n, nnz, d_rowptr, d_colidx, d_values, values_dtype, storage_dtype,
                                           nullptr, stream, out);
}

spaden_status_t spaden_convert_csr_to_bitmap_ex(int64_t m, int64_t n, int64_t nnz, const int32_t *d_rowptr,
                                                const int32_t *d_colidx, const void *d_values,
                                                spaden_dtype_t values_dtype, spaden_dtype_t storage_dtype,
                                                const spaden_convert_opts_t *opts, void *stream,
                                                spaden_matrix_t *out) {
    SPADEN_NVTX("spaden_convert_csr_to_bitmap_ex");
    g_last_error.clear();
    int res_t = 0;
    float auto_fill = 0.f;
    if (opts) {
        if (opts->struct_size != (int32_t)sizeof(spaden_convert_opts_t) || opts->residual_max_popc < -1 ||
            opts->residual_max_popc > 64) {
            if (out) *out = nullptr;
            set_error("bad spaden_convert_opts_t (struct_size or residual_max_popc not in [-1, 64])");
            return SPADEN_ERR_INVALID_ARGUMENT;
        }
        res_t = opts->residual_max_popc;
        auto_fill = opts->auto_mean_fill;
        if (!(auto_fill >= 0.f && auto_fill <= 64.f)) {
            if (out) *out = nullptr;
            set_error("bad spaden_convert_opts_t.auto_mean_fill (must be in [0, 64])");
            return SPADEN_ERR_INVALID_ARGUMENT;
        }
    }
    if (!out) {
        set_error("out must not be NULL");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    *out = nullptr;
    if (m < 0 || n < 0 || nnz < 0) {
        set_error("m, n, nnz must be >= 0");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (m >= (1LL << 31) - 8 || n >= (1LL << 31) - 8 || nnz >= (1LL << 31) - 1) {
        set_error("m, n, nnz must be < 2^31 (int32 indices)");
        return SPADEN_ERR_UNSUPPORTED;
    }
    if ((values_dtype != SPADEN_R_32F && values_dtype != SPADEN_R_16F) ||
        (storage_dtype != SPADEN_R_32F && storage_dtype != SPADEN_R_16F)) {
        set_error("dtype must be SPADEN_R_32F or SPADEN_R_16F");
        return SPADEN_ERR_UNSUPPORTED;
    }
    if (!d_rowptr || (nnz > 0 && (!d_colidx || !d_values))) {
        set_error("NULL rowptr (or colidx/values with nnz > 0)");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_status(e, "cudaGetDevice");
    spaden_status_t s = check_device_ptr(d_rowptr, "rowptr", dev);
    if (s == SPADEN_OK && nnz > 0) s = check_device_ptr(d_colidx, "colidx", dev);
    if (s == SPADEN_OK && nnz > 0) s = check_device_ptr(d_values, "values", dev);
    if (s != SPADEN_OK) return s;

    Matrix *A = new (std::nothrow) Matrix();
    if (!A) {
        set_error("host allocation failed");
        return SPADEN_ERR_OUT_OF_MEMORY;
    }
    A->device = dev;
    s = convert_csr(m, n, nnz, d_rowptr, d_colidx, d_values, values_dtype, storage_dtype, res_t, auto_fill,
                    (cudaStream_t)stream, A);
    if (s != SPADEN_OK) {
        cudaStreamSynchronize((cudaStream_t)stream);
        release(A);
        return s;
    }
    *out = A;
    return SPADEN_OK;
}

namespace spaden_capi_kernels {
__global__ void k_col_range(int64_t nnz, int64_t n, const int32_t *__restrict__ colidx, uint32_t *flag) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x)
        if (colidx[e] < 0 || colidx[e] >= n) atomicOr(flag, 1u);
}
}  // namespace spaden_capi_kernels

spaden_status_t spaden_degree_order(int64_t m, const int32_t *d_rowptr, int32_t *d_perm, void *stream) {
    SPADEN_NVTX("spaden_degree_order");
    g_last_error.clear();
    if (m < 0 || m >= (1LL << 31) - 8) {
        set_error("m must be in [0, 2^31)");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (m == 0) return SPADEN_OK;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_status(e, "cudaGetDevice");
    spaden_status_t s = check_device_ptr(d_rowptr, "rowptr", dev);
    if (s == SPADEN_OK) s = check_device_ptr(d_perm, "perm", dev);
    if (s != SPADEN_OK) return s;
    return degree_order(m, d_rowptr, d_perm, (cudaStream_t)stream);
}

spaden_status_t spaden_permute_csr(int64_t m, int64_t nnz, const int32_t *d_rowptr, const int32_t *d_colidx,
                                   const void *d_values, spaden_dtype_t dtype, const int32_t *d_perm,
                                   int32_t *d_out_rowptr, int32_t *d_out_colidx, void *d_out_values,
                                   void *stream) {
    SPADEN_NVTX("spaden_permute_csr");
    g_last_error.clear();
    if (m < 0 || nnz < 0 || m >= (1LL << 31) - 8 || nnz >= (1LL << 31) - 1) {
        set_error("m, nnz must be in [0, 2^31)");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (dtype != SPADEN_R_32F && dtype != SPADEN_R_16F) {
        set_error("dtype must be SPADEN_R_32F or SPADEN_R_16F");
        return SPADEN_ERR_UNSUPPORTED;
    }
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_status(e, "cudaGetDevice");
    spaden_status_t s = check_device_ptr(d_rowptr, "rowptr", dev);
    if (s == SPADEN_OK) s = check_device_ptr(d_out_rowptr, "out_rowptr", dev);
    if (s == SPADEN_OK && m > 0) s = check_device_ptr(d_perm, "perm", dev);
    if (s == SPADEN_OK && nnz > 0) s = check_device_ptr(d_colidx, "colidx", dev);
    if (s == SPADEN_OK && nnz > 0) s = check_device_ptr(d_values, "values", dev);
    if (s == SPADEN_OK && nnz > 0) s = check_device_ptr(d_out_colidx, "out_colidx", dev);
    if (s == SPADEN_OK && nnz > 0) s = check_device_ptr(d_out_values, "out_values", dev);
    if (s != SPADEN_OK) return s;
    cudaStream_t st = (cudaStream_t)stream;
    if (nnz > 0) {
        uint32_t *flag = nullptr, h = 0;
        e = dmalloc(&flag, sizeof(uint32_t), st);
        if (e == cudaSuccess) e = cudaMemsetAsync(flag, 0, sizeof(uint32_t), st);
        if (e == cudaSuccess) {
            spaden_capi_kernels::k_col_range<<<(unsigned)std::min<int64_t>((nnz + 255) / 256, 148 * 64), 256, 0, st>>>(nnz, m, d_colidx,
                                                                                                   flag);
            e = cudaMemcpyAsync(&h, flag, sizeof(h), cudaMemcpyDeviceToHost, st);
        }
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
        dev_free(flag, st);
        if (e != cudaSuccess) return cuda_status(e, "checking column range");
        if (h) {
            set_error("a column index is outside [0, m)");
            return SPADEN_ERR_INDEX_OUT_OF_RANGE;
        }
    }
    return permute_csr(m, nnz, d_rowptr, d_colidx, d_values, dtype == SPADEN_R_16F ? 2 : 4, d_perm, d_out_rowptr,
                       d_out_colidx, d_out_values, st);
}

spaden_status_t spaden_count_blocks(int64_t m, int64_t n, int64_t nnz, const int32_t *d_rowptr,
                                    const int32_t *d_colidx, void *stream, int64_t *Bnnz) {
    SPADEN_NVTX("spaden_count_blocks");
    g_last_error.clear();
    if (!Bnnz) {
        set_error("Bnnz must not be NULL");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    *Bnnz = 0;
    if (m < 0 || n < 0 || nnz < 0) {
        set_error("m, n, nnz must be >= 0");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (m >= (1LL << 31) - 8 || n >= (1LL << 31) - 8 || nnz >= (1LL << 31) - 1) {
        set_error("m, n, nnz must be < 2^31 (int32 indices)");
        return SPADEN_ERR_UNSUPPORTED;
    }
    if (!d_rowptr || (nnz > 0 && !d_colidx)) {
        set_error("NULL rowptr (or colidx with nnz > 0)");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_status(e, "cudaGetDevice");
    spaden_status_t s = check_device_ptr(d_rowptr, "rowptr", dev);
    if (s == SPADEN_OK && nnz > 0) s = check_device_ptr(d_colidx, "colidx", dev);
    if (s != SPADEN_OK) return s;
    Matrix tmp;
    tmp.device = dev;
    s = convert_csr(m, n, nnz, d_rowptr, d_colidx, nullptr, SPADEN_R_32F, SPADEN_R_32F, 0, 0.f,
                    (cudaStream_t)stream, &tmp, /*count_only=*/true);
    if (s == SPADEN_OK) *Bnnz = tmp.Bnnz;
    return s;
}

spaden_status_t spaden_spmv(spaden_matrix_t A, float alpha, const float *d_x, float beta, float *d_y,
                            void *stream) {
    SPADEN_NVTX("spaden_spmv");
    if (!A) {
        set_error("NULL matrix handle");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if ((A->m > 0 && !d_y) || (A->Bnnz > 0 && !d_x)) {
        set_error("NULL x or y");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (d_x && d_y && A->m > 0 && A->n > 0) {
        const char *xb = (const char *)d_x, *xe = xb + 4 * A->n;
        const char *yb = (const char *)d_y, *ye = yb + 4 * A->m;
        if (xb < ye && yb < xe) {
            set_error("x and y must not overlap");
            return SPADEN_ERR_INVALID_ARGUMENT;
        }
    }
    return spmv_launch(*A, alpha, d_x, beta, d_y, (cudaStream_t)stream);
}

spaden_status_t spaden_spmv_scatter(spaden_matrix_t A, float alpha, const float *d_x, float beta, float *d_y,
                                    float *const *h_out_ptrs, int32_t npeers, int64_t out_offset, void *stream) {
    SPADEN_NVTX("spaden_spmv_scatter");
    if (!A || npeers < 1 || npeers > kMaxPeers || !h_out_ptrs || out_offset < 0 ||
        (A->Bnnz > 0 && !d_x) || (beta != 0.f && A->m > 0 && !d_y)) {
        set_error("bad arguments (handle, 1 <= npeers <= 8, out pointers, x, y with beta != 0)");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    PeerOut po{};
    for (int p = 0; p < npeers; ++p) {
        if (!h_out_ptrs[p]) {
            set_error("NULL destination pointer");
            return SPADEN_ERR_INVALID_ARGUMENT;
        }
        po.ptr[p] = h_out_ptrs[p];
    }
    po.n = npeers;
    po.offset = out_offset;
    return spmv_launch(*A, alpha, d_x, beta, d_y, (cudaStream_t)stream, &po);
}

spaden_status_t spaden_spmm(spaden_matrix_t A, float alpha, const float *d_X, int64_t ldx, int32_t k, float beta,
                            float *d_Y, int64_t ldy, void *stream) {
    SPADEN_NVTX("spaden_spmm");
    if (!A || k < 0 || ldx < A->n || ldy < A->m || (k > 0 && ((A->m > 0 && !d_Y) || (A->Bnnz > 0 && !d_X)))) {
        set_error("NULL handle/matrices, k < 0, or ldx < n / ldy < m");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (k > 0 && d_X && d_Y && A->m > 0 && A->n > 0) {
        const char *xb = (const char *)d_X, *xe = (const char *)(d_X + (int64_t)(k - 1) * ldx + A->n);
        const char *yb = (const char *)d_Y, *ye = (const char *)(d_Y + (int64_t)(k - 1) * ldy + A->m);
        if (xb < ye && yb < xe) {
            set_error("X and Y must not overlap");
            return SPADEN_ERR_INVALID_ARGUMENT;
        }
    }
    if (k == 0) return SPADEN_OK;
    return spmm_launch(*A, alpha, d_X, ldx, k, beta, d_Y, ldy, (cudaStream_t)stream);
}

int64_t spaden_spmm_tc_xb_bytes(int64_t n, int32_t k) {
    if (n <= 0 || k <= 0) return 0;
    return 2048 * ((n + 7) / 8) * (((int64_t)k + 127) / 128);
}

spaden_status_t spaden_spmm_tc_pack_x(int64_t n, int32_t k, const float *d_X, int64_t ldx, void *d_Xb,
                                      void *stream) {
    SPADEN_NVTX("spaden_spmm_tc_pack_x");
    g_last_error.clear();
    if (n < 0 || k < 0 || ldx < n || (n > 0 && k > 0 && (!d_X || !d_Xb)) || ((uintptr_t)d_Xb & 15u)) {
        set_error("bad arguments (n, k >= 0, ldx >= n, non-NULL 16-byte aligned d_Xb)");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    return spmm_tc_pack_x(n, k, d_X, ldx, d_Xb, (cudaStream_t)stream);
}

spaden_status_t spaden_spmm_tc(spaden_matrix_t A, float alpha, const void *d_Xb, int32_t k, float beta, float *d_Y,
                               int64_t ldy, void *stream) {
    SPADEN_NVTX("spaden_spmm_tc");
    g_last_error.clear();
    if (!A || k < 0 || ldy < A->m || (k > 0 && A->m > 0 && (!d_Y || !d_Xb)) || ((uintptr_t)d_Xb & 15u)) {
        set_error("NULL handle/matrices, k < 0, ldy < m, or d_Xb not 16-byte aligned");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (A->storage != SPADEN_R_16F || A->res_max_popc > 0) {
        set_error("spaden_spmm_tc needs a pure bitBSR handle with fp16 storage");
        return SPADEN_ERR_UNSUPPORTED;
    }
    if (k > 0 && A->m > 0 && A->n > 0) {
        const char *xb = (const char *)d_Xb, *xe = xb + spaden_spmm_tc_xb_bytes(A->n, k);
        const char *yb = (const char *)d_Y, *ye = (const char *)(d_Y + (int64_t)(k - 1) * ldy + A->m);
        if (xb < ye && yb < xe) {
            set_error("X slabs and Y must not overlap");
            return SPADEN_ERR_INVALID_ARGUMENT;
        }
    }
    return spmm_tc_launch(*A, alpha, d_Xb, k, beta, d_Y, ldy, (cudaStream_t)stream);
}

spaden_status_t spaden_spmv_host(spaden_matrix_t A, float alpha, const float *h_x, float beta, float *h_y,
                                 void *stream) {
    SPADEN_NVTX("spaden_spmv_host");
    if (!A || (A->n > 0 && !h_x) || (A->m > 0 && !h_y)) {
        set_error("NULL handle or host vector");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    cudaStream_t st = (cudaStream_t)stream;
    if (!A->stage_x && A->n > 0) SPADEN_CUDA_TRY(dmalloc(&A->stage_x, pad16(4 * A->n), st));
    if (!A->stage_y && A->m > 0) SPADEN_CUDA_TRY(dmalloc(&A->stage_y, pad16(4 * A->m), st));
    if (A->n > 0)
        SPADEN_CUDA_TRY(cudaMemcpyAsync(A->stage_x, h_x, 4 * A->n, cudaMemcpyHostToDevice, st));
    if (beta != 0.f && A->m > 0)
        SPADEN_CUDA_TRY(cudaMemcpyAsync(A->stage_y, h_y, 4 * A->m, cudaMemcpyHostToDevice, st));
    spaden_status_t s = spmv_launch(*A, alpha, A->stage_x, beta, A->stage_y, st);
    if (s != SPADEN_OK) return s;
    if (A->m > 0)
        SPADEN_CUDA_TRY(cudaMemcpyAsync(h_y, A->stage_y, 4 * A->m, cudaMemcpyDeviceToHost, st));
    SPADEN_CUDA_TRY(cudaStreamSynchronize(st));
    return SPADEN_OK;
}

spaden_status_t spaden_spmv_host_batched(spaden_matrix_t A, float alpha, const float *h_x, int64_t ldx,
                                         float beta, float *h_y, int64_t ldy, int64_t nvec, void *stream) {
    SPADEN_NVTX("spaden_spmv_host_batched");
    if (!A || nvec < 0 || (nvec > 0 && ((A->n > 0 && !h_x) || (A->m > 0 && !h_y))) || ldx < A->n ||
        ldy < A->m) {
        set_error("NULL handle/vectors, nvec < 0, or ldx < n / ldy < m");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    if (nvec == 0) return SPADEN_OK;
    spaden_status_t s = ensure_pipeline(A);
    if (s != SPADEN_OK) return s;
    cudaStream_t cs = (cudaStream_t)stream;
    const int S = A->pipe_slots;
    cudaEvent_t *in_ready = A->ev, *computed = A->ev + S, *drained = A->ev + 2 * S;
    cudaEvent_t ev_start = A->ev[3 * S], ev_end = A->ev[3 * S + 1];
    // slot k%S: H2D(x_k[, y_k]) on s_h2d -> SpMV on cs -> D2H(y_k) on s_d2h.  A
    // slot is refilled only after the SpMV of vector k-S consumed it and its y
    // left the device, so H2D(k+1), SpMV(k) and D2H(k-1) run concurrently.
    SPADEN_CUDA_TRY(cudaEventRecord(ev_start, cs));
    SPADEN_CUDA_TRY(cudaStreamWaitEvent(A->s_h2d, ev_start, 0));
    SPADEN_CUDA_TRY(cudaStreamWaitEvent(A->s_d2h, ev_start, 0));
    for (int64_t k = 0; k < nvec; ++k) {
        const int j = (int)(k % S);
        float *dx = A->pipe_x[j], *dy = A->pipe_y[j];
        if (k >= S) SPADEN_CUDA_TRY(cudaStreamWaitEvent(A->s_h2d, drained[j], 0));
        if (A->n > 0)
            SPADEN_CUDA_TRY(cudaMemcpyAsync(dx, h_x + k * ldx, 4 * A->n, cudaMemcpyHostToDevice, A->s_h2d));
        if (beta != 0.f && A->m > 0)
            SPADEN_CUDA_TRY(cudaMemcpyAsync(dy, h_y + k * ldy, 4 * A->m, cudaMemcpyHostToDevice, A->s_h2d));
        SPADEN_CUDA_TRY(cudaEventRecord(in_ready[j], A->s_h2d));
        SPADEN_CUDA_TRY(cudaStreamWaitEvent(cs, in_ready[j], 0));
        if (k >= S && beta == 0.f) SPADEN_CUDA_TRY(cudaStreamWaitEvent(cs, drained[j], 0));
        s = spmv_launch(*A, alpha, dx, beta, dy, cs);
        if (s != SPADEN_OK) return s;
        SPADEN_CUDA_TRY(cudaEventRecord(computed[j], cs));
        SPADEN_CUDA_TRY(cudaStreamWaitEvent(A->s_d2h, computed[j], 0));
        if (A->m > 0)
            SPADEN_CUDA_TRY(cudaMemcpyAsync(h_y + k * ldy, dy, 4 * A->m, cudaMemcpyDeviceToHost, A->s_d2h));
        SPADEN_CUDA_TRY(cudaEventRecord(drained[j], A->s_d2h));
    }
    SPADEN_CUDA_TRY(cudaEventRecord(ev_end, A->s_d2h));
    SPADEN_CUDA_TRY(cudaStreamWaitEvent(cs, ev_end, 0));
    SPADEN_CUDA_TRY(cudaStreamSynchronize(cs));
    return SPADEN_OK;
}

spaden_status_t spaden_free(spaden_matrix_t A) {
    SPADEN_NVTX("spaden_free");
    if (!A) return SPADEN_OK;
    int cur = 0;
    const int dev = A->device;
    cudaGetDevice(&cur);
    if (cur != dev) cudaSetDevice(dev);
    cudaError_t e = cudaDeviceSynchronize();
    release(A);
    if (cur != dev) cudaSetDevice(cur);
    if (e != cudaSuccess) return cuda_status(e, "cudaDeviceSynchronize in spaden_free");
    return SPADEN_OK;
}

spaden_status_t spaden_spmv_launch_count(spaden_matrix_t A, float beta, int32_t *count) {
    if (!A || !count) {
        set_error("NULL handle or count");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    *count = spmv_launch_count(*A, beta);
    return SPADEN_OK;
}

spaden_status_t spaden_get_info(spaden_matrix_t A, spaden_info_t *info) {
    if (!A || !info) {
        set_error("NULL handle or info");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    const int64_t sv = A->storage == SPADEN_R_16F ? 2 : 4;
    info->m = A->m;
    info->n = A->n;
    info->nnz = A->nnz;
    info->Bnrow = A->Bnrow;
    info->Bnnz = A->Bnnz;
    info->storage_dtype = (int32_t)A->storage;
    info->device = A->device;
    info->format_bytes = 4 * (A->Bnrow + 1) + 4 * A->Bnnz + 8 * A->Bnnz + 4 * (A->Bnnz + 1) +
                         sv * (A->nnz - A->res_nnz);
    if (A->res_max_popc > 0) info->format_bytes += 4 * (A->m + 1) + (4 + sv) * A->res_nnz;
    info->residual_nnz = A->res_nnz;
    info->residual_max_popc = A->res_max_popc;
    info->residual_parts = A->n_res_parts;
    info->aux_bytes = A->aux_bytes + A->res_aux_bytes;
    info->n_tiles = A->n_tiles;
    info->n_long = A->n_long;
    return SPADEN_OK;
}

spaden_status_t spaden_get_arrays(spaden_matrix_t A, spaden_arrays_t *v) {
    if (!A || !v) {
        set_error("NULL handle or arrays");
        return SPADEN_ERR_INVALID_ARGUMENT;
    }
    v->blk_rowptr = A->blk_rowptr;
    v->blk_col = A->blk_col;
    v->bitmap = A->bitmap;
    v->blk_offset = A->blk_offset;
    v->values = A->values;
    // the residual CSR (NULL when it is split into column parts)
    const bool one = A->n_res_parts == 1;
    v->res_rowptr = one ? A->res[0].rowptr : nullptr;
    v->res_colidx = one ? A->res[0].colidx : nullptr;
    v->res_values = one ? A->res[0].values : nullptr;
    return SPADEN_OK;
}

}  // extern "C"
