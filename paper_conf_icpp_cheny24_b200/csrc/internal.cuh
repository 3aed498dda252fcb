// internal.cuh -- shared declarations of the libspaden.so implementation.
// Product code only: nothing here is shared with oracle/.
#pragma once

#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <stdint.h>
#include <atomic>
#include <string>

#include "spaden.h"

// One SpMV tile: block-rows [br0, br1), their blocks [b0, b1), values [v0, v1).
struct alignas(32) spaden_tile_desc_s {
    int32_t br0, br1, b0, b1, v0, v1, pad0, pad1;
};

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

    // SpMV schedule (aux, schedule.cu)
    int64_t aux_bytes = 0;
    int64_t n_tiles = 0;                       // whole-block-row tiles
    int64_t n_long = 0;                        // block-rows too large for a tile
    int tile_cfg = 0;                          // spaden::tile_cfg index the schedule was built for
    struct spaden_tile_desc_s *tiles = nullptr; // [n_tiles] (spaden::TileDesc)
    uint8_t *rot = nullptr;                    // [Bnnz] per-block row rotation of the slot decode (bank
                                               // conflicts, schedule.cu) or NULL (no rotation)
    int32_t *long_rows = nullptr;              // [n_long]
    int64_t n_chunks = 0;                      // kLongChunk-block chunks of the long rows
    int32_t *chunk_start = nullptr;            // [n_long+1] first chunk of each long row
    int32_t *chunk_row = nullptr;              // [n_chunks] index into long_rows
    float *carry = nullptr;                    // [kScratchSlots][n_chunks*8] per-chunk row partials
    int32_t *chunk_done = nullptr;             // [kScratchSlots][n_long] chunks finished per long row (0 between calls)
    // long-row scratch: one of kScratchSlots sets per spmv call (round robin), so
    // up to kScratchSlots calls on one handle may run concurrently on different streams
    static constexpr int kScratchSlots = 4;
    mutable std::atomic<uint32_t> scratch_next{0};

    // SpMM schedules for K = 2, 4 right-hand sides (index 0, 1; built lazily by spaden_spmm)
    struct spaden_tile_desc_s *spmm_tiles[3] = {};
    int64_t spmm_ntiles[3] = {};
    int spmm_state[3] = {};                    // 0 not built, 1 built, -1 unsupported
    // tensor-core SpMM chunk schedule (spmm_tc.cu, built by the first spaden_spmm_tc call)
    void *tc_chunks = nullptr;                 // [tc_nchunks] chunk descriptors
    int32_t *tc_cta_start = nullptr;           // [tc_grid + 1] first chunk of each CTA
    int tc_grid = 0;                           // CTAs the schedule was built for (0 = not built)
    int64_t tc_nchunks = 0;

    // hybrid residual (csrc/hybrid.cu), empty in pure bitBSR mode: a CSR with
    // global columns, split into column segments (parts) when x is larger than
    // kXSegBytes so that each part's x gathers stay L2-resident
    int64_t res_nnz = 0;
    int res_max_popc = 0;
    struct ResBins {                     // class c: perm[row_start[c], row_start[c+1]), CTAs from cta_start[c]
        int64_t row_start[8], cta_start[8];  // classes 0..kResClasses (the last: empty / long rows)
    };
    struct ResPart {
        int64_t col0 = 0, col1 = 0, nnz = 0;  // columns [col0, col1) of the residual
        int32_t *rowptr = nullptr;           // [m+1]
        int32_t *colidx = nullptr;           // [nnz]
        void *values = nullptr;              // [nnz]
        int64_t n_long = 0;                  // rows longer than kResLongRow (chunked)
        int64_t n_chunks = 0;
        int32_t *long_rows = nullptr;        // [n_long]
        int32_t *chunk_start = nullptr;      // [n_long+1]
        int32_t *chunk_row = nullptr;        // [n_chunks] index into long_rows
        float *carry = nullptr;              // [kScratchSlots][n_chunks]
        int32_t *done = nullptr;             // [kScratchSlots][n_long] chunks finished per long row (0 between calls)
        int32_t *perm = nullptr;             // all rows, grouped by length class (then empty / long rows)
        ResBins bins = {};
    };
    static constexpr int kMaxResParts = 16;
    ResPart res[kMaxResParts];
    int n_res_parts = 0;
    int64_t res_aux_bytes = 0;           // perms, long-row chunk lists, per-part rowptrs beyond the first

    // host-API staging buffers (lazily allocated): [2] slots for the batched pipeline
    float *stage_x = nullptr;          // spaden_spmv_host
    float *stage_y = nullptr;
    static constexpr int kMaxPipe = 8;  // spaden_spmv_host_batched: up to kMaxPipe slots
    int pipe_slots = 0;                 // slots in use (SPADEN_PIPE_SLOTS, default kDefaultPipe)
    float *pipe_x[kMaxPipe] = {};
    float *pipe_y[kMaxPipe] = {};
    cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
    cudaEvent_t ev[3 * kMaxPipe + 2] = {};
};

namespace spaden {

using Matrix = ::spaden_matrix_s;

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
// Launch shape of the tiled SpMV kernel: CTAs per SM, consumer warps per CTA,
// pipeline stages and bytes per stage.  A tile (whole block-rows) must fit one
// stage including the 16-byte alignment slack of its regions.
struct TileCfg {
    int ctas_per_sm, consumers, stages, stage_bytes;
};
constexpr int kMaxStages = 8;
// the launch shapes k_spmv_tiled is instantiated for (SPADEN_TILE_CFG selects one;
// every stage holds a block-row of kLongRowBytes plus kStageSlack)
inline bool tile_cfg_valid(int i) {
    switch (i) {
    case 1: case 2: case 3: case 5: case 6: case 7: case 10: case 14: case 15: case 16: return true;
    default: return false;
    }
}
__host__ __device__ inline TileCfg tile_cfg(int i) {
    switch (i) {
    case 1: return TileCfg{2, 16, 3, 36 * 1024};
    case 3: return TileCfg{4, 8, 2, 27 * 1024};
    case 5: return TileCfg{3, 8, 4, 18 * 1024};
    case 6: return TileCfg{2, 16, 6, 18 * 1024};
    case 7: return TileCfg{4, 8, 3, 18 * 1024};
    // 4 consumer warps per CTA: half the warps share (and wait on) each tile
    case 10: return TileCfg{6, 4, 2, 18 * 1024};
    // 2 CTAs per SM, deeper rings (4 stages)
    case 14: return TileCfg{2, 12, 4, 24 * 1024};
    case 15: return TileCfg{2, 16, 4, 27 * 1024};
    case 16: return TileCfg{2, 8, 4, 27 * 1024};
    default: return TileCfg{3, 8, 3, 24 * 1024};  // cfg 2
    }
}
int default_tile_cfg(int64_t format_bytes, int value_bytes);  // SPADEN_TILE_CFG override, else by matrix size
constexpr int kStageSlack = 384;
constexpr int64_t kSmallMatrixBytes = 64ll << 20;  // below: kSmallTileCfg
constexpr int kSmallTileCfg = 5;  // measured L2-flushed: fem62k 16.3 -> 15.1 us
// shared-memory bytes a block occupies in a stage: bitmap 8 + blk_col 4 +
// blk_offset 4 (copied) + 8 fp32 row partials at a 9-word stride (scratch)
constexpr int kBlockStageBytes = 16 + 36;
// + 1 byte per block when the schedule carries row rotations (the rotation region);
// the long-row cost (kLongRowBytes) is computed with kBlockStageBytes alone
constexpr int kBlockRotBytes = 1;
// row-rotated decode stores a block's 8 row partials as two 16-byte stores
// (spmv.cu block_slots_rot_v4): the rotation pass then models the value loads only
#ifndef SPADEN_ROT_V4
#define SPADEN_ROT_V4 1
#endif
// A block-row whose stage cost (kBlockStageBytes per block + its values + 4)
// exceeds kLongRowBytes is "long" (chunk path) whatever the tile config: the
// split between the tile path and the chunk path -- two different summation
// orders -- is then a function of the block-row alone, so y is bitwise the
// same for every 8-row-aligned partition (slices of different sizes pick
// different tile configs).  Every tile config holds such a row in one stage.
constexpr int64_t kLongRowBytes = 9 * 1024;
// long block-rows are split into chunks of this many blocks (relative to the
// block-row start, so the split depends only on the row itself)
#ifndef SPADEN_LONG_CHUNK
#define SPADEN_LONG_CHUNK 128
#endif
constexpr int kLongChunk = SPADEN_LONG_CHUNK;
// With at most this many chunks (latency-bound: about one wave of warps) the
// warp finishing a long row's last chunk does its fix-up; with more, a separate
// fix-up kernel runs after the chunks (the per-chunk fence + counter atomic
// costs more than the launch when chunks are many: DESIGN.md §5)
#ifndef SPADEN_FUSED_FIXUP_MAX
#define SPADEN_FUSED_FIXUP_MAX 8192
#endif
constexpr int64_t kFusedFixupMaxChunks = SPADEN_FUSED_FIXUP_MAX;
int64_t fused_fixup_max();  // kFusedFixupMaxChunks, or the SPADEN_FUSED_FIXUP_MAX environment override
// at most this many block-rows per tile: phase 2 of a tile runs on one warp, so
// runs of (nearly) empty block-rows are cut into many tiles
constexpr int kMaxTileRows = 128;
// hybrid residual rows: fixed 1024-entry chunks; rows above kResLongRow entries
// have their chunks processed in parallel (carry + ordered fix-up)
#ifndef SPADEN_RES_CHUNK
#define SPADEN_RES_CHUNK 256
#endif
constexpr int kResChunk = SPADEN_RES_CHUNK;
// lanes per residual row (the per-row summation tree has log2 of this many levels)
#ifndef SPADEN_RES_LANES
#define SPADEN_RES_LANES 16
#endif
constexpr int kResLanes = SPADEN_RES_LANES;
constexpr int kResLongRow = 4096;
// x bytes per residual column segment (part): a part's x slice plus the stream
// must stay in the 126 MB L2; larger x is split (SPADEN_XSEG_COLS overrides the
// columns per part, tests)
constexpr int64_t kXSegBytes = 64ll << 20;
// length classes of the binned residual pass: class c (L = 2^c lanes per row)
// holds rows of len entries with 4*2^(c-1) < len <= 4*2^c; the last class takes
// everything up to kResLongRow
constexpr int kResClasses = 6;
__host__ __device__ inline int res_class(int len) {
    int c = 0;
    while (c < kResClasses - 1 && len > (4 << c)) ++c;
    return c;
}
// mean nonzeros per block from which the predicated-slot decode is used
constexpr int kSlotsMinFill = 8;
// hybrid threshold of the automatic choice (residual_max_popc = -1)
constexpr int kAutoResidualPopc = 4;
// decode used above that fill (1 = lane per block, 2 = lane per block row)
constexpr int kDenseDecode = 1;

using TileDesc = ::spaden_tile_desc_s;
using ResBins = ::spaden_matrix_s::ResBins;
using ResPart = ::spaden_matrix_s::ResPart;

spaden_status_t build_schedule(Matrix *A, cudaStream_t stream);
spaden_status_t build_spmm_schedule(Matrix *A, int kidx, int K, cudaStream_t stream);


// Fused SpMV + all-gather: besides (or instead of) y,
// every y value is stored at ptr[p][offset + row] for each of the n peer
// buffers (NVLink-mapped x_next slices of the other GPUs, plus the local one).
constexpr int kMaxPeers = 8;
struct PeerOut {
    float *ptr[kMaxPeers];
    int32_t n;
    int32_t pad;
    int64_t offset;
};

// converter (convert.cu)
spaden_status_t convert_csr(int64_t m, int64_t n, int64_t nnz, const int32_t *rowptr,
                            const int32_t *colidx, const void *values, spaden_dtype_t vdt,
                            spaden_dtype_t sdt, int residual_max_popc, float auto_mean_fill,
                            cudaStream_t stream, Matrix *A, bool count_only = false);

// hybrid split (hybrid.cu): move blocks with popc <= t into a CSR residual
spaden_status_t split_residual(Matrix *A, int t, cudaStream_t stream);
// hybrid SpMV, first part: y = beta*y + alpha*A_res*x on every row (y not read
// when beta = 0); the bitBSR kernels follow with beta = 1
// (*launched: whether it launched any kernel -- later kernels of the call use
// programmatic dependent launch only then)
cudaError_t residual_first(const Matrix &A, float alpha, const float *x, float beta, float *y, cudaStream_t stream,
                           int slot, bool *launched);
// scratch set of one spmv call (Matrix::kScratchSlots round robin)
inline int pick_scratch(const Matrix &A) {
    return (int)(A.scratch_next.fetch_add(1u, std::memory_order_relaxed) % (uint32_t)Matrix::kScratchSlots);
}
bool residual_binned_enabled(const Matrix &A);  // binned residual kernel (not the SPADEN_RES=fixed ablation)

// SpMV (spmv.cu)
spaden_status_t spmv_launch(const Matrix &A, float alpha, const float *x, float beta, float *y,
                            cudaStream_t stream, const PeerOut *peers = nullptr);
int spmv_launch_count(const Matrix &A, float beta);  // launches of one spmv_launch (no peers)
// SpMM: k column-major vectors (spmv.cu)
spaden_status_t spmm_launch(Matrix &A, float alpha, const float *X, int64_t ldx, int k, float beta, float *Y,
                            int64_t ldy, cudaStream_t stream);

// tensor-core SpMM (spmm_tc.cu)
spaden_status_t spmm_tc_pack_x(int64_t n, int32_t k, const float *X, int64_t ldx, void *Xb, cudaStream_t stream);
spaden_status_t spmm_tc_launch(Matrix &A, float alpha, const void *Xb, int32_t k, float beta, float *Y,
                               int64_t ldy, cudaStream_t stream);  // builds the chunk schedule at the first call

// reordering (reorder.cu)
spaden_status_t degree_order(int64_t m, const int32_t *rowptr, int32_t *perm, cudaStream_t st);
spaden_status_t permute_csr(int64_t m, int64_t nnz, const int32_t *rowptr, const int32_t *colidx, const void *values,
                            int value_bytes, const int32_t *perm, int32_t *out_rowptr, int32_t *out_colidx,
                            void *out_values, cudaStream_t st);

// exclusive scan of int32 (scan.cu): out[i] = sum_{j<i} in[j], out[count] = total.
// `in` and `out` may alias.  tmp must hold scan_tmp_ints(count) int32.
size_t scan_tmp_ints(int64_t count);
cudaError_t exclusive_scan_i32(const int32_t *in, int32_t *out, int64_t count, int32_t *tmp,
                               cudaStream_t stream);

// Programmatic dependent launch (PDL): a kernel launched with launch_k(dep =
// true, ...) may start while the previous kernel of the same SpMV call still
// runs (its prologue and the work that reads only A and x overlap the
// predecessor's tail); it calls pdl_wait() before touching anything the
// predecessor writes (y, chunk carries).  Only kernels that follow another
// kernel of the same call use it, so x -- produced before the call -- is
// complete.  Both device calls are no-ops under a normal launch.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
bool pdl_enabled();  // SPADEN_PDL=0 disables (A/B), read per call
template <typename... KArgs, typename... Args>
cudaError_t launch_k(bool dep, void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                     Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    if (dep && pdl_enabled()) {
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
    }
    return cudaLaunchKernelEx(&cfg, kernel, args...);
}

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

// Device memory of handles and conversion scratch: stream-ordered allocations
// from a library-private pool per device (capi.cu) that keeps up to
// kPoolKeepBytes of freed memory mapped, so converting again after
// spaden_free does not pay the driver's map/unmap (conversion time is then
// stable from the second conversion on).  dev_free is stream ordered as well.
constexpr uint64_t kPoolKeepBytes = 4ull << 30;
cudaError_t dev_alloc(void **ptr, size_t bytes, cudaStream_t st);
void dev_free(void *ptr, cudaStream_t st);
template <typename T> inline cudaError_t dmalloc(T **ptr, size_t bytes, cudaStream_t st) {
    return dev_alloc(reinterpret_cast<void **>(ptr), bytes, st);
}

}  // namespace spaden
