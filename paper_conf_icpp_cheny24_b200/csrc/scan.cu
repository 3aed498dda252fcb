// scan.cu -- exclusive prefix sum of int32 counts (steps C2 and C4 of the
// converter: block-rowptr scan and per-chunk block/value offsets
// "computed with exclusive scan to determine the offset").
//
// Reduce-then-scan in three launches: per-tile sums, one CTA scanning the tile
// sums, per-tile scan + carry-in.  Tiles are 4096 ints (1024 threads x 4).
#include "internal.cuh"

namespace spaden {
namespace {

constexpr int kThreads = 1024;
constexpr int kItems = 4;
constexpr int kTile = kThreads * kItems;

__device__ __forceinline__ int block_excl_scan(int v, int *smem_warp, int *total) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    int wt;
    int ex = warp_excl_scan_i32(v, lane, &wt);
    if (lane == 0) smem_warp[warp] = wt;
    __syncthreads();
    if (warp == 0) {
        int s = smem_warp[lane];
        int t;
        int e = warp_excl_scan_i32(s, lane, &t);
        smem_warp[lane] = e;
        if (lane == 0) smem_warp[32] = t;
    }
    __syncthreads();
    int r = ex + smem_warp[warp];
    *total = smem_warp[32];
    __syncthreads();
    return r;
}

__global__ void __launch_bounds__(kThreads) k_tile_sums(const int32_t *__restrict__ in, int64_t count,
                                                        int32_t *__restrict__ sums) {
    __shared__ int sm[33];
    int64_t base = (int64_t)blockIdx.x * kTile;
    int v = 0;
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
        int64_t k = base + (int64_t)i * kThreads + threadIdx.x;
        if (k < count) v += in[k];
    }
    int tot;
    block_excl_scan(v, sm, &tot);
    if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

// single CTA: exclusive scan of `n` tile sums in place, total appended at sums[n]
__global__ void __launch_bounds__(kThreads) k_scan_sums(int32_t *sums, int64_t n) {
    __shared__ int sm[33];
    int carry = 0;
    for (int64_t base = 0; base < n; base += kThreads) {
        int64_t k = base + threadIdx.x;
        int v = k < n ? sums[k] : 0;
        int tot;
        int e = block_excl_scan(v, sm, &tot);
        if (k < n) sums[k] = carry + e;
        carry += tot;
    }
    if (threadIdx.x == 0) sums[n] = carry;
}

__global__ void __launch_bounds__(kThreads) k_tile_scan(const int32_t *in, int32_t *out, int64_t count,
                                                        const int32_t *__restrict__ sums) {
    __shared__ int sm[33];
    int64_t base = (int64_t)blockIdx.x * kTile + (int64_t)threadIdx.x * kItems;  // blocked layout
    int v[kItems];
    int local = 0;
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
        int64_t k = base + i;
        v[i] = k < count ? in[k] : 0;
        local += v[i];
    }
    int tot;
    int run = block_excl_scan(local, sm, &tot) + sums[blockIdx.x];
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
        int64_t k = base + i;
        if (k < count) out[k] = run;
        run += v[i];
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) out[count] = sums[gridDim.x];
}

}  // namespace

size_t scan_tmp_ints(int64_t count) { return (size_t)((count + kTile - 1) / kTile) + 2; }

cudaError_t exclusive_scan_i32(const int32_t *in, int32_t *out, int64_t count, int32_t *tmp,
                               cudaStream_t stream) {
    if (count <= 0) return cudaMemsetAsync(out, 0, sizeof(int32_t), stream);
    int64_t tiles = (count + kTile - 1) / kTile;
    k_tile_sums<<<(unsigned)tiles, kThreads, 0, stream>>>(in, count, tmp);
    k_scan_sums<<<1, kThreads, 0, stream>>>(tmp, tiles);
    k_tile_scan<<<(unsigned)tiles, kThreads, 0, stream>>>(in, out, count, tmp);
    return cudaGetLastError();
}

}  // namespace spaden
