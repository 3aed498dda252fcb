// spmv.cu -- y = alpha*A*x + beta*y over bitBSR on sm_100a CUDA cores
// (§4.3).
//
// v0 mapping ("row-byte lanes"): one warp per block-row ("each row of
// blocks ... is computed with a segment of x with length 8, producing a segment
// of y with length 8").  The warp walks the block-row four blocks at a time; the
// 8 lanes of group g = lane/8 take block b0+g+4i and lane r = lane%8 owns row r of
// that block, i.e. byte r of the bitmap.  Its first value sits at
// blk_offset[b] + popc(bitmap & ((1<<8r)-1)) (popcount rank, reading R1 of
// Alg. 2); the 8 bit slots are unrolled and predicated on the byte,
// so structural zeros are neither loaded nor multiplied (reading R11).
// x[8*bc .. 8*bc+7] is one 32-byte sector read as two float4 broadcasts
// (Alg. 2 lines 7-10).  Each lane accumulates its row over the
// block-row in fp32; the four groups are combined with two xor-shuffles in a
// fixed order, so the result depends only on the block-row's own blocks.
#include "internal.cuh"

namespace spaden {
namespace {

constexpr unsigned kFull = 0xffffffffu;

template <typename V> __device__ __forceinline__ float ldv(const V *p);
template <> __device__ __forceinline__ float ldv<float>(const float *p) { return __ldg(p); }
template <> __device__ __forceinline__ float ldv<__half>(const __half *p) {
    return __half2float(__ldg(p));
}

template <typename V>
__global__ void __launch_bounds__(256)
k_spmv_v0(int64_t m, int64_t n, int64_t Bnrow, const int32_t *__restrict__ blk_rowptr,
          const int32_t *__restrict__ blk_col, const uint64_t *__restrict__ bitmap,
          const int32_t *__restrict__ blk_offset, const V *__restrict__ vals,
          const float *__restrict__ x, bool x_vec, float alpha, float beta, float *__restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int g = lane >> 3, r = lane & 7;
    const int64_t nwarps = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t br = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); br < Bnrow;
         br += nwarps) {
        const int b0 = __ldg(blk_rowptr + br), b1 = __ldg(blk_rowptr + br + 1);
        float acc = 0.f;
        for (int b = b0 + g; b < b1; b += 4) {
            const uint64_t bmp = __ldg(bitmap + b);
            const int bc = __ldg(blk_col + b);
            const int off = __ldg(blk_offset + b);
            const uint32_t byte = (uint32_t)(bmp >> (8 * r)) & 0xffu;
            int p = off + __popcll(bmp & ((1ull << (8 * r)) - 1ull));
            const float *xs = x + 8 * (int64_t)bc;
            float xv[8];
            if (x_vec && 8 * (int64_t)bc + 8 <= n) {
                const float4 lo = __ldg(reinterpret_cast<const float4 *>(xs));
                const float4 hi = __ldg(reinterpret_cast<const float4 *>(xs) + 1);
                xv[0] = lo.x; xv[1] = lo.y; xv[2] = lo.z; xv[3] = lo.w;
                xv[4] = hi.x; xv[5] = hi.y; xv[6] = hi.z; xv[7] = hi.w;
            } else {  // ragged last block column / unaligned x: read only referenced entries
#pragma unroll
                for (int c = 0; c < 8; ++c) xv[c] = ((byte >> c) & 1u) ? __ldg(xs + c) : 0.f;
            }
#pragma unroll
            for (int c = 0; c < 8; ++c) {
                if ((byte >> c) & 1u) {
                    acc = fmaf(ldv<V>(vals + p), xv[c], acc);
                    ++p;
                }
            }
        }
        acc += __shfl_xor_sync(kFull, acc, 8);
        acc += __shfl_xor_sync(kFull, acc, 16);
        const int64_t row = 8 * br + r;
        if (g == 0 && row < m) {
            float o = alpha * acc;
            if (beta != 0.f) o = fmaf(beta, y[row], o);
            y[row] = o;
        }
    }
}

}  // namespace

spaden_status_t spmv_launch(const Matrix &A, float alpha, const float *x, float beta, float *y,
                            cudaStream_t st) {
    if (A.m == 0) return SPADEN_OK;
    const int threads = 256;
    const int64_t want = (A.Bnrow + 7) / 8;
    const unsigned grid = (unsigned)std::min<int64_t>(want, 148LL * 64);
    const bool x_vec = ((uintptr_t)x & 15u) == 0;
    if (A.storage == SPADEN_R_16F)
        k_spmv_v0<__half><<<grid, threads, 0, st>>>(A.m, A.n, A.Bnrow, A.blk_rowptr, A.blk_col, A.bitmap,
                                                   A.blk_offset, (const __half *)A.values, x, x_vec, alpha, beta, y);
    else
        k_spmv_v0<float><<<grid, threads, 0, st>>>(A.m, A.n, A.Bnrow, A.blk_rowptr, A.blk_col, A.bitmap,
                                                  A.blk_offset, (const float *)A.values, x, x_vec, alpha, beta, y);
    SPADEN_CUDA_TRY(cudaGetLastError());
    return SPADEN_OK;
}

}  // namespace spaden
