// spmv.cu -- y = alpha*A*x + beta*y over bitBSR on sm_100a CUDA cores
// (§4.3).
//
// k_spmv_tiled: persistent CTAs fed by a TMA bulk-copy pipeline, and
// k_spmv_long_chunks (chunks + fused fix-up) for block-rows too large for a
// pipeline stage.
//
// Decode (both kernels follow PAPER.md §4.3.1 / Alg. 2 semantics):
// bit 8r+c of a block's bitmap is entry (r, c); its value is the
// next one in the block's packed run because values are stored in ascending
// bit order ("stored consecutively") -- i.e. the value index of a set
// bit is blk_offset + popcount of the lower bits (reading R1 of Alg. 2 lines
// 5-6).  Only set bits load a value or touch x ("zero elements are calculated
// instead of loading from memory"): structural zeros are never
// multiplied (reading R11).  x[8bc .. 8bc+7] is the block's 8-element segment
// (Alg. 2 lines 7-10).
#include <mutex>
#include <cstddef>
#include <cstdlib>

#include "internal.cuh"

namespace spaden {
namespace {

constexpr unsigned kFull = 0xffffffffu;

template <typename V> __device__ __forceinline__ float ldv(const V *p);
template <> __device__ __forceinline__ float ldv<float>(const float *p) { return __ldg(p); }
template <> __device__ __forceinline__ float ldv<__half>(const __half *p) {
    return __half2float(__ldg(p));
}

// ==========================================================================
// Tiled kernel: persistent CTAs, TMA bulk-copy pipeline through shared memory.
//
// Warp 0 (one elected lane) is the producer; warps 1..CONSUMERS consume.
// Tiles (schedule.cu: runs of whole block-rows) go round-robin to CTAs,
// tile t -> CTA t % gridDim.x.  Per tile the producer waits for the ring slot
// (mbarrier "empty"), writes a header, and issues cp.async.bulk copies of the
// bitmap, blk_col, blk_offset, blk_rowptr and value slices (16-byte-aligned
// supersets) completing on the slot's "full" mbarrier (complete_tx), with an
// L2 evict-first policy (the matrix is streamed once; x stays resident).
//
// Phase 1 (decode): the tile's blocks are cut into units of 32 consecutive
// blocks, grabbed dynamically by the consumer warps (shared counter).  One
// lane per block: it walks the 64 bit slots in ascending bit order (predicated,
// or a set-bit loop for low-fill matrices -- same arithmetic) and writes the
// block's 8 row partials to a scratch area of the stage.
// Phase 2 (reduce): the warp whose completion count finishes the tile sums, for each
// block-row and row, the block partials in a fixed order (4 interleaved chains
// by block index within the block-row, then (c0+c1)+(c2+c3)) and stores y.
// The summation order depends only on the block-row, so any 8-row-aligned row
// partition of A produces bitwise identical y.
// ==========================================================================


__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
// try_wait suspends the warp (up to the hint) instead of spinning: waiting
// warps then cost no issue slots
constexpr uint32_t kSuspendHintNs = 0x989680;
#ifndef SPADEN_AVAIL_SLEEP_NS
#define SPADEN_AVAIL_SLEEP_NS 64  // back-off of a consumer waiting for its unit's tile to be published
#endif
__device__ __forceinline__ bool mbar_try_wait(uint32_t bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(ok)
        : "r"(bar), "r"(parity), "r"(kSuspendHintNs)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar,
                                         uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], "
        "%4;" ::"r"(dst),
        "l"(src), "r"(bytes), "r"(bar), "l"(policy)
        : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint2 lds_u2(uint32_t a) {
    uint2 v;
    asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}
__device__ __forceinline__ int lds_i32(uint32_t a) {
    int v;
    asm("ld.shared.s32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ float lds_f32(uint32_t a) {
    float v;
    asm("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u8(uint32_t a) {
    unsigned short v;
    asm("ld.shared.u8 %0, [%1];" : "=h"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ float lds_f16(uint32_t a) {
    unsigned short h;
    asm("ld.shared.u16 %0, [%1];" : "=h"(h) : "r"(a));
    return __half2float(__ushort_as_half(h));
}
// header loads must stay below the full-barrier wait: volatile + memory clobber
__device__ __forceinline__ int4 lds_i4_volatile(uint32_t a) {
    int4 v;
    asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ int atom_add_shared(uint32_t a, int v) {
    int old;
    asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(a), "r"(v) : "memory");
    return old;
}
__device__ __forceinline__ void sts_f32(uint32_t a, float v) {
    asm volatile("st.shared.f32 [%0], %1;" ::"r"(a), "f"(v) : "memory");
}
// row partials of a block: 8 floats at a 9-word stride (bank-conflict-free
// per-lane stores and phase-2 reads)
constexpr uint32_t kPartStride = 36;
// row-rotated decode (ROT): the 8 row partials of a block, un-rotated in
// registers, leave as two 16-byte stores at a 32-byte stride (conflict free)
constexpr bool kRotV4 = SPADEN_ROT_V4 != 0;
constexpr uint32_t kPartStrideV4 = 32;

// Value source of a block's packed run: shared-memory stage or global memory.
template <typename V> struct SmemVals {
    using P = uint32_t;  // shared byte address
    static __device__ __forceinline__ float get(P p) {
        if constexpr (sizeof(V) == 2) return lds_f16(p);
        else return lds_f32(p);
    }
    static constexpr uint32_t step = sizeof(V);
};
template <typename V> struct GlobalVals {
    using P = const V *;
    static __device__ __forceinline__ float get(P p) { return ldv<V>(p); }
    static constexpr int step = 1;
};

struct XSeg {
    float v[8];
};

// nbc_vec = number of leading block columns whose x segment may be read as one
// 32-byte vector (n/8 when x is 32-byte aligned, else 0); other segments read only the
// columns referenced by `cols` (bit c set = column c used by the block).
// texx != 0: x is also bound to a 1-D float4 texture; aligned segments are then
// fetched through the texture pipe (TLD), which has its own L1TEX data path, so
// the LSU data pipe -- the kernel's bottleneck, saturated by the shared-memory
// value loads -- only carries smem traffic.
__device__ __forceinline__ void load_x(XSeg &xs, const float *__restrict__ x, int bc, int nbc_vec, uint32_t cols,
                                       unsigned long long texx = 0ull, int tex_off = 0) {
    const float *p = x + 8 * (int64_t)bc;
    if (texx && bc < nbc_vec) {  // tex_off: float4 index of x in the texture (SpMM vector j)
        const float4 a = tex1Dfetch<float4>((cudaTextureObject_t)texx, tex_off + 2 * bc);
        const float4 b = tex1Dfetch<float4>((cudaTextureObject_t)texx, tex_off + 2 * bc + 1);
        xs.v[0] = a.x, xs.v[1] = a.y, xs.v[2] = a.z, xs.v[3] = a.w;
        xs.v[4] = b.x, xs.v[5] = b.y, xs.v[6] = b.z, xs.v[7] = b.w;
    } else if (bc < nbc_vec) {  // one 32-byte sector, one 256-bit load (LDG.E.ENL2.256)
        asm("ld.global.nc.v8.f32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
            : "=f"(xs.v[0]), "=f"(xs.v[1]), "=f"(xs.v[2]), "=f"(xs.v[3]), "=f"(xs.v[4]), "=f"(xs.v[5]),
              "=f"(xs.v[6]), "=f"(xs.v[7])
            : "l"(p));
    } else {
#pragma unroll
        for (int c = 0; c < 8; ++c) xs.v[c] = ((cols >> c) & 1u) ? __ldg(p + c) : 0.f;
    }
}

__device__ __forceinline__ uint32_t used_cols(uint2 bm) {
    uint32_t w = bm.x | bm.y;
    w |= w >> 16;
    w |= w >> 8;
    return w & 0xffu;
}

// Row partials of one block, 64 predicated slots in ascending bit order.  Each
// row starts at its own popcount rank (P:L138 exclusive counts), so the eight
// rows are independent dependency chains of at most 8 slots.  pA / pB: first
// value of rows 0-3 / rows 4-7 of the half-words bm.x / bm.y (block_slots_at
// lets a caller hand in the two bitmap halves swapped, see SwapHalves).
template <class VS>
__device__ __forceinline__ void block_slots_at(uint2 bm, typename VS::P pA, typename VS::P pB, const XSeg &xs,
                                               float acc[8]) {
#pragma unroll
    for (int r = 0; r < 8; ++r) {
        const uint32_t w = r < 4 ? bm.x : bm.y;
        const uint32_t byte = (w >> (8 * (r & 3))) & 0xffu;
        const int below = (r & 3) == 0 ? 0 : __popc(w & ((1u << (8 * (r & 3))) - 1u));
        typename VS::P p = (r < 4 ? pA : pB) + below * VS::step;
        float a = 0.f;
#pragma unroll
        for (int c = 0; c < 8; ++c) {
            if ((byte >> c) & 1u) {
                a = fmaf(VS::get(p), xs.v[c], a);
                p += VS::step;
            }
        }
        acc[r] = a;
    }
}

// Slot decode of one block walking its rows in the cyclic order rho, rho+1, ...
// (rho from the schedule's bank-conflict pass, schedule.cu): step t decodes
// original row (t + rho) & 7, whose values start at popcount rank
// below(row) = (below_rot(t) + below(rho)) mod popc(bm).  Each row is still one
// fma chain over its columns in ascending order, stored to its own partial
// slot, so the result does not depend on rho.  Partials go to q + 4*row.
template <class VS>
__device__ __forceinline__ void block_slots_rot(uint2 bm, uint32_t rho, typename VS::P p0, const XSeg &xs,
                                                uint32_t q) {
    const uint64_t b = ((uint64_t)bm.y << 32) | bm.x;
    const uint32_t sh = 8u * rho;
    const uint64_t rb = sh ? ((b >> sh) | (b << (64u - sh))) : b;  // row t of rb = row (t+rho)&7 of b
    const int P = __popcll(b);
    const int B = __popcll(b & ((1ull << sh) - 1ull));             // values of rows < rho
    const uint32_t rlo = (uint32_t)rb, rhi = (uint32_t)(rb >> 32);
#pragma unroll
    for (int t = 0; t < 8; ++t) {
        const uint32_t w = t < 4 ? rlo : rhi;
        const uint32_t byte = (w >> (8 * (t & 3))) & 0xffu;
        int below = (t & 3) == 0 ? 0 : __popc(w & ((1u << (8 * (t & 3))) - 1u));
        if (t >= 4) below += __popc(rlo);
        int start = below + B;
        start = start >= P ? start - P : start;  // rows of the wrapped part
        typename VS::P p = p0 + start * VS::step;
        float a = 0.f;
#pragma unroll
        for (int c = 0; c < 8; ++c) {
            if ((byte >> c) & 1u) {
                a = fmaf(VS::get(p), xs.v[c], a);
                p += VS::step;
            }
        }
        sts_f32(q + 4u * ((uint32_t)(t + rho) & 7u), a);
    }
}

__device__ __forceinline__ void sts_v4(uint32_t a, float x, float y, float z, float w) {
    asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(a), "f"(x), "f"(y), "f"(z), "f"(w) : "memory");
}

// block_slots_rot with the partials kept in registers: step t computes original
// row (t + rho) & 7; a two-stage select network rotates the 8 sums back into
// row order (by rho & 3), rotation by 4 swaps the two 16-byte stores.  Same
// fma chains as block_slots_rot.
template <class VS>
__device__ __forceinline__ void block_slots_rot_v4(uint2 bm, uint32_t rho, typename VS::P p0, const XSeg &xs,
                                                   uint32_t q) {
    const uint64_t b = ((uint64_t)bm.y << 32) | bm.x;
    const uint32_t sh = 8u * rho;
    const uint64_t rb = sh ? ((b >> sh) | (b << (64u - sh))) : b;
    const int P = __popcll(b);
    const int B = __popcll(b & ((1ull << sh) - 1ull));
    const uint32_t rlo = (uint32_t)rb, rhi = (uint32_t)(rb >> 32);
    float acc[8];
#pragma unroll
    for (int t = 0; t < 8; ++t) {
        const uint32_t w = t < 4 ? rlo : rhi;
        const uint32_t byte = (w >> (8 * (t & 3))) & 0xffu;
        int below = (t & 3) == 0 ? 0 : __popc(w & ((1u << (8 * (t & 3))) - 1u));
        if (t >= 4) below += __popc(rlo);
        int start = below + B;
        start = start >= P ? start - P : start;
        typename VS::P p = p0 + start * VS::step;
        float a = 0.f;
#pragma unroll
        for (int c = 0; c < 8; ++c) {
            if ((byte >> c) & 1u) {
                a = fmaf(VS::get(p), xs.v[c], a);
                p += VS::step;
            }
        }
        acc[t] = a;
    }
    // row r = (t + rho) & 7 holds acc[t]: o[r] = acc[(r - rho) & 7]
    float s1[8], s2[8];
    const bool r1 = rho & 1u, r2 = rho & 2u;
#pragma unroll
    for (int i = 0; i < 8; ++i) s1[i] = r1 ? acc[(i + 7) & 7] : acc[i];
#pragma unroll
    for (int i = 0; i < 8; ++i) s2[i] = r2 ? s1[(i + 6) & 7] : s1[i];
    const uint32_t lo = (rho & 4u) ? 16u : 0u;
    sts_v4(q + lo, s2[0], s2[1], s2[2], s2[3]);
    sts_v4(q + (16u - lo), s2[4], s2[5], s2[6], s2[7]);
}

template <class VS>
__device__ __forceinline__ void block_slots(uint2 bm, typename VS::P p0, const XSeg &xs, float acc[8]) {
    block_slots_at<VS>(bm, p0, p0 + __popc(bm.x) * VS::step, xs, acc);
}

// Bank-conflict breaker for 2-byte values: lanes with bit 1 of
// the lane index set walk rows 4-7 before rows 0-3.  Neighbouring blocks have
// similar bitmaps and fp16 runs ~11 words apart, so at a given slot their
// value loads otherwise collide in the same banks far more often than at
// random; the swap breaks that correlation (simulated 4.31 -> 3.88 wavefronts
// per block on fem62k).  Each row keeps its own fma order: y is unchanged.
struct SwapHalves {
    bool on;
    __device__ __forceinline__ uint2 bitmap(uint2 bm) const { return on ? make_uint2(bm.y, bm.x) : bm; }
    // shared byte offset of the partial of the decoded row index r
    __device__ __forceinline__ uint32_t part_off(int r) const { return 4u * (uint32_t)(on ? (r ^ 4) : r); }
};

// The same partials by iterating the set bits (fewer instructions when the
// block holds few nonzeros); identical fma sequence per row.
template <class VS>
__device__ __forceinline__ void block_bits(uint2 bm, typename VS::P p, const float *__restrict__ xseg,
                                           float acc[8]) {
#pragma unroll
    for (int r = 0; r < 8; ++r) {
        uint32_t byte = ((r < 4 ? bm.x : bm.y) >> (8 * (r & 3))) & 0xffu;
        float a = 0.f;
        while (byte) {
            const int c = __ffs(byte) - 1;
            byte &= byte - 1;
            a = fmaf(VS::get(p), __ldg(xseg + c), a);
            p += VS::step;
        }
        acc[r] = a;
    }
}

// Final store of y[row]: local y, and/or the peer buffers of the fused
// all-gather (plain st.global through NVLink-mapped addresses).
__device__ __forceinline__ void store_y(float *__restrict__ y, int64_t row, float o, const PeerOut &po) {
    if (po.n == 0) {
        y[row] = o;
        return;
    }
    if (y) y[row] = o;
#pragma unroll
    for (int p = 0; p < kMaxPeers; ++p)
        if (p < po.n) po.ptr[p][po.offset + row] = o;
}

// Phase 2: y for every block-row of a tile from the per-block row partials
// (9-word stride), 4 block-rows x 8 rows per warp pass, 4 chains per row
// indexed by block position within the block-row, combined (c0+c1)+(c2+c3).
template <uint32_t kStride = kPartStride>
__device__ __forceinline__ void reduce_tile(uint32_t a_rp, uint32_t a_part, int nbr, int b0, int br0, int lane,
                                            int64_t m, float alpha, float beta, float *__restrict__ y,
                                            const PeerOut &po) {
    const int r = lane & 7;
    for (int base = 0; base < nbr; base += 4) {
        const int brl = base + (lane >> 3);
        if (brl < nbr) {
            const int k0 = lds_i32(a_rp + 4u * brl) - b0;
            const int k1 = lds_i32(a_rp + 4u * (brl + 1)) - b0;
            float c0 = 0.f, c1 = 0.f, c2 = 0.f, c3 = 0.f;
            uint32_t q = a_part + kStride * k0 + 4u * r;
            int k = k0;
            for (; k + 3 < k1; k += 4, q += 4 * kStride) {
                c0 += lds_f32(q);
                c1 += lds_f32(q + kStride);
                c2 += lds_f32(q + 2 * kStride);
                c3 += lds_f32(q + 3 * kStride);
            }
            if (k < k1) c0 += lds_f32(q);
            if (k + 1 < k1) c1 += lds_f32(q + kStride);
            if (k + 2 < k1) c2 += lds_f32(q + 2 * kStride);
            const float sum = (c0 + c1) + (c2 + c3);
            const int64_t row = 8 * ((int64_t)br0 + brl) + r;
            if (row < m) {
                float o = alpha * sum;
                if (beta != 0.f) o = fmaf(beta, y[row], o);
                store_y(y, row, o, po);
            }
        }
    }
}

// Phase 2 for K right-hand sides: partials of a block are [r][j] at a
// 4(8K+1)-byte stride; entry idx = (block-row, r, j); same chain order as
// reduce_tile, so column j equals the SpMV of vector j bitwise.
template <int K>
__device__ __forceinline__ void reduce_tile_k(uint32_t a_rp, uint32_t a_part, int nbr, int b0, int br0, int lane,
                                              int64_t m, float alpha, float beta, float *__restrict__ y,
                                              int64_t ldy) {
    constexpr uint32_t PS = 4u * (8 * K + 1);
    for (int idx = lane; idx < nbr * 8 * K; idx += 32) {
        const int brl = idx / (8 * K), rj = idx % (8 * K);
        const int r = rj / K, j = rj % K;
        const int k0 = lds_i32(a_rp + 4u * brl) - b0;
        const int k1 = lds_i32(a_rp + 4u * (brl + 1)) - b0;
        float c0 = 0.f, c1 = 0.f, c2 = 0.f, c3 = 0.f;
        uint32_t q = a_part + PS * k0 + 4u * rj;
        int k = k0;
        for (; k + 3 < k1; k += 4, q += 4 * PS) {
            c0 += lds_f32(q);
            c1 += lds_f32(q + PS);
            c2 += lds_f32(q + 2 * PS);
            c3 += lds_f32(q + 3 * PS);
        }
        if (k < k1) c0 += lds_f32(q);
        if (k + 1 < k1) c1 += lds_f32(q + PS);
        if (k + 2 < k1) c2 += lds_f32(q + 2 * PS);
        const float sum = (c0 + c1) + (c2 + c3);
        const int64_t row = 8 * ((int64_t)br0 + brl) + r;
        if (row < m) {
            float *yp = y + (int64_t)j * ldy + row;
            float o = alpha * sum;
            if (beta != 0.f) o = fmaf(beta, *yp, o);
            *yp = o;
        }
    }
}

// Phase 1 for K right-hand sides: one lane per block, 64 predicated slots, each
// loaded value multiplied into K accumulators (per-row, same fma order as
// block_slots for every vector); partials stored [r][j].
template <class VS, int K>
__device__ __forceinline__ void block_slots_k(uint2 bm, typename VS::P p0, const XSeg (&xs)[K], uint32_t q) {
    const int plo = __popc(bm.x);
#pragma unroll
    for (int r = 0; r < 8; ++r) {
        const uint32_t w = r < 4 ? bm.x : bm.y;
        const uint32_t byte = (w >> (8 * (r & 3))) & 0xffu;
        const int below = ((r & 3) == 0 ? 0 : __popc(w & ((1u << (8 * (r & 3))) - 1u))) + (r < 4 ? 0 : plo);
        typename VS::P p = p0 + below * VS::step;
        float a[K];
#pragma unroll
        for (int j = 0; j < K; ++j) a[j] = 0.f;
#pragma unroll
        for (int c = 0; c < 8; ++c) {
            if ((byte >> c) & 1u) {
                const float v = VS::get(p);
#pragma unroll
                for (int j = 0; j < K; ++j) a[j] = fmaf(v, xs[j].v[c], a[j]);
                p += VS::step;
            }
        }
#pragma unroll
        for (int j = 0; j < K; ++j) sts_f32(q + 4u * (r * K + j), a[j]);
    }
}

__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
    unsigned short h;
    asm("ld.shared.u16 %0, [%1];" : "=h"(h) : "r"(a));
    return h;
}

__device__ __forceinline__ uint32_t pack_f16x2(float lo, float hi) {
    uint32_t r;
    asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
    return r;
}

__device__ __forceinline__ float2 unpack_f16x2(uint32_t v) {
    return __half22float2(*reinterpret_cast<__half2 *>(&v));
}

__device__ __forceinline__ void mma16816(float d[4], const uint32_t a[4], uint32_t b0, uint32_t b1) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

// One 32-block unit through tensor cores (fp16 values): 8 MMAs of 4 blocks.
__device__ __forceinline__ void mma_unit(int lb0, int nb, int lane, uint32_t a_bmp, uint32_t a_col, uint32_t a_off,
                                         uint32_t a_val, int v0, uint32_t a_part, const float *__restrict__ x,
                                         int nbc_vec) {
    const int g = lane >> 2, t = lane & 3;
    const uint32_t mlo = lane < 16 ? (1u << (2 * lane)) - 1u : 0xffffffffu;
    const uint32_t mhi = lane < 16 ? 0u : (1u << (2 * lane - 32)) - 1u;
    const int sh = (2 * lane) & 31;
#pragma unroll 1
    for (int q = 0; q < 8; ++q) {
        uint32_t a[4];
        // fragment register order: {TL, BL, TR, BR} = blocks {P, R, Q, S} = {4q, 4q+2, 4q+1, 4q+3}
        const int order[4] = {0, 2, 1, 3};
#pragma unroll
        for (int f = 0; f < 4; ++f) {
            const int lb = lb0 + 4 * q + order[f];
            uint32_t reg = 0u;
            if (lb < nb) {
                const uint2 bm = lds_u2(a_bmp + 8u * lb);
                const uint32_t two = ((lane < 16 ? bm.x : bm.y) >> sh) & 3u;
                if (two) {
                    const int rank = __popc(bm.x & mlo) + __popc(bm.y & mhi);
                    const uint32_t p = a_val + 2u * (uint32_t)(lds_i32(a_off + 4u * lb) - v0 + rank);
                    const uint32_t h0 = (two & 1u) ? lds_u16(p) : 0u;
                    const uint32_t h1 = (two & 2u) ? lds_u16(p + 2u * (two & 1u)) : 0u;
                    reg = h0 | (h1 << 16);
                }
            }
            a[f] = reg;
        }
        // B: column g (< 4) holds block (4q+g)'s x segment in its k-half
        uint32_t bh0 = 0u, bh1 = 0u, bl0 = 0u, bl1 = 0u;
        const int lbx = lb0 + 4 * q + g;
        if (g < 4 && lbx < nb) {
            const int bc = lds_i32(a_col + 4u * lbx);
            const float *xp = x + 8 * (int64_t)bc + 2 * t;
            const uint2 bm = lds_u2(a_bmp + 8u * lbx);
            const uint32_t cols = used_cols(bm);
            float x0 = 0.f, x1 = 0.f;
            if (bc < nbc_vec) {
                const float2 v = __ldg(reinterpret_cast<const float2 *>(xp));
                x0 = v.x;
                x1 = v.y;
            } else {
                if ((cols >> (2 * t)) & 1u) x0 = __ldg(xp);
                if ((cols >> (2 * t + 1)) & 1u) x1 = __ldg(xp + 1);
            }
            const uint32_t hi = pack_f16x2(x0, x1);
            const float2 hf = unpack_f16x2(hi);
            const uint32_t lo = pack_f16x2(x0 - hf.x, x1 - hf.y);
            if (g & 1) {
                bh1 = hi;
                bl1 = lo;
            } else {
                bh0 = hi;
                bl0 = lo;
            }
        }
        float d[4] = {0.f, 0.f, 0.f, 0.f};
        mma16816(d, a, bh0, bh1);
        mma16816(d, a, bl0, bl1);
        // P row g = C[g][0], Q row g = C[g][1] (t = 0); R row g = C[g+8][2], S = C[g+8][3] (t = 1)
        if (t < 2) {
            const int lbA = lb0 + 4 * q + 2 * t, lbB = lbA + 1;
            const float vA = t == 0 ? d[0] : d[2], vB = t == 0 ? d[1] : d[3];
            if (lbA < nb) sts_f32(a_part + kPartStride * lbA + 4u * g, vA);
            if (lbB < nb) sts_f32(a_part + kPartStride * lbB + 4u * g, vB);
        }
    }
}

// per-stage tile header; the first 32 bytes are what every consumer warp needs
// to decode (two 16-byte loads), the next 16 only the phase-2 warp
struct alignas(16) StageHdr {
    int v0, nb;                                // first value, blocks
    uint32_t a_rot;                            // shared address of the row-rotation bytes (ROT)
    uint32_t a_val;                            // shared address of the value slice
    uint32_t a_bmp, a_col, a_off, a_part;      // ... of bitmap / blk_col / blk_offset; row-partial scratch
    int br0, nbr, b0;                          // tile block-rows, first block (phase 2)
    uint32_t a_rp;                             // ... of the blk_rowptr slice
};

// DEC: 0 = set-bit loop, 1 = 64 predicated slots per lane (lane = block; with
// ROT the rows in the schedule's bank-conflict rotation), 4 = tensor-core
// ablation (fp16).
//
// Work split inside a CTA: the producer lane stages the CTA's tiles through an
// S-stage ring; their 32-block units form one queue (numbered in tile order).
// A consumer warp takes the next unit number from a shared counter, waits
// until the producer has published the tile holding it (units_avail), finds
// its stage by unit range, waits for the data (full mbarrier), decodes the
// unit and counts it done on the stage; the warp that completes a tile runs
// its phase 2 and alone releases the stage (empty mbarrier, one arrival).  A
// warp therefore only touches the tiles it works on, and idle warps take the
// units of tiles whose other warps are still busy.
struct alignas(16) StageRange {
    int ustart, uend;  // the stage's tile holds queue units [ustart, uend)
    int parity, pad;   // full-barrier phase parity of that fill
};

template <typename V, int DEC, int CONSUMERS, int MINB, int K = 1, bool ROT = false>
__global__ void __launch_bounds__(32 * (CONSUMERS + 1), MINB)
k_spmv_tiled(int stages, int stage_bytes, int64_t m, const TileDesc *__restrict__ tiles, int ntiles, const int32_t *__restrict__ blk_rowptr,
             const int32_t *__restrict__ blk_col, const uint64_t *__restrict__ bitmap,
             const int32_t *__restrict__ blk_offset, const V *__restrict__ vals, const float *__restrict__ x,
             int nbc_vec, float alpha, float beta, float *__restrict__ y, int64_t ldx, int64_t ldy,
             const PeerOut po, unsigned long long texx, int wait_y, const uint8_t *__restrict__ rot) {
    // a unit is BPL * 32 consecutive blocks: the slot decode handles two blocks per
    // lane (the second block's x fetch is issued before the first is decoded)
    constexpr int BPL = 1;  // 2 measured slower (fewer units per tile: fem1p5m fp32 0.1146 -> 0.1227 ms)
    constexpr int UB = 32 * BPL;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t full_bar[kMaxStages], empty_bar[kMaxStages];
    __shared__ StageHdr hdr[kMaxStages];
    __shared__ StageRange range[kMaxStages];
    __shared__ int unit_done[kMaxStages];
    __shared__ int unit_next, units_avail;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    pdl_trigger();
    if (threadIdx.x == 0) {
        for (int s = 0; s < stages; ++s) {
            mbar_init(smem_u32(&full_bar[s]), 1);
            mbar_init(smem_u32(&empty_bar[s]), 1);
            range[s] = StageRange{0, 0, 0, 0};
            unit_done[s] = 0;
        }
        unit_next = 0;
        units_avail = 0;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const uint32_t sbase = smem_u32(smem);

    if (warp == 0) {  // ---------------------------------------------- producer
        if (lane == 0) {
            const uint64_t pol = policy_evict_first();
            int i = 0, s = 0, U = 0;
            uint32_t ph = 0;
            // tile descriptors are loaded one tile ahead (the load latency then
            // overlaps the wait for a free stage)
            int4 nd0 = make_int4(0, 0, 0, 0);
            int2 nd1 = make_int2(0, 0);
            if (blockIdx.x < ntiles) {
                nd0 = __ldg(reinterpret_cast<const int4 *>(tiles + blockIdx.x));
                nd1 = __ldg(reinterpret_cast<const int2 *>(tiles + blockIdx.x) + 2);
            }
            for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++i, s = (s + 1 == stages) ? (ph ^= 1u, 0) : s + 1) {
                const int4 d0 = nd0;
                const int2 d1 = nd1;
                if (t + (int)gridDim.x < ntiles) {
                    nd0 = __ldg(reinterpret_cast<const int4 *>(tiles + t + gridDim.x));
                    nd1 = __ldg(reinterpret_cast<const int2 *>(tiles + t + gridDim.x) + 2);
                }
                const int br0 = d0.x, br1 = d0.y, b0 = d0.z, b1 = d0.w, v0 = d1.x, v1 = d1.y;
                if (i >= stages) mbar_wait(smem_u32(&empty_bar[s]), ph ^ 1u);
                const uint32_t stage = sbase + (uint32_t)s * (uint32_t)stage_bytes;
                uint32_t cur = stage;
                struct Reg {
                    uintptr_t src;
                    uint32_t sz;
                };
                auto region = [&](const void *lo_p, size_t len, uint32_t *addr_out) {
                    const uintptr_t lo = (uintptr_t)lo_p, hi = lo + len;
                    const uintptr_t alo = lo & ~(uintptr_t)15, ahi = (hi + 15) & ~(uintptr_t)15;
                    *addr_out = cur + (uint32_t)(lo - alo);
                    const Reg r{alo, len > 0 ? (uint32_t)(ahi - alo) : 0u};
                    cur += r.sz;
                    return r;
                };
                StageHdr h;
                h.br0 = br0;
                h.nbr = br1 - br0;
                h.b0 = b0;
                h.v0 = v0;
                h.nb = b1 - b0;
                h.a_rot = 0;
                // the value slice first: its bank layout is the one the rotation
                // pass assumed (16-byte aligned start of the stage)
                const Reg rs[6] = {region(vals + v0, sizeof(V) * (size_t)(v1 - v0), &h.a_val),
                                   region(bitmap + b0, 8u * (b1 - b0), &h.a_bmp),
                                   region(blk_col + b0, 4u * (b1 - b0), &h.a_col),
                                   region(blk_offset + b0, 4u * (b1 - b0), &h.a_off),
                                   region(blk_rowptr + br0, 4u * (br1 - br0 + 1), &h.a_rp),
                                   ROT ? region(rot + b0, (size_t)(b1 - b0), &h.a_rot) : Reg{0, 0u}};
                const uint32_t bytes = cur - stage;
                h.a_part = cur;  // kPartStride bytes of row partials per block (not copied)
                hdr[s] = h;
                const int units = max(1, (h.nb + UB - 1) / UB);
                asm volatile("st.shared.v4.s32 [%0], {%1, %2, %3, %4};" ::"r"(smem_u32(&range[s])), "r"(U),
                             "r"(U + units), "r"((int)ph), "r"(0)
                             : "memory");  // one 16-byte store: consumers never see a torn range
                unit_done[s] = 0;
                U += units;
                const uint32_t fb = smem_u32(&full_bar[s]);
                mbar_arrive_expect_tx(fb, bytes);
                uint32_t dst = stage;
#pragma unroll
                for (int k = 0; k < 6; ++k) {
                    if (rs[k].sz) bulk_g2s(dst, (const void *)rs[k].src, rs[k].sz, fb, pol);
                    dst += rs[k].sz;
                }
                // publish the tile's units (after its header, range and counter)
                asm volatile("st.release.cta.shared.s32 [%0], %1;" ::"r"(smem_u32(&units_avail)), "r"(U) : "memory");
            }
        }
        pdl_wait();  // a PDL-launched grid completes only after its predecessor
        return;
    }

    // ------------------------------------------------------------ consumers
    // the CTA's unit count (its tiles t = blockIdx.x + k*gridDim.x)
    int total = 0;
    for (int t = blockIdx.x + lane * gridDim.x; t < ntiles; t += 32 * gridDim.x) {
        const int2 bb = __ldg(reinterpret_cast<const int2 *>(tiles + t) + 1);  // b0, b1
        total += max(1, (bb.y - bb.x + UB - 1) / UB);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) total += __shfl_xor_sync(kFull, total, o);
    const uint32_t a_avail = smem_u32(&units_avail), a_unext = smem_u32(&unit_next);
    const uint32_t a_range0 = smem_u32(&range[0]), a_full0 = smem_u32(&full_bar[0]);
    const uint32_t a_hdr0 = smem_u32(&hdr[0]), a_done0 = smem_u32(&unit_done[0]);
    int avail = 0;
    while (true) {
        int g = 0;
        if (lane == 0) g = atom_add_shared(a_unext, 1);
        g = __shfl_sync(kFull, g, 0);
        if (g >= total) break;
        while (avail <= g) {  // the producer has not published the tile yet
            asm volatile("ld.acquire.cta.shared.s32 %0, [%1];" : "=r"(avail) : "r"(a_avail) : "memory");
            if (avail <= g) __nanosleep(SPADEN_AVAIL_SLEEP_NS);
        }
        int s = 0, us = 0, par = 0;
        for (; s < stages; ++s) {  // the stage whose tile holds unit g (its current fill:
            const int4 rg = lds_i4_volatile(a_range0 + 16u * s);  // a stage is refilled
            if (rg.x <= g && g < rg.y) {                          // only after its tile is done)
                us = rg.x;
                par = rg.z;
                break;
            }
        }
        const uint32_t a_hdr = a_hdr0 + (uint32_t)(s * sizeof(StageHdr));
        mbar_wait(a_full0 + 8u * s, (uint32_t)par);
        const int4 h0 = lds_i4_volatile(a_hdr);
        const int4 h1 = lds_i4_volatile(a_hdr + 16u);
        const int v0 = h0.x, nb = h0.y;
        const int units = max(1, (nb + UB - 1) / UB);
        const uint32_t a_rot = (uint32_t)h0.z, a_val = (uint32_t)h0.w;
        const uint32_t a_bmp = h1.x, a_col = h1.y, a_off = h1.z, a_part = h1.w;
        const int ul = g - us;
        if constexpr (K > 1) {  // SpMM: K right-hand sides
            const int lb = ul * 32 + lane;
            if (lb < nb) {
                const uint2 bm = lds_u2(a_bmp + 8u * lb);
                const int bc = lds_i32(a_col + 4u * lb);
                const uint32_t p = a_val + (uint32_t)(lds_i32(a_off + 4u * lb) - v0) * (uint32_t)sizeof(V);
                const uint32_t cols = used_cols(bm);
                XSeg xs[K];
#pragma unroll
                for (int j = 0; j < K; ++j) load_x(xs[j], x + j * ldx, bc, nbc_vec, cols, texx, (int)(j * ldx / 4));
                block_slots_k<SmemVals<V>, K>(bm, p, xs, a_part + 4u * (8 * K + 1) * lb);
            }
        } else if constexpr (DEC == 4) {
            // tensor-core ablation (SURVEY.md §8(f) NEXT-3, fp16 values): the
            // paper's fragment trick on mma.sync.m16n8k16 -- four
            // blocks per MMA, block P/Q/R/S in the TL/TR/BL/BR quadrants, lane l
            // owns bits 2l, 2l+1 of each (Alg. 2 mapping); x split
            // into fp16 hi + lo parts (two MMAs) to keep ~22 bits of x.
            mma_unit(ul * 32, nb, lane, a_bmp, a_col, a_off, a_val, v0, a_part, x, nbc_vec);
        } else {
            if constexpr (DEC == 1) {  // phase 1: BPL blocks per lane, all loads first
                int lbs[BPL];
                uint2 bms[BPL];
                uint32_t ps[BPL], rhos[BPL];
                XSeg xss[BPL];
#pragma unroll
                for (int h = 0; h < BPL; ++h) {
                    const int lb = ul * UB + 32 * h + lane;
                    lbs[h] = lb;
                    if (lb < nb) {
                        bms[h] = lds_u2(a_bmp + 8u * lb);
                        const int bc = lds_i32(a_col + 4u * lb);
                        ps[h] = a_val + (uint32_t)(lds_i32(a_off + 4u * lb) - v0) * (uint32_t)sizeof(V);
                        rhos[h] = ROT ? lds_u8(a_rot + (uint32_t)lb) : 0u;
                        load_x(xss[h], x, bc, nbc_vec, used_cols(bms[h]), texx);
                    }
                }
#pragma unroll
                for (int h = 0; h < BPL; ++h) {
                    const int lb = lbs[h];
                    if (lb >= nb) continue;
                    if constexpr (ROT && kRotV4) {
                        block_slots_rot_v4<SmemVals<V>>(bms[h], rhos[h], ps[h], xss[h], a_part + kPartStrideV4 * lb);
                    } else if constexpr (ROT) {
                        block_slots_rot<SmemVals<V>>(bms[h], rhos[h], ps[h], xss[h], a_part + kPartStride * lb);
                    } else {
                        const uint32_t q = a_part + kPartStride * lb;
                        float acc[8];
                        const uint2 bm = bms[h];
                        const SwapHalves sw{sizeof(V) == 2 && ((lane >> 1) & 1)};
                        const uint32_t plo = (uint32_t)__popc(bm.x) * (uint32_t)sizeof(V);
                        block_slots_at<SmemVals<V>>(sw.bitmap(bm), sw.on ? ps[h] + plo : ps[h], sw.on ? ps[h] : ps[h] + plo,
                                                    xss[h], acc);
#pragma unroll
                        for (int r = 0; r < 8; ++r) sts_f32(q + sw.part_off(r), acc[r]);
                    }
                }
            } else {
            const int lb = ul * 32 + lane;
            if (lb < nb) {  // phase 1: one block per lane
                const uint2 bm = lds_u2(a_bmp + 8u * lb);
                const int bc = lds_i32(a_col + 4u * lb);
                const uint32_t p = a_val + (uint32_t)(lds_i32(a_off + 4u * lb) - v0) * (uint32_t)sizeof(V);
                float acc[8];
                const uint32_t q = a_part + kPartStride * lb;
                if constexpr (false) {
                } else if constexpr (DEC == 1) {
                    XSeg xs;
                    load_x(xs, x, bc, nbc_vec, used_cols(bm), texx);
                    const SwapHalves sw{sizeof(V) == 2 && ((lane >> 1) & 1)};
                    const uint32_t plo = (uint32_t)__popc(bm.x) * (uint32_t)sizeof(V);
                    block_slots_at<SmemVals<V>>(sw.bitmap(bm), sw.on ? p + plo : p, sw.on ? p : p + plo, xs, acc);
#pragma unroll
                    for (int r = 0; r < 8; ++r) sts_f32(q + sw.part_off(r), acc[r]);
                } else {
                    block_bits<SmemVals<V>>(bm, p, x + 8 * (int64_t)bc, acc);
#pragma unroll
                    for (int r = 0; r < 8; ++r) sts_f32(q + 4u * r, acc[r]);
                }
            }
            }
        }
        __syncwarp();
        int last = 0;
        if (lane == 0) {
            __threadfence_block();
            last = (atom_add_shared(a_done0 + 4u * s, 1) + 1 == units);
        }
        if (__shfl_sync(kFull, last, 0)) {  // phase 2: this warp completed the tile
            __threadfence_block();
            if (wait_y) pdl_wait();  // y of the previous kernels (hybrid residual pass)
            const int4 h2 = lds_i4_volatile(a_hdr + 32u);  // br0, nbr, b0, a_rp
            if constexpr (K > 1)
                reduce_tile_k<K>((uint32_t)h2.w, a_part, h2.y, h2.z, h2.x, lane, m, alpha, beta, y, ldy);
            else if constexpr (DEC == 1 && ROT && kRotV4)
                reduce_tile<kPartStrideV4>((uint32_t)h2.w, a_part, h2.y, h2.z, h2.x, lane, m, alpha, beta, y, po);
            else
                reduce_tile((uint32_t)h2.w, a_part, h2.y, h2.z, h2.x, lane, m, alpha, beta, y, po);
            __syncwarp();
            if (lane == 0) mbar_arrive(smem_u32(&empty_bar[s]));  // release the stage
        }
    }
    pdl_wait();  // a PDL-launched grid completes only after its predecessor
}

// fix-up of long block-row j by one warp: lane l adds the 8-float partials of
// chunks l, l+32, ... in order, then a fixed xor tree (a function of the row's
// chunk count).  Carries are read from L2 (__ldcg): they were written by other SMs.
__device__ __forceinline__ void long_fixup_row(int64_t m, int j, int lane, const int32_t *__restrict__ long_rows,
                                               const int32_t *__restrict__ chunk_start, const float *carry,
                                               float alpha, float beta, float *__restrict__ y, const PeerOut &po) {
    float tot[8];
#pragma unroll
    for (int r = 0; r < 8; ++r) tot[r] = 0.f;
    for (int c = chunk_start[j] + lane; c < chunk_start[j + 1]; c += 32) {
        const float4 *c4 = reinterpret_cast<const float4 *>(carry + 8 * (int64_t)c);
        const float4 lo = __ldcg(c4), hi = __ldcg(c4 + 1);
        tot[0] += lo.x, tot[1] += lo.y, tot[2] += lo.z, tot[3] += lo.w;
        tot[4] += hi.x, tot[5] += hi.y, tot[6] += hi.z, tot[7] += hi.w;
    }
#pragma unroll
    for (int r = 0; r < 8; ++r) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) tot[r] += __shfl_xor_sync(kFull, tot[r], o);
    }
    if (lane == 0) {
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            const int64_t row = 8 * (int64_t)long_rows[j] + r;
            if (row < m) {
                float o = alpha * tot[r];
                if (beta != 0.f) o = fmaf(beta, y[row], o);
                store_y(y, row, o, po);
            }
        }
    }
}

// separate fix-up launch (more than kFusedFixupMaxChunks chunks)
__global__ void __launch_bounds__(256)
k_spmv_long_fixup(int64_t m, int nlong, const int32_t *__restrict__ long_rows,
                  const int32_t *__restrict__ chunk_start, const float *carry, float alpha, float beta,
                  float *__restrict__ y, const PeerOut po) {
    pdl_wait();
    const int64_t j = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (j < nlong) long_fixup_row(m, (int)j, threadIdx.x & 31, long_rows, chunk_start, carry, alpha, beta, y, po);
}

// Long block-rows (too large for a stage), straight from global memory.
// k_spmv_long_chunks: one warp per kLongChunk-block chunk; lane j takes blocks
// j, j+32, ... of the chunk (same per-block arithmetic as the tiled kernel),
// sums them in that order, then a fixed xor tree over the lanes gives the
// chunk's 8 row partials (carry).  The warp that finishes a row's last chunk
// runs the fix-up (long_fixup_row): lane l adds the carries of chunks l, l+32,
// ... in order, then a fixed xor tree over the lanes.  The order depends only
// on the block-row (its chunk count), not on which warp finishes last.
template <typename V, bool SLOTS, bool FUSED>
__global__ void __launch_bounds__(256)
k_spmv_long_chunks(int nchunks, const int32_t *__restrict__ long_rows, const int32_t *__restrict__ chunk_start,
                   const int32_t *__restrict__ chunk_row, const int32_t *__restrict__ blk_rowptr,
                   const int32_t *__restrict__ blk_col, const uint64_t *__restrict__ bitmap,
                   const int32_t *__restrict__ blk_offset, const V *__restrict__ vals, const float *__restrict__ x,
                   int nbc_vec, float *carry, int32_t *__restrict__ done, int64_t m, float alpha, float beta,
                   float *__restrict__ y, const PeerOut po) {
    pdl_trigger();
    const int w = (int)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    const int lane = threadIdx.x & 31;
    if (w >= nchunks) return;
    const int j = chunk_row[w];
    const int br = long_rows[j];
    const int cb0 = blk_rowptr[br] + (w - chunk_start[j]) * kLongChunk;
    const int cb1 = min(blk_rowptr[br + 1], cb0 + kLongChunk);
    float tot[8];
#pragma unroll
    for (int r = 0; r < 8; ++r) tot[r] = 0.f;
    for (int b = cb0 + lane; b < cb1; b += 32) {
        const uint64_t w64 = __ldg(bitmap + b);
        const uint2 bm = make_uint2((uint32_t)w64, (uint32_t)(w64 >> 32));
        const int bc = __ldg(blk_col + b);
        const V *p = vals + __ldg(blk_offset + b);
        float acc[8];
        if constexpr (SLOTS) {
            XSeg xs;
            load_x(xs, x, bc, nbc_vec, used_cols(bm));
            block_slots<GlobalVals<V>>(bm, p, xs, acc);
        } else {
            block_bits<GlobalVals<V>>(bm, p, x + 8 * (int64_t)bc, acc);
        }
#pragma unroll
        for (int r = 0; r < 8; ++r) tot[r] += acc[r];
    }
#pragma unroll
    for (int r = 0; r < 8; ++r) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) tot[r] += __shfl_xor_sync(kFull, tot[r], o);
    }
    // FUSED (few chunks): the warp that completes the row's last
    // chunk does the fix-up (threadfence + completion counter, reset for the
    // next call); otherwise k_spmv_long_fixup runs after this launch
    int last = 0;
    if (lane == 0) {
        float4 *c4 = reinterpret_cast<float4 *>(carry + 8 * (int64_t)w);
        __stcg(c4, make_float4(tot[0], tot[1], tot[2], tot[3]));
        __stcg(c4 + 1, make_float4(tot[4], tot[5], tot[6], tot[7]));
        if constexpr (FUSED) {
            __threadfence();
            last = atomicAdd(done + j, 1) == chunk_start[j + 1] - chunk_start[j] - 1;
        }
    }
    pdl_wait();  // fix-up below reads y; unfused: still complete only after the predecessor
    if (FUSED && __shfl_sync(kFull, last, 0)) {
        __threadfence();
        long_fixup_row(m, j, lane, long_rows, chunk_start, carry, alpha, beta, y, po);
        if (lane == 0) done[j] = 0;
    }
}

int sm_count() {
    static int c = [] {
        int dev = 0, n = 148;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        return n;
    }();
    return c;
}

// Texture objects binding x (n4 float4 elements from x) for load_x, cached per
// (device, pointer, length); SPADEN_XTEX=0 disables (LDG path, ablation).
// Entries are never destroyed while the library is loaded (a CUDA graph or an
// in-flight kernel may hold one); once kTexCache distinct vectors are bound,
// further vectors use the LDG path (same values, load_x's other branch).
constexpr int kTexCache = 256;
unsigned long long x_texture(const float *x, int64_t n4) {
    const char *env = getenv("SPADEN_XTEX");  // read per call (tests toggle it)
    if ((env && env[0] == '0') || n4 <= 0) return 0ull;
    static std::mutex mu;
    struct Entry {
        const float *x;
        int dev;
        int64_t n4;
        cudaTextureObject_t obj;
    };
    static Entry cache[kTexCache] = {};
    static int used = 0;
    static int max_width[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lock(mu);
    for (int i = 0; i < used; ++i)
        if (cache[i].x == x && cache[i].dev == dev && cache[i].n4 == n4) return cache[i].obj;
    if (used == kTexCache || dev < 0 || dev >= 64) return 0ull;
    if (max_width[dev] == 0 &&
        cudaDeviceGetAttribute(&max_width[dev], cudaDevAttrMaxTexture1DLinearWidth, dev) != cudaSuccess)
        max_width[dev] = -1;
    if (n4 > (int64_t)max_width[dev]) return 0ull;
    cudaResourceDesc rd{};
    rd.resType = cudaResourceTypeLinear;
    rd.res.linear.devPtr = const_cast<float *>(x);
    rd.res.linear.desc = cudaCreateChannelDesc<float4>();
    rd.res.linear.sizeInBytes = (size_t)n4 * 16;
    cudaTextureDesc td{};
    td.readMode = cudaReadModeElementType;
    cudaTextureObject_t o = 0;
    if (cudaCreateTextureObject(&o, &rd, &td, nullptr) != cudaSuccess) {
        cudaGetLastError();
        return 0ull;
    }
    cache[used++] = Entry{x, dev, n4, o};
    return o;
}

// Resident CTAs per SM of a kernel at a dynamic shared-memory size, capped at
// `cap`; sets the kernel's max dynamic smem attribute first.  Cached per
// (kernel, smem, device) behind a mutex (thread-safe; several handles and
// streams may launch concurrently).
int occupancy(const void *kern, int threads, size_t smem, int cap, cudaError_t *err) {
    static std::mutex mu;
    struct Key {
        const void *k;
        size_t smem;
        int dev;
        int occ;
    };
    static Key cache[64];
    static int used = 0;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lock(mu);
    for (int i = 0; i < used; ++i)
        if (cache[i].k == kern && cache[i].smem == smem && cache[i].dev == dev) return cache[i].occ;
    int occ = 0;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, threads, smem);
    if (e != cudaSuccess) {
        *err = e;
        return 0;
    }
    occ = std::max(1, std::min(occ, cap));
    if (used < 64) cache[used++] = Key{kern, smem, dev, occ};
    return occ;
}

// long block-rows after (or, few chunks, before and beside) the tile kernel
template <typename V, bool SLOTS>
cudaError_t launch_long_rows(const Matrix &A, int slot, float alpha, const float *x, int nbc_vec, float beta,
                             float *y, cudaStream_t st, const PeerOut &po, bool dep, bool fused) {
    float *carry = A.carry + (size_t)slot * 8 * (size_t)std::max<int64_t>(1, A.n_chunks);
    int32_t *done = A.chunk_done + (size_t)slot * (size_t)A.n_long;
    const unsigned g = (unsigned)((32 * A.n_chunks + 255) / 256);
    cudaError_t e = launch_k(dep, fused ? k_spmv_long_chunks<V, SLOTS, true> : k_spmv_long_chunks<V, SLOTS, false>,
                             dim3(g), dim3(256), 0, st, (int)A.n_chunks, (const int32_t *)A.long_rows,
                             (const int32_t *)A.chunk_start, (const int32_t *)A.chunk_row,
                             (const int32_t *)A.blk_rowptr, (const int32_t *)A.blk_col, (const uint64_t *)A.bitmap,
                             (const int32_t *)A.blk_offset, (const V *)A.values, x, nbc_vec, carry, done,
                             (int64_t)A.m, alpha, beta, y, po);
    if (e == cudaSuccess && !fused)
        e = launch_k(true, k_spmv_long_fixup, dim3((unsigned)((32 * A.n_long + 255) / 256)), dim3(256), 0, st,
                     (int64_t)A.m, (int)A.n_long, (const int32_t *)A.long_rows, (const int32_t *)A.chunk_start,
                     (const float *)carry, alpha, beta, y, po);
    return e;
}

template <typename V, int DEC, int CONSUMERS, int MINB, bool ROT>
cudaError_t launch_tiled_rot(const Matrix &A, int slot, const TileCfg &cfg, float alpha, const float *x, float beta,
                             float *y, cudaStream_t st, const PeerOut &po, bool dep) {
    const int nbc_vec = ((uintptr_t)x & 31u) == 0 ? (int)(A.n / 8) : 0;
    const size_t smem = (size_t)cfg.stages * cfg.stage_bytes;
    auto kern = k_spmv_tiled<V, DEC, CONSUMERS, MINB, 1, ROT>;
    cudaError_t e = cudaSuccess;
    const int occ = occupancy((const void *)kern, 32 * (CONSUMERS + 1), smem, MINB, &e);
    if (e != cudaSuccess) return e;
    const bool hyb = A.res_max_popc > 0;  // the residual pass wrote y before these kernels
    const bool fused = A.n_long > 0 && A.n_chunks <= fused_fixup_max();
    // few long-row chunks (one wave): launch them first, the tiled kernel then
    // starts (PDL) while they run -- their rows are disjoint, so it waits for
    // them only before exiting.  Many chunks: tiled kernel, then the chunks as a
    // normal launch (an early-launched grid of many waves would park finished
    // CTAs in pdl_wait next to the tiled kernel: rmat22 pure 1.33 -> 2.20 ms),
    // then the separate fix-up.
    if (fused) {
        e = launch_long_rows<V, (DEC != 0)>(A, slot, alpha, x, nbc_vec, beta, y, st, po, dep, true);
        dep = true;
    }
    if (A.n_tiles > 0 && e == cudaSuccess) {
        const int grid = (int)std::min<int64_t>(A.n_tiles, (int64_t)sm_count() * occ);
        const unsigned long long texx = x_texture(x, 2 * (int64_t)nbc_vec);
        e = launch_k(dep, kern, dim3(grid), dim3(32 * (CONSUMERS + 1)), smem, st,
                     cfg.stages, cfg.stage_bytes, (int64_t)A.m, (const TileDesc *)A.tiles, (int)A.n_tiles,
                     (const int32_t *)A.blk_rowptr, (const int32_t *)A.blk_col, (const uint64_t *)A.bitmap,
                     (const int32_t *)A.blk_offset, (const V *)A.values, x, nbc_vec, alpha, beta, y, (int64_t)0,
                     (int64_t)0, po, texx, (int)hyb, (const uint8_t *)A.rot);
        dep = true;
    }
    if (A.n_long > 0 && !fused && e == cudaSuccess)
        e = launch_long_rows<V, (DEC != 0)>(A, slot, alpha, x, nbc_vec, beta, y, st, po, false, false);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

template <typename V, int DEC, int CONSUMERS, int MINB>
cudaError_t launch_tiled_cfg(const Matrix &A, int slot, const TileCfg &cfg, float alpha, const float *x, float beta,
                             float *y, cudaStream_t st, const PeerOut &po, bool dep) {
    if constexpr (DEC == 1) {
        if (A.rot) return launch_tiled_rot<V, DEC, CONSUMERS, MINB, true>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    }
    return launch_tiled_rot<V, DEC, CONSUMERS, MINB, false>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
}

template <typename V, int DEC>
cudaError_t launch_tiled(const Matrix &A, int slot, float alpha, const float *x, float beta, float *y,
                         cudaStream_t st, const PeerOut &po, bool dep) {
    const TileCfg cfg = tile_cfg(A.tile_cfg);
    switch (A.tile_cfg) {
    case 5: return launch_tiled_cfg<V, DEC, 8, 3>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    case 6: return launch_tiled_cfg<V, DEC, 16, 2>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    case 7: return launch_tiled_cfg<V, DEC, 8, 4>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    case 10: return launch_tiled_cfg<V, DEC, 4, 6>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    case 14: return launch_tiled_cfg<V, DEC, 12, 2>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    case 15: return launch_tiled_cfg<V, DEC, 16, 2>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    case 16: return launch_tiled_cfg<V, DEC, 8, 2>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    case 1: return launch_tiled_cfg<V, DEC, 16, 2>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    case 3: return launch_tiled_cfg<V, DEC, 8, 4>(A, slot, cfg, alpha, x, beta, y, st, po, dep);
    default: return launch_tiled_cfg<V, DEC, 8, 3>(A, slot, cfg, alpha, x, beta, y, st, po, dep);  // cfg 2
    }
}

template <typename V, int K, int CONSUMERS, int MINB>
cudaError_t launch_spmm_cfg(const Matrix &A, int slot, const TileCfg &cfg, const TileDesc *tiles, int64_t ntiles, float alpha,
                            const float *X, int64_t ldx, float beta, float *Y, int64_t ldy, cudaStream_t st) {
    const bool aligned = ((uintptr_t)X & 31u) == 0 && ((ldx * 4) % 32) == 0;
    const int nbc_vec = aligned ? (int)(A.n / 8) : 0;
    const size_t smem = (size_t)cfg.stages * cfg.stage_bytes;
    cudaError_t oe = cudaSuccess;
    const int occ = occupancy((const void *)k_spmv_tiled<V, 1, CONSUMERS, MINB, K>, 32 * (CONSUMERS + 1), smem,
                              MINB, &oe);
    if (oe != cudaSuccess) return oe;
    if (ntiles > 0) {
        const int grid = (int)std::min<int64_t>(ntiles, (int64_t)sm_count() * occ);
        const unsigned long long texx = nbc_vec ? x_texture(X, 2 * (int64_t)nbc_vec + (K - 1) * (ldx / 4)) : 0ull;
        k_spmv_tiled<V, 1, CONSUMERS, MINB, K><<<grid, 32 * (CONSUMERS + 1), smem, st>>>(
            cfg.stages, cfg.stage_bytes, A.m, tiles, (int)ntiles, A.blk_rowptr, A.blk_col, A.bitmap,
            A.blk_offset, (const V *)A.values, X, nbc_vec, alpha, beta, Y, ldx, ldy, PeerOut{}, texx, 1,
            (const uint8_t *)nullptr);
    }
    if (A.n_long > 0) {  // long block-rows: the SpMV chunk path, once per vector (same arithmetic)
        const int nbc1 = ((uintptr_t)X & 31u) == 0 && ((ldx * 4) % 32) == 0 ? (int)(A.n / 8) : 0;
        const bool fused = A.n_chunks <= fused_fixup_max();
        for (int j = 0; j < K; ++j) {
            cudaError_t e = launch_long_rows<V, true>(A, slot, alpha, X + j * ldx, nbc1, beta, Y + j * ldy, st,
                                                      PeerOut{}, false, fused);
            if (e != cudaSuccess) return e;
        }
    }
    return cudaGetLastError();
}

template <typename V, int K>
cudaError_t launch_spmm(const Matrix &A, int slot, const TileDesc *tiles, int64_t ntiles, float alpha, const float *X,
                        int64_t ldx, float beta, float *Y, int64_t ldy, cudaStream_t st) {
    const TileCfg cfg = tile_cfg(A.tile_cfg);
    // same stage geometry as the SpMV schedule; fewer CTAs per SM so the K
    // accumulators and x segments fit in registers without spilling
    switch (A.tile_cfg) {
    case 0: case 1: case 6:
        return launch_spmm_cfg<V, K, 16, 1>(A, slot, cfg, tiles, ntiles, alpha, X, ldx, beta, Y, ldy, st);
    default: return launch_spmm_cfg<V, K, 8, 2>(A, slot, cfg, tiles, ntiles, alpha, X, ldx, beta, Y, ldy, st);
    }
}

}  // namespace

bool pdl_enabled() {
    const char *e = getenv("SPADEN_PDL");
    return !(e && e[0] == '0');
}

int64_t fused_fixup_max() {  // SPADEN_FUSED_FIXUP_MAX overrides (tests), read per call
    const char *e = getenv("SPADEN_FUSED_FIXUP_MAX");
    return e ? atoll(e) : kFusedFixupMaxChunks;
}


spaden_status_t spmm_launch(Matrix &A, float alpha, const float *X, int64_t ldx, int k, float beta, float *Y,
                            int64_t ldy, cudaStream_t st) {
    int j = 0;
    while (j < k) {
        const int left = k - j;
        // groups of 4 (measured best: 8 needs more registers than 2 CTAs/SM allow
        // and smaller tiles)
        const int K = left >= 4 ? 4 : left >= 2 ? 2 : 1;
        const int kidx = K == 4 ? 1 : 0;
        if (K > 1 && A.m > 0 && A.spmm_state[kidx] == 0) build_spmm_schedule(&A, kidx, K, st);
        if (K == 1 || A.spmm_state[kidx] != 1 || A.m == 0) {  // one SpMV per vector
            for (int q = 0; q < K; ++q) {
                spaden_status_t s = spmv_launch(A, alpha, X + (j + q) * ldx, beta, Y + (j + q) * ldy, st);
                if (s != SPADEN_OK) return s;
            }
        } else {
            const TileDesc *tiles = A.spmm_tiles[kidx];
            const int64_t nt = A.spmm_ntiles[kidx];
            const float *Xj = X + j * ldx;
            float *Yj = Y + j * ldy;
            cudaError_t e = cudaSuccess;
            float beta_bit = beta;  // hybrid: residual pass first (y = beta*y + alpha*A_res*x), then accumulate
            const int slot = pick_scratch(A);
            if (A.res_max_popc > 0) {
                bool launched = false;
                for (int q = 0; q < K && e == cudaSuccess; ++q)
                    e = residual_first(A, alpha, Xj + q * ldx, beta, Yj + q * ldy, st, slot, &launched);
                beta_bit = 1.f;
            }
            if (e != cudaSuccess) return cuda_status(e, "launching the residual pass");
            if (A.storage == SPADEN_R_16F)
                e = K == 4 ? launch_spmm<__half, 4>(A, slot, tiles, nt, alpha, Xj, ldx, beta_bit, Yj, ldy, st)
                           : launch_spmm<__half, 2>(A, slot, tiles, nt, alpha, Xj, ldx, beta_bit, Yj, ldy, st);
            else
                e = K == 4 ? launch_spmm<float, 4>(A, slot, tiles, nt, alpha, Xj, ldx, beta_bit, Yj, ldy, st)
                           : launch_spmm<float, 2>(A, slot, tiles, nt, alpha, Xj, ldx, beta_bit, Yj, ldy, st);
            if (e != cudaSuccess) return cuda_status(e, "launching SpMM");
        }
        j += K;
    }
    return SPADEN_OK;
}

// launches issued by spmv_launch (mirrors its dispatch; spaden_spmv_launch_count)
int spmv_launch_count(const Matrix &A, float beta) {
    if (A.m == 0) return 0;
    int n = 0;
    if (A.res_max_popc > 0) {  // residual_first
        const bool binned = residual_binned_enabled(A);
        for (int q = 0; q < A.n_res_parts; ++q) {
            const ResPart &P = A.res[q];
            const float b = q == 0 ? beta : 1.f;
            if (binned) n += P.bins.cta_start[b == 1.f ? kResClasses : kResClasses + 1] > 0 ? 1 : 0;
            else n += (b != 1.f ? 1 : 0) + (P.nnz > 0 ? 1 : 0);
            if (P.n_long > 0) n += 1 + (P.n_chunks > fused_fixup_max() ? 1 : 0);
        }
    }
    n += A.n_tiles > 0 ? 1 : 0;
    if (A.n_long > 0) n += 1 + (A.n_chunks > fused_fixup_max() ? 1 : 0);
    return n;
}

spaden_status_t spmv_launch(const Matrix &A, float alpha, const float *x, float beta, float *y,
                            cudaStream_t st, const PeerOut *peers) {
    if (A.m == 0) return SPADEN_OK;
    const PeerOut po = peers ? *peers : PeerOut{};
    if (po.n > 0 && A.res_max_popc > 0) {
        set_error("the fused all-gather store needs a pure bitBSR handle (no hybrid residual)");
        return SPADEN_ERR_UNSUPPORTED;
    }
    // hybrid (NEXT-1): the residual pass runs first and applies beta to every row
    // (y = beta*y + alpha*A_res*x); the bitBSR kernels then accumulate (beta = 1)
    // over the block-rows that hold blocks (the schedule skips the others)
    bool dep = false;  // bitBSR kernels follow a residual kernel of this call (PDL)
    const int slot = pick_scratch(A);
    if (A.res_max_popc > 0) {
        SPADEN_CUDA_TRY(residual_first(A, alpha, x, beta, y, st, slot, &dep));
        beta = 1.f;
    }
    // decode style from the mean block fill (predicated slots for dense-ish blocks)
    const int decode_env = [] {  // SPADEN_DECODE=bits|slots|rows|mma overrides (ablation), read per call
        const char *e = getenv("SPADEN_DECODE");
        if (e && e[0] == 'b') return 0;
        if (e && e[0] == 's') return 1;
        if (e && e[0] == 'm') return 4;
        return -1;
    }();
    const int dec = decode_env >= 0 ? decode_env
                                    : ((A.Bnnz == 0 || A.nnz >= (int64_t)kSlotsMinFill * A.Bnnz) ? kDenseDecode : 0);
    cudaError_t e;
    if (A.storage == SPADEN_R_16F) {
        switch (dec) {
        case 0: e = launch_tiled<__half, 0>(A, slot, alpha, x, beta, y, st, po, dep); break;
        case 4: e = launch_tiled<__half, 4>(A, slot, alpha, x, beta, y, st, po, dep); break;
        default: e = launch_tiled<__half, 1>(A, slot, alpha, x, beta, y, st, po, dep);
        }
    } else {  // (the tensor-core ablation exists for fp16 values only)
        switch (dec) {
        case 0: e = launch_tiled<float, 0>(A, slot, alpha, x, beta, y, st, po, dep); break;
        default: e = launch_tiled<float, 1>(A, slot, alpha, x, beta, y, st, po, dep);
        }
    }
    if (e != cudaSuccess) return cuda_status(e, "launching k_spmv_tiled");
    return SPADEN_OK;
}

}  // namespace spaden
