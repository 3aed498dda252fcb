// spmm_tc.cu -- bitBSR SpMM on the 5th-generation tensor cores (tcgen05 / TMEM),
// SURVEY.md §8(f) NEXT-4, the paper's future work "adaptation of bitBSR for
// other sparse operations on dense matrix units, including SpMM".
//
//   Y[:, j] = alpha * A X[:, j] + beta * Y[:, j],  j < k,
//
// with A in bitBSR (fp16 values) and X given as fp16 "slabs": the 8 x entries
// of block column bc for every vector, Xb[bc][j][0..7] (spaden_spmm_tc_pack_x).
// fp16 x is the paper's tensor-core input precision (inputs half,
// outputs fp32); accumulation is fp32 in TMEM.
//
// For a block-row br with blocks b_1 .. b_nb the 8 x k slab of Y is
//   Y_br^T (k x 8) = sum over pairs (b_2p+1, b_2p+2) of  Xs_pair^T (k x 16) . A_pair^T (16 x 8)
// i.e. one tcgen05.mma (M = 128 vectors, N = 8 rows, K = 16 = two blocks' 8
// columns) per pair of blocks (a lone last block pairs with a zero tile and a
// zero slab).  Operands, both K-major without swizzle:
//   A operand: the two blocks' x slabs, [128 vectors][8 fp16] = 16 rows of 8x16 B
//              core matrices (SBO = 128 B between 8-vector groups, LBO = slab2 -
//              slab1), staged by cp.async.bulk straight from Xb;
//   B operand: the two blocks decoded into dense 8x8 fp16 tiles (row-major, one
//              core matrix each, LBO = tile2 - tile1): 8 lanes per block, lane
//              r walking row r's bits in column order (value index = offset +
//              popcount rank, P:L138 / Alg. 2 semantics P:L172-177) and storing
//              the dense row as one 16-byte store (a warp decodes 4 blocks at
//              once; the paper's lane-per-2-bits mapping took 20 instructions
//              per block instead of ~7: K = 64 1.221 -> 1.187 ms).
// The pairs of a block-row accumulate in its own 8 TMEM columns in block order
// (deterministic, a function of the block-row alone); the epilogue reads the
// 128 x 8 fp32 accumulator with tcgen05.ld and writes alpha*D + beta*Y.
//
// Work split: each CTA (one per SM) owns a contiguous range of block-rows
// holding ~Bnnz/grid blocks (whole block-rows: an accumulator never spans two
// CTAs), cut into chunks of up to kTcPairs block pairs by a schedule built on
// the GPU at the handle's first spaden_spmm_tc call.  A chunk is a run of
// consecutive blocks [B0, B1); block-rows [brA, brE) end in it, a block-row
// may start in an earlier chunk (pair pA) and continue into the next (pE).
// Roles per CTA:
//   warp 9     producer lane: bulk-copies the chunk's MMA record (TcRec,
//              precomputed with the schedule), blk_rowptr, bitmap, blk_col,
//              blk_offset and value slices (4-chunk ring);
//   warp 10    x slabs: once a chunk's arrays have landed, its lanes issue one
//              cp.async.bulk per block (3 slab buffers);
//   warps 4-7  decode the blocks into dense tiles (4-chunk ring);
//   warps 8, 11  MMA issue, alternate chunks (warp 8 also allocates TMEM): one elected lane issues the MMAs
//              (pair o's descriptors are base + o * stride: blocks sit in pair
//              order, see TcRec; the per-block-row slot comes through redux.sync
//              so every MMA operand is warp-uniform);
//   warps 0-3  epilogue (TMEM lanes 32w..32w+31 = vectors): tcgen05.ld of the
//              accumulators of the block-rows ending in the chunk, alpha*D +
//              beta*Y written as two 16-byte stores per vector and block-row.
// mbarriers per ring slot: arrays landed, arrays free (epilogue done with the
// record), tiles written, MMAs complete (tcgen05.commit: tiles free +
// accumulators ready), epilogue done; per slab buffer: slabs landed, MMAs
// reading it complete.  The MMAs of chunk c wait for the epilogue of chunk
// c-3, so at most 3 * kTcPairs < kTcSlots accumulators are live.
// History (fem1p5m, K = 128, per chunk of ~13 MMAs): a producer lane walking
// blk_rowptr into the MMA list at run time set the pace (1.81 ms); moving the
// walk to the schedule left the MMA lane at ~100 cycles per MMA (a per-MMA
// ELECT loop for non-uniform operands) and the decode warps busy with 16-byte
// cp.async slab pieces and a proxy fence per chunk (traced with
// -DSPADEN_TC_TRACE, tools/tc_trace.py).
#include <algorithm>

#include "internal.cuh"

namespace spaden {
namespace {

constexpr int kTcM = 128;         // vectors per MMA (UMMA M)
constexpr int kTcN = 8;           // rows of a block-row (UMMA N)
constexpr int kTcPairs = 15;      // block pairs per chunk (4 chunks start < kTcSlots block-rows)
constexpr int kTcBlocks = 2 * kTcPairs;
constexpr int kTcRows = 48;       // block-rows touched by one chunk (incl. empty ones)
constexpr int kTcSlots = 64;      // TMEM accumulator slots (8 columns each, 512 columns)
constexpr int kSlabBytes = kTcM * 16;
constexpr int kTileBytes = 128;
constexpr int kTcRecBytes = 160;  // a chunk's MMA record (TcRec)
constexpr int kTcArrBytes = 5120; // one chunk's staged arrays (record, brp, bitmap, blk_col, blk_offset, values)
#ifndef SPADEN_TC_RING
#define SPADEN_TC_RING 4
#endif
#ifndef SPADEN_TC_SLABS
#define SPADEN_TC_SLABS 3
#endif
constexpr int kTcRing = SPADEN_TC_RING;  // arrays, tiles and accumulator hand-off: chunks in flight
constexpr int kTcSlabBufs = SPADEN_TC_SLABS;  // x slabs: chunks (the big buffers)
#ifndef SPADEN_TC_DECODE_WARPS
#define SPADEN_TC_DECODE_WARPS 4  // 8 measured slower once a warp decodes 4 blocks at a time
#endif
constexpr int kTcDecodeWarps = SPADEN_TC_DECODE_WARPS;
constexpr int kTcSlabBytes = kTcBlocks * kSlabBytes;
constexpr int kTcTileBytes = kTcBlocks * kTileBytes;
constexpr int kTcSmem = kTcSlabBufs * kTcSlabBytes + kTcRing * (kTcTileBytes + kTcArrBytes);
constexpr int kTcThreads = (4 + kTcDecodeWarps + 4) * 32;

// one chunk of the schedule (48 bytes)
struct alignas(16) TcChunk {
    int brA, pA;     // first block-row touched, its first pair in this chunk
    int brE, pE;     // block-rows [brA, brE) end here; block-row brE continues (pE pairs done) if pE > 0
    int B0, B1;      // blocks [B0, B1)
    int seq0;        // accumulator sequence number of the first non-empty block-row touched
    int V0, V1;      // values [V0, V1) = blk_offset[B0], blk_offset[B1]
    int pad0, pad1, pad2;
};

// A chunk's MMAs and finished block-rows, precomputed with the schedule and
// staged with the chunk's arrays (so no thread walks blk_rowptr at run time).
// The chunk's blocks are placed in *pair order*: pair o of the chunk uses tile
// and slab positions 2o, 2o+1 (a block-row's lone last block has a zero tile
// as partner), so the MMA descriptors of pair o are base + o * stride and the
// issue loop needs no per-MMA operand from memory.
//   seg[s]  = slot | accumulate << 6 | pairs << 7  (the s-th non-empty block-row
//             of the chunk: TMEM slot, whether it continues an earlier chunk's
//             accumulation, its pairs in this chunk)
//   lone    = bit o: pair o has no second block
//   pos[q]  = position of the chunk's block q
//   end[e]  = i | (slot + 1) << 6  (block-row brA + i ends in the chunk; 0 = empty row)
struct alignas(16) TcRec {
    uint8_t nseg, nends;
    uint16_t lone;
    uint16_t seg[kTcPairs];
    uint8_t pos[kTcBlocks];
    uint16_t end[kTcRows];
};
static_assert(sizeof(TcRec) == kTcRecBytes && offsetof(TcRec, seg) == 4 && offsetof(TcRec, pos) == 34 &&
                  offsetof(TcRec, end) == 64,
              "TcRec layout");
// worst case of one chunk's staged regions (each rounded out to 16 bytes on both ends)
static_assert(kTcRecBytes + (4 * (kTcRows + 1) + 30) + (8 * kTcBlocks + 30) + 2 * (4 * kTcBlocks + 30) +
                      (2 * 64 * kTcBlocks + 30) <= kTcArrBytes,
              "kTcArrBytes too small");

#ifdef SPADEN_TC_TRACE  // experiment builds only (tools/exp_build.sh): per-role timestamps of CTA 0
__device__ long long *g_tc_trace;
constexpr int kTrChunks = 512, kTrEv = 8;
#define TR(role, c, ev)                                                                         \
    do {                                                                                        \
        if (trp && (c) < kTrChunks) trp[((role) * kTrChunks + (c)) * kTrEv + (ev)] = clock64(); \
    } while (0)
#else
#define TR(role, c, ev) \
    do {                \
    } while (0)
#endif

__device__ __forceinline__ uint32_t s_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void tc_mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void tc_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tc_arrive_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tc_wait(uint32_t bar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok) {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(ok)
            : "r"(bar), "r"(parity), "r"(0x989680u)
            : "memory");
    }
}
// MMA-issue warps: poll without the suspend hint and back off with __nanosleep
// (their polls otherwise take issue slots from the decode warps)
#ifndef SPADEN_TC_MMA_BACKOFF
#define SPADEN_TC_MMA_BACKOFF 64
#endif
__device__ __forceinline__ void tc_wait_mma(uint32_t bar, uint32_t parity) {
    if (!SPADEN_TC_MMA_BACKOFF) {
        tc_wait(bar, parity);
        return;
    }
    uint32_t ok = 0, ns = 32;
    while (true) {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(ok)
            : "r"(bar), "r"(parity)
            : "memory");
        if (ok) return;
        __nanosleep(ns);
        ns = ns < SPADEN_TC_MMA_BACKOFF ? 2 * ns : ns;
    }
}
__device__ __forceinline__ void tc_bulk(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
        "l"(src), "r"(bytes), "r"(bar)
        : "memory");
}
__device__ __forceinline__ uint32_t tc_lds8(uint32_t a) {
    uint16_t v;
    asm volatile("ld.shared.u8 %0, [%1];" : "=h"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t tc_lds(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}
// UMMA shared-memory descriptor, K-major, no swizzle (SM100 version 1)
__device__ __forceinline__ uint64_t umma_desc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((addr & 0x3FFFFu) >> 4) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}
// high word of every descriptor here (SBO = 128 bytes, version 1): the MMA
// lists carry only the low words
constexpr uint32_t kDescHi = ((128u >> 4) & 0x3FFFu) | (1u << 14);
// instruction descriptor: kind::f16, A = B = F16 (K-major), D = F32, M = 128, N = 8
constexpr uint32_t kTcIdesc = (1u << 4) | ((uint32_t)(kTcN >> 3) << 17) | ((uint32_t)(kTcM >> 4) << 24);

// issued by the whole (converged) warp, one elected lane executes the MMA; the
// operands must be warp-uniform (see the MMA warp: passed through redux.sync,
// whose result ptxas keeps in uniform registers, so no per-MMA ELECT loop)
__device__ __forceinline__ void umma_f16_elect(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t accumulate) {
    asm volatile(
        "{\n .reg .pred p, e;\n setp.ne.b32 p, %4, 0;\n elect.sync _|e, 0xffffffff;\n"
        " @e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(kTcIdesc), "r"(accumulate)
        : "memory");
}

// staged arrays of a chunk inside its buffer (16-byte aligned regions)
struct TcArr {
    uint32_t brp, bmp, col, off, val, rec;  // shared addresses of element 0 of each slice, of the record
};

// Chunk schedule (built once per handle on the GPU).  Block-rows are grouped in
// order into units of whole block-rows holding <= kTcPairs pairs (a block-row
// with more pairs is a unit of its own, cut into several chunks); units go to
// the CTAs round robin, so all CTAs sweep the matrix together and the x slabs
// of the band they touch stay in L2.  A unit never spans two CTAs, so an
// accumulator never does.  One thread walks the block-rows (count pass:
// out == nullptr counts chunks per CTA).
__global__ void k_tc_sched(const int32_t *__restrict__ brp, const int32_t *__restrict__ boff, int64_t Bnrow, int G,
                           int32_t *__restrict__ counts,
                           int32_t *__restrict__ fill, const int32_t *__restrict__ cta_start,
                           TcChunk *__restrict__ out) {
    if (blockIdx.x != 0 || threadIdx.x != 0) return;
    if (!out)
        for (int c = 0; c < G; ++c) counts[c] = 0;
    else
        for (int c = 0; c < G; ++c) fill[c] = 0;
    int seq[1024];  // accumulator sequence per CTA (G <= 1024)
    for (int c = 0; c < G && c < 1024; ++c) seq[c] = 0;
    int64_t br = 0;
    int unit = 0;
    while (br < Bnrow) {
        const int cta = unit % G;
        ++unit;
        // a unit: whole block-rows up to kTcPairs pairs / kTcRows rows, or one long block-row
        TcChunk ch;
        ch.brA = (int)br;
        ch.pA = 0;
        ch.seq0 = seq[cta];
        ch.B0 = brp[br];
        ch.pad0 = ch.pad1 = ch.pad2 = 0;
        int np = 0;
        while (br < Bnrow && br - ch.brA < kTcRows - 1) {
            const int nb = brp[br + 1] - brp[br];
            const int npr = (nb + 1) >> 1;
            if (np > 0 && np + npr > kTcPairs) break;  // next block-row goes to the next unit
            if (npr > kTcPairs) {                      // long block-row: chunks of kTcPairs pairs
                for (int p = 0; p < npr; p += kTcPairs) {
                    TcChunk lc = ch;
                    lc.brA = (int)br;
                    lc.pA = p;
                    lc.B0 = brp[br] + 2 * p;
                    const int pe = min(npr, p + kTcPairs);
                    lc.brE = pe == npr ? (int)br + 1 : (int)br;
                    lc.pE = pe == npr ? 0 : pe;
                    lc.B1 = min(brp[br] + 2 * pe, brp[br + 1]);
                    lc.seq0 = seq[cta];
                    lc.V0 = boff[lc.B0];
                    lc.V1 = boff[lc.B1];
                    if (out) out[cta_start[cta] + fill[cta]++] = lc;
                    else counts[cta]++;
                }
                ++seq[cta];
                ++br;
                np = -1;  // unit done
                break;
            }
            np += npr;
            if (nb > 0) ++seq[cta];
            ++br;
        }
        if (np < 0) continue;
        ch.brE = (int)br;
        ch.pE = 0;
        ch.B1 = brp[br];
        ch.V0 = boff[ch.B0];
        ch.V1 = boff[ch.B1];
        if (out) out[cta_start[cta] + fill[cta]++] = ch;
        else counts[cta]++;
    }
}

// one thread per chunk: its MMA record (the block-rows it touches, in order)
__global__ void k_tc_ops(const int32_t *__restrict__ brp, const TcChunk *__restrict__ chunks, int64_t nchunks,
                         TcRec *__restrict__ recs) {
    const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nchunks) return;
    const TcChunk ch = chunks[c];
    TcRec r;
    const int rows = ch.brE - ch.brA + (ch.pE > 0 ? 1 : 0);
    int seq = ch.seq0, ne = 0, ns = 0, o = 0;
    r.lone = 0;
    for (int q = 0; q < kTcBlocks; ++q) r.pos[q] = 0;
    for (int i = 0; i < rows; ++i) {
        const int s0 = brp[ch.brA + i], nb = brp[ch.brA + i + 1] - s0;
        const int slot = seq % kTcSlots;
        if (ch.brA + i < ch.brE) r.end[ne++] = (uint16_t)(i | ((nb ? slot + 1 : 0) << 6));
        if (nb == 0) continue;
        const int npr = (nb + 1) >> 1;
        const int pb = i == 0 ? ch.pA : 0;
        const int pe = (ch.brA + i < ch.brE) ? npr : ch.pE;
        r.seg[ns++] = (uint16_t)(slot | ((pb > 0 ? 1 : 0) << 6) | ((pe - pb) << 7));
        for (int p = pb; p < pe; ++p, ++o) {
            const int q1 = s0 + 2 * p - ch.B0;
            r.pos[q1] = (uint8_t)(2 * o);
            if (2 * p + 1 < nb) r.pos[q1 + 1] = (uint8_t)(2 * o + 1);
            else r.lone |= (uint16_t)(1u << o);
        }
        if (ch.brA + i < ch.brE) ++seq;
    }
    r.nseg = (uint8_t)ns;
    r.nends = (uint8_t)ne;
    for (int e = ne; e < kTcRows; ++e) r.end[e] = 0;
    for (int t = ns; t < kTcPairs; ++t) r.seg[t] = 0;
    const uint4 *src = reinterpret_cast<const uint4 *>(&r);
    uint4 *dst = reinterpret_cast<uint4 *>(recs + c);
#pragma unroll
    for (int w = 0; w < kTcRecBytes / 16; ++w) dst[w] = src[w];
}

__global__ void __launch_bounds__(kTcThreads, 1)
k_spmm_tc(int64_t m, const TcChunk *__restrict__ chunks, const TcRec *__restrict__ recs,
          const int32_t *__restrict__ cta_start,
          const int32_t *__restrict__ brp, const int32_t *__restrict__ bcol, const uint64_t *__restrict__ bitmap,
          const int32_t *__restrict__ boff, const __half *__restrict__ vals, const __half *__restrict__ Xb,
          int64_t nbcx, int32_t j0, int32_t kv, float alpha, float beta, float *__restrict__ Y, int64_t ldy) {
    extern __shared__ __align__(1024) unsigned char smem[];
    __shared__ TcChunk cdesc[kTcRing];
    __shared__ TcArr arr[kTcRing];
    // a = c % kTcRing (arrays, tiles, accumulator hand-off), b = c % kTcSlabBufs (x slabs)
    __shared__ __align__(8) uint64_t bar_arr[kTcRing];    // arrays landed (producer, tx)
    __shared__ __align__(8) uint64_t bar_afree[kTcRing];  // arrays of chunk c no longer read (4 epilogue warps)
    __shared__ __align__(8) uint64_t bar_epi[kTcRing];    // epilogue done with chunk c (4 warps)
    __shared__ __align__(8) uint64_t bar_tiles[kTcRing];  // tiles decoded (decode warps)
    __shared__ __align__(8) uint64_t bar_mma[kTcRing];    // chunk's MMAs complete (commit): tiles free,
                                                          // accumulators ready
    __shared__ __align__(8) uint64_t bar_sfree[kTcSlabBufs];  // MMAs reading the slabs complete (commit)
    __shared__ __align__(8) uint64_t bar_slab[kTcSlabBufs];   // slab bulk copies landed (producer, tx)
    __shared__ uint32_t tmem_base_sh;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t sb = s_u32(smem);
    const uint32_t tiles0 = sb + (uint32_t)kTcSlabBufs * kTcSlabBytes;
    const uint32_t arr0 = tiles0 + (uint32_t)kTcRing * kTcTileBytes;
    const int c0 = cta_start[blockIdx.x], nch = cta_start[blockIdx.x + 1] - c0;
    const int kMma = 4 + kTcDecodeWarps, kProd = kMma + 1, kSlab = kMma + 2, kMma2 = kMma + 3;

    if (threadIdx.x == 0) {
        for (int a = 0; a < kTcRing; ++a) {
            tc_mbar_init(s_u32(&bar_arr[a]), 1);
            tc_mbar_init(s_u32(&bar_afree[a]), 4);
            tc_mbar_init(s_u32(&bar_epi[a]), 4);
            tc_mbar_init(s_u32(&bar_tiles[a]), kTcDecodeWarps);
            tc_mbar_init(s_u32(&bar_mma[a]), 1);  // tcgen05.commit
        }
        for (int b = 0; b < kTcSlabBufs; ++b) {
            tc_mbar_init(s_u32(&bar_sfree[b]), 1);
            tc_mbar_init(s_u32(&bar_slab[b]), 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    // the slab buffers start zeroed: a lone block's partner position (zero tile)
    // then only ever holds zeros or earlier finite slabs, never NaN patterns
    for (int i = threadIdx.x; i < kTcSlabBufs * kTcSlabBytes / 16; i += blockDim.x)
        asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(sb + 16u * i), "r"(0u) : "memory");
    if (warp == kMma) {  // TMEM: 512 columns = kTcSlots accumulators of 8 fp32 columns
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(s_u32(&tmem_base_sh))
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // zeroed slabs -> tensor core
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#ifdef SPADEN_TC_TRACE
    long long *const trp = blockIdx.x == 0 ? g_tc_trace : nullptr;
#endif
    const uint32_t tmem = tmem_base_sh;
    const uint32_t tmem_u = __reduce_or_sync(0xffffffffu, tmem);  // warp-uniform copy (MMA operands)
    auto slab_of = [&](int b, int q) { return sb + (uint32_t)b * kTcSlabBytes + (uint32_t)q * kSlabBytes; };
    auto tile_of = [&](int a, int q) { return tiles0 + (uint32_t)a * kTcTileBytes + (uint32_t)q * kTileBytes; };
    auto ring_ph = [](int c) { return (uint32_t)((c / kTcRing) & 1); };
    auto slab_ph = [](int c) { return (uint32_t)((c / kTcSlabBufs) & 1); };

    if (warp == kProd) {  // ---------------------------------------------- producer: arrays
        TcChunk next = nch > 0 ? chunks[c0] : TcChunk{};  // descriptors one chunk ahead
        for (int c = 0; c < nch; ++c) {
            if (lane == 0) {  // the chunk's record and array slices (one lane)
                const int a = c % kTcRing;
                const TcChunk ch = next;
                if (c + 1 < nch) next = chunks[c0 + c + 1];
                TR(0, c, 0);
                if (c >= kTcRing) tc_wait(s_u32(&bar_afree[a]), ring_ph(c - kTcRing));
                TR(0, c, 1);
                cdesc[a] = ch;
                const int nrows = ch.brE - ch.brA + (ch.pE > 0 ? 1 : 0);
                const int v0 = ch.V0, v1 = ch.V1;
                uint32_t cur = arr0 + (uint32_t)a * kTcArrBytes;
                uint32_t total = 0;
                const void *srcs[6] = {recs + c0 + c, brp + ch.brA, bitmap + ch.B0, bcol + ch.B0, boff + ch.B0,
                                       vals + v0};
                const uint32_t lens[6] = {(uint32_t)kTcRecBytes, 4u * (uint32_t)(nrows + 1),
                                          8u * (uint32_t)(ch.B1 - ch.B0), 4u * (uint32_t)(ch.B1 - ch.B0),
                                          4u * (uint32_t)(ch.B1 - ch.B0), 2u * (uint32_t)(v1 - v0)};
                uint32_t addr[6], asrc[6], asz[6];
                for (int r = 0; r < 6; ++r) {
                    const uintptr_t lo = (uintptr_t)srcs[r];
                    const uintptr_t alo = lo & ~(uintptr_t)15;
                    asz[r] = lens[r] ? (uint32_t)(((lo + lens[r] + 15) & ~(uintptr_t)15) - alo) : 0u;
                    asrc[r] = (uint32_t)(lo - alo);
                    addr[r] = cur + asrc[r];
                    cur += asz[r];
                    total += asz[r];
                }
                arr[a] = TcArr{addr[1], addr[2], addr[3], addr[4], addr[5], addr[0]};
                const uint32_t fb = s_u32(&bar_arr[a]);
                tc_arrive_tx(fb, total);
                uint32_t dst = arr0 + (uint32_t)a * kTcArrBytes;
                for (int r = 0; r < 6; ++r) {
                    if (asz[r]) tc_bulk(dst, (const void *)((uintptr_t)srcs[r] - asrc[r]), asz[r], fb);
                    dst += asz[r];
                }
                TR(0, c, 2);
            }
        }
    } else if (warp == kSlab) {  // ------------------------------------------------ x slabs
        for (int cs = 0; cs < nch; ++cs) {
            {  // one bulk copy per block, lane per block
                const int a = cs % kTcRing, b = cs % kTcSlabBufs;
                tc_wait(s_u32(&bar_arr[a]), ring_ph(cs));
                if (cs >= kTcSlabBufs) tc_wait(s_u32(&bar_sfree[b]), slab_ph(cs - kTcSlabBufs));
                const TcArr ar = arr[a];
                const int nblk = cdesc[a].B1 - cdesc[a].B0;
                const uint32_t sbar = s_u32(&bar_slab[b]);
                if (lane == 0) tc_arrive_tx(sbar, (uint32_t)nblk * (uint32_t)kSlabBytes);
                __syncwarp();
                // runs of consecutive block columns at consecutive positions are one copy
                // (a group's slabs are adjacent in Xb)
                const __half *xg = Xb + (int64_t)(j0 / kTcM) * nbcx * (kTcM * 8);
                for (int q = lane; q < nblk; q += 32) {
                    const int bc = (int)tc_lds(ar.col + 4u * q);
                    const int pos = (int)tc_lds8(ar.rec + 34u + (uint32_t)q);
                    auto continues = [&](int r, int bcr, int posr) {  // block r extends block r-1's run
                        return (int)tc_lds(ar.col + 4u * (r - 1)) == bcr - 1 &&
                               (int)tc_lds8(ar.rec + 34u + (uint32_t)(r - 1)) == posr - 1;
                    };
                    if (q > 0 && continues(q, bc, pos)) continue;  // inside a run
                    int len = 1;
                    while (q + len < nblk) {
                        const int r = q + len;
                        if (!continues(r, (int)tc_lds(ar.col + 4u * r), (int)tc_lds8(ar.rec + 34u + (uint32_t)r))) break;
                        ++len;
                    }
                    tc_bulk(slab_of(b, pos), xg + (int64_t)bc * (kTcM * 8), (uint32_t)(len * kSlabBytes), sbar);
                }
            }
        }
    } else if (warp >= 4 && warp < kMma) {  // --------------------------------- decode
        const int dw = warp - 4;
        for (int c = 0; c < nch; ++c) {
            const int a = c % kTcRing;
            if (lane == 0 && dw == 0) TR(1, c, 0);
            tc_wait(s_u32(&bar_arr[a]), ring_ph(c));
            if (lane == 0 && dw == 0) TR(1, c, 1);
            const TcChunk ch = cdesc[a];
            const TcArr ar = arr[a];
            const int nblk = ch.B1 - ch.B0;
            if (lane == 0 && dw == 0) TR(1, c, 3);
            if (c >= kTcRing) tc_wait(s_u32(&bar_mma[a]), ring_ph(c - kTcRing));  // tile slot free
            if (lane == 0 && dw == 0) TR(1, c, 4);
            const int v0 = (int)tc_lds(ar.off);  // blk_offset of the chunk's first block
            // 8 lanes per block, lane = row r: the row's set bits in ascending
            // column order take the row's values (popcount rank of the row start,
            // P:L138), the dense 8-half row leaves as one 16-byte store; a warp
            // decodes 4 blocks per step
            {
                const int qs = lane >> 3, r = lane & 7;
                for (int qb = 4 * dw; qb < nblk; qb += 4 * kTcDecodeWarps) {
                    const int q = qb + qs;
                    if (q < nblk) {
                        const uint32_t lo = tc_lds(ar.bmp + 8u * q), hi = tc_lds(ar.bmp + 8u * q + 4u);
                        const int off = (int)tc_lds(ar.off + 4u * q) - v0;
                        const uint32_t pos = tc_lds8(ar.rec + 34u + (uint32_t)q);
                        const uint64_t bm = ((uint64_t)hi << 32) | lo;
                        const uint32_t byte = (uint32_t)(bm >> (8 * r)) & 0xffu;
                        uint32_t va = ar.val + 2u * (uint32_t)(off + __popcll(bm & ((1ull << (8 * r)) - 1ull)));
                        uint32_t w[4];
#pragma unroll
                        for (int c2 = 0; c2 < 4; ++c2) {
                            uint16_t h0 = 0, h1 = 0;
                            if ((byte >> (2 * c2)) & 1u) {
                                asm volatile("ld.shared.u16 %0, [%1];" : "=h"(h0) : "r"(va) : "memory");
                                va += 2u;
                            }
                            if ((byte >> (2 * c2 + 1)) & 1u) {
                                asm volatile("ld.shared.u16 %0, [%1];" : "=h"(h1) : "r"(va) : "memory");
                                va += 2u;
                            }
                            w[c2] = (uint32_t)h0 | ((uint32_t)h1 << 16);
                        }
                        asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(tile_of(a, (int)pos) + 16u * (uint32_t)r),
                                     "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3])
                                     : "memory");
                    }
                }
            }
            // zero tiles for the partners of lone blocks (pair o: position 2o+1)
            for (uint32_t lone = tc_lds(ar.rec) >> 16; lone; lone &= lone - 1) {
                const int o = __ffs(lone) - 1;
                if (o % kTcDecodeWarps == dw)
                    asm volatile("st.shared.u32 [%0], %1;" ::"r"(tile_of(a, 2 * o + 1) + 4u * lane), "r"(0u) : "memory");
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // tiles -> tensor core
            __syncwarp();
            if (lane == 0) tc_arrive(s_u32(&bar_tiles[a]));
            if (lane == 0 && dw == 0) TR(1, c, 5);
        }
    } else if (warp == kMma || warp == kMma2) {  // ------------------------------- MMA issue
        // two issuing warps take alternate chunks: one chunk's waits and record
        // reads overlap the other's MMAs (each commits its own MMAs)
        for (int c = warp == kMma ? 0 : 1; c < nch; c += 2) {
            const int a = c % kTcRing, b = c % kTcSlabBufs;
            if (lane == 0) TR(2, c, 0);
            tc_wait_mma(s_u32(&bar_arr[a]), ring_ph(c));
            if (lane == 0) TR(2, c, 1);
            tc_wait_mma(s_u32(&bar_tiles[a]), ring_ph(c));
            if (lane == 0) TR(2, c, 2);
            tc_wait_mma(s_u32(&bar_slab[b]), slab_ph(c));
            if (lane == 0) TR(2, c, 3);
            // accumulator slots: the epilogue has finished chunk c-3
            // (chunks c-2 .. c hold at most 3 * kTcPairs < kTcSlots started block-rows)
            if (c >= 3) tc_wait_mma(s_u32(&bar_epi[(c - 3) % kTcRing]), ring_ph(c - 3));
            // a block-row continued from the previous chunk accumulates after that
            // chunk's MMAs (issued by the other warp) have completed
            if (c >= 1 && cdesc[a].pA > 0) tc_wait_mma(s_u32(&bar_mma[(c - 1) % kTcRing]), ring_ph(c - 1));
            if (lane == 0) TR(2, c, 4);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            // the record's head and segments (bytes 0..33): three loads in flight at once
            const uint32_t rec = arr[a].rec;
            uint32_t r0, r1, r2, r3, r4, r5, r6, r7, r8;
            asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                         : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
                         : "r"(rec)
                         : "memory");
            asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                         : "=r"(r4), "=r"(r5), "=r"(r6), "=r"(r7)
                         : "r"(rec + 16u)
                         : "memory");
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(r8) : "r"(rec + 32u) : "memory");
            // segments: warp-uniform through redux.sync (one per non-empty block-row);
            // seg[t] is the low half of word 1 + t/2 for even t, the high half for odd t
            const uint32_t nseg = __reduce_or_sync(0xffffffffu, r0 & 0xffu);
            TR(2, c, 5);
            // pair o: slabs at positions 2o, 2o+1 (LBO one slab), tiles at 2o, 2o+1 (LBO one tile)
            const uint32_t ad0 = (uint32_t)umma_desc(slab_of(b, 0), (uint32_t)kSlabBytes, 128u);
            const uint32_t bd0 = (uint32_t)umma_desc(tile_of(a, 0), (uint32_t)kTileBytes, 128u);
            uint32_t o = 0;
#pragma unroll 1
            for (uint32_t t = 0; t < nseg; ++t) {
                const uint32_t i = t >> 1;
                const uint32_t w = i < 4 ? (i < 2 ? (i == 0 ? r1 : r2) : (i == 2 ? r3 : r4))
                                         : (i < 6 ? (i == 4 ? r5 : r6) : (i == 6 ? r7 : r8));
                const uint32_t sg = __reduce_or_sync(0xffffffffu, (t & 1u) ? (w >> 16) : (w & 0xffffu));
                const uint32_t d = tmem_u + (sg & 63u) * (uint32_t)kTcN;
                const uint32_t acc0 = (sg >> 6) & 1u, np = sg >> 7;
                // descriptors of pair o: base + o * stride (two MMAs per step)
                uint32_t ad = ad0 + o * (2u * kSlabBytes >> 4), bd = bd0 + o * (2u * kTileBytes >> 4);
                uint32_t p = 0;
#pragma unroll 1
                for (; p + 1 < np; p += 2) {
                    umma_f16_elect(d, ((uint64_t)kDescHi << 32) | ad, ((uint64_t)kDescHi << 32) | bd, p > 0 ? 1u : acc0);
                    umma_f16_elect(d, ((uint64_t)kDescHi << 32) | (ad + (2u * kSlabBytes >> 4)),
                                   ((uint64_t)kDescHi << 32) | (bd + (2u * kTileBytes >> 4)), 1u);
                    ad += 2u * (2u * kSlabBytes >> 4);
                    bd += 2u * (2u * kTileBytes >> 4);
                }
                if (p < np)
                    umma_f16_elect(d, ((uint64_t)kDescHi << 32) | ad, ((uint64_t)kDescHi << 32) | bd, p > 0 ? 1u : acc0);
                o += np;
            }
            if (lane == 0) {
                // completion of every MMA issued so far: slabs of buffer b free, tiles of
                // slot a free + accumulators of the chunk ready
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                                 s_u32(&bar_sfree[b]))
                             : "memory");
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                                 s_u32(&bar_mma[a]))
                             : "memory");
                TR(2, c, 6);
            }
            __syncwarp();
        }
    } else if (warp < 4) {  // ------------------------------------------------ epilogue
        const int vec = warp * 32 + lane;  // TMEM lane = vector within the group
        for (int c = 0; c < nch; ++c) {
            const int a = c % kTcRing;
            if (threadIdx.x == 0) TR(3, c, 0);
            tc_wait(s_u32(&bar_mma[a]), ring_ph(c));
            if (threadIdx.x == 0) TR(3, c, 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            // block-rows ending in this chunk, from the staged record
            const uint32_t rec = arr[a].rec;
            const int ne = (int)((tc_lds(rec) >> 8) & 0xffu);
            const int brA = cdesc[a].brA;
            for (int e = 0; e < ne; ++e) {
                const uint32_t ea = rec + 64u + 2u * (uint32_t)e;
                const uint32_t w = tc_lds(ea & ~3u);
                const uint32_t en = (ea & 2u) ? (w >> 16) : (w & 0xffffu);
                const int br = brA + (int)(en & 63u), slot = (int)(en >> 6) - 1;
                float v[8];
                if (slot >= 0) {
                    uint32_t r[8];
                    const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)(slot * kTcN);
                    asm volatile(
                        "tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
                          "=r"(r[7])
                        : "r"(taddr)
                        : "memory");
                    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
                    for (int t = 0; t < 8; ++t) v[t] = __uint_as_float(r[t]);
                } else {
#pragma unroll
                    for (int t = 0; t < 8; ++t) v[t] = 0.f;  // empty block-row: y = beta * y
                }
                if (vec < kv) {
                    float *yp = Y + (int64_t)(j0 + vec) * ldy + 8 * (int64_t)br;
                    const int64_t left = m - 8 * (int64_t)br;
                    if (left >= 8 && ((uintptr_t)yp & 15u) == 0) {  // two full 16-byte stores (one sector)
                        float4 lo = make_float4(alpha * v[0], alpha * v[1], alpha * v[2], alpha * v[3]);
                        float4 hi = make_float4(alpha * v[4], alpha * v[5], alpha * v[6], alpha * v[7]);
                        if (beta != 0.f) {
                            const float4 ol = *reinterpret_cast<const float4 *>(yp);
                            const float4 oh = *reinterpret_cast<const float4 *>(yp + 4);
                            lo = make_float4(fmaf(beta, ol.x, lo.x), fmaf(beta, ol.y, lo.y), fmaf(beta, ol.z, lo.z),
                                             fmaf(beta, ol.w, lo.w));
                            hi = make_float4(fmaf(beta, oh.x, hi.x), fmaf(beta, oh.y, hi.y), fmaf(beta, oh.z, hi.z),
                                             fmaf(beta, oh.w, hi.w));
                        }
                        *reinterpret_cast<float4 *>(yp) = lo;
                        *reinterpret_cast<float4 *>(yp + 4) = hi;
                    } else {
                        const int rows = (int)(left < 8 ? left : 8);
#pragma unroll
                        for (int t = 0; t < 8; ++t) {
                            if (t < rows) {
                                float o = alpha * v[t];
                                if (beta != 0.f) o = fmaf(beta, yp[t], o);
                                yp[t] = o;
                            }
                        }
                    }
                }
            }
            asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
            __syncwarp();
            if (lane == 0) {
                tc_arrive(s_u32(&bar_epi[a]));
                tc_arrive(s_u32(&bar_afree[a]));  // the chunk's staged arrays and record are no longer read
            }
            if (threadIdx.x == 0) TR(3, c, 2);
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (warp == kMma)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem) : "memory");
}

// Xb[g][bc][jj][c] = fp16(X[(128g + jj)*ldx + 8bc + c]) (round to nearest even),
// 0 past n and past k.  A transpose through shared memory: a CTA takes 32
// vectors x 16 block columns, reads each vector's 128 consecutive floats
// coalesced, and writes each block column's 32 slab rows (512 contiguous bytes)
// as 16-byte stores.
constexpr int kPackJ = 32, kPackBC = 16, kPackRow = 8 * kPackBC + 8;  // halves per smem row (+8: no conflicts)
__global__ void __launch_bounds__(256) k_pack_x_f16(int64_t n, int32_t k, const float *__restrict__ X, int64_t ldx,
                                                    __half *__restrict__ Xb) {
    __shared__ __align__(16) __half sh[kPackJ * kPackRow];
    const int64_t nbc = (n + 7) / 8;
    const int64_t bc0 = (int64_t)blockIdx.x * kPackBC;
    const int j0 = blockIdx.y * kPackJ;  // vectors up to the padded group end (a multiple of 128)
#pragma unroll 4
    for (int idx = threadIdx.x; idx < kPackJ * 8 * kPackBC; idx += 256) {
        const int r = idx / (8 * kPackBC), c = idx % (8 * kPackBC);
        const int j = j0 + r;
        const int64_t f = 8 * bc0 + c;
        float v = 0.f;
        if (j < k && f < n) v = __ldg(X + (int64_t)j * ldx + f);
        sh[r * kPackRow + c] = __float2half_rn(v);
    }
    __syncthreads();
    for (int idx = threadIdx.x; idx < kPackJ * kPackBC; idx += 256) {
        const int b = idx / kPackJ, r = idx % kPackJ;
        const int j = j0 + r;
        const int64_t bc = bc0 + b;
        if (bc < nbc) {
            const int64_t slot = ((int64_t)(j / kTcM) * nbc + bc) * kTcM + (j % kTcM);
            *reinterpret_cast<uint4 *>(Xb + slot * 8) = *reinterpret_cast<const uint4 *>(sh + r * kPackRow + 8 * b);
        }
    }
}

}  // namespace

spaden_status_t spmm_tc_pack_x(int64_t n, int32_t k, const float *X, int64_t ldx, void *Xb, cudaStream_t st) {
    const int64_t nbc = (n + 7) / 8;
    if (nbc == 0 || k == 0) return SPADEN_OK;
    const int64_t kpad = ((int64_t)k + kTcM - 1) / kTcM * kTcM;  // groups are zero-padded to 128 vectors
    const dim3 grid((unsigned)((nbc + kPackBC - 1) / kPackBC), (unsigned)(kpad / kPackJ));
    k_pack_x_f16<<<grid, 256, 0, st>>>(n, k, X, ldx, (__half *)Xb);
    SPADEN_CUDA_TRY(cudaGetLastError());
    return SPADEN_OK;
}

static spaden_status_t build_tc_schedule(Matrix &A, int G, cudaStream_t st) {
    int32_t *cnt = nullptr;
    SPADEN_CUDA_TRY(dmalloc(&A.tc_cta_start, sizeof(int32_t) * (G + 1), st));
    const size_t ntmp = scan_tmp_ints(G + 1);
    SPADEN_CUDA_TRY(cudaMallocAsync(&cnt, sizeof(int32_t) * (ntmp + G + 1), st));
    k_tc_sched<<<1, 1, 0, st>>>(A.blk_rowptr, A.blk_offset, A.Bnrow, G, A.tc_cta_start, nullptr, nullptr, nullptr);
    cudaError_t e = exclusive_scan_i32(A.tc_cta_start, A.tc_cta_start, G, cnt, st);
    int32_t total = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(&total, A.tc_cta_start + G, sizeof(int32_t), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    // chunk descriptors, then the chunks' MMA records (16-byte aligned: bulk-copied)
    const size_t rec_off = (sizeof(TcChunk) * (size_t)std::max(1, total) + 127) & ~(size_t)127;
    if (e == cudaSuccess) e = dmalloc(&A.tc_chunks, rec_off + sizeof(TcRec) * (size_t)std::max(1, total), st);
    if (e == cudaSuccess) {
        k_tc_sched<<<1, 1, 0, st>>>(A.blk_rowptr, A.blk_offset, A.Bnrow, G, nullptr, cnt + ntmp, A.tc_cta_start,
                                    (TcChunk *)A.tc_chunks);
        if (total > 0)
            k_tc_ops<<<(unsigned)((total + 255) / 256), 256, 0, st>>>(
                A.blk_rowptr, (const TcChunk *)A.tc_chunks, total, (TcRec *)((char *)A.tc_chunks + rec_off));
        e = cudaGetLastError();
    }
    cudaFreeAsync(cnt, st);
    if (e != cudaSuccess) return cuda_status(e, "tensor-core SpMM schedule");
    A.tc_nchunks = total;
    A.tc_grid = G;
    A.aux_bytes += (int64_t)(rec_off + sizeof(TcRec) * (size_t)total + sizeof(int32_t) * (G + 1));
    return SPADEN_OK;
}

#ifdef SPADEN_TC_TRACE
extern "C" __attribute__((visibility("default"))) int spaden_debug_tc_trace(void *buf) {
    return (int)cudaMemcpyToSymbol(g_tc_trace, &buf, sizeof(buf));
}
#endif

spaden_status_t spmm_tc_launch(Matrix &A, float alpha, const void *Xb, int32_t k, float beta, float *Y,
                               int64_t ldy, cudaStream_t st) {
    if (A.m == 0 || k == 0) return SPADEN_OK;
    static bool attr_set[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64 && !attr_set[dev]) {
        SPADEN_CUDA_TRY(cudaFuncSetAttribute(k_spmm_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, kTcSmem));
        attr_set[dev] = true;
    }
    if (A.tc_grid == 0) {  // first call: the chunk schedule (one host synchronisation)
        int sms = 148;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        const spaden_status_t s =
            build_tc_schedule(A, (int)std::max<int64_t>(1, std::min<int64_t>(std::min(sms, 1024), A.Bnrow)), st);
        if (s != SPADEN_OK) return s;
    }
    for (int32_t j0 = 0; j0 < k; j0 += kTcM) {
        const int32_t kv = std::min<int32_t>(kTcM, k - j0);
        const size_t rec_off = (sizeof(TcChunk) * (size_t)std::max<int64_t>(1, A.tc_nchunks) + 127) & ~(size_t)127;
        k_spmm_tc<<<A.tc_grid, kTcThreads, kTcSmem, st>>>(A.m, (const TcChunk *)A.tc_chunks,
                                                            (const TcRec *)((const char *)A.tc_chunks + rec_off),
                                                            A.tc_cta_start,
                                                            A.blk_rowptr, A.blk_col, A.bitmap, A.blk_offset,
                                                            (const __half *)A.values, (const __half *)Xb, (A.n + 7) / 8, j0, kv,
                                                            alpha, beta, Y, ldy);
        SPADEN_CUDA_TRY(cudaGetLastError());
    }
    return SPADEN_OK;
}

}  // namespace spaden
