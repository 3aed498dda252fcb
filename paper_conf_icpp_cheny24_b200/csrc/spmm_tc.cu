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
//              core matrix each, LBO = tile2 - tile1): a warp decodes a block
//              with lane l owning bits 2l, 2l+1 -- exactly the paper's Alg. 2
//              lane mapping, value index = offset + popcount rank.
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
//   warp 13    producer lane: bulk-copies the chunk's blk_rowptr, bitmap,
//              blk_col, blk_offset and value slices (4-chunk ring) and, one
//              chunk behind, walks the staged blk_rowptr into the chunk's MMA
//              list and the list of block-rows ending in it;
//   warps 4-11 copy the x slabs of the chunk's blocks (cp.async, 3 slab
//              buffers) and decode the blocks into dense tiles (4-chunk ring);
//   warp 12    TMEM allocation + the MMA issue thread;
//   warps 0-3  epilogue (TMEM lanes 32w..32w+31 = vectors): tcgen05.ld of the
//              accumulators of the block-rows ending in the chunk, alpha*D +
//              beta*Y written as two 16-byte stores per vector and block-row.
// mbarriers per ring slot: arrays landed, MMA list written, tiles written,
// MMAs complete (tcgen05.commit: tiles free + accumulators ready), epilogue
// done; per slab buffer: slab copies landed (cp.async.mbarrier.arrive), MMAs
// reading it complete.  The MMAs of chunk c wait for the epilogue of chunk
// c-3, so at most 3 * kTcPairs < kTcSlots accumulators are live.
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
constexpr int kTcArrBytes = 5120; // one chunk's staged arrays (brp, bitmap, blk_col, blk_offset, values)
constexpr int kTcRing = 4;        // arrays, tiles and accumulator hand-off: 4 chunks in flight
constexpr int kTcSlabBufs = 3;    // x slabs: 3 chunks (the big buffers)
constexpr int kTcDecodeWarps = 8;
constexpr int kTcSlabBytes = kTcBlocks * kSlabBytes;
constexpr int kTcTileBytes = kTcBlocks * kTileBytes;
constexpr int kTcSmem = kTcSlabBufs * kTcSlabBytes + kTcRing * (kTcTileBytes + kTcArrBytes) + kSlabBytes + kTileBytes;
constexpr int kTcThreads = (4 + kTcDecodeWarps + 2) * 32;

// one chunk of the schedule (48 bytes)
struct alignas(16) TcChunk {
    int brA, pA;     // first block-row touched, its first pair in this chunk
    int brE, pE;     // block-rows [brA, brE) end here; block-row brE continues (pE pairs done) if pE > 0
    int B0, B1;      // blocks [B0, B1)
    int seq0;        // accumulator sequence number of the first non-empty block-row touched
    int V0, V1;      // values [V0, V1) = blk_offset[B0], blk_offset[B1]
    int pad0, pad1, pad2;
};

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
__device__ __forceinline__ void tc_bulk(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
        "l"(src), "r"(bytes), "r"(bar)
        : "memory");
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
// instruction descriptor: kind::f16, A = B = F16 (K-major), D = F32, M = 128, N = 8
constexpr uint32_t kTcIdesc = (1u << 4) | ((uint32_t)(kTcN >> 3) << 17) | ((uint32_t)(kTcM >> 4) << 24);

__device__ __forceinline__ void umma_f16(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t accumulate) {
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
        " tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(kTcIdesc), "r"(accumulate)
        : "memory");
}

// staged arrays of a chunk inside its buffer (16-byte aligned regions)
struct TcArr {
    uint32_t brp, bmp, col, off, val;  // shared addresses of element 0 of each slice
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

__global__ void __launch_bounds__(kTcThreads, 1)
k_spmm_tc(int64_t m, const TcChunk *__restrict__ chunks, const int32_t *__restrict__ cta_start,
          const int32_t *__restrict__ brp, const int32_t *__restrict__ bcol, const uint64_t *__restrict__ bitmap,
          const int32_t *__restrict__ boff, const __half *__restrict__ vals, const __half *__restrict__ Xb,
          int32_t k, int32_t j0, int32_t kv, float alpha, float beta, float *__restrict__ Y, int64_t ldy) {
    extern __shared__ __align__(1024) unsigned char smem[];
    __shared__ TcChunk cdesc[kTcRing];
    __shared__ TcArr arr[kTcRing];
    // a = c % kTcRing (arrays, tiles, accumulator hand-off), b = c % kTcSlabBufs (x slabs)
    __shared__ __align__(8) uint64_t bar_arr[kTcRing];    // arrays landed (producer, tx)
    __shared__ __align__(8) uint64_t bar_afree[kTcRing];  // arrays of chunk c no longer read (MMA issued)
    __shared__ __align__(8) uint64_t bar_epi[kTcRing];    // epilogue done with chunk c (4 warps)
    __shared__ int2 ends[kTcRing][kTcRows];               // (block-row, slot or -1) ending in chunk c
    __shared__ int nends[kTcRing];
    __shared__ uint4 ops[kTcRing][kTcPairs][2];           // the chunk's MMAs: (adesc, bdesc), (d, accumulate)
    __shared__ int nops[kTcRing];
    __shared__ __align__(8) uint64_t bar_ops[kTcRing];    // MMA list and ends of chunk c written (producer)
    __shared__ __align__(8) uint64_t bar_tiles[kTcRing];  // tiles decoded (decode warps)
    __shared__ __align__(8) uint64_t bar_mma[kTcRing];    // chunk's MMAs complete (commit): tiles free,
                                                          // accumulators ready
    __shared__ __align__(8) uint64_t bar_sfree[kTcSlabBufs];  // MMAs reading the slabs complete (commit)
    __shared__ __align__(8) uint64_t bar_slab[kTcSlabBufs];   // slab cp.asyncs landed (every decode thread)
    __shared__ uint32_t tmem_base_sh;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t sb = s_u32(smem);
    const uint32_t tiles0 = sb + (uint32_t)kTcSlabBufs * kTcSlabBytes;
    const uint32_t arr0 = tiles0 + (uint32_t)kTcRing * kTcTileBytes;
    const uint32_t zero_slab = arr0 + (uint32_t)kTcRing * kTcArrBytes, zero_tile = zero_slab + kSlabBytes;
    const int c0 = cta_start[blockIdx.x], nch = cta_start[blockIdx.x + 1] - c0;
    const int kMma = 4 + kTcDecodeWarps, kProd = kMma + 1;

    if (threadIdx.x == 0) {
        for (int a = 0; a < kTcRing; ++a) {
            tc_mbar_init(s_u32(&bar_arr[a]), 1);
            tc_mbar_init(s_u32(&bar_afree[a]), 1);
            tc_mbar_init(s_u32(&bar_ops[a]), 1);
            tc_mbar_init(s_u32(&bar_epi[a]), 4);
            tc_mbar_init(s_u32(&bar_tiles[a]), kTcDecodeWarps);
            tc_mbar_init(s_u32(&bar_mma[a]), 2);  // tcgen05.commit + the MMA thread's own arrive (ends list)
        }
        for (int b = 0; b < kTcSlabBufs; ++b) {
            tc_mbar_init(s_u32(&bar_sfree[b]), 1);
            tc_mbar_init(s_u32(&bar_slab[b]), kTcDecodeWarps * 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    // zero slab + zero tile (the partner of a block-row's lone last block)
    for (int i = threadIdx.x; i < (kSlabBytes + kTileBytes) / 16; i += blockDim.x)
        asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(zero_slab + 16u * i), "r"(0u) : "memory");
    if (warp == kMma) {  // TMEM: 512 columns = kTcSlots accumulators of 8 fp32 columns
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(s_u32(&tmem_base_sh))
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // zero slab/tile -> tensor core
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tmem_base_sh;
    auto slab_of = [&](int b, int q) { return sb + (uint32_t)b * kTcSlabBytes + (uint32_t)q * kSlabBytes; };
    auto tile_of = [&](int a, int q) { return tiles0 + (uint32_t)a * kTcTileBytes + (uint32_t)q * kTileBytes; };
    auto ring_ph = [](int c) { return (uint32_t)((c / kTcRing) & 1); };
    auto slab_ph = [](int c) { return (uint32_t)((c / kTcSlabBufs) & 1); };

    if (warp == kProd) {  // ------------------------------- producer: arrays, then x slabs
        if (lane == 0) {
            // the MMA list and the block-rows ending in chunk cw (walk of its staged
            // blk_rowptr, one chunk behind the copies); ops / ends of its ring slot were
            // last read by the MMA thread and the epilogue of chunk cw - kTcRing
            auto walk = [&](int cw) {
                const int a = cw % kTcRing, b = cw % kTcSlabBufs;
                tc_wait(s_u32(&bar_arr[a]), ring_ph(cw));
                if (cw >= kTcRing) tc_wait(s_u32(&bar_epi[a]), ring_ph(cw - kTcRing));
                const TcChunk ch = cdesc[a];
                const TcArr ar = arr[a];
                const int rows = ch.brE - ch.brA + (ch.pE > 0 ? 1 : 0);
                int seq = ch.seq0, ne = 0, no = 0;
                for (int i = 0; i < rows; ++i) {
                    const int s0 = (int)tc_lds(ar.brp + 4u * i), nb = (int)tc_lds(ar.brp + 4u * i + 4u) - s0;
                    if (ch.brA + i < ch.brE) ends[a][ne++] = make_int2(ch.brA + i, nb ? seq % kTcSlots : -1);
                    if (nb == 0) continue;
                    const int npr = (nb + 1) >> 1;
                    const int pb = i == 0 ? ch.pA : 0;
                    const int pe = (ch.brA + i < ch.brE) ? npr : ch.pE;
                    const uint32_t d = tmem + (uint32_t)((seq % kTcSlots) * kTcN);
                    for (int p = pb; p < pe; ++p) {
                        const int q1 = s0 + 2 * p - ch.B0;
                        const bool two = 2 * p + 1 < nb;
                        const uint32_t s1 = slab_of(b, q1), t1 = tile_of(a, q1);
                        const uint32_t s2 = two ? slab_of(b, q1 + 1) : zero_slab;
                        const uint32_t t2 = two ? tile_of(a, q1 + 1) : zero_tile;
                        const uint64_t ad = umma_desc(s1, s2 - s1, 128u), bd = umma_desc(t1, t2 - t1, 128u);
                        ops[a][no][0] = make_uint4((uint32_t)ad, (uint32_t)(ad >> 32), (uint32_t)bd, (uint32_t)(bd >> 32));
                        ops[a][no][1] = make_uint4(d, p > 0 ? 1u : 0u, 0u, 0u);
                        ++no;
                    }
                    if (ch.brA + i < ch.brE) ++seq;
                }
                nends[a] = ne;
                nops[a] = no;
                tc_arrive(s_u32(&bar_ops[a]));
            };
            TcChunk next = nch > 0 ? chunks[c0] : TcChunk{};  // descriptors one chunk ahead
            for (int c = 0; c < nch; ++c) {
                const int a = c % kTcRing;
                const TcChunk ch = next;
                if (c + 1 < nch) next = chunks[c0 + c + 1];
                if (c >= kTcRing) tc_wait(s_u32(&bar_afree[a]), ring_ph(c - kTcRing));
                cdesc[a] = ch;
                const int nrows = ch.brE - ch.brA + (ch.pE > 0 ? 1 : 0);
                const int v0 = ch.V0, v1 = ch.V1;
                uint32_t cur = arr0 + (uint32_t)a * kTcArrBytes;
                uint32_t total = 0;
                const void *srcs[5] = {brp + ch.brA, bitmap + ch.B0, bcol + ch.B0, boff + ch.B0, vals + v0};
                const uint32_t lens[5] = {4u * (uint32_t)(nrows + 1), 8u * (uint32_t)(ch.B1 - ch.B0),
                                          4u * (uint32_t)(ch.B1 - ch.B0), 4u * (uint32_t)(ch.B1 - ch.B0),
                                          2u * (uint32_t)(v1 - v0)};
                uint32_t addr[5], asrc[5], asz[5];
                for (int r = 0; r < 5; ++r) {
                    const uintptr_t lo = (uintptr_t)srcs[r];
                    const uintptr_t alo = lo & ~(uintptr_t)15;
                    asz[r] = lens[r] ? (uint32_t)(((lo + lens[r] + 15) & ~(uintptr_t)15) - alo) : 0u;
                    asrc[r] = (uint32_t)(lo - alo);
                    addr[r] = cur + asrc[r];
                    cur += asz[r];
                    total += asz[r];
                }
                arr[a] = TcArr{addr[0], addr[1], addr[2], addr[3], addr[4]};
                const uint32_t fb = s_u32(&bar_arr[a]);
                tc_arrive_tx(fb, total);
                uint32_t dst = arr0 + (uint32_t)a * kTcArrBytes;
                for (int r = 0; r < 5; ++r) {
                    if (asz[r]) tc_bulk(dst, (const void *)((uintptr_t)srcs[r] - asrc[r]), asz[r], fb);
                    dst += asz[r];
                }
                if (c >= 1) walk(c - 1);
            }
            if (nch > 0) walk(nch - 1);
        }
    } else if (warp >= 4 && warp < kMma) {  // --------------------------------- decode
        const int dw = warp - 4;
        for (int c = 0; c < nch; ++c) {
            const int a = c % kTcRing, b = c % kTcSlabBufs;
            tc_wait(s_u32(&bar_arr[a]), ring_ph(c));
            const TcChunk ch = cdesc[a];
            const TcArr ar = arr[a];
            const int nblk = ch.B1 - ch.B0;
            // x slabs: cp.async by the decode warps, a warp per block's slab (16 bytes per
            // lane and step); many small bulk copies serialise in the copy engine
            if (c >= kTcSlabBufs) tc_wait(s_u32(&bar_sfree[b]), slab_ph(c - kTcSlabBufs));
            {
                // this warp's blocks q = dw + 8i: all their pieces in flight at once
                // (distinct address registers: an LDGSTS holds its operands until
                // the data returns, so a reused register would serialise the slabs)
                constexpr int kPer = (kTcBlocks + kTcDecodeWarps - 1) / kTcDecodeWarps;
                uint64_t srcs[kPer];
                uint32_t dsts[kPer];
#pragma unroll
                for (int i = 0; i < kPer; ++i) {
                    const int q = dw + kTcDecodeWarps * i;
                    const int bc = q < nblk ? (int)tc_lds(ar.col + 4u * q) : 0;
                    srcs[i] = (uint64_t)(Xb + ((int64_t)bc * k + j0) * 8);
                    dsts[i] = slab_of(b, q);
                }
#pragma unroll
                for (int r = 0; r < kTcM / 32; ++r) {
                    const int piece = lane + 32 * r;
#pragma unroll
                    for (int i = 0; i < kPer; ++i) {
                        if (dw + kTcDecodeWarps * i < nblk && piece < kv)
                            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dsts[i] + 16u * piece),
                                         "l"(srcs[i] + 16ull * piece)
                                         : "memory");
                    }
                }
                // the slab buffer's barrier completes when every decode thread's copies
                // have landed; the decode warps move on without waiting
                asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(s_u32(&bar_slab[b]))
                             : "memory");
            }
            if (c >= kTcRing) tc_wait(s_u32(&bar_mma[a]), ring_ph(c - kTcRing));  // tile slot free
            const int v0 = (int)tc_lds(ar.off);  // blk_offset of the chunk's first block
            // a warp per block, lane l -> bits 2l, 2l+1 (row l/4, columns 2(l%4), 2(l%4)+1)
            for (int q = dw; q < nblk; q += kTcDecodeWarps) {
                const uint32_t lo = tc_lds(ar.bmp + 8u * q), hi = tc_lds(ar.bmp + 8u * q + 4u);
                const uint64_t bm = ((uint64_t)hi << 32) | lo;
                const int off = (int)tc_lds(ar.off + 4u * q) - v0;
                const int bit = 2 * lane;
                const uint32_t two = (uint32_t)(bm >> bit) & 3u;
                uint32_t word = 0;
                if (two) {
                    const int idx = off + __popcll(bm & ((1ull << bit) - 1ull));
                    const uint32_t a0 = ar.val + 2u * (uint32_t)idx;
                    uint16_t h0 = 0, h1 = 0;
                    if (two & 1u) asm volatile("ld.shared.u16 %0, [%1];" : "=h"(h0) : "r"(a0) : "memory");
                    if (two & 2u)
                        asm volatile("ld.shared.u16 %0, [%1];" : "=h"(h1) : "r"(a0 + 2u * (two & 1u)) : "memory");
                    word = (uint32_t)h0 | ((uint32_t)h1 << 16);
                }
                asm volatile("st.shared.u32 [%0], %1;" ::"r"(tile_of(a, q) + 4u * lane), "r"(word) : "memory");
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // tiles -> tensor core
            __syncwarp();
            if (lane == 0) tc_arrive(s_u32(&bar_tiles[a]));
        }
    } else if (warp == kMma) {  // ------------------------------------------- MMA issue
        for (int c = 0; c < nch; ++c) {
            const int a = c % kTcRing, b = c % kTcSlabBufs;
            tc_wait(s_u32(&bar_tiles[a]), ring_ph(c));
            tc_wait(s_u32(&bar_ops[a]), ring_ph(c));
            tc_wait(s_u32(&bar_slab[b]), slab_ph(c));
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // cp.async slabs -> tensor core
            // accumulator slots: the epilogue has finished chunk c-3 (chunks c-2 .. c
            // hold at most 3 * kTcPairs < kTcSlots started block-rows)
            if (c >= 3) tc_wait(s_u32(&bar_epi[(c - 3) % kTcRing]), ring_ph(c - 3));
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            if (lane == 0) {
                tc_arrive(s_u32(&bar_afree[a]));  // decoding is done: the staged arrays are free
                const int no = nops[a];
                for (int o = 0; o < no; ++o) {
                    const uint4 dd = ops[a][o][0], dx = ops[a][o][1];
                    umma_f16(dx.x, ((uint64_t)dd.y << 32) | dd.x, ((uint64_t)dd.w << 32) | dd.z, dx.y);
                }
                // completion of every MMA issued so far: slabs of buffer b free, tiles of
                // slot a free + accumulators of the chunk ready
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                                 s_u32(&bar_sfree[b]))
                             : "memory");
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                                 s_u32(&bar_mma[a]))
                             : "memory");
                tc_arrive(s_u32(&bar_mma[a]));  // release: the ends list written above
            }
            __syncwarp();
        }
    } else if (warp < 4) {  // ------------------------------------------------ epilogue
        const int vec = warp * 32 + lane;  // TMEM lane = vector within the group
        for (int c = 0; c < nch; ++c) {
            const int a = c % kTcRing;
            tc_wait(s_u32(&bar_mma[a]), ring_ph(c));
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const int ne = nends[a];
            for (int e = 0; e < ne; ++e) {  // block-rows ending in this chunk
                const int2 en = ends[a][e];
                const int br = en.x;
                float v[8];
                if (en.y >= 0) {
                    uint32_t r[8];
                    const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)(en.y * kTcN);
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
            if (lane == 0) tc_arrive(s_u32(&bar_epi[a]));
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (warp == kMma)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem) : "memory");
}

// Xb[bc][j][c] = fp16(X[j*ldx + 8bc + c]) (round to nearest even), 0 past n
__global__ void k_pack_x_f16(int64_t n, int32_t k, const float *__restrict__ X, int64_t ldx, __half *__restrict__ Xb) {
    const int64_t nbc = (n + 7) / 8;
    const int64_t total = nbc * (int64_t)k;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t bc = t / k;
        const int j = (int)(t - bc * k);
        const float *src = X + (int64_t)j * ldx + 8 * bc;
        __align__(16) __half h[8];
#pragma unroll
        for (int c = 0; c < 8; ++c) h[c] = (8 * bc + c < n) ? __float2half_rn(src[c]) : __float2half_rn(0.f);
        *reinterpret_cast<uint4 *>(Xb + t * 8) = *reinterpret_cast<const uint4 *>(h);
    }
}

}  // namespace

spaden_status_t spmm_tc_pack_x(int64_t n, int32_t k, const float *X, int64_t ldx, void *Xb, cudaStream_t st) {
    const int64_t total = ((n + 7) / 8) * (int64_t)k;
    if (total == 0) return SPADEN_OK;
    const unsigned grid = (unsigned)std::min<int64_t>((total + 255) / 256, 148 * 32);
    k_pack_x_f16<<<grid, 256, 0, st>>>(n, k, X, ldx, (__half *)Xb);
    SPADEN_CUDA_TRY(cudaGetLastError());
    return SPADEN_OK;
}

static spaden_status_t build_tc_schedule(Matrix &A, int G, cudaStream_t st) {
    int32_t *cnt = nullptr;
    SPADEN_CUDA_TRY(cudaMalloc(&A.tc_cta_start, sizeof(int32_t) * (G + 1)));
    const size_t ntmp = scan_tmp_ints(G + 1);
    SPADEN_CUDA_TRY(cudaMallocAsync(&cnt, sizeof(int32_t) * (ntmp + G + 1), st));
    k_tc_sched<<<1, 1, 0, st>>>(A.blk_rowptr, A.blk_offset, A.Bnrow, G, A.tc_cta_start, nullptr, nullptr, nullptr);
    cudaError_t e = exclusive_scan_i32(A.tc_cta_start, A.tc_cta_start, G, cnt, st);
    int32_t total = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(&total, A.tc_cta_start + G, sizeof(int32_t), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e == cudaSuccess) e = cudaMalloc(&A.tc_chunks, sizeof(TcChunk) * (size_t)std::max(1, total));
    if (e == cudaSuccess) {
        k_tc_sched<<<1, 1, 0, st>>>(A.blk_rowptr, A.blk_offset, A.Bnrow, G, nullptr, cnt + ntmp, A.tc_cta_start,
                                    (TcChunk *)A.tc_chunks);
        e = cudaGetLastError();
    }
    cudaFreeAsync(cnt, st);
    if (e != cudaSuccess) return cuda_status(e, "tensor-core SpMM schedule");
    A.tc_nchunks = total;
    A.tc_grid = G;
    A.aux_bytes += (int64_t)(sizeof(TcChunk) * (size_t)total + sizeof(int32_t) * (G + 1));
    return SPADEN_OK;
}

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
        k_spmm_tc<<<A.tc_grid, kTcThreads, kTcSmem, st>>>(A.m, (const TcChunk *)A.tc_chunks, A.tc_cta_start,
                                                            A.blk_rowptr, A.blk_col, A.bitmap, A.blk_offset,
                                                            (const __half *)A.values, (const __half *)Xb, k, j0, kv,
                                                            alpha, beta, Y, ldy);
        SPADEN_CUDA_TRY(cudaGetLastError());
    }
    return SPADEN_OK;
}

}  // namespace spaden
