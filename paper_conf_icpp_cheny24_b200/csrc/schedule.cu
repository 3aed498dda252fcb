// schedule.cu -- SpMV work schedule, built once at conversion time.
//
// The v1 SpMV kernel streams the bitBSR arrays through shared memory in
// "tiles": runs of WHOLE block-rows [br0, br1) whose blocks, values and
// blk_rowptr slice fit one pipeline stage (TileCfg::stage_bytes).  Keeping block-rows
// whole keeps each row's summation order a function of that block-row alone
// (deterministic and independent of how rows are partitioned across GPUs).
// A block-row too large for half a stage is "long": it is listed separately,
// cut into kLongChunk-block chunks (counted from the row start) processed
// straight from global memory by k_spmv_long_chunks, and its chunk partials are
// summed in chunk order by k_spmv_long_fixup.
//
// Tiles are packed greedily inside segments of kSeg block-rows (one thread per
// segment; two passes: count, then write after a scan of the counts).
#include <cstdlib>

#include "internal.cuh"

namespace spaden {
namespace {

constexpr int kSeg = 256;

// stage bytes of a block-row: `blk_bytes` per block (copied metadata + partial
// scratch), its values, its blk_rowptr entry
__device__ __forceinline__ int64_t br_cost(const int32_t *brp, const int32_t *boff, int64_t br, int sv,
                                           int blk_bytes, int32_t *nb_out, int32_t *nv_out) {
    const int b0 = brp[br], b1 = brp[br + 1];
    const int nv = boff[b1] - boff[b0];
    *nb_out = b1 - b0;
    *nv_out = nv;
    return (int64_t)blk_bytes * (b1 - b0) + (int64_t)sv * nv + 4;
}

// Long rows are classified with the SpMV cost (kBlockStageBytes per block) so
// SpMV and SpMM schedules (pack_blk_bytes = 16 + 4(8K+1)) share one long-row set;
// a normal row that does not fit a stage under the pack cost sets *too_big.
template <bool WRITE>
__global__ void k_pack(int64_t Bnrow, const int32_t *__restrict__ brp, const int32_t *__restrict__ boff,
                       int sv, int64_t cap, int64_t long_cost, int pack_blk_bytes, bool skip_empty,
                       uint32_t *too_big,
                       int32_t *__restrict__ seg_tiles,
                       int32_t *__restrict__ seg_long, const int32_t *__restrict__ tile_start,
                       const int32_t *__restrict__ long_start, TileDesc *__restrict__ tiles,
                       int32_t *__restrict__ long_rows) {
    const int64_t seg = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nseg = (Bnrow + kSeg - 1) / kSeg;
    if (seg >= nseg) return;
    const int64_t s0 = seg * kSeg, s1 = min(Bnrow, s0 + kSeg);
    int nt = 0, nl = 0;
    int64_t open_br = -1, open_cost = 0;
    int32_t tbase = WRITE ? tile_start[seg] : 0;
    int32_t lbase = WRITE ? long_start[seg] : 0;
    auto close = [&](int64_t br_end) {
        if (open_br >= 0) {
            if (WRITE) {
                TileDesc d;
                d.br0 = (int32_t)open_br;
                d.br1 = (int32_t)br_end;
                d.b0 = brp[open_br];
                d.b1 = brp[br_end];
                d.v0 = boff[d.b0];
                d.v1 = boff[d.b1];
                d.pad0 = d.pad1 = 0;
                tiles[tbase + nt] = d;
            }
            ++nt;
            open_br = -1;
            open_cost = 0;
        }
    };
    for (int64_t br = s0; br < s1; ++br) {
        int32_t nb, nv;
        if (br_cost(brp, boff, br, sv, kBlockStageBytes, &nb, &nv) > long_cost) {
            close(br);
            if (WRITE && long_rows) long_rows[lbase + nl] = (int32_t)br;
            ++nl;
            continue;
        }
        if (skip_empty && nb == 0) {  // hybrid: y of block-rows without blocks is done by the residual pass
            close(br);
            continue;
        }
        const int64_t c = br_cost(brp, boff, br, sv, pack_blk_bytes, &nb, &nv);
        if (c > cap && too_big) atomicOr(too_big, 1u);
        if (open_br >= 0 && (open_cost + c > cap || br - open_br >= kMaxTileRows)) close(br);
        if (open_br < 0) open_br = br;
        open_cost += c;
    }
    close(s1);
    if (!WRITE) {
        seg_tiles[seg] = nt;
        seg_long[seg] = nl;
    }
}

// ---------------------------------------------------------------------------
// Row rotations of the slot decode (bank conflicts).  The tiled kernel decodes a
// 32-block unit with one lane per block and one predicated shared-memory load
// per bit slot: instruction i = 8t + c reads, in every lane whose block has that
// bit, the block's value at its popcount rank.  Lanes whose values sit in the
// same bank at different words serialise (one wavefront per distinct word).  A
// lane may walk its block's rows in any cyclic order -- row (t + rho) & 7 at
// step t -- without changing any row's own fma order, so y is bitwise the same
// for every rho.  This pass picks rho per block greedily, lanes in order: for
// each lane the rotation that adds the fewest wavefronts given the lanes before
// it (a warp per tile; lanes evaluate the 8 rotations x 64 slots in parallel,
// per-(instruction, bank) word counts in shared memory).  Banks are taken
// relative to the tile's value region, which the kernel copies from a 16-byte
// aligned start (a constant bank shift per tile, invisible to the conflicts).
constexpr int kRotWarps = 8;

template <int SV>
__global__ void __launch_bounds__(32 * kRotWarps)
k_rot_greedy(const TileDesc *__restrict__ tiles, int ntiles, const uint64_t *__restrict__ bitmap,
             const int32_t *__restrict__ blk_offset, uint8_t *__restrict__ rot, int passes) {
    __shared__ uint8_t load[kRotWarps][64][32];  // words per (slot instruction, bank) so far
    __shared__ uint8_t rho_s[kRotWarps][32];     // the unit's chosen rotations (local-search passes)
    __shared__ uint8_t mx[kRotWarps][64];        // max over banks = wavefronts of the instruction
    __shared__ uint8_t sload[kRotWarps][8][32];  // the 8 partial stores (step t -> row (t+rho)&7)
    __shared__ uint8_t smx[kRotWarps][8];
    const int w = threadIdx.x >> 5, j = threadIdx.x & 31;
    const int t = blockIdx.x * kRotWarps + w;
    if (t >= ntiles) return;
    const int b0 = tiles[t].b0, b1 = tiles[t].b1;
    uint32_t *lw = reinterpret_cast<uint32_t *>(&load[w][0][0]);
    const int r = j & 7;
    for (int ub = b0; ub < b1; ub += 32) {
        for (int q = j; q < 64 * 32 / 4; q += 32) lw[q] = 0u;
        for (int q = j; q < 8 * 32 / 4; q += 32) reinterpret_cast<uint32_t *>(&sload[w][0][0])[q] = 0u;
        if (j < 16) reinterpret_cast<uint32_t *>(&mx[w][0])[j] = 0u;
        if (j < 2) reinterpret_cast<uint32_t *>(&smx[w][0])[j] = 0u;
        __syncwarp();
        const int nbu = min(32, b1 - ub);
        for (int l = 0; l < nbu; ++l) {
            const uint64_t bm = __ldg(bitmap + ub + l);
            const int off = __ldg(blk_offset + ub + l);
            int delta = 0;
#pragma unroll 4
            for (int k = 0; k < 16; ++k) {
                const int sl = (j >> 3) + 4 * k;
                if ((bm >> sl) & 1ull) {
                    const int rank = __popcll(bm & ((1ull << sl) - 1ull));
                    const int bank = (int)((((int64_t)off + rank) * SV) >> 2) & 31;
                    const int ins = 8 * (((sl >> 3) - r) & 7) + (sl & 7);
                    delta += (load[w][ins][bank] + 1 > mx[w][ins]) ? 1 : 0;
                }
            }
            // the block's partial stores: step t writes row (t + r) & 7 at word
            // 9 * lane + row of the unit's scratch (kPartStride = 36 bytes); the
            // vectorised stores (SPADEN_ROT_V4) are conflict free whatever r
#pragma unroll
            for (int h = 0; h < (SPADEN_ROT_V4 ? 0 : 2); ++h) {
                const int tt = 2 * (j >> 3) + h;
                const int bank = (9 * l + ((tt + r) & 7)) & 31;
                delta += (sload[w][tt][bank] + 1 > smx[w][tt]) ? 1 : 0;
            }
            delta += __shfl_xor_sync(0xffffffffu, delta, 8);
            delta += __shfl_xor_sync(0xffffffffu, delta, 16);
            int key = delta * 8 + r;  // fewest added wavefronts, then the smallest rotation
            key = min(key, __shfl_xor_sync(0xffffffffu, key, 1));
            key = min(key, __shfl_xor_sync(0xffffffffu, key, 2));
            key = min(key, __shfl_xor_sync(0xffffffffu, key, 4));
            const int best = key & 7;
#pragma unroll
            for (int h = 0; h < 2; ++h) {  // lane j commits slots j and j + 32 (distinct instructions)
                const int sl = j + 32 * h;
                if ((bm >> sl) & 1ull) {
                    const int rank = __popcll(bm & ((1ull << sl) - 1ull));
                    const int bank = (int)((((int64_t)off + rank) * SV) >> 2) & 31;
                    const int ins = 8 * (((sl >> 3) - best) & 7) + (sl & 7);
                    const int nl = load[w][ins][bank] + 1;
                    load[w][ins][bank] = (uint8_t)nl;
                    if (nl > mx[w][ins]) mx[w][ins] = (uint8_t)nl;
                }
            }
            if (j < 8) {
                const int bank = (9 * l + ((j + best) & 7)) & 31;
                const int nl = sload[w][j][bank] + 1;
                sload[w][j][bank] = (uint8_t)nl;
                if (nl > smx[w][j]) smx[w][j] = (uint8_t)nl;
            }
            if (j == 0) {
                rot[ub + l] = (uint8_t)best;
                rho_s[w][l] = (uint8_t)best;
            }
            __syncwarp();
        }
        // local search (value loads only, SPADEN_ROT_V4): take each lane's block out
        // again, recompute the maxima it may have set, and re-pick its rotation
        // against all the other lanes of the unit (never worse than the greedy)
        for (int pass = 0; SPADEN_ROT_V4 && pass < passes; ++pass) {
            for (int l = 0; l < nbu; ++l) {
                const uint64_t bm = __ldg(bitmap + ub + l);
                const int off = __ldg(blk_offset + ub + l);
                const int cur = rho_s[w][l];
                int touched[2] = {-1, -1};  // instructions this lane's slots j, j + 32 used
#pragma unroll
                for (int h = 0; h < 2; ++h) {  // remove
                    const int sl = j + 32 * h;
                    if ((bm >> sl) & 1ull) {
                        const int rank = __popcll(bm & ((1ull << sl) - 1ull));
                        const int bank = (int)((((int64_t)off + rank) * SV) >> 2) & 31;
                        const int ins = 8 * (((sl >> 3) - cur) & 7) + (sl & 7);
                        load[w][ins][bank] = (uint8_t)(load[w][ins][bank] - 1);
                        touched[h] = ins;
                    }
                }
                __syncwarp();
#pragma unroll
                for (int h = 0; h < 2; ++h) {  // new maxima of the instructions the block left
                    const int ins = touched[h];
                    if (ins >= 0) {
                        int mm = 0;
                        for (int bk = 0; bk < 32; ++bk) mm = max(mm, (int)load[w][ins][(bk + j) & 31]);
                        mx[w][ins] = (uint8_t)mm;
                    }
                }
                __syncwarp();
                int delta = 0;
#pragma unroll 4
                for (int k = 0; k < 16; ++k) {
                    const int sl = (j >> 3) + 4 * k;
                    if ((bm >> sl) & 1ull) {
                        const int rank = __popcll(bm & ((1ull << sl) - 1ull));
                        const int bank = (int)((((int64_t)off + rank) * SV) >> 2) & 31;
                        const int ins = 8 * (((sl >> 3) - r) & 7) + (sl & 7);
                        delta += (load[w][ins][bank] + 1 > mx[w][ins]) ? 1 : 0;
                    }
                }
                delta += __shfl_xor_sync(0xffffffffu, delta, 8);
                delta += __shfl_xor_sync(0xffffffffu, delta, 16);
                // prefer the current rotation on ties (the search then only moves downhill)
                int key = delta * 16 + (r == cur ? 0 : 8) + r;
                key = min(key, __shfl_xor_sync(0xffffffffu, key, 1));
                key = min(key, __shfl_xor_sync(0xffffffffu, key, 2));
                key = min(key, __shfl_xor_sync(0xffffffffu, key, 4));
                const int best = key & 7;
                __syncwarp();
#pragma unroll
                for (int h = 0; h < 2; ++h) {  // add back with the chosen rotation
                    const int sl = j + 32 * h;
                    if ((bm >> sl) & 1ull) {
                        const int rank = __popcll(bm & ((1ull << sl) - 1ull));
                        const int bank = (int)((((int64_t)off + rank) * SV) >> 2) & 31;
                        const int ins = 8 * (((sl >> 3) - best) & 7) + (sl & 7);
                        const int nl = load[w][ins][bank] + 1;
                        load[w][ins][bank] = (uint8_t)nl;
                        if (nl > mx[w][ins]) mx[w][ins] = (uint8_t)nl;
                    }
                }
                if (j == 0) {
                    rot[ub + l] = (uint8_t)best;
                    rho_s[w][l] = (uint8_t)best;
                }
                __syncwarp();
            }
        }
    }
}

int rotation_passes() {  // SPADEN_ROT_PASSES: local-search passes after the greedy (default 1), read per conversion
    const char *e = getenv("SPADEN_ROT_PASSES");
    return e ? atoi(e) : 1;
}

bool rotation_enabled() {  // SPADEN_ROT=0 disables (A/B, tests), read per conversion
    const char *e = getenv("SPADEN_ROT");
    return !(e && e[0] == '0');
}

__global__ void k_long_chunks(int nlong, const int32_t *__restrict__ long_rows, const int32_t *__restrict__ brp,
                              int32_t *__restrict__ cnt) {
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j < nlong) {
        const int br = long_rows[j];
        cnt[j] = (brp[br + 1] - brp[br] + kLongChunk - 1) / kLongChunk;
    }
}

__global__ void k_chunk_rows(int nlong, const int32_t *__restrict__ chunk_start, int32_t *__restrict__ chunk_row) {
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j < nlong)
        for (int c = chunk_start[j]; c < chunk_start[j + 1]; ++c) chunk_row[c] = j;
}

__global__ void k_sched_summary(const int32_t *tile_total, const int32_t *long_total, int32_t *out) {
    out[0] = *tile_total;
    out[1] = *long_total;
}

}  // namespace

int default_tile_cfg(int64_t format_bytes, int value_bytes) {
    const char *e = getenv("SPADEN_TILE_CFG");
    if (e && e[0] >= '0' && e[0] <= '9') {
        const int c = atoi(e);
        if (tile_cfg_valid(c)) return c;
    }
    // measured best on fem1p5m: fp32 values 3 CTAs/SM x 8 consumers
    // x 3 x 24 KB, fp16 values 2 x 16 x 4 x 27 KB; small matrices need smaller stages to
    // give every CTA several tiles
    if (format_bytes < kSmallMatrixBytes) return kSmallTileCfg;
    return 15;  // fp32 and fp16 values (fp32: cfg2 0.1151 ms, cfg15 0.1131 ms on fem1p5m)
}

spaden_status_t build_schedule(Matrix *A, cudaStream_t st) {
    const int64_t Bnrow = A->Bnrow;
    const int sv = A->storage == SPADEN_R_16F ? 2 : 4;
    const int64_t nseg = (Bnrow + kSeg - 1) / kSeg;
    const int sv_b = A->storage == SPADEN_R_16F ? 2 : 4;
    A->tile_cfg = default_tile_cfg(4 * (A->Bnrow + 1) + 16 * A->Bnnz + (int64_t)sv_b * A->nnz, sv_b);
    const TileCfg cfg = tile_cfg(A->tile_cfg);
    const int64_t stage_cap = cfg.stage_bytes - kStageSlack;
    // long rows: one constant for every config (partition invariance, internal.cuh);
    const int64_t long_cost = kLongRowBytes;
    const int64_t cap = stage_cap;
    if (stage_cap < long_cost) {
        set_error("tile config stage smaller than the long-row threshold");
        return SPADEN_ERR_UNSUPPORTED;
    }
    const bool hyb = A->res_max_popc > 0;  // hybrid: tiles skip block-rows without blocks
    if (Bnrow == 0) return SPADEN_OK;
    // row rotations: CTA-pipeline configs with the predicated-slot decode (mean
    // block fill >= kSlotsMinFill, spmv.cu); one byte per block in the stage
    const int64_t bit_nnz = A->nnz - A->res_nnz;
    const bool use_rot = rotation_enabled() && A->Bnnz > 0 &&
                         bit_nnz >= (int64_t)kSlotsMinFill * A->Bnnz;
    const int pack_blk = kBlockStageBytes + (use_rot ? kBlockRotBytes : 0);

    const size_t n_tmp = scan_tmp_ints(nseg + 1);
    const size_t ints = 2 * (size_t)(nseg + 1) + n_tmp + 4;
    int32_t *tmp = nullptr;
    SPADEN_CUDA_TRY(cudaMallocAsync(&tmp, ints * sizeof(int32_t), st));
    int32_t *seg_tiles = tmp, *seg_long = tmp + (nseg + 1), *scan_tmp = tmp + 2 * (nseg + 1);
    int32_t *summary = scan_tmp + n_tmp;
    const unsigned grid = (unsigned)((nseg + 127) / 128);
    k_pack<false><<<grid, 128, 0, st>>>(Bnrow, A->blk_rowptr, A->blk_offset, sv, cap, long_cost, pack_blk,
                                        hyb, nullptr, seg_tiles, seg_long, nullptr, nullptr, nullptr, nullptr);
    cudaError_t e = exclusive_scan_i32(seg_tiles, seg_tiles, nseg, scan_tmp, st);
    if (e == cudaSuccess) e = exclusive_scan_i32(seg_long, seg_long, nseg, scan_tmp, st);
    int32_t h[2] = {0, 0};
    if (e == cudaSuccess) {
        k_sched_summary<<<1, 1, 0, st>>>(seg_tiles + nseg, seg_long + nseg, summary);
        e = cudaMemcpyAsync(h, summary, sizeof(h), cudaMemcpyDeviceToHost, st);
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) {
        cudaFreeAsync(tmp, st);
        return cuda_status(e, "building SpMV schedule");
    }
    A->n_tiles = h[0];
    A->n_long = h[1];
    const size_t tile_bytes = sizeof(TileDesc) * (size_t)std::max<int64_t>(1, A->n_tiles + 1);
    const size_t long_bytes = sizeof(int32_t) * (size_t)std::max<int64_t>(1, A->n_long);
    e = dmalloc(&A->tiles, tile_bytes, st);
    if (e == cudaSuccess) e = dmalloc(&A->long_rows, long_bytes, st);
    if (e != cudaSuccess) {
        cudaFreeAsync(tmp, st);
        return cuda_status(e, "allocating SpMV schedule");
    }
    A->aux_bytes = (int64_t)(tile_bytes + long_bytes);
    k_pack<true><<<grid, 128, 0, st>>>(Bnrow, A->blk_rowptr, A->blk_offset, sv, cap, long_cost, pack_blk,
                                       hyb, nullptr, nullptr, nullptr, seg_tiles, seg_long, A->tiles, A->long_rows);
    e = cudaGetLastError();
    cudaFreeAsync(tmp, st);
    if (e != cudaSuccess) return cuda_status(e, "packing SpMV schedule");
    if (use_rot && A->n_tiles > 0 && A->Bnnz > 0) {  // bank-conflict row rotations (slot decode)
        e = dmalloc(&A->rot, pad16((size_t)A->Bnnz), st);
        if (e == cudaSuccess) e = cudaMemsetAsync(A->rot, 0, pad16((size_t)A->Bnnz), st);
        if (e == cudaSuccess) {
            const unsigned g = (unsigned)((A->n_tiles + kRotWarps - 1) / kRotWarps);
            if (sv == 2)
                k_rot_greedy<2><<<g, 32 * kRotWarps, 0, st>>>(A->tiles, (int)A->n_tiles, A->bitmap, A->blk_offset, A->rot,
                                                              rotation_passes());
            else
                k_rot_greedy<4><<<g, 32 * kRotWarps, 0, st>>>(A->tiles, (int)A->n_tiles, A->bitmap, A->blk_offset, A->rot,
                                                              rotation_passes());
            e = cudaGetLastError();
        }
        if (e != cudaSuccess) return cuda_status(e, "row-rotation schedule");
        A->aux_bytes += (int64_t)pad16((size_t)A->Bnnz);
    }
    if (A->n_long == 0) return SPADEN_OK;

    // long block-rows -> fixed kLongChunk-block chunks (+ carry slots)
    const int nl = (int)A->n_long;
    int32_t *ltmp = nullptr;
    const size_t lt = scan_tmp_ints(nl + 1);
    SPADEN_CUDA_TRY(cudaMallocAsync(&ltmp, (lt + 4) * sizeof(int32_t), st));
    e = dmalloc(&A->chunk_start, sizeof(int32_t) * (nl + 1), st);
    if (e == cudaSuccess) {
        k_long_chunks<<<(nl + 255) / 256, 256, 0, st>>>(nl, A->long_rows, A->blk_rowptr, A->chunk_start);
        e = exclusive_scan_i32(A->chunk_start, A->chunk_start, nl, ltmp, st);
    }
    int32_t nch = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(&nch, A->chunk_start + nl, sizeof(int32_t), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    cudaFreeAsync(ltmp, st);
    if (e == cudaSuccess) {
        A->n_chunks = nch;
        e = dmalloc(&A->chunk_row, sizeof(int32_t) * std::max(1, nch), st);
    }
    constexpr int SL = Matrix::kScratchSlots;
    if (e == cudaSuccess) e = dmalloc(&A->carry, sizeof(float) * 8 * std::max(1, nch) * SL, st);
    if (e == cudaSuccess) e = dmalloc(&A->chunk_done, sizeof(int32_t) * nl * SL, st);
    if (e == cudaSuccess) e = cudaMemsetAsync(A->chunk_done, 0, sizeof(int32_t) * nl * SL, st);
    if (e == cudaSuccess) {
        k_chunk_rows<<<(nl + 255) / 256, 256, 0, st>>>(nl, A->chunk_start, A->chunk_row);
        e = cudaGetLastError();
    }
    if (e != cudaSuccess) return cuda_status(e, "long-row chunk schedule");
    A->aux_bytes += (int64_t)sizeof(int32_t) * (2 * nl + 1 + nch) + (int64_t)(sizeof(float) * 8 * nch + 4 * nl) * SL;
    return SPADEN_OK;
}

// SpMM schedule for K right-hand sides (built lazily by spaden_spmm): same
// stage size and long-row set as the SpMV schedule, tiles packed with the
// larger per-block partial scratch.  Returns UNSUPPORTED when some normal
// block-row cannot fit a stage with K vectors (the caller then runs K SpMVs).
spaden_status_t build_spmm_schedule(Matrix *A, int kidx, int K, cudaStream_t st) {
    const int64_t Bnrow = A->Bnrow;
    const int sv = A->storage == SPADEN_R_16F ? 2 : 4;
    const TileCfg cfg = tile_cfg(A->tile_cfg);
    const int64_t cap = cfg.stage_bytes - kStageSlack;
    const int64_t long_cost = kLongRowBytes;  // same long-row set as the SpMV schedule
    const int pack_bytes = 16 + 4 * (8 * K + 1);
    const bool hyb = A->res_max_popc > 0;
    const int64_t nseg = (Bnrow + kSeg - 1) / kSeg;
    A->spmm_state[kidx] = -1;
    if (Bnrow == 0) return SPADEN_ERR_UNSUPPORTED;
    const size_t n_tmp = scan_tmp_ints(nseg + 1);
    int32_t *tmp = nullptr;
    SPADEN_CUDA_TRY(cudaMallocAsync(&tmp, (2 * (size_t)(nseg + 1) + n_tmp + 8) * sizeof(int32_t), st));
    int32_t *seg_tiles = tmp, *seg_long = tmp + (nseg + 1), *scan_tmp = tmp + 2 * (nseg + 1);
    int32_t *summary = scan_tmp + n_tmp;
    uint32_t *too_big = (uint32_t *)(summary + 4);
    cudaMemsetAsync(too_big, 0, 4, st);
    const unsigned grid = (unsigned)((nseg + 127) / 128);
    k_pack<false><<<grid, 128, 0, st>>>(Bnrow, A->blk_rowptr, A->blk_offset, sv, cap, long_cost, pack_bytes, hyb,
                                        too_big, seg_tiles, seg_long, nullptr, nullptr, nullptr, nullptr);
    cudaError_t e = exclusive_scan_i32(seg_tiles, seg_tiles, nseg, scan_tmp, st);
    int32_t h[2] = {0, 0};
    if (e == cudaSuccess) {
        k_sched_summary<<<1, 1, 0, st>>>(seg_tiles + nseg, (const int32_t *)too_big, summary);
        e = cudaMemcpyAsync(h, summary, sizeof(h), cudaMemcpyDeviceToHost, st);
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess || h[1] != 0) {
        cudaFreeAsync(tmp, st);
        if (e != cudaSuccess) return cuda_status(e, "building SpMM schedule");
        set_error("a block-row does not fit a pipeline stage with this many right-hand sides");
        return SPADEN_ERR_UNSUPPORTED;
    }
    const size_t tile_bytes = sizeof(TileDesc) * (size_t)std::max(1, h[0] + 1);
    e = dmalloc(&A->spmm_tiles[kidx], tile_bytes, st);
    if (e == cudaSuccess) {
        k_pack<true><<<grid, 128, 0, st>>>(Bnrow, A->blk_rowptr, A->blk_offset, sv, cap, long_cost, pack_bytes,
                                           hyb, nullptr, nullptr, nullptr, seg_tiles, seg_long, A->spmm_tiles[kidx],
                                           nullptr);
        e = cudaGetLastError();
    }
    cudaFreeAsync(tmp, st);
    if (e != cudaSuccess) return cuda_status(e, "packing SpMM schedule");
    A->spmm_ntiles[kidx] = h[0];
    A->spmm_state[kidx] = 1;
    A->aux_bytes += (int64_t)tile_bytes;
    return SPADEN_OK;
}

}  // namespace spaden
