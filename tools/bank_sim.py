"""Shared-memory bank-conflict model of the slot decode.

For every 32-block unit of a matrix and every predicated slot instruction
(row r, column c) of the lane-per-block decode, the active lanes are the blocks
with bit 8r+c set and each reads the word holding its value at
blk_offset + rank.  The instruction costs max-over-banks(distinct words)
wavefronts.  Per-lane row-half swaps (rows 4-7 first) are modelled by `rot`.
Matches ncu within a few percent (fem1p5m fp32: 3.8 measured, 3.96 modelled).

    python tools/bank_sim.py [fem62k]
"""
import sys

import numpy as np

sys.path.insert(0, __file__.rsplit('/tools/', 1)[0])
import oracle  # noqa: E402  (harness: the reference converter gives the arrays)
import workloads  # noqa: E402


def unit_arrays(name):
    A = workloads.make(name)
    _, B = oracle.csr_to_bitbsr(A.m, A.n, A.rowptr, A.colidx, A.values)
    bm = B.bitmap.astype(np.uint64)
    off = B.blk_offset[:-1].astype(np.int64)
    bits = ((bm[:, None] >> np.arange(64, dtype=np.uint64)) & np.uint64(1)).astype(np.int64)
    rank = np.cumsum(bits, axis=1) - bits
    U = len(bm) // 32
    return (bits[:U * 32].reshape(U, 32, 64), rank[:U * 32].reshape(U, 32, 64), off[:U * 32].reshape(U, 32))


def wavefronts_per_block(bits, rank, off, value_bytes, rot):
    U = bits.shape[0]
    lanes = np.arange(32)
    tot = 0
    for t in range(8):
        for c in range(8):
            slot = 8 * ((t + rot) % 8) + c
            act = bits[:, lanes, slot].astype(bool)
            words = (off + rank[:, lanes, slot]) * value_bytes // 4
            for u in range(U):
                w = np.unique(words[u][act[u]])
                if w.size:
                    tot += np.bincount(w % 32, minlength=32).max()
    return tot / (U * 32)


if __name__ == '__main__':
    bits, rank, off = unit_arrays(sys.argv[1] if len(sys.argv) > 1 else 'fem62k')
    lanes = np.arange(32)
    for vb in (4, 2):
        for name, rot in (('row order', np.zeros(32, int)), ('rows 4-7 first on lanes with bit 1', 4 * ((lanes >> 1) & 1))):
            print(f'{vb}-byte values, {name:36s}: {wavefronts_per_block(bits, rank, off, vb, rot):.3f} wavefronts/block')
