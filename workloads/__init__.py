"""Seeded synthetic input generators shared by the oracle tests, the CUDA parity
tests and bench.py.

This module holds NONE of the method's arithmetic (no tiling, no bitmaps, no
SpMV): it only produces canonical CSR matrices (row-sorted, duplicate-free,
int32 indices, float32 values) and dense vectors, with the shapes and value
distributions of the paper's workloads (§5.1, Table 1).
The recipes and their calibration are in DESIGN.md §"Input recipe" and
SURVEY.md §8(d).

Every generator is deterministic in its seed.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class CSR:
    """Canonical CSR (§2.1): rowptr[m+1], colidx[nnz], values[nnz]."""

    m: int
    n: int
    rowptr: np.ndarray  # int32 [m+1]
    colidx: np.ndarray  # int32 [nnz]
    values: np.ndarray  # float32 (or float16) [nnz]

    @property
    def nnz(self) -> int:
        return int(self.colidx.shape[0])

    def row_slice(self, r0: int, r1: int) -> "CSR":
        """Rows [r0, r1) with global columns (the multi-GPU row partition)."""
        r1 = min(r1, self.m)
        r0 = min(r0, r1)
        a, b = int(self.rowptr[r0]), int(self.rowptr[r1])
        rp = (self.rowptr[r0:r1 + 1] - a).astype(np.int32)
        return CSR(r1 - r0, self.n, rp, self.colidx[a:b].copy(), self.values[a:b].copy())


def from_coo(m: int, n: int, rows, cols, vals, dtype=np.float32) -> CSR:
    """Canonical CSR from COO triples (sorted by (row, col); duplicates must not occur)."""
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    vals = np.asarray(vals, dtype=dtype)
    order = np.lexsort((cols, rows))
    rows, cols, vals = rows[order], cols[order], vals[order]
    if rows.size > 1:
        dup = (rows[1:] == rows[:-1]) & (cols[1:] == cols[:-1])
        if dup.any():
            raise ValueError("duplicate (row, col) in COO input")
    counts = np.bincount(rows, minlength=m) if rows.size else np.zeros(m, np.int64)
    rowptr = np.zeros(m + 1, np.int64)
    np.cumsum(counts, out=rowptr[1:])
    return CSR(m, n, rowptr.astype(np.int32), cols.astype(np.int32), vals)


def from_dense(a: np.ndarray, dtype=np.float32, keep_explicit: np.ndarray | None = None) -> CSR:
    """CSR of the nonzeros of a dense matrix (plus any positions in keep_explicit)."""
    mask = a != 0
    if keep_explicit is not None:
        mask |= keep_explicit
    r, c = np.nonzero(mask)
    return from_coo(a.shape[0], a.shape[1], r, c, a[r, c], dtype)


# --------------------------------------------------------------------------
# Hand-worked examples (expected arrays in tests/golden)
# --------------------------------------------------------------------------

def h1() -> CSR:
    ent = [(0, 0, 1), (0, 9, 2), (1, 1, 3), (3, 7, 4), (7, 7, 5), (7, 8, 6),
           (9, 2, 7), (12, 3, -1), (15, 15, 8)]
    r, c, v = zip(*ent)
    return from_coo(16, 16, r, c, v)


def h2() -> CSR:
    ent = [(0, 12, 1.5), (3, 4, 0.0), (8, 0, 2), (9, 9, -3), (9, 12, 0.5)]
    r, c, v = zip(*ent)
    return from_coo(10, 13, r, c, v)


# --------------------------------------------------------------------------
# Closed-form matrices
# --------------------------------------------------------------------------

def identity(n: int) -> CSR:
    i = np.arange(n)
    return from_coo(n, n, i, i, np.ones(n))


def diagonal(n: int, seed: int = 0) -> CSR:
    rng = np.random.default_rng(seed)
    i = np.arange(n)
    return from_coo(n, n, i, i, rng.uniform(-2, 2, n).astype(np.float32))


def permutation(perm: np.ndarray) -> CSR:
    """P with P[i, perm[i]] = 1, so (P x)_i = x[perm[i]]."""
    n = perm.shape[0]
    return from_coo(n, n, np.arange(n), perm, np.ones(n))


def reversal(n: int) -> CSR:
    return permutation(np.arange(n)[::-1].copy())


def random_perm(n: int, seed: int = 0) -> np.ndarray:
    return np.random.default_rng(seed).permutation(n)


def dense_block(m: int, n: int, seed: int = 0) -> CSR:
    rng = np.random.default_rng(seed)
    a = rng.uniform(0.5, 1.5, (m, n)).astype(np.float32)
    return from_dense(a)


def random_sparse(m: int, n: int, density: float, seed: int = 0,
                  dist: str = "uniform", dtype=np.float32) -> CSR:
    """Uniform random pattern with the given density (exact nnz = round(density*m*n))."""
    rng = np.random.default_rng(seed)
    total = m * n
    nnz = int(round(density * total))
    if total == 0 or nnz == 0:
        return CSR(m, n, np.zeros(m + 1, np.int32), np.zeros(0, np.int32), np.zeros(0, dtype))
    flat = rng.choice(total, size=nnz, replace=False)
    r, c = np.divmod(flat, n)
    if dist == "int":
        v = rng.integers(-4, 5, nnz).astype(dtype)
        v[v == 0] = 1
    else:
        v = rng.uniform(-1, 1, nnz).astype(dtype)
    return from_coo(m, n, r, c, v, dtype)


# --------------------------------------------------------------------------
# BASELINE.json configs
# --------------------------------------------------------------------------

def tiny(seed: int = 0) -> CSR:
    """configs[0]: 1024x1024, 10,000 distinct uniform positions (seed 0), U(-1,1) values (seed 1)."""
    m = n = 1024
    flat = np.random.default_rng(seed).choice(m * n, size=10_000, replace=False)
    r, c = np.divmod(flat, n)
    v = np.random.default_rng(seed + 1).uniform(-1, 1, flat.size).astype(np.float32)
    return from_coo(m, n, r, c, v)


def _splitmix64(z: np.ndarray) -> np.ndarray:
    """Counter-based hash (SplitMix64 finaliser) on uint64 arrays."""
    with np.errstate(over="ignore"):
        z = z + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def fem(nx: int, ny: int, nz: int, keep: float = 0.85, dof: int = 3, seed: int = 0,
        value_seed: int | None = None) -> CSR:
    """FEM-like matrix (cant-shaped, Table 1): an nx*ny*nz node grid with
    27-point node adjacency (including self); each undirected neighbour pair is
    kept with probability `keep` (symmetric pattern, decided by a counter-based
    hash of the pair); `dof` degrees of freedom per node give dense dof x dof
    couplings; node-major ordering (row = dof*node + d). Values N(0,1) float32.
    """
    N = nx * ny * nz
    node = np.arange(N, dtype=np.int64)
    x = node % nx
    y = (node // nx) % ny
    z = node // (nx * ny)
    offs = [(dz, dy, dx) for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
    J = np.empty((N, 27), dtype=np.int64)
    M = np.empty((N, 27), dtype=bool)
    seed_u = np.uint64(seed * 0x1000193 + 7)
    for s, (dz, dy, dx) in enumerate(offs):
        xx, yy, zz = x + dx, y + dy, z + dz
        inb = (xx >= 0) & (xx < nx) & (yy >= 0) & (yy < ny) & (zz >= 0) & (zz < nz)
        j = (zz * ny + yy) * nx + xx
        lo = np.minimum(node, j).astype(np.uint64)
        hi = np.maximum(node, j).astype(np.uint64)
        h = _splitmix64(lo * np.uint64(0x100000001B3) ^ (hi + seed_u))
        u = (h >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)
        kept = (u < keep) | (j == node)
        J[:, s] = np.where(inb, j, 0)
        M[:, s] = inb & kept
    # entries in (node, d, s, d') order == row-major with ascending columns
    cols = (dof * J[:, None, :, None] + np.arange(dof)[None, None, None, :])
    mask = np.broadcast_to(M[:, None, :, None], (N, dof, 27, dof))
    cols = np.broadcast_to(cols, (N, dof, 27, dof))[mask].astype(np.int32)
    per_row = np.repeat(M.sum(axis=1) * dof, dof)
    rowptr = np.zeros(N * dof + 1, np.int64)
    np.cumsum(per_row, out=rowptr[1:])
    rng = np.random.default_rng(seed + 1 if value_seed is None else value_seed)
    vals = rng.standard_normal(cols.shape[0], dtype=np.float32)
    return CSR(N * dof, N * dof, rowptr.astype(np.int32), cols, vals)


def rmat_edges(scale: int, edge_factor: int, seed: int = 0,
               abcd=(0.57, 0.19, 0.19, 0.05), relabel: bool = False):
    """R-MAT edge stream (Graph500-style quadrant recursion), numpy version.
    Returns (src, dst) int64 arrays; duplicates not removed."""
    rng = np.random.default_rng(seed)
    ne = edge_factor << scale
    a, b, c, _ = abcd
    src = np.zeros(ne, np.int64)
    dst = np.zeros(ne, np.int64)
    for level in range(scale):
        u = rng.random(ne)
        bit_dst = (u >= a) & (u < a + b) | (u >= a + b + c)   # quadrants b, d -> dst bit
        bit_src = (u >= a + b)                                # quadrants c, d -> src bit
        src |= bit_src.astype(np.int64) << level
        dst |= bit_dst.astype(np.int64) << level
    if relabel:
        p = rng.permutation(1 << scale)
        src, dst = p[src], p[dst]
    return src, dst


def powerlaw(scale: int = 20, edge_factor: int = 5, seed: int = 0, relabel: bool = False) -> CSR:
    """configs[2] (web-Google-shaped): R-MAT(.57,.19,.19,.05), A[src][dst] = 1.0,
    duplicates removed, natural vertex order by default."""
    n = 1 << scale
    src, dst = rmat_edges(scale, edge_factor, seed, relabel=relabel)
    key = np.unique(src * n + dst)
    r, c = np.divmod(key, n)
    counts = np.bincount(r, minlength=n)
    rowptr = np.zeros(n + 1, np.int64)
    np.cumsum(counts, out=rowptr[1:])
    return CSR(n, n, rowptr.astype(np.int32), c.astype(np.int32), np.ones(key.size, np.float32))


def pagerank_matrix(n: int, src: np.ndarray, dst: np.ndarray) -> CSR:
    """Column-stochastic A[dst][src] = 1/outdeg(src) over unique edges (rmat25's
    PageRank-style iteration). Dangling sources contribute nothing."""
    key = np.unique(dst.astype(np.int64) * n + src.astype(np.int64))
    r, c = np.divmod(key, n)
    outdeg = np.bincount(c, minlength=n)
    vals = (1.0 / outdeg[c]).astype(np.float32)
    counts = np.bincount(r, minlength=n)
    rowptr = np.zeros(n + 1, np.int64)
    np.cumsum(counts, out=rowptr[1:])
    return CSR(n, n, rowptr.astype(np.int32), c.astype(np.int32), vals)


def vector(n: int, seed: int = 2, lo: float = -1.0, hi: float = 1.0) -> np.ndarray:
    return np.random.default_rng(seed).uniform(lo, hi, n).astype(np.float32)


# Names mirror BASELINE.json:configs.
CONFIGS = {
    "tiny": lambda: tiny(0),
    "fem62k": lambda: fem(27, 27, 28, keep=0.85, seed=0),
    "powerlaw1m": lambda: powerlaw(20, 5, seed=0),
    "fem1p5m": lambda: fem(80, 80, 78, keep=0.85, seed=0),
}


def make(name: str) -> CSR:
    return CONFIGS[name]()


# --------------------------------------------------------------------------
# R-MAT on the GPU (rmat25: ~1.07B edges; numpy is far too slow at that size)
# --------------------------------------------------------------------------

def rmat_torch(scale: int, edge_factor: int, seed: int = 0, device="cuda", relabel: bool = True,
               abcd=(0.57, 0.19, 0.19, 0.05), chunk: int = 1 << 26):
    """Graph500-style R-MAT edge stream generated with torch on `device` in fixed
    chunks from one seeded generator, so every rank that calls it with the same
    arguments gets the same stream.  Returns (src, dst) int64 tensors."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    n = 1 << scale
    ne = edge_factor << scale
    a, b, c, _ = abcd
    src = torch.empty(ne, dtype=torch.int64, device=device)
    dst = torch.empty(ne, dtype=torch.int64, device=device)
    for s0 in range(0, ne, chunk):
        k = min(chunk, ne - s0)
        s = torch.zeros(k, dtype=torch.int64, device=device)
        d = torch.zeros(k, dtype=torch.int64, device=device)
        for level in range(scale):
            u = torch.rand(k, generator=g, device=device)
            bit_d = ((u >= a) & (u < a + b)) | (u >= a + b + c)
            bit_s = u >= a + b
            s |= bit_s.to(torch.int64) << level
            d |= bit_d.to(torch.int64) << level
        src[s0:s0 + k] = s
        dst[s0:s0 + k] = d
    if relabel:
        perm = torch.randperm(n, generator=g, device=device)
        src = perm[src]
        dst = perm[dst]
    return src, dst


def pagerank_slice_torch(scale: int, edge_factor: int, r0: int, r1: int, seed: int = 0, device="cuda"):
    """Rows [r0, r1) of the column-stochastic PageRank matrix A[dst][src] =
    1/outdeg(src) over the unique edges of rmat_torch(...) (global columns).
    Returns torch CSR pieces (rowptr int32[r1-r0+1], colidx int32, values fp32)
    on `device`, and the global n and nnz."""
    import torch
    n = 1 << scale
    src, dst = rmat_torch(scale, edge_factor, seed, device)
    key = torch.unique(dst * n + src)          # sorted by (dst, src), duplicates removed
    del src, dst
    s = key % n
    outdeg = torch.bincount(s, minlength=n)
    nnz_total = int(key.numel())
    lo = torch.searchsorted(key, torch.tensor([r0 * n, r1 * n], device=device))
    ks = key[int(lo[0]):int(lo[1])]
    rows = (ks // n - r0)
    cols = (ks % n)
    vals = (1.0 / outdeg[cols].to(torch.float64)).to(torch.float32)
    counts = torch.bincount(rows, minlength=r1 - r0)
    rowptr = torch.zeros(r1 - r0 + 1, dtype=torch.int64, device=device)
    rowptr[1:] = torch.cumsum(counts, 0)
    return rowptr.to(torch.int32), cols.to(torch.int32), vals, n, nnz_total
