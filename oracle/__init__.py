"""Python wrapper (ctypes + numpy) around oracle/oracle.c.

TEST INFRASTRUCTURE ONLY: may be imported by tests/, __graft_entry__.smoke()
and bench.py's cpu_baseline / --impl reference legs, nothing else.  It never
imports the product package and the product package never imports it.

Each function cites the PAPER.md passage it follows (see oracle.c's header).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

ORC_OK, ORC_BAD_ROWPTR, ORC_COL_RANGE, ORC_UNSORTED, ORC_NOMEM = range(5)


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain -O2, no fast-math, no FP contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-fPIC", "-shared",
                               "-ffp-contract=off", "-fno-fast-math", "-fopenmp", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        _lib.oracle_csr_spmv_f64.argtypes = [I64, P, P, P, P, P, P]
        _lib.oracle_csr_spmv_f64_omp.argtypes = [I64, P, P, P, P, P, P]
        _lib.oracle_csr_spmv_f64_omp.restype = ctypes.c_int
        _lib.oracle_bitbsr_count.argtypes = [I64, I64, I64, P, P, P]
        _lib.oracle_bitbsr_count.restype = ctypes.c_int
        _lib.oracle_csr_to_bitbsr.argtypes = [I64, I64, I64, P, P, P, ctypes.c_int, P, P, P, P, P]
        _lib.oracle_csr_to_bitbsr.restype = ctypes.c_int
        _lib.oracle_bitbsr_to_csr.argtypes = [I64, P, P, P, P, P, ctypes.c_int, P, P, P]
        _lib.oracle_f32_to_f16_rne.argtypes = [I64, P, P]
        _lib.oracle_pagerank_f64.argtypes = [I64, P, P, P, ctypes.c_double, ctypes.c_int, P, P]
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def spmv(rowptr, colidx, values, x):
    """Algorithm 1 in fp64: returns (y, s) with y_i = sum v*x and
    s_i = sum |v*x|.  values / x are upcast exactly to float64 (fp16 and fp32
    both embed exactly)."""
    rowptr = _c(rowptr, np.int64)
    colidx = _c(colidx, np.int32)
    v = _c(np.asarray(values).astype(np.float64), np.float64)
    xx = _c(np.asarray(x).astype(np.float64), np.float64)
    m = rowptr.shape[0] - 1
    y = np.zeros(m, np.float64)
    s = np.zeros(m, np.float64)
    lib().oracle_csr_spmv_f64(m, _p(rowptr), _p(colidx), _p(v), _p(xx), _p(y), _p(s))
    return y, s


def spmv_omp(rowptr, colidx, values, x):
    """spmv() with the row loop on all host cores (OpenMP, static schedule);
    bitwise equal to spmv().  Returns (y, s, threads)."""
    rowptr = _c(rowptr, np.int64)
    colidx = _c(colidx, np.int32)
    v = _c(np.asarray(values).astype(np.float64), np.float64)
    xx = _c(np.asarray(x).astype(np.float64), np.float64)
    m = rowptr.shape[0] - 1
    y = np.zeros(m, np.float64)
    s = np.zeros(m, np.float64)
    t = lib().oracle_csr_spmv_f64_omp(m, _p(rowptr), _p(colidx), _p(v), _p(xx), _p(y), _p(s))
    return y, s, int(t)


def f32_to_f16(values) -> np.ndarray:
    """IEEE round-to-nearest-even to binary16 (reading R10); returns float16 array."""
    v = _c(values, np.float32)
    out = np.zeros(v.shape[0], np.uint16)
    lib().oracle_f32_to_f16_rne(v.shape[0], _p(v), _p(out))
    return out.view(np.float16)


class BitBSR:
    """Host copy of the five bitBSR arrays (Fig. 4)."""

    def __init__(self, m, n, blk_rowptr, blk_col, bitmap, blk_offset, values):
        self.m, self.n = m, n
        self.blk_rowptr, self.blk_col, self.bitmap = blk_rowptr, blk_col, bitmap
        self.blk_offset, self.values = blk_offset, values

    @property
    def Bnrow(self):
        return (self.m + 7) // 8

    @property
    def Bnnz(self):
        return int(self.blk_col.shape[0])


def csr_to_bitbsr(m, n, rowptr, colidx, values):
    """Reference converter.  Returns (status, BitBSR|None).  values may be
    float32 or float16; they are moved as raw bits."""
    rowptr = _c(rowptr, np.int64)
    colidx = _c(colidx, np.int32)
    values = np.ascontiguousarray(values)
    vb = values.dtype.itemsize
    assert vb in (2, 4)
    raw = values.view(np.uint16 if vb == 2 else np.uint32)
    nnz = colidx.shape[0]
    bnnz = ctypes.c_int64(0)
    st = lib().oracle_bitbsr_count(m, n, nnz, _p(rowptr), _p(colidx), ctypes.byref(bnnz))
    if st != ORC_OK:
        return st, None
    B = bnnz.value
    Bnrow = (m + 7) // 8
    brp = np.zeros(Bnrow + 1, np.int64)
    bcol = np.zeros(B, np.int32)
    bmp = np.zeros(B, np.uint64)
    boff = np.zeros(B + 1, np.int64)
    vout = np.zeros(nnz, raw.dtype)
    st = lib().oracle_csr_to_bitbsr(m, n, nnz, _p(rowptr), _p(colidx), _p(raw), vb,
                                    _p(brp), _p(bcol), _p(bmp), _p(boff), _p(vout))
    if st != ORC_OK:
        return st, None
    return ORC_OK, BitBSR(m, n, brp, bcol, bmp, boff, vout.view(values.dtype))


def bitbsr_to_csr(A: BitBSR):
    """Reference decoder (reading R1: value index = popcount rank of the bit)."""
    nnz = int(A.blk_offset[-1]) if A.blk_offset.shape[0] else 0
    vb = A.values.dtype.itemsize
    rowptr = np.zeros(A.m + 1, np.int64)
    colidx = np.zeros(nnz, np.int32)
    vout = np.zeros(nnz, np.uint16 if vb == 2 else np.uint32)
    raw = np.ascontiguousarray(A.values).view(vout.dtype)
    lib().oracle_bitbsr_to_csr(A.m, _p(_c(A.blk_rowptr, np.int64)), _p(_c(A.blk_col, np.int32)),
                               _p(_c(A.bitmap, np.uint64)), _p(_c(A.blk_offset, np.int64)),
                               _p(raw), vb, _p(rowptr), _p(colidx), _p(vout))
    return rowptr, colidx, vout.view(A.values.dtype)


def pagerank(rowptr, colidx, values, d: float, iters: int, x0):
    rowptr = _c(rowptr, np.int64)
    colidx = _c(colidx, np.int32)
    v = _c(np.asarray(values).astype(np.float64), np.float64)
    x0 = _c(np.asarray(x0).astype(np.float64), np.float64)
    n = rowptr.shape[0] - 1
    out = np.zeros(n, np.float64)
    lib().oracle_pagerank_f64(n, _p(rowptr), _p(colidx), _p(v), d, iters, _p(x0), _p(out))
    return out


def bitbsr_bytes(m: int, bnnz: int, nnz: int, value_bytes: int) -> int:
    """Stored footprint of bitBSR: int32 blk_rowptr[Bnrow+1], int32 blk_col[Bnnz],
    uint64 bitmap[Bnnz], int32 blk_offset[Bnnz+1], values[nnz].  With fp16 values
    this reproduces the paper's 2.85 B/nnz over Table 1."""
    Bnrow = (m + 7) // 8
    return 4 * (Bnrow + 1) + 4 * bnnz + 8 * bnnz + 4 * (bnnz + 1) + value_bytes * nnz


def componentwise_error(y_hat, y_star, s) -> float:
    """max_i |y_hat_i - y*_i| / s_i with 0/0 := 0."""
    d = np.abs(np.asarray(y_hat, np.float64) - y_star)
    s = np.asarray(s, np.float64)
    with np.errstate(divide="ignore", invalid="ignore"):
        r = np.where(s > 0, d / np.where(s > 0, s, 1), np.where(d > 0, np.inf, 0))
    return float(r.max()) if r.size else 0.0


def normwise_error(y_hat, y_star, a_inf: float, x_inf: float) -> float:
    """||y_hat - y*||_inf / (||A||_inf ||x||_inf)  (BASELINE north_star fp16 tolerance)."""
    d = np.abs(np.asarray(y_hat, np.float64) - y_star)
    den = a_inf * x_inf
    if d.size == 0:
        return 0.0
    return float(d.max() / den) if den > 0 else float(d.max())


def csr_inf_norm(rowptr, values) -> float:
    """||A||_inf = max_i sum_k |a_ik|."""
    v = np.abs(np.asarray(values, np.float64))
    rp = np.asarray(rowptr, np.int64)
    if v.size == 0:
        return 0.0
    c = np.concatenate([[0.0], np.cumsum(v)])
    return float((c[rp[1:]] - c[rp[:-1]]).max())


def hybrid_split(m, n, rowptr, colidx, values, t: int):
    """Hybrid format reference: an entry goes
    to the CSR residual iff its 8x8 block (row//8, col//8) holds at most t
    entries; all other entries stay in bitBSR.  Returns (kept CSR, residual CSR)
    as (rowptr int64[m+1], colidx int32, values) tuples, both row-sorted."""
    rowptr = np.asarray(rowptr, np.int64)
    colidx = np.asarray(colidx, np.int32)
    values = np.asarray(values)
    rows = np.repeat(np.arange(m, dtype=np.int64), np.diff(rowptr))
    nbc = (n + 7) // 8
    key = (rows // 8) * max(nbc, 1) + colidx.astype(np.int64) // 8
    if key.size:
        _, inv, cnt = np.unique(key, return_inverse=True, return_counts=True)
        res = cnt[inv] <= t
    else:
        res = np.zeros(0, bool)

    def sub(mask):
        counts = np.bincount(rows[mask], minlength=m) if m else np.zeros(0, np.int64)
        rp = np.zeros(m + 1, np.int64)
        np.cumsum(counts, out=rp[1:])
        return rp, colidx[mask], values[mask]

    return sub(~res), sub(res)


def degree_order(rowptr) -> np.ndarray:
    """Degree ordering (SURVEY.md §8(f) NEXT-1 reordering; degree-based ordering is
    one of the remedies PAPER.md §6 cites): perm[k] = the row placed k-th,
    rows by descending degree rowptr[i+1]-rowptr[i], equal degrees in ascending
    row order (a stable sort of -degree).  Definition only."""
    deg = np.diff(np.asarray(rowptr, dtype=np.int64))
    return np.argsort(-deg, kind="stable").astype(np.int32)


def permute_csr(rowptr, colidx, values, perm):
    """Symmetric permutation B = P A P^T of a square CSR matrix, written from its
    definition B[k, l] = A[perm[k], perm[l]]: every entry (i, j, v) of A becomes
    (iperm[i], iperm[j], v) with iperm[perm[k]] = k, entries then in (row, column)
    order.  Returns (rowptr, colidx, values) numpy arrays."""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    m = rowptr.size - 1
    perm = np.asarray(perm, dtype=np.int64)
    iperm = np.empty(m, dtype=np.int64)
    iperm[perm] = np.arange(m, dtype=np.int64)
    rows = np.repeat(np.arange(m, dtype=np.int64), np.diff(rowptr))
    nr = iperm[rows]
    nc = iperm[np.asarray(colidx, dtype=np.int64)]
    order = np.lexsort((nc, nr))
    counts = np.bincount(nr, minlength=m) if m else np.zeros(0, np.int64)
    rp = np.zeros(m + 1, np.int64)
    np.cumsum(counts, out=rp[1:])
    return rp.astype(np.int32), nc[order].astype(np.int32), np.asarray(values)[order]
