"""Pins of the CPU oracle (oracle/) against things other than itself:
hand-worked examples (tests/golden), dense brute force, closed
forms, Table 1, numpy's float16 rounding and a dense
linear solve for the PageRank fixed point.  CPU only."""
import json
import os

import numpy as np
import pytest

import oracle
import workloads as W

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def golden_csr(g):
    r, c, v = zip(*g["entries"])
    return W.from_coo(g["m"], g["n"], r, c, v)


# ---------------------------------------------------------------- H1 / H2
@pytest.mark.parametrize("name", ["h1.json", "h2.json"])
def test_hand_worked_conversion(name):
    g = load(name)
    A = golden_csr(g)
    st, B = oracle.csr_to_bitbsr(A.m, A.n, A.rowptr, A.colidx, A.values)
    assert st == oracle.ORC_OK
    assert B.blk_rowptr.tolist() == g["blk_rowptr"]
    assert B.blk_col.tolist() == g["blk_col"]
    assert [int(h, 16) for h in g["bitmap"]] == [int(b) for b in B.bitmap]
    assert B.blk_offset.tolist() == g["blk_offset"]
    assert B.values.tolist() == [float(v) for v in g["values"]]


@pytest.mark.parametrize("name", ["h1.json", "h2.json"])
def test_hand_worked_spmv(name):
    g = load(name)
    A = golden_csr(g)
    x = np.arange(1, A.n + 1, dtype=np.float32)
    y, s = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    assert y.tolist() == [float(v) for v in g["y"]]
    assert (s >= np.abs(y)).all()


def test_fig4_row0_is_low_byte():
    """a block whose row0 holds only its first element -> row0 == 0x01."""
    A = W.from_coo(8, 8, [0, 2, 2], [0, 1, 6], [1.0, 2.0, 3.0])
    st, B = oracle.csr_to_bitbsr(8, 8, A.rowptr, A.colidx, A.values)
    assert st == 0
    bmp = int(B.bitmap[0])
    assert bmp & 0xFF == 0x01
    assert (bmp >> 16) & 0xFF == 0b01000010


# ---------------------------------------------------------- brute force
def dense_of(A):
    D = np.zeros((A.m, A.n), np.float64)
    for i in range(A.m):
        for k in range(A.rowptr[i], A.rowptr[i + 1]):
            D[i, A.colidx[k]] = A.values[k]
    return D


@pytest.mark.parametrize("m,n,dens,seed", [(1, 1, 1.0, 0), (7, 9, 0.3, 1), (64, 64, 0.05, 2),
                                           (255, 129, 0.01, 3), (256, 256, 0.3, 4),
                                           (100, 3, 0.5, 5), (3, 200, 0.2, 6)])
def test_spmv_vs_dense_bruteforce(m, n, dens, seed):
    A = W.random_sparse(m, n, dens, seed)
    x = W.vector(n, seed + 10)
    y, s = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    ref = dense_of(A) @ x.astype(np.float64)
    np.testing.assert_allclose(y, ref, rtol=1e-13, atol=1e-13)
    ref_s = np.abs(dense_of(A)) @ np.abs(x.astype(np.float64))
    np.testing.assert_allclose(s, ref_s, rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("m,n,dens,seed", [(0, 5, 0.1, 0), (255, 129, 0.01, 3), (256, 256, 0.3, 4)])
def test_spmv_omp_vs_dense_and_serial(m, n, dens, seed):
    """The all-cores oracle (bench cpu_baseline arm) against the dense product,
    and bitwise against the serial Alg. 1 (same per-row order)."""
    A = W.random_sparse(m, n, dens, seed)
    x = W.vector(n, seed + 10)
    y, s, threads = oracle.spmv_omp(A.rowptr, A.colidx, A.values, x)
    assert threads >= 1
    ref = dense_of(A) @ x.astype(np.float64)
    np.testing.assert_allclose(y, ref, rtol=1e-13, atol=1e-13)
    y1, s1 = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    assert np.array_equal(y, y1) and np.array_equal(s, s1)


def tiles_bruteforce(A):
    """Independent bitBSR builder from the dense view: walk every 8x8 tile of
    the dense pattern in (tile-row, tile-col) order, bit = 8r + c."""
    P = np.zeros((A.m, A.n), bool)
    V = np.zeros((A.m, A.n), np.float64)
    for i in range(A.m):
        for k in range(A.rowptr[i], A.rowptr[i + 1]):
            P[i, A.colidx[k]] = True
            V[i, A.colidx[k]] = A.values[k]
    brp, bcol, bmp, boff, vals = [0], [], [], [0], []
    for br in range((A.m + 7) // 8):
        for bc in range((A.n + 7) // 8):
            word = 0
            for r in range(8):
                for c in range(8):
                    i, j = 8 * br + r, 8 * bc + c
                    if i < A.m and j < A.n and P[i, j]:
                        word |= 1 << (8 * r + c)
                        vals.append(V[i, j])
            if word:
                bcol.append(bc)
                bmp.append(word)
                boff.append(len(vals))
        brp.append(len(bcol))
    return brp, bcol, bmp, boff, vals


@pytest.mark.parametrize("m,n,dens,seed", [(9, 17, 0.2, 0), (40, 40, 0.1, 1), (33, 70, 0.05, 2),
                                           (16, 16, 1.0, 3), (1, 1, 1.0, 4), (64, 8, 0.5, 5)])
def test_conversion_vs_dense_tiles(m, n, dens, seed):
    A = W.random_sparse(m, n, dens, seed)
    st, B = oracle.csr_to_bitbsr(A.m, A.n, A.rowptr, A.colidx, A.values)
    assert st == 0
    brp, bcol, bmp, boff, vals = tiles_bruteforce(A)
    assert B.blk_rowptr.tolist() == brp
    assert B.blk_col.tolist() == bcol
    assert [int(b) for b in B.bitmap] == bmp
    assert B.blk_offset.tolist() == boff
    assert B.values.astype(np.float64).tolist() == vals


@pytest.mark.parametrize("dtype", [np.float32, np.float16])
def test_decode_roundtrip(dtype):
    for seed, (m, n, d) in enumerate([(100, 90, 0.05), (1024, 1024, 0.01), (31, 1000, 0.1)]):
        A = W.random_sparse(m, n, d, seed)
        vals = A.values.astype(dtype)
        st, B = oracle.csr_to_bitbsr(m, n, A.rowptr, A.colidx, vals)
        assert st == 0
        rp, ci, vv = oracle.bitbsr_to_csr(B)
        assert np.array_equal(rp, A.rowptr.astype(np.int64))
        assert np.array_equal(ci, A.colidx)
        assert np.array_equal(vv.view(np.uint16 if dtype == np.float16 else np.uint32),
                              vals.view(np.uint16 if dtype == np.float16 else np.uint32))


def test_signed_zero_and_nan_bits_roundtrip():
    v = np.array([0.0, -0.0, np.nan, 1e-45, -np.inf], np.float32)
    v[2] = np.frombuffer(np.uint32(0x7FC00123).tobytes(), np.float32)[0]
    A = W.CSR(1, 5, np.array([0, 5], np.int32), np.arange(5, dtype=np.int32), v)
    st, B = oracle.csr_to_bitbsr(1, 5, A.rowptr, A.colidx, A.values)
    assert st == 0 and int(B.bitmap[0]) == 0x1F
    assert np.array_equal(B.values.view(np.uint32), v.view(np.uint32))


# ---------------------------------------------------------- closed forms
@pytest.mark.parametrize("n", [1, 7, 8, 9, 1023, 1024])
def test_identity_closed_form(n):
    A = W.identity(n)
    st, B = oracle.csr_to_bitbsr(n, n, A.rowptr, A.colidx, A.values)
    assert st == 0
    assert B.Bnnz == (n + 7) // 8
    full = 0x8040201008040201
    for b, word in enumerate(B.bitmap):
        k = min(8, n - 8 * b)
        expect = full if k == 8 else sum(1 << (9 * i) for i in range(k))
        assert int(word) == expect
    if n % 8 == 3:
        assert int(B.bitmap[-1]) == 0x40201
    x = W.vector(n, 3)
    y, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    assert np.array_equal(y, x.astype(np.float64))


def test_reversal_closed_form():
    n = 64
    A = W.reversal(n)
    st, B = oracle.csr_to_bitbsr(n, n, A.rowptr, A.colidx, A.values)
    assert st == 0
    assert all(int(w) == 0x0102040810204080 for w in B.bitmap)
    assert B.blk_col.tolist() == [n // 8 - 1 - br for br in range(n // 8)]
    x = W.vector(n, 4)
    y, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    assert np.array_equal(y, x[::-1].astype(np.float64))


@pytest.mark.parametrize("n", [9, 1000])
def test_permutation_and_diagonal(n):
    perm = W.random_perm(n, 1)
    P = W.permutation(perm)
    x = W.vector(n, 5)
    y, _ = oracle.spmv(P.rowptr, P.colidx, P.values, x)
    assert np.array_equal(y, x[perm].astype(np.float64))
    D = W.diagonal(n, 2)
    y, _ = oracle.spmv(D.rowptr, D.colidx, D.values, x)
    assert np.array_equal(y, D.values.astype(np.float64) * x.astype(np.float64))


def test_dense_tile_full_bitmap():
    A = W.dense_block(8, 8)
    st, B = oracle.csr_to_bitbsr(8, 8, A.rowptr, A.colidx, A.values)
    assert st == 0 and B.Bnnz == 1 and int(B.bitmap[0]) == 0xFFFFFFFFFFFFFFFF
    A = W.dense_block(64, 64, 1)
    st, B = oracle.csr_to_bitbsr(64, 64, A.rowptr, A.colidx, A.values)
    assert B.Bnnz == 64 and all(int(w) == 0xFFFFFFFFFFFFFFFF for w in B.bitmap)
    assert B.blk_offset.tolist() == list(range(0, 64 * 65, 64))


def test_small_integer_exact():
    A = W.random_sparse(200, 150, 0.1, 9, dist="int")
    x = np.random.default_rng(1).integers(-8, 9, 150).astype(np.float32)
    y, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    ref = dense_of(A).astype(np.int64) @ x.astype(np.int64)
    assert np.array_equal(y, ref.astype(np.float64))


def test_empty_and_degenerate():
    for m, n in [(0, 0), (0, 5), (5, 0), (8, 8)]:
        A = W.CSR(m, n, np.zeros(m + 1, np.int32), np.zeros(0, np.int32), np.zeros(0, np.float32))
        st, B = oracle.csr_to_bitbsr(m, n, A.rowptr, A.colidx, A.values)
        assert st == 0 and B.Bnnz == 0
        assert B.blk_rowptr.tolist() == [0] * ((m + 7) // 8 + 1)
        assert B.blk_offset.tolist() == [0]
        y, _ = oracle.spmv(A.rowptr, A.colidx, A.values, np.zeros(n, np.float32))
        assert y.shape == (m,) and not y.any()


def test_empty_middle_and_last_block_rows():
    A = W.from_coo(40, 40, [0, 30], [39, 0], [1.0, 2.0])
    st, B = oracle.csr_to_bitbsr(40, 40, A.rowptr, A.colidx, A.values)
    assert B.blk_rowptr.tolist() == [0, 1, 1, 1, 2, 2]
    assert int(B.bitmap[0]) == 1 << 7 and int(B.bitmap[1]) == 1 << (8 * 6)


@pytest.mark.parametrize("kind,code", [("unsorted", oracle.ORC_UNSORTED), ("dup", oracle.ORC_UNSORTED),
                                       ("col_n", oracle.ORC_COL_RANGE), ("col_neg", oracle.ORC_COL_RANGE),
                                       ("rowptr", oracle.ORC_BAD_ROWPTR), ("rowptr_end", oracle.ORC_BAD_ROWPTR)])
def test_rejects_bad_csr(kind, code):
    rp = np.array([0, 2, 4], np.int32)
    ci = np.array([1, 3, 0, 2], np.int32)
    if kind == "unsorted":
        ci = np.array([3, 1, 0, 2], np.int32)
    elif kind == "dup":
        ci = np.array([1, 1, 0, 2], np.int32)
    elif kind == "col_n":
        ci = np.array([1, 4, 0, 2], np.int32)
    elif kind == "col_neg":
        ci = np.array([-1, 3, 0, 2], np.int32)
    elif kind == "rowptr":
        rp = np.array([0, 3, 2], np.int32)
    elif kind == "rowptr_end":
        rp = np.array([0, 2, 3], np.int32)
    st, B = oracle.csr_to_bitbsr(2, 4, rp, ci, np.ones(4, np.float32))
    assert st == code and B is None


# ------------------------------------------------------------ Table 1
def test_table1_invariants_and_footprint():
    t = load("table1.json")
    rows = t["rows"]
    for name, nrow, nnz, bnrow, bnnz in rows:
        assert bnrow == -(-nrow // 8), name                  # Bnrow = ceil(nrow/8)
        assert 1 <= nnz / bnnz <= 64, name                   # 1 <= fill <= 64
    raef = rows[0]
    assert raef[2] == 64 * raef[4]                           # raefsky3: every block full
    ev = rows[: t["evaluated"]]
    spaden = np.mean([oracle.bitbsr_bytes(r[1], r[4], r[2], 2) / r[2] for r in ev])
    csr = np.mean([(4 * (r[1] + 1) + 8 * r[2]) / r[2] for r in ev])
    bsr = np.mean([(4 * (r[3] + 1) + 4 * r[4] + 64 * 4 * r[4]) / r[2] for r in ev])
    assert abs(spaden - t["bytes_per_nnz"]["spaden"]) < 0.005, spaden
    assert abs(csr - t["bytes_per_nnz"]["csr"]) < 0.005, csr
    assert abs(bsr - t["bytes_per_nnz"]["bsr"]) < 0.005, bsr
    # with fp32 values the same format could not reach the paper's number
    sp32 = np.mean([oracle.bitbsr_bytes(r[1], r[4], r[2], 4) / r[2] for r in ev])
    assert sp32 > 4.5


# ------------------------------------------------------------ fp16 RNE
def test_f16_rne_matches_numpy():
    rng = np.random.default_rng(0)
    v = np.concatenate([rng.standard_normal(10000).astype(np.float32),
                        rng.uniform(-70000, 70000, 1000).astype(np.float32),
                        (rng.standard_normal(1000) * 1e-6).astype(np.float32),
                        np.array([0.0, -0.0, 65504.0, 65520.0, 65519.99, 1e-8, 6e-8, 2.0 ** -24,
                                  1 + 2.0 ** -11, 1 + 3 * 2.0 ** -11, np.inf, -np.inf], np.float32)])
    ours = oracle.f32_to_f16(v)
    ref = v.astype(np.float16)
    assert np.array_equal(ours.view(np.uint16), ref.view(np.uint16))
    # ties to even: 1 + 2^-11 -> 1.0, 1 + 3*2^-11 -> 1 + 2^-9
    assert float(oracle.f32_to_f16(np.array([1 + 2.0 ** -11], np.float32))[0]) == 1.0
    assert float(oracle.f32_to_f16(np.array([1 + 3 * 2.0 ** -11], np.float32))[0]) == 1 + 2.0 ** -9


# ------------------------------------------------------------ PageRank
def test_pagerank_fixed_point_dense_solve():
    n = 300
    src, dst = W.rmat_edges(8, 8, seed=3, relabel=True)
    src = np.concatenate([src, np.arange(256)])               # no dangling nodes:
    dst = np.concatenate([dst, (np.arange(256) + 1) % 256])   # add a ring
    n = 256
    A = W.pagerank_matrix(n, src, dst)
    d = 0.85
    x0 = np.full(n, 1.0 / n)
    x = oracle.pagerank(A.rowptr, A.colidx, A.values.astype(np.float64), d, 300, x0)
    D = dense_of(A)
    Dd = np.zeros((n, n))
    # recompute exact 1/outdeg in fp64 for the fixed point
    Dd[D != 0] = 1.0
    Dd = Dd / Dd.sum(axis=0, keepdims=True)
    xs = np.linalg.solve(np.eye(n) - d * Dd, np.full(n, (1 - d) / n))
    np.testing.assert_allclose(x, xs, rtol=1e-6)              # fp32-rounded 1/outdeg values
    assert abs(x.sum() - 1.0) < 1e-6


def test_pagerank_cycle_uniform():
    n = 50
    src = np.arange(n)
    dst = (src + 1) % n
    A = W.pagerank_matrix(n, src, dst)
    x = oracle.pagerank(A.rowptr, A.colidx, A.values, 0.85, 20, np.random.default_rng(0).dirichlet(np.ones(n)))
    xs = oracle.pagerank(A.rowptr, A.colidx, A.values, 0.85, 400, np.full(n, 1.0 / n))
    np.testing.assert_allclose(xs, np.full(n, 1.0 / n), rtol=1e-14)
    assert abs(x.sum() - 1) < 1e-12


# ------------------------------------------------------------ error metrics
def test_error_metrics():
    assert oracle.componentwise_error([1.0, 0.0], np.array([1.0, 0.0]), np.array([2.0, 0.0])) == 0.0
    assert oracle.componentwise_error([1.5], np.array([1.0]), np.array([2.0])) == 0.25
    assert oracle.componentwise_error([1e-30], np.array([0.0]), np.array([0.0])) == np.inf
    assert oracle.normwise_error([1.0, 2.5], np.array([1.0, 2.0]), 2.0, 1.0) == 0.25
    assert oracle.csr_inf_norm(np.array([0, 2, 3]), np.array([1.0, -2.0, 5.0])) == 5.0


def test_fem62k_invariants():
    """Converter invariants on the cant-shaped config (SURVEY.md §8(c) Invariants)."""
    A = W.make("fem62k")
    st, B = oracle.csr_to_bitbsr(A.m, A.n, A.rowptr, A.colidx, A.values)
    assert st == 0
    pc = np.array([bin(int(w)).count("1") for w in B.bitmap[:20000]])
    assert pc.min() >= 1 and pc.max() <= 64
    assert np.array_equal(np.diff(B.blk_offset[:20001]), pc)
    assert B.blk_offset[-1] == A.nnz
    assert B.Bnrow == (A.m + 7) // 8
    assert np.array_equal(B.blk_offset[B.blk_rowptr[:-1]], A.rowptr[0:A.m:8].astype(np.int64))
    d = np.diff(B.blk_col.astype(np.int64))
    starts = np.zeros(B.Bnnz, bool)
    starts[B.blk_rowptr[:-1][B.blk_rowptr[:-1] < B.Bnnz]] = True
    assert (d[~starts[1:]] > 0).all()
    fill = A.nnz / B.Bnnz
    assert 18 < fill < 26   # cant: 22.25 (Table 1)


# ------------------------------------------------------------ hybrid (NEXT-1)
def test_hybrid_split_hand_worked():
    """H1 with t = 2: only block (0,0) (4 entries) stays bitBSR (worked by hand)."""
    A = W.h1()
    (krp, kci, kv), (rrp, rci, rv) = oracle.hybrid_split(A.m, A.n, A.rowptr, A.colidx, A.values, 2)
    st, B = oracle.csr_to_bitbsr(A.m, A.n, krp, kci, kv)
    assert B.blk_rowptr.tolist() == [0, 1, 1] and B.blk_col.tolist() == [0]
    assert [int(w) for w in B.bitmap] == [0x8000000080000201]
    assert B.values.tolist() == [1, 3, 4, 5]
    assert rrp.tolist() == [0, 1, 1, 1, 1, 1, 1, 1, 2, 2, 3, 3, 3, 4, 4, 4, 5]
    assert rci.tolist() == [9, 8, 2, 3, 15] and rv.tolist() == [2, 6, 7, -1, 8]
    # t = 1: only the single-entry block (1,1) -> residual
    (krp, kci, kv), (rrp, rci, rv) = oracle.hybrid_split(A.m, A.n, A.rowptr, A.colidx, A.values, 1)
    assert rci.tolist() == [15] and rv.tolist() == [8] and rrp[-1] == 1


@pytest.mark.parametrize("t", [1, 2, 5, 64])
def test_hybrid_split_partitions_entries(t):
    A = W.random_sparse(300, 250, 0.03, 4)
    (krp, kci, kv), (rrp, rci, rv) = oracle.hybrid_split(A.m, A.n, A.rowptr, A.colidx, A.values, t)
    D = dense_of(A)
    K = dense_of(W.CSR(A.m, A.n, krp.astype(np.int32), kci, kv))
    R = dense_of(W.CSR(A.m, A.n, rrp.astype(np.int32), rci, rv))
    assert np.array_equal(K + R, D)
    assert not ((K != 0) & (R != 0)).any()
    st, B = oracle.csr_to_bitbsr(A.m, A.n, krp, kci, kv)
    pc = np.array([bin(int(w)).count("1") for w in B.bitmap])
    assert (pc > t).all()
    x = W.vector(A.n, 1)
    y, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    yk, _ = oracle.spmv(krp, kci, kv, x)
    yr, _ = oracle.spmv(rrp, rci, rv, x)
    np.testing.assert_allclose(yk + yr, y, rtol=1e-12, atol=1e-12)


# ------------------------------------------------ reordering (NEXT-1)
def test_degree_order_hand_worked():
    """Degrees [1, 3, 0, 3, 2] -> descending, ties in ascending row order:
    rows 1, 3 (degree 3), 4 (2), 0 (1), 2 (0)."""
    rp = np.array([0, 1, 4, 4, 7, 9], np.int32)
    assert oracle.degree_order(rp).tolist() == [1, 3, 4, 0, 2]


def test_degree_order_closed_forms():
    n = 37
    eye = W.from_dense(np.eye(n, dtype=np.float32))
    assert np.array_equal(oracle.degree_order(eye.rowptr), np.arange(n))        # all equal: identity
    low = W.from_dense(np.tril(np.ones((n, n), np.float32)))
    assert np.array_equal(oracle.degree_order(low.rowptr), np.arange(n)[::-1])  # degree i+1: reversal
    assert oracle.degree_order(np.zeros(1, np.int32)).size == 0                  # m = 0


@pytest.mark.parametrize("m,dens,seed", [(1, 1.0, 0), (13, 0.3, 1), (64, 0.08, 2), (200, 0.02, 3)])
def test_permute_csr_vs_dense(m, dens, seed):
    """B = P A P^T against dense indexing B = A[perm][:, perm] (a different
    mechanism than the oracle's entry relabelling + lexsort), and the SpMV
    identity B (P x) = P (A x)."""
    A = W.random_sparse(m, m, dens, seed)
    for perm in (oracle.degree_order(A.rowptr), W.random_perm(m, seed + 7)):
        rp, ci, v = oracle.permute_csr(A.rowptr, A.colidx, A.values, perm)
        B = W.CSR(m, m, rp, ci, v)
        dense_a = np.zeros((m, m), np.float32)
        for i in range(m):
            dense_a[i, A.colidx[A.rowptr[i]:A.rowptr[i + 1]]] = A.values[A.rowptr[i]:A.rowptr[i + 1]]
        dense_b = np.zeros((m, m), np.float32)
        for i in range(m):
            dense_b[i, ci[rp[i]:rp[i + 1]]] = v[rp[i]:rp[i + 1]]
        assert np.array_equal(dense_b, dense_a[perm][:, perm])
        assert all(np.all(np.diff(ci[rp[i]:rp[i + 1]]) > 0) for i in range(m))   # canonical rows
        x = W.vector(m, seed)
        y, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x)
        yb, _ = oracle.spmv(rp, ci, v, x[perm])
        assert np.allclose(yb, y[perm], rtol=1e-12, atol=1e-12)
