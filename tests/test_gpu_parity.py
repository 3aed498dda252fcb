"""Parity of the CUDA path (through the C ABI) against the CPU oracle.

Conversion: bit-exact (memcmp of all five bitBSR arrays against oracle/'s
reference converter, plus oracle decode back to the input CSR).
SpMV: fp32 values componentwise |y - y*| / s <= 1e-5; fp16 values componentwise
1e-5 against the oracle on the stored fp16 values and normwise 1e-2 against the
original fp32 values (BASELINE north_star).  Closed
forms (identity / permutation / diagonal / small integers / H1 / H2) bitwise.
"""
import ctypes

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

TOL32 = 1e-5
TOL16_NORM = 1e-2


@pytest.fixture(scope="module")
def sp():
    import paper_conf_icpp_cheny24_b200 as sp
    return sp


@pytest.fixture(scope="module")
def torch():
    import torch
    assert torch.cuda.is_available()
    return torch


def dev(torch, A, values=None):
    vals = A.values if values is None else values
    return (torch.from_numpy(np.ascontiguousarray(A.rowptr)).cuda(),
            torch.from_numpy(np.ascontiguousarray(A.colidx)).cuda(),
            torch.from_numpy(np.ascontiguousarray(vals)).cuda())


def convert(sp, torch, A, values=None, storage=None):
    rp, ci, v = dev(torch, A, values)
    M = sp.convert(rp, ci, v, A.n, storage=storage)
    torch.cuda.synchronize()
    return M


def host_arrays(torch, M):
    return {k: t.cpu().numpy() for k, t in M.arrays().items()}


def assert_format_parity(torch, M, A, values):
    st, B = oracle.csr_to_bitbsr(A.m, A.n, A.rowptr, A.colidx, values)
    assert st == 0
    h = host_arrays(torch, M)
    i = M.info
    assert (i.m, i.n, i.nnz, i.Bnrow, i.Bnnz) == (A.m, A.n, A.nnz, B.Bnrow, B.Bnnz)
    assert np.array_equal(h["blk_rowptr"].astype(np.int64), B.blk_rowptr)
    if B.Bnnz:
        assert np.array_equal(h["blk_col"], B.blk_col)
        assert np.array_equal(h["bitmap"].view(np.uint64), B.bitmap)
    assert np.array_equal(h["blk_offset"].astype(np.int64), B.blk_offset)
    if A.nnz:
        ub = np.uint16 if values.dtype == np.float16 else np.uint32
        assert np.array_equal(h["values"].view(ub), np.ascontiguousarray(B.values).view(ub))
    # footprint formula
    assert i.format_bytes == oracle.bitbsr_bytes(A.m, B.Bnnz, A.nnz, values.dtype.itemsize)
    # decode(GPU arrays) == input CSR, bit for bit
    G = oracle.BitBSR(A.m, A.n, h["blk_rowptr"].astype(np.int64), h["blk_col"] if B.Bnnz else B.blk_col,
                      h["bitmap"].view(np.uint64) if B.Bnnz else B.bitmap,
                      h["blk_offset"].astype(np.int64), h["values"] if A.nnz else values[:0])
    rp, ci, vv = oracle.bitbsr_to_csr(G)
    assert np.array_equal(rp, A.rowptr.astype(np.int64))
    assert np.array_equal(ci, A.colidx)
    ub = np.uint16 if values.dtype == np.float16 else np.uint32
    assert np.array_equal(np.ascontiguousarray(vv).view(ub), np.ascontiguousarray(values).view(ub))
    return B


def gpu_spmv(torch, M, x, alpha=1.0, beta=0.0, y0=None):
    xd = torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).cuda()
    yd = torch.from_numpy(np.ascontiguousarray(y0, dtype=np.float32)).cuda() if y0 is not None else None
    y = M.spmv(xd, yd, alpha=alpha, beta=beta)
    torch.cuda.synchronize()
    return y.cpu().numpy()


CASES = {
    "h1": lambda: W.h1(),
    "h2": lambda: W.h2(),
    "identity1": lambda: W.identity(1),
    "identity7": lambda: W.identity(7),
    "identity9": lambda: W.identity(9),
    "identity1023": lambda: W.identity(1023),
    "reversal64": lambda: W.reversal(64),
    "perm1000": lambda: W.permutation(W.random_perm(1000, 3)),
    "diag1024": lambda: W.diagonal(1024, 1),
    "dense8": lambda: W.dense_block(8, 8),
    "dense64": lambda: W.dense_block(64, 64, 2),
    "corner": lambda: W.from_coo(13, 21, [12], [20], [3.0]),
    "empty_middle_last": lambda: W.from_coo(40, 40, [0, 30], [39, 0], [1.0, 2.0]),
    "rand_rect": lambda: W.random_sparse(333, 517, 0.02, 5),
    "rand_dense": lambda: W.random_sparse(129, 65, 0.6, 6),
    "tiny": lambda: W.tiny(0),
    "hub": lambda: hub_matrix(),
}


def hub_matrix(m=64, n=100_003, hub_rows=(3, 9, 60), hub_nnz=30_000, seed=7):
    """A few hub rows spanning many block columns (forces the chunked converter path)."""
    rng = np.random.default_rng(seed)
    rows, cols = [], []
    for r in hub_rows:
        c = rng.choice(n, hub_nnz, replace=False)
        rows.append(np.full(c.size, r))
        cols.append(c)
    for r in range(m):
        c = rng.choice(n, 5, replace=False)
        rows.append(np.full(5, r))
        cols.append(c)
    rows = np.concatenate(rows)
    cols = np.concatenate(cols)
    key = np.unique(rows.astype(np.int64) * n + cols)
    r, c = np.divmod(key, n)
    return W.from_coo(m, n, r, c, rng.uniform(-1, 1, key.size))


@pytest.mark.parametrize("name", sorted(CASES))
@pytest.mark.parametrize("mode", ["f32>f32", "f32>f16", "f16>f16", "f16>f32"])
def test_conversion_bit_exact(sp, torch, name, mode):
    A = CASES[name]()
    vin = A.values.astype(np.float16) if mode.startswith("f16") else A.values
    if mode == "f32>f16":
        stored = oracle.f32_to_f16(A.values)
    elif mode == "f16>f32":
        stored = vin.astype(np.float32)
    else:
        stored = vin
    M = convert(sp, torch, A, values=vin, storage="fp16" if mode.endswith("f16") else "fp32")
    h = host_arrays(torch, M)
    # the reference converter applied to the oracle-rounded values
    Aref = W.CSR(A.m, A.n, A.rowptr, A.colidx, stored)
    assert_format_parity(torch, M, Aref, stored)
    M.free()


@pytest.mark.parametrize("m,n", [(0, 0), (0, 7), (7, 0), (8, 8), (17, 3)])
def test_empty_matrices(sp, torch, m, n):
    A = W.CSR(m, n, np.zeros(m + 1, np.int32), np.zeros(0, np.int32), np.zeros(0, np.float32))
    rp = torch.zeros(m + 1, dtype=torch.int32, device="cuda")
    ci = torch.zeros(1, dtype=torch.int32, device="cuda")
    v = torch.zeros(1, dtype=torch.float32, device="cuda")
    h = ctypes.c_void_p()
    st = sp.spaden_convert_csr_to_bitmap(m, n, 0, rp.data_ptr(), ci.data_ptr(), v.data_ptr(), 0, 0,
                                         torch.cuda.current_stream().cuda_stream, ctypes.byref(h))
    assert st == 0
    M = sp.Matrix(h, rp.device)
    assert M.info.Bnnz == 0 and M.info.Bnrow == (m + 7) // 8
    if m:
        x = torch.ones(max(n, 1), device="cuda")[:n].contiguous() if n else torch.zeros(0, device="cuda")
        y0 = torch.full((m,), float("nan"), device="cuda")
        st = sp.spaden_spmv(M.handle, 1.0, x.data_ptr() or None, 0.0, y0.data_ptr(), None)
        torch.cuda.synchronize()
        assert st == 0 and (y0 == 0).all()
        y1 = torch.full((m,), 2.0, device="cuda")
        sp.spaden_spmv(M.handle, 1.0, x.data_ptr() or None, 0.5, y1.data_ptr(), None)
        torch.cuda.synchronize()
        assert (y1 == 1.0).all()
    M.free()


def bad_inputs():
    rp = np.array([0, 2, 4], np.int32)
    ci = np.array([1, 3, 0, 2], np.int32)
    yield "unsorted", rp, np.array([3, 1, 0, 2], np.int32), 3
    yield "dup", rp, np.array([1, 1, 0, 2], np.int32), 3
    yield "col_n", rp, np.array([1, 4, 0, 2], np.int32), 2
    yield "col_neg", rp, np.array([-1, 3, 0, 2], np.int32), 2
    yield "rowptr_nonmono", np.array([0, 3, 2], np.int32), ci, 1
    yield "rowptr_end", np.array([0, 2, 3], np.int32), ci, 1
    yield "rowptr_start", np.array([1, 2, 4], np.int32), ci, 1


@pytest.mark.parametrize("case", list(bad_inputs()), ids=lambda c: c[0])
def test_rejects_invalid_csr(sp, torch, case):
    _, rp, ci, code = case
    rpd, cid = torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda()
    v = torch.ones(4, device="cuda")
    h = ctypes.c_void_p()
    st = sp.spaden_convert_csr_to_bitmap(2, 4, 4, rpd.data_ptr(), cid.data_ptr(), v.data_ptr(), 0, 0,
                                         None, ctypes.byref(h))
    assert st == code and h.value is None


def test_rejects_unsorted_hub_row_and_host_pointer(sp, torch):
    A = hub_matrix()
    ci = A.colidx.copy()
    k = int(A.rowptr[9]) + 20_000          # inside a chunked hub row
    ci[k], ci[k + 1] = ci[k + 1], ci[k]
    h = ctypes.c_void_p()
    rp, cid, v = dev(torch, A)
    cid.copy_(torch.from_numpy(ci))
    st = sp.spaden_convert_csr_to_bitmap(A.m, A.n, A.nnz, rp.data_ptr(), cid.data_ptr(), v.data_ptr(), 0, 0,
                                         None, ctypes.byref(h))
    assert st == sp.SPADEN_ERR_UNSORTED_OR_DUPLICATE
    host_rp = np.zeros(A.m + 1, np.int32)
    st = sp.spaden_convert_csr_to_bitmap(A.m, A.n, 0, host_rp.ctypes.data, None, None, 0, 0, None,
                                         ctypes.byref(h))
    assert st == sp.SPADEN_ERR_INVALID_ARGUMENT


# ------------------------------------------------------------------ SpMV
def check_spmv(A, y, stored, x):
    ys, s = oracle.spmv(A.rowptr, A.colidx, stored, x)
    err = oracle.componentwise_error(y, ys, s)
    assert err <= TOL32, err
    return ys


@pytest.mark.parametrize("name", sorted(CASES))
def test_spmv_fp32(sp, torch, name):
    A = CASES[name]()
    M = convert(sp, torch, A)
    x = W.vector(A.n, 11)
    y = gpu_spmv(torch, M, x)
    check_spmv(A, y, A.values, x)


@pytest.mark.parametrize("name", sorted(CASES))
def test_spmv_fp16(sp, torch, name):
    A = CASES[name]()
    M = convert(sp, torch, A, storage="fp16")
    x = W.vector(A.n, 12)
    y = gpu_spmv(torch, M, x)
    stored = oracle.f32_to_f16(A.values)
    check_spmv(A, y, stored, x)
    y32, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    nerr = oracle.normwise_error(y, y32, oracle.csr_inf_norm(A.rowptr, A.values), float(np.abs(x).max(initial=0)))
    assert nerr <= TOL16_NORM


@pytest.mark.parametrize("name", ["h1", "h2"])
def test_spmv_hand_worked_exact(sp, torch, name):
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", name + ".json")))
    A = CASES[name]()
    M = convert(sp, torch, A)
    y = gpu_spmv(torch, M, np.arange(1, A.n + 1, dtype=np.float32))
    assert y.tolist() == [float(v) for v in g["y"]]


def test_spmv_closed_forms_bitwise(sp, torch):
    for n in (1, 7, 8, 9, 1023, 1024):
        x = W.vector(n, n)
        assert np.array_equal(gpu_spmv(torch, convert(sp, torch, W.identity(n)), x), x)
        perm = W.random_perm(n, n)
        assert np.array_equal(gpu_spmv(torch, convert(sp, torch, W.permutation(perm)), x), x[perm])
        D = W.diagonal(n, n)
        assert np.array_equal(gpu_spmv(torch, convert(sp, torch, D), x), (D.values * x).astype(np.float32))
    A = W.random_sparse(300, 280, 0.2, 1, dist="int")
    x = np.random.default_rng(2).integers(-8, 9, 280).astype(np.float32)
    y = gpu_spmv(torch, convert(sp, torch, A), x)
    ys, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    assert np.array_equal(y.astype(np.float64), ys)


def test_alpha_beta_and_nan_semantics(sp, torch):
    A = W.random_sparse(200, 190, 0.05, 4)
    M = convert(sp, torch, A)
    x = W.vector(190, 1)
    y0 = W.vector(200, 2)
    y = gpu_spmv(torch, M, x, alpha=2.0, beta=0.5, y0=y0)
    ys, s = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    ref = 2.0 * ys + 0.5 * y0.astype(np.float64)
    assert oracle.componentwise_error(y, ref, 2.0 * s + 0.5 * np.abs(y0)) <= TOL32
    # beta == 0: y's old contents (NaN) are ignored
    y = gpu_spmv(torch, M, x, beta=0.0, y0=np.full(200, np.nan, np.float32))
    assert np.isfinite(y).all()
    # a NaN in x only reaches rows that reference that column (structural zeros never multiplied)
    j = int(A.colidx[0])
    xn = x.copy()
    xn[j] = np.nan
    y = gpu_spmv(torch, M, xn)
    dense_ref = np.zeros(200, bool)
    for i in range(200):
        dense_ref[i] = j in A.colidx[A.rowptr[i]:A.rowptr[i + 1]]
    assert np.array_equal(np.isnan(y), dense_ref)


def test_unaligned_x(sp, torch):
    A = W.random_sparse(100, 97, 0.1, 3)
    M = convert(sp, torch, A)
    x = W.vector(97, 4)
    buf = torch.zeros(98, device="cuda")
    buf[1:].copy_(torch.from_numpy(x))
    xv = buf[1:]
    y = M.spmv(xv)
    torch.cuda.synchronize()
    check_spmv(A, y.cpu().numpy(), A.values, x)


def test_deterministic_and_partition_invariant(sp, torch):
    A = W.make("fem62k")
    x = W.vector(A.n, 5)
    M = convert(sp, torch, A)
    y1 = gpu_spmv(torch, M, x)
    y2 = gpu_spmv(torch, M, x)
    assert np.array_equal(y1, y2)
    parts = []
    bounds = [0, 8 * 1000, 8 * 3001, 8 * 5000, A.m]
    for r0, r1 in zip(bounds[:-1], bounds[1:]):
        S = A.row_slice(r0, r1)
        parts.append(gpu_spmv(torch, convert(sp, torch, S), x))
    assert np.array_equal(np.concatenate(parts), y1)
    check_spmv(A, y1, A.values, x)


def test_spmv_host_matches_device(sp, torch):
    A = W.tiny(0)
    M = convert(sp, torch, A)
    x = W.vector(A.n, 8)
    yd = gpu_spmv(torch, M, x)
    xh = torch.from_numpy(x).pin_memory()
    yh = torch.empty(A.m, dtype=torch.float32).pin_memory()
    M.spmv_host(xh, yh)
    assert np.array_equal(yh.numpy(), yd)


def test_cuda_graph_capture(sp, torch):
    A = W.tiny(1)
    M = convert(sp, torch, A)
    x = torch.from_numpy(W.vector(A.n, 9)).cuda()
    y = torch.empty(A.m, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        M.spmv(x, y)
    torch.cuda.synchronize()
    ref = y.clone()
    y.zero_()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        M.spmv(x, y, stream=s)
    g.replay()
    torch.cuda.synchronize()
    assert torch.equal(y, ref)


@pytest.mark.parametrize("t", [0, 2])
def test_cuda_graph_capture_chain(sp, torch, t):
    """The multi-kernel chains (hybrid residual pass, long-row chunks with the
    fused fix-up, programmatic dependent launches) captured in a CUDA graph and
    replayed repeatedly give the eager result bitwise, with alpha/beta."""
    A = hub_matrix(m=96, n=200_003, hub_rows=(3, 60, 61), hub_nnz=60_000, seed=5)
    rp, ci, v = dev(torch, A)
    M = sp.convert(rp, ci, v, A.n, residual_max_popc=t)
    torch.cuda.synchronize()
    assert M.info.n_long >= 1 or M.info.residual_nnz > 0
    x = torch.from_numpy(W.vector(A.n, 19)).cuda()
    y0 = torch.from_numpy(W.vector(A.m, 20)).cuda()
    s = torch.cuda.Stream()
    y = y0.clone()
    with torch.cuda.stream(s):
        M.spmv(x, y, alpha=0.5, beta=-2.0, stream=s)
    torch.cuda.synchronize()
    ref = y.clone()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        M.spmv(x, y, alpha=0.5, beta=-2.0, stream=s)
    for _ in range(3):
        y.copy_(y0)
        g.replay()
        torch.cuda.synchronize()
        assert torch.equal(y, ref)


@pytest.mark.parametrize("storage", ["fp32", "fp16"])
@pytest.mark.parametrize("fixup", ["fused", "separate"])
@pytest.mark.parametrize("seg_cols", [3000, 20_011 // 2 + 1, 64])
def test_residual_column_parts(sp, torch, storage, fixup, seg_cols, monkeypatch):
    """Residual split into column parts (as for x > 32 MB; forced here with
    SPADEN_XSEG_COLS): every part's rows binned, parts added in column order.
    Within tolerance of the oracle, deterministic, 8-row-partition invariant,
    alpha/beta, launch count = CUDA-graph nodes."""
    monkeypatch.setenv("SPADEN_XSEG_COLS", str(seg_cols))
    if fixup == "separate":
        monkeypatch.setenv("SPADEN_FUSED_FIXUP_MAX", "0")
    A = binned_rows_matrix(seed=13)
    stored = A.values if storage == "fp32" else oracle.f32_to_f16(A.values)
    x = W.vector(A.n, 43)
    rp, ci, v = dev(torch, A)
    M = sp.convert(rp, ci, v, A.n, storage=storage, residual_max_popc=64)
    assert M.info.residual_nnz == A.nnz and M.info.Bnnz == 0
    assert "res_rowptr" not in M.arrays()  # split into parts
    y = gpu_spmv(torch, M, x)
    assert np.array_equal(y, gpu_spmv(torch, M, x))
    check_spmv(A, y, stored, x)
    y0 = W.vector(A.m, 44)
    ys, s = oracle.spmv(A.rowptr, A.colidx, stored, x)
    y2 = gpu_spmv(torch, M, x, alpha=0.5, beta=-1.5, y0=y0)
    assert oracle.componentwise_error(y2, 0.5 * ys - 1.5 * y0, 0.5 * s + 1.5 * np.abs(y0)) <= TOL32
    cut = (A.m // 16) * 8
    parts = []
    for r0, r1 in ((0, cut), (cut, A.m)):
        S = A.row_slice(r0, r1)
        r, c, vv = dev(torch, S)
        parts.append(gpu_spmv(torch, sp.convert(r, c, vv, S.n, storage=storage, residual_max_popc=64), x))
    assert np.array_equal(np.concatenate(parts), y)
    xd = torch.from_numpy(x).cuda()
    yd = torch.from_numpy(y0).cuda()
    assert graph_nodes(torch, lambda st: M.spmv(xd, yd, alpha=1.0, beta=0.5, stream=st)) == M.launch_count(0.5)


def test_hybrid_auto_threshold(sp, torch):
    """residual_max_popc = -1: hybrid (t = 4) for low mean block fill, pure bitBSR
    for FEM-like blocks; the choice is reported in spaden_info_t; results within
    tolerance; values outside [-1, 64] are rejected."""
    for A, want in ((W.powerlaw(13, 6, seed=1), 4), (W.fem(6, 7, 8, seed=2), 0)):
        rp, ci, v = dev(torch, A)
        M = sp.convert(rp, ci, v, A.n, residual_max_popc=-1)
        assert M.info.residual_max_popc == want
        assert (M.info.residual_nnz > 0) == (want > 0)
        assert M.info.residual_parts == (1 if want else 0)
        x = W.vector(A.n, 45)
        check_spmv(A, gpu_spmv(torch, M, x), A.values, x)
    A = W.tiny(0)
    rp, ci, v = dev(torch, A)
    for bad in (-2, 65):
        with pytest.raises(sp.SpadenError):
            sp.convert(rp, ci, v, A.n, residual_max_popc=bad)


def graph_nodes(torch, fn):
    """Number of nodes (kernel launches, memsets) fn() puts on a captured stream."""
    rt = pytest.importorskip("cuda.bindings.runtime")
    s = torch.cuda.Stream()
    fn(s)  # eager warm-up (lazy module loading outside the capture)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph(keep_graph=True)
    with torch.cuda.graph(g, stream=s):
        fn(s)
    out = rt.cudaGraphGetNodes(rt.cudaGraph_t(init_value=g.raw_cuda_graph()))
    assert int(out[0]) == 0
    return int(out[-1])


@pytest.mark.parametrize("case", ["fem", "hub_fused", "hub_separate", "hyb_long", "hyb_long_sep", "hyb_fixed"])
@pytest.mark.parametrize("beta", [0.0, 0.5, 1.0])
def test_launch_count_matches_graph(sp, torch, case, beta, monkeypatch):
    """spaden_spmv_launch_count (the bench's gpu_launches) equals the number of
    nodes a captured spaden_spmv puts in a CUDA graph."""
    if case.endswith("sep"):
        monkeypatch.setenv("SPADEN_FUSED_FIXUP_MAX", "0")
    if case == "hub_separate":
        monkeypatch.setenv("SPADEN_FUSED_FIXUP_MAX", "0")
    if case == "hyb_fixed":
        monkeypatch.setenv("SPADEN_RES", "fixed")
    A = W.fem(6, 7, 8, seed=2) if case == "fem" else (
        binned_rows_matrix() if case.startswith("hyb") else hub_matrix(m=40, n=70_001, hub_rows=(3, 30), hub_nnz=40_000))
    t = 2 if case.startswith("hyb") else 0
    rp, ci, v = dev(torch, A)
    M = sp.convert(rp, ci, v, A.n, residual_max_popc=t)
    x = torch.from_numpy(W.vector(A.n, 3)).cuda()
    y = torch.from_numpy(W.vector(A.m, 4)).cuda()
    n = graph_nodes(torch, lambda s: M.spmv(x, y, alpha=1.0, beta=beta, stream=s))
    assert n == M.launch_count(beta) >= 1


@pytest.mark.parametrize("t", [0, 3])
def test_pdl_off_bitwise_equal(sp, torch, t, monkeypatch):
    """Programmatic dependent launch only changes when kernels may start:
    SPADEN_PDL=0 (plain stream order) gives the same y bitwise."""
    A = W.powerlaw(14, 6, seed=3)
    rp, ci, v = dev(torch, A)
    M = sp.convert(rp, ci, v, A.n, residual_max_popc=t)
    x = W.vector(A.n, 21)
    y0 = W.vector(A.m, 22)
    ref = gpu_spmv(torch, M, x, alpha=1.25, beta=0.5, y0=y0)
    monkeypatch.setenv("SPADEN_PDL", "0")
    assert np.array_equal(gpu_spmv(torch, M, x, alpha=1.25, beta=0.5, y0=y0), ref)
    ys, s = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    assert oracle.componentwise_error(ref, 1.25 * ys + 0.5 * y0, 1.25 * s + 0.5 * np.abs(y0)) <= TOL32


@pytest.mark.parametrize("name", ["fem62k", "powerlaw1m"])
def test_configs_full(sp, torch, name):
    A = W.make(name)
    M = convert(sp, torch, A)
    assert_format_parity(torch, M, A, A.values)
    x = W.vector(A.n, 21)
    check_spmv(A, gpu_spmv(torch, M, x), A.values, x)
    M16 = convert(sp, torch, A, storage="fp16")
    y = gpu_spmv(torch, M16, x)
    check_spmv(A, y, oracle.f32_to_f16(A.values), x)


@pytest.mark.slow
def test_fem1p5m_full(sp, torch):
    """BASELINE configs[3] at full size, in the launch configuration bench.py times."""
    A = W.make("fem1p5m")
    x = W.vector(A.n, 31)
    for storage, stored in (("fp32", A.values), ("fp16", oracle.f32_to_f16(A.values))):
        M = convert(sp, torch, A, storage=storage)
        i = M.info
        assert i.nnz == A.nnz and i.Bnrow == (A.m + 7) // 8
        assert i.format_bytes == oracle.bitbsr_bytes(A.m, i.Bnnz, A.nnz, 2 if storage == "fp16" else 4)
        check_spmv(A, gpu_spmv(torch, M, x), stored, x)
        # sampled block-rows of the format against the reference converter on a row slice
        h = M.arrays()
        rng = np.random.default_rng(0)
        for br in rng.choice(i.Bnrow, 64, replace=False):
            S = A.row_slice(8 * int(br), 8 * int(br) + 8)
            st, B = oracle.csr_to_bitbsr(S.m, S.n, S.rowptr, S.colidx, stored[A.rowptr[8 * br]:A.rowptr[min(8 * br + 8, A.m)]])
            b0, b1 = [int(v) for v in h["blk_rowptr"][br:br + 2].cpu()]
            assert b1 - b0 == B.Bnnz
            assert np.array_equal(h["blk_col"][b0:b1].cpu().numpy(), B.blk_col)
            assert np.array_equal(h["bitmap"][b0:b1].cpu().numpy().view(np.uint64), B.bitmap)
            off = h["blk_offset"][b0:b1 + 1].cpu().numpy().astype(np.int64)
            assert np.array_equal(off - off[0], B.blk_offset)
            assert off[0] == A.rowptr[8 * br]
        M.free()


def test_rmat25_full_hybrid_sampled(sp, torch):
    """BASELINE configs[4] (R-MAT scale 25, edge factor 32, 1.05B nnz, PageRank
    values) at full size on one GPU, converted as bench.py does (automatic
    hybrid: t = 4, residual split into 2 column parts because x is 134 MB): y on
    4096 sampled rows (incl. the longest ones) against the fp64 oracle on those rows."""
    rp, ci, v, n, nnz = W.pagerank_slice_torch(25, 32, 0, 1 << 25, seed=0, device="cuda")
    M = sp.convert(rp, ci, v, n, residual_max_popc=-1)
    torch.cuda.synchronize()
    i = M.info
    assert i.nnz == nnz and i.residual_max_popc == 4 and i.residual_parts == 2
    g = torch.Generator(device="cuda")
    g.manual_seed(7)
    x = torch.rand(n, generator=g, device="cuda")
    y = M.spmv(x)
    torch.cuda.synchronize()
    rph = rp.cpu().numpy().astype(np.int64)
    lens = np.diff(rph)
    rng = np.random.default_rng(3)
    rows = np.unique(np.concatenate([rng.choice(n, 4064, replace=False), np.argsort(lens)[-32:]]))
    sub_rp = np.zeros(rows.size + 1, np.int64)
    sub_rp[1:] = np.cumsum(lens[rows])
    idx = torch.from_numpy(np.concatenate([np.arange(rph[r], rph[r + 1]) for r in rows])).cuda()
    cols = ci[idx].cpu().numpy()
    vals = v[idx].cpu().numpy()
    ys, s = oracle.spmv(sub_rp, cols, vals, x.cpu().numpy())
    err = oracle.componentwise_error(y[torch.from_numpy(rows).cuda()].cpu().numpy(), ys, s)
    assert err <= TOL32, err
    M.free()


def test_tile_row_cap_empty_block_rows(sp, torch):
    """Long runs of empty block-rows (more than the 128 block-rows a tile may
    hold) between a few populated ones: y is exact (small integers) and rows
    with no entries are exactly beta*y0."""
    m, n = 8 * 1000 + 5, 4096
    rows = np.array([0, 3, 8 * 300 + 1, 8 * 300 + 1, 8 * 999 + 7, m - 1])
    cols = np.array([0, 4095, 17, 18, 2048, 5])
    vals = np.array([1, 2, 3, 4, 5, 6], dtype=np.float32)
    A = W.from_coo(m, n, rows, cols, vals)
    x = (np.arange(n) % 7 + 1).astype(np.float32)
    M = convert(sp, torch, A)
    y = gpu_spmv(torch, M, x)
    ref = np.zeros(m, np.float32)
    np.add.at(ref, rows, vals * x[cols])
    assert np.array_equal(y, ref)
    y0 = W.vector(m, 5)
    y2 = gpu_spmv(torch, M, x, alpha=1.0, beta=0.5, y0=y0)
    empty = np.setdiff1d(np.arange(m), rows)
    assert np.array_equal(y2[empty], (np.float32(0.5) * y0[empty]).astype(np.float32))


@pytest.mark.parametrize("fixup", ["fused", "separate"])
def test_long_rows_deterministic_and_partition_invariant(sp, torch, fixup, monkeypatch):
    """Block-rows far larger than a pipeline stage (hub rows) go through the
    chunked long-row path; y is deterministic, within tolerance, and identical
    under an 8-row-aligned row split -- with the fix-up fused into the chunk
    kernel (last warp per row) and as a separate launch, bitwise equal."""
    A = hub_matrix(m=96, n=400_003, hub_rows=(3, 9, 60, 61), hub_nnz=120_000, seed=11)
    M = convert(sp, torch, A)
    assert M.info.n_long >= 2
    x = W.vector(A.n, 13)
    ref = gpu_spmv(torch, M, x)
    if fixup == "separate":
        monkeypatch.setenv("SPADEN_FUSED_FIXUP_MAX", "0")
    y1 = gpu_spmv(torch, M, x)
    assert np.array_equal(y1, ref)
    y2 = gpu_spmv(torch, M, x, alpha=2.0, beta=-1.0, y0=y1)
    assert np.array_equal(gpu_spmv(torch, M, x, alpha=2.0, beta=-1.0, y0=y1), y2)
    check_spmv(A, y1, A.values, x)
    parts = [gpu_spmv(torch, convert(sp, torch, A.row_slice(r0, r1)), x) for r0, r1 in ((0, 56), (56, 96))]
    assert np.array_equal(np.concatenate(parts), y1)


def test_pagerank_iteration_vs_oracle(sp, torch):
    """rmat-style PageRank (x <- 0.85 A x + 0.15/n) through the CUDA path and the
    row-partition driver vs the fp64 oracle iteration."""
    from paper_conf_icpp_cheny24_b200.dist import IteratedSpMV, RowPartition
    scale, K = 14, 20
    rp, ci, v, n, nnz = W.pagerank_slice_torch(scale, 16, 0, 1 << scale, seed=3, device="cuda")
    M = sp.convert(rp, ci, v, n)
    part = RowPartition(n, 1)
    it = IteratedSpMV(part, n, lambda xx, yy, a, b: M.spmv(xx, yy, alpha=a, beta=b),
                      torch.full((n,), 1.0 / n, device="cuda"), 0)
    for _ in range(K):
        x = it.step(0.85, 0.15 / n)
    torch.cuda.synchronize()
    ref = oracle.pagerank(rp.cpu().numpy(), ci.cpu().numpy(), v.cpu().numpy(), 0.85, K, np.full(n, 1.0 / n))
    got = x[:n].cpu().numpy().astype(np.float64)
    rel = np.abs(got - ref) / np.abs(ref)
    assert rel.max() <= 1e-5, rel.max()


TILE_CFGS = [1, 2, 3, 5, 6, 7, 10, 14, 15, 16]  # internal.cuh tile_cfg_valid


@pytest.mark.parametrize("rot", ["1", "0"])
@pytest.mark.parametrize("cfg", TILE_CFGS)
def test_every_tile_config_same_result(sp, torch, cfg, rot, monkeypatch):
    """All launch shapes (SPADEN_TILE_CFG), with and without the bank-conflict row
    rotations (SPADEN_ROT), give the oracle's y within tolerance and bitwise the
    same y: the long-row split is a constant and a rotation only reorders rows."""
    monkeypatch.setenv("SPADEN_ROT", rot)
    A = W.make("fem62k")
    x = W.vector(A.n, 17)
    monkeypatch.setenv("SPADEN_TILE_CFG", str(cfg))
    for storage, stored in (("fp32", A.values), ("fp16", oracle.f32_to_f16(A.values))):
        M = convert(sp, torch, A, storage=storage)
        y = gpu_spmv(torch, M, x)
        check_spmv(A, y, stored, x)
        monkeypatch.setenv("SPADEN_TILE_CFG", "3")
        monkeypatch.setenv("SPADEN_ROT", "0")
        y3 = gpu_spmv(torch, convert(sp, torch, A, storage=storage), x)
        monkeypatch.setenv("SPADEN_TILE_CFG", str(cfg))
        monkeypatch.setenv("SPADEN_ROT", rot)
        assert np.array_equal(y, y3)
    H = hub_matrix()
    M = convert(sp, torch, H)
    check_spmv(H, gpu_spmv(torch, M, W.vector(H.n, 3)), H.values, W.vector(H.n, 3))


@pytest.mark.parametrize("beta", [0.0, 0.5])
@pytest.mark.parametrize("slots", [None, 2, 8])
def test_spmv_host_batched(sp, torch, beta, slots, monkeypatch):
    if slots is not None:  # read when the handle first builds its pipeline
        monkeypatch.setenv("SPADEN_PIPE_SLOTS", str(slots))
    A = W.make("fem62k")
    M = convert(sp, torch, A)
    K = 11  # > 8 slots: every slot is reused
    X = torch.from_numpy(np.stack([W.vector(A.n, 40 + k) for k in range(K)])).pin_memory()
    Y0 = np.stack([W.vector(A.m, 60 + k) for k in range(K)])
    Y = torch.from_numpy(Y0.copy()).pin_memory()
    M.spmv_host_batched(X, Y, alpha=1.5, beta=beta)
    for k in range(K):
        yd = gpu_spmv(torch, M, X[k].numpy(), alpha=1.5, beta=beta, y0=Y0[k])
        assert np.array_equal(Y[k].numpy(), yd)


# ------------------------------------------------------------ hybrid (NEXT-1)
HYB_CASES = {"h1": W.h1, "tiny": lambda: W.tiny(0), "hub": lambda: hub_matrix(),
             # residual hub rows of ~100k entries: ~100 chunks, several per fix-up lane
             "bighub": lambda: hub_matrix(m=40, n=900_007, hub_rows=(0, 17, 33), hub_nnz=100_000, seed=3),
             "pl14": lambda: W.powerlaw(14, 5, seed=1), "fem": lambda: W.fem(6, 7, 8, seed=2)}


@pytest.mark.parametrize("name", sorted(HYB_CASES))
@pytest.mark.parametrize("t", [1, 2, 4])
@pytest.mark.parametrize("storage", ["fp32", "fp16"])
def test_hybrid_conversion_bit_exact(sp, torch, name, t, storage):
    A = HYB_CASES[name]()
    stored = A.values if storage == "fp32" else oracle.f32_to_f16(A.values)
    rp, ci, v = dev(torch, A)
    M = sp.convert(rp, ci, v, A.n, storage=storage, residual_max_popc=t)
    torch.cuda.synchronize()
    (krp, kci, kv), (rrp, rci, rv) = oracle.hybrid_split(A.m, A.n, A.rowptr, A.colidx, stored, t)
    st, B = oracle.csr_to_bitbsr(A.m, A.n, krp, kci, kv)
    h = host_arrays(torch, M)
    i = M.info
    ub = np.uint16 if storage == "fp16" else np.uint32
    assert i.residual_nnz == rci.size and i.Bnnz == B.Bnnz
    assert np.array_equal(h["blk_rowptr"].astype(np.int64), B.blk_rowptr)
    assert np.array_equal(h["blk_offset"].astype(np.int64), B.blk_offset)
    if B.Bnnz:
        assert np.array_equal(h["blk_col"], B.blk_col)
        assert np.array_equal(h["bitmap"].view(np.uint64), B.bitmap)
        assert np.array_equal(h["values"].view(ub), np.ascontiguousarray(B.values).view(ub))
    assert np.array_equal(h["res_rowptr"].astype(np.int64), rrp)
    assert np.array_equal(h["res_colidx"], rci)
    assert np.array_equal(h["res_values"].view(ub), np.ascontiguousarray(rv).view(ub))
    sv = 2 if storage == "fp16" else 4
    assert i.format_bytes == oracle.bitbsr_bytes(A.m, B.Bnnz, kci.size, sv) + 4 * (A.m + 1) + (4 + sv) * rci.size


@pytest.mark.parametrize("name", sorted(HYB_CASES))
def test_hybrid_spmv(sp, torch, name):
    A = HYB_CASES[name]()
    x = W.vector(A.n, 23)
    rp, ci, v = dev(torch, A)
    M = sp.convert(rp, ci, v, A.n, residual_max_popc=2)
    y1 = gpu_spmv(torch, M, x)
    assert np.array_equal(y1, gpu_spmv(torch, M, x))
    check_spmv(A, y1, A.values, x)
    y0 = W.vector(A.m, 24)
    y2 = gpu_spmv(torch, M, x, alpha=0.5, beta=2.0, y0=y0)
    ys, s = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    assert oracle.componentwise_error(y2, 0.5 * ys + 2.0 * y0, 0.5 * s + 2.0 * np.abs(y0)) <= TOL32
    if A.m >= 16:   # 8-row-aligned split gives identical y
        cut = (A.m // 16) * 8
        parts = []
        for r0, r1 in ((0, cut), (cut, A.m)):
            S = A.row_slice(r0, r1)
            r, c, vv = dev(torch, S)
            parts.append(gpu_spmv(torch, sp.convert(r, c, vv, S.n, residual_max_popc=2), x))
        assert np.array_equal(np.concatenate(parts), y1)


def binned_rows_matrix(seed=11):
    """Residual rows at every length-class boundary of the binned residual pass
    (1, 4 | 5, 8 | 9, 16 | 17, 32 | 33, 64 | 65 .. 4096 | > 4096 long rows) plus
    empty rows, in shuffled row order; with t = 64 every block is residual."""
    rng = np.random.default_rng(seed)
    lens = [0, 1, 2, 3, 4, 5, 7, 8, 9, 15, 16, 17, 31, 32, 33, 63, 64, 65, 100, 127, 128, 129, 1000, 4095, 4096,
            4097, 9000]
    lens = np.array(lens * 3)
    rng.shuffle(lens)
    n = 20_011
    rows, cols = [], []
    for r, k in enumerate(lens):
        c = np.sort(rng.choice(n, int(k), replace=False))
        rows.append(np.full(c.size, r))
        cols.append(c)
    rows, cols = np.concatenate(rows), np.concatenate(cols)
    return W.from_coo(lens.size, n, rows, cols, rng.uniform(-1, 1, rows.size))


@pytest.mark.parametrize("storage", ["fp32", "fp16"])
@pytest.mark.parametrize("t", [2, 64])
@pytest.mark.parametrize("fixup", ["fused", "separate"])
def test_residual_length_classes(sp, torch, storage, t, fixup, monkeypatch):
    """Binned residual pass: every length class and the long-row path against the
    oracle, bitwise deterministic, 8-row-partition invariant, and within tolerance
    of the fixed 16-lane residual kernel (SPADEN_RES=fixed)."""
    if fixup == "separate":  # long-row fix-up as its own launch (as with many chunks)
        monkeypatch.setenv("SPADEN_FUSED_FIXUP_MAX", "0")
    A = binned_rows_matrix()
    stored = A.values if storage == "fp32" else oracle.f32_to_f16(A.values)
    x = W.vector(A.n, 41)
    rp, ci, v = dev(torch, A)
    M = sp.convert(rp, ci, v, A.n, storage=storage, residual_max_popc=t)
    if t == 64:
        assert M.info.Bnnz == 0 and M.info.residual_nnz == A.nnz
    y = gpu_spmv(torch, M, x)
    assert np.array_equal(y, gpu_spmv(torch, M, x))
    check_spmv(A, y, stored, x)
    y0 = W.vector(A.m, 42)
    ys, s = oracle.spmv(A.rowptr, A.colidx, stored, x)
    y2 = gpu_spmv(torch, M, x, alpha=-0.75, beta=0.5, y0=y0)
    assert oracle.componentwise_error(y2, -0.75 * ys + 0.5 * y0, 0.75 * s + 0.5 * np.abs(y0)) <= TOL32
    cut = (A.m // 16) * 8
    parts = []
    for r0, r1 in ((0, cut), (cut, A.m)):
        S = A.row_slice(r0, r1)
        r, c, vv = dev(torch, S)
        parts.append(gpu_spmv(torch, sp.convert(r, c, vv, S.n, storage=storage, residual_max_popc=t), x))
    assert np.array_equal(np.concatenate(parts), y)
    monkeypatch.setenv("SPADEN_RES", "fixed")
    check_spmv(A, gpu_spmv(torch, M, x), stored, x)


@pytest.mark.parametrize("decode", ["slots", "bits", "mma"])
@pytest.mark.parametrize("name", ["fem62k_small", "hub", "tiny", "h2"])
def test_decode_ablations_fp16(sp, torch, decode, name, monkeypatch):
    """Every decode variant (SPADEN_DECODE) on fp16 storage, including the
    tensor-core ablation (mma.sync m16n8k16, x split into fp16 hi+lo)."""
    A = W.fem(9, 9, 10, seed=4) if name == "fem62k_small" else CASES[name]()
    monkeypatch.setenv("SPADEN_DECODE", decode)
    M = convert(sp, torch, A, storage="fp16")
    x = W.vector(A.n, 29)
    y = gpu_spmv(torch, M, x)
    check_spmv(A, y, oracle.f32_to_f16(A.values), x)


@pytest.mark.parametrize("decode", ["bits"])
@pytest.mark.parametrize("storage", ["fp32", "fp16"])
def test_decodes_bitwise_equal_to_slots(sp, torch, decode, storage, monkeypatch):
    """Every CUDA-core decode computes the same per-block row partials in the same
    order, so y is bitwise identical to the default decode."""
    A = W.fem(9, 9, 10, seed=5)
    x = W.vector(A.n, 31)
    monkeypatch.setenv("SPADEN_DECODE", "slots")
    M = convert(sp, torch, A, storage=storage)
    ref = gpu_spmv(torch, M, x)
    monkeypatch.setenv("SPADEN_DECODE", decode)
    assert np.array_equal(gpu_spmv(torch, M, x), ref)


def random_cases(count=24, seed=123):
    rng = np.random.default_rng(seed)
    for i in range(count):
        m = int(rng.choice([1, 2, 7, 8, 9, 63, 64, 65, 300, 1000, 4099]))
        n = int(rng.choice([1, 3, 8, 15, 64, 129, 1000, 5000, 70_001]))
        dens = float(rng.choice([0.001, 0.01, 0.05, 0.3, 1.0]))
        dens = min(dens, 200_000 / max(1, m * n))
        yield i, m, n, dens


@pytest.mark.parametrize("case", list(random_cases()), ids=lambda c: f"r{c[0]}_{c[1]}x{c[2]}")
def test_random_shapes_all_modes(sp, torch, case):
    """Randomised shapes (1xN, Nx1, ragged, dense, very sparse) through every
    storage mode and the hybrid split: conversion exact, SpMV within tolerance."""
    i, m, n, dens = case
    A = W.random_sparse(m, n, dens, seed=1000 + i)
    x = W.vector(n, 2000 + i)
    for storage in ("fp32", "fp16"):
        stored = A.values if storage == "fp32" else oracle.f32_to_f16(A.values)
        M = convert(sp, torch, A, storage=storage)
        assert_format_parity(torch, M, W.CSR(A.m, A.n, A.rowptr, A.colidx, stored), stored)
        check_spmv(A, gpu_spmv(torch, M, x), stored, x)
        rp, ci, v = dev(torch, A)
        H = sp.convert(rp, ci, v, n, storage=storage, residual_max_popc=int(1 + i % 4))
        check_spmv(A, gpu_spmv(torch, H, x), stored, x)


# ------------------------------------------------------------ SpMM (NEXT-4)
@pytest.mark.parametrize("k", [1, 2, 3, 4, 7, 8, 13])
@pytest.mark.parametrize("name", ["fem", "hub", "tiny", "h2"])
@pytest.mark.parametrize("storage", ["fp32", "fp16"])
def test_spmm_columns_equal_spmv(sp, torch, k, name, storage):
    """spaden_spmm: column j equals spaden_spmv on vector j bitwise, and the
    oracle within tolerance (fp32/fp16 values, long rows, ragged shapes)."""
    A = {"fem": lambda: W.fem(7, 8, 9, seed=6), "hub": hub_matrix, "tiny": lambda: W.tiny(2), "h2": W.h2}[name]()
    M = convert(sp, torch, A, storage=storage)
    X = torch.from_numpy(np.stack([W.vector(A.n, 300 + j) for j in range(k)])).cuda()
    Y0 = torch.from_numpy(np.stack([W.vector(A.m, 400 + j) for j in range(k)])).cuda()
    Y = M.spmm(X, Y0.clone(), alpha=0.75, beta=0.5)
    torch.cuda.synchronize()
    stored = A.values if storage == "fp32" else oracle.f32_to_f16(A.values)
    for j in range(k):
        yj = M.spmv(X[j].contiguous(), Y0[j].clone(), alpha=0.75, beta=0.5)
        torch.cuda.synchronize()
        assert torch.equal(Y[j], yj), j
        ys, s = oracle.spmv(A.rowptr, A.colidx, stored, X[j].cpu().numpy())
        y0 = Y0[j].cpu().numpy().astype(np.float64)
        assert oracle.componentwise_error(Y[j].cpu().numpy(), 0.75 * ys + 0.5 * y0, 0.75 * s + 0.5 * np.abs(y0)) <= TOL32


def test_spmm_hybrid(sp, torch):
    A = hub_matrix()
    rp, ci, v = dev(torch, A)
    M = sp.convert(rp, ci, v, A.n, residual_max_popc=2)
    X = torch.from_numpy(np.stack([W.vector(A.n, 500 + j) for j in range(4)])).cuda()
    Y = M.spmm(X)
    for j in range(4):
        assert torch.equal(Y[j], M.spmv(X[j].contiguous()))


@pytest.mark.parametrize("npeers", [1, 3, 8])
@pytest.mark.parametrize("name", ["fem", "hub", "tiny", "h2", "empty"])
@pytest.mark.parametrize("storage", ["fp32", "fp16"])
def test_spmv_scatter_virtual_peers(sp, torch, npeers, name, storage):
    """NEXT-2 fused SpMV + all-gather store: every destination buffer ("virtual
    peers" on one GPU) receives y at out_offset bitwise equal to spaden_spmv,
    nothing outside [offset, offset+m) is touched, and the local y is written
    too when given (alpha/beta honoured)."""
    A = {"fem": lambda: W.fem(7, 8, 9, seed=6), "hub": hub_matrix, "tiny": lambda: W.tiny(2), "h2": W.h2,
         "empty": lambda: W.from_coo(17, 5, [], [], [])}[name]()
    M = convert(sp, torch, A, storage=storage)
    x = torch.from_numpy(W.vector(A.n, 61)).cuda()
    y0 = torch.from_numpy(W.vector(A.m, 62)).cuda()
    off = 13
    total = A.m + off + 29
    bufs = [torch.full((total,), float(p) - 7.0, device="cuda") for p in range(npeers)]
    y = y0.clone()
    M.spmv_scatter(x, [b.data_ptr() for b in bufs], off, y=y, alpha=0.75, beta=0.5)
    ref = M.spmv(x, y0.clone(), alpha=0.75, beta=0.5)
    torch.cuda.synchronize()
    assert torch.equal(y, ref)
    for p, b in enumerate(bufs):
        assert torch.equal(b[off:off + A.m], ref), p
        assert bool((b[:off] == float(p) - 7.0).all()) and bool((b[off + A.m:] == float(p) - 7.0).all())
    # beta == 0 without a local y: peers only
    bufs2 = [torch.zeros(total, device="cuda") for _ in range(npeers)]
    M.spmv_scatter(x, [b.data_ptr() for b in bufs2], off)
    torch.cuda.synchronize()
    ref0 = M.spmv(x)
    for b in bufs2:
        assert torch.equal(b[off:off + A.m], ref0)


def test_spmv_scatter_rejects(sp, torch):
    A = W.tiny(1)
    M = convert(sp, torch, A)
    x = torch.from_numpy(W.vector(A.n, 1)).cuda()
    b = torch.zeros(A.m, device="cuda")
    with pytest.raises(sp.SpadenError):
        M.spmv_scatter(x, [b.data_ptr()] * 9, 0)
    with pytest.raises(sp.SpadenError):
        M.spmv_scatter(x, [b.data_ptr()], 0, beta=0.5)          # beta != 0 needs y
    H = hub_matrix()
    rp, ci, v = dev(torch, H)
    Mh = sp.convert(rp, ci, v, H.n, residual_max_popc=2)
    bh = torch.zeros(H.m, device="cuda")
    with pytest.raises(sp.SpadenError):                          # hybrid: unsupported
        Mh.spmv_scatter(torch.from_numpy(W.vector(H.n, 1)).cuda(), [bh.data_ptr()], 0)


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_fused_iterated_spmv_emulated_ranks(sp, torch, world):
    """dist.FusedIteratedSpMV with `world` ranks emulated on one GPU (peer views =
    plain device buffers, stepped rank by rank): after every PageRank-style step
    each rank's x is bitwise equal to the unfused single-rank IteratedSpMV."""
    from paper_conf_icpp_cheny24_b200 import dist
    src, dst = W.rmat_edges(12, 8, seed=5, relabel=True)
    A = W.pagerank_matrix(1 << 12, src, dst)
    x0 = torch.full((A.n,), 1.0 / A.n, device="cuda")
    alpha, c = 0.85, 0.15 / A.n
    full = convert(sp, torch, A)
    ref = dist.IteratedSpMV(dist.RowPartition(A.m, 1), A.n,
                            lambda x, y, a, b: full.spmv(x, y, alpha=a, beta=b), x0, 0)
    part = dist.RowPartition(A.m, world)
    L = max(part.padded, A.n)
    bufs = ([torch.zeros(L, device="cuda") for _ in range(world)],
            [torch.zeros(L, device="cuda") for _ in range(world)])
    ranks = []
    for r in range(world):
        r0, r1 = part.range(r)
        M = convert(sp, torch, A.row_slice(r0, r1))
        ranks.append(dist.FusedIteratedSpMV(part, A.n, M, x0, r, buffers=(*bufs, lambda: None)))
    for _ in range(6):
        xr = ref.step(alpha, c)
        for rk in ranks:
            rk.step(alpha, c)
        torch.cuda.synchronize()
        for rk in ranks:
            assert torch.equal(rk.x[: A.n], xr[: A.n])


@pytest.mark.parametrize("storage", ["fp32", "fp16"])
def test_x_texture_path_bitwise_equal_to_ldg(sp, torch, storage, monkeypatch):
    """x fetched through the texture pipe (default) and through LDG (SPADEN_XTEX=0)
    give bitwise identical y, for SpMV and SpMM, aligned and unaligned x."""
    A = W.fem(7, 8, 9, seed=6)
    M = convert(sp, torch, A, storage=storage)
    xb = torch.from_numpy(W.vector(A.n + 1, 71)).cuda()
    X = torch.from_numpy(np.stack([W.vector(A.n, 80 + j) for j in range(4)])).cuda()
    outs = {}
    for mode in ("1", "0"):
        monkeypatch.setenv("SPADEN_XTEX", mode)
        outs[mode] = (M.spmv(xb[:A.n]), M.spmv(xb[1:].contiguous()), M.spmv(xb[1:]), M.spmm(X))
        torch.cuda.synchronize()
    for a, b in zip(outs["1"], outs["0"]):
        assert torch.equal(a, b)


# ---------------------------------------------------------------- round 2
def mid_cost_matrix(nbr, seed, lo_blocks=120, hi_blocks=175, fill=(6, 12), short_frac=0.3):
    """Block-rows whose stage cost (52 B per block + values) straddles the long-row
    threshold (kLongRowBytes = 9 KB) -- the regime where the round-1 cutoff
    (half a stage) depended on the tile config, i.e. on the slice size -- plus a
    share of short block-rows.  nbr block-rows of 8 rows, n = 64k columns."""
    rng = np.random.default_rng(seed)
    n = 1 << 16
    short = rng.random(nbr) < short_frac
    nbs = np.where(short, rng.integers(10, 40, nbr), rng.integers(lo_blocks, hi_blocks, nbr))
    br_of = np.repeat(np.arange(nbr), nbs)
    bc = np.concatenate([np.sort(rng.choice(n // 8, k, replace=False)) for k in nbs])
    p = rng.uniform(fill[0] / 64, fill[1] / 64, bc.size)
    bits = rng.random((bc.size, 64)) < p[:, None]
    bits[:, 0] |= ~bits.any(1)                       # no empty block
    blk, bit = np.nonzero(bits)
    r = (8 * br_of[blk] + bit // 8).astype(np.int64)
    c = (8 * bc[blk] + bit % 8).astype(np.int64)
    v = rng.standard_normal(r.size).astype(np.float32)
    return W.from_coo(8 * nbr, n, r, c, v)


@pytest.mark.slow
@pytest.mark.parametrize("storage", ["fp32", "fp16"])
def test_partition_invariance_across_tile_config_switch(sp, torch, storage):
    """A > 64 MB matrix (large-matrix tile config) cut into 8-row-aligned slices
    below 64 MB (small-matrix config, smaller stages) gives bitwise the same y:
    the tile/long-row split is one constant (kLongRowBytes), not half a stage.
    Also against the fp64 oracle on the stored values."""
    nbr = 12500 if storage == "fp32" else 19000
    A = mid_cost_matrix(nbr, seed=11)
    vals = A.values if storage == "fp32" else oracle.f32_to_f16(A.values)
    M = convert(sp, torch, A, storage=storage)
    assert M.info.format_bytes > 64 << 20 and M.info.n_long > 0
    x = W.vector(A.n, 5)
    y = gpu_spmv(torch, M, x)
    check_spmv(A, y, vals, x)
    M.free()
    bounds = [0, 8 * (nbr // 4), 8 * (nbr // 2 + 7), 8 * (3 * nbr // 4), A.m]
    parts = []
    for r0, r1 in zip(bounds[:-1], bounds[1:]):
        S = A.row_slice(r0, r1)
        Ms = convert(sp, torch, S, storage=storage)
        assert Ms.info.format_bytes < 64 << 20
        parts.append(gpu_spmv(torch, Ms, x))
        Ms.free()
    assert np.array_equal(np.concatenate(parts).view(np.uint32), y.view(np.uint32))


def test_auto_hybrid_takes_the_whole_matrix_fill(sp, torch):
    """residual_max_popc = -1 on row slices: with auto_mean_fill = the whole
    matrix's fill (count_blocks summed over the slices), every slice takes the
    same t as the whole matrix, so the concatenated y is bitwise the whole-matrix
    y even though one slice alone would have chosen differently."""
    F = W.fem(8, 8, 8, seed=3)                       # fill ~20: alone -> pure bitBSR
    P = W.powerlaw(14, 5, seed=2)                    # fill ~1:  alone -> t = 4
    m = F.m + P.m
    m8 = -(-F.m // 8) * 8
    rows = np.concatenate([np.repeat(np.arange(F.m), np.diff(F.rowptr)),
                           m8 + np.repeat(np.arange(P.m), np.diff(P.rowptr))])
    n = max(F.n, P.n)
    A = W.from_coo(m8 + P.m, n, rows, np.concatenate([F.colidx, P.colidx]),
                   np.concatenate([F.values, P.values]))
    rp, ci, v = dev(torch, A)
    whole = sp.convert(rp, ci, v, A.n, residual_max_popc=-1)
    t_whole = whole.info.residual_max_popc
    x = W.vector(A.n, 9)
    y = gpu_spmv(torch, whole, x)
    check_spmv(A, y, A.values, x)
    slices = [A.row_slice(0, m8), A.row_slice(m8, A.m)]
    devs = [dev(torch, S) for S in slices]
    bnnz = sum(sp.count_blocks(r, c, A.n) for r, c, _ in devs)
    fill = A.nnz / bnnz
    own = [sp.convert(r, c, vv, A.n, residual_max_popc=-1).info.residual_max_popc for r, c, vv in devs]
    assert len(set(own)) == 2, own                   # the slices alone disagree
    parts = []
    for (r, c, vv) in devs:
        Ms = sp.convert(r, c, vv, A.n, residual_max_popc=-1, auto_mean_fill=fill)
        assert Ms.info.residual_max_popc == t_whole
        parts.append(gpu_spmv(torch, Ms, x))
    assert np.array_equal(np.concatenate(parts).view(np.uint32), y.view(np.uint32))


@pytest.mark.parametrize("name", ["fem62k", "tiny", "hub", "rand_rect", "empty_middle_last"])
def test_count_blocks_matches_oracle(sp, torch, name):
    A = W.make(name) if name == "fem62k" else CASES[name]()
    st, B = oracle.csr_to_bitbsr(A.m, A.n, A.rowptr, A.colidx, A.values)
    r, c, _ = dev(torch, A)
    assert sp.count_blocks(r, c, A.n) == B.Bnnz


def test_count_blocks_rejects_bad_csr(sp, torch):
    A = W.from_coo(16, 16, [0, 0], [3, 2], [1.0, 2.0])   # row 0 columns 3, 2 (built sorted)
    r, c, _ = dev(torch, A)
    c2 = c.clone()
    c2[0], c2[1] = c[1], c[0]                             # unsorted
    with pytest.raises(sp.SpadenError):
        sp.count_blocks(r, c2, A.n)


@pytest.mark.parametrize("npeers", [1, 3])
@pytest.mark.parametrize("name", ["fem", "hub", "empty_rows"])
def test_spmv_scatter_vs_oracle(sp, torch, npeers, name):
    """NEXT-2 peer-store epilogue against the fp64 oracle (not against the CUDA
    SpMV): every destination buffer holds alpha*A x + beta*y0 within the fp32
    tolerance, including rows of empty block-rows (beta*y0 exactly)."""
    A = {"fem": lambda: W.fem(7, 8, 9, seed=6), "hub": hub_matrix,
         "empty_rows": lambda: W.from_coo(90, 70, [0, 41, 89], [5, 69, 0], [1.5, -2.0, 3.0])}[name]()
    M = convert(sp, torch, A)
    xn = W.vector(A.n, 61)
    y0n = W.vector(A.m, 62)
    x = torch.from_numpy(xn).cuda()
    off = 5
    bufs = [torch.full((A.m + off + 3,), 99.0, device="cuda") for _ in range(npeers)]
    y = torch.from_numpy(y0n).cuda()
    M.spmv_scatter(x, [b.data_ptr() for b in bufs], off, y=y, alpha=0.75, beta=0.5)
    torch.cuda.synchronize()
    ys, s = oracle.spmv(A.rowptr, A.colidx, A.values, xn)
    ref = 0.75 * ys + 0.5 * y0n.astype(np.float64)
    sc = 0.75 * s + 0.5 * np.abs(y0n.astype(np.float64))
    for b in bufs:
        got = b[off:off + A.m].cpu().numpy()
        assert oracle.componentwise_error(got, ref, sc) <= TOL32
        assert bool((b[:off] == 99.0).all()) and bool((b[off + A.m:] == 99.0).all())


@pytest.mark.parametrize("world", [2, 3, 8])
def test_fused_iterated_spmv_vs_oracle_pagerank(sp, torch, world):
    """dist.FusedIteratedSpMV (NEXT-2, ranks emulated on one GPU) against the
    fp64 PageRank iteration of the oracle: every rank's x after K steps within
    1e-5 componentwise (all-positive iterates: relative error)."""
    from paper_conf_icpp_cheny24_b200 import dist
    src, dst = W.rmat_edges(12, 8, seed=5, relabel=True)
    A = W.pagerank_matrix(1 << 12, src, dst)
    K = 8
    x0 = torch.full((A.n,), 1.0 / A.n, device="cuda")
    part = dist.RowPartition(A.m, world)
    L = max(part.padded, A.n)
    bufs = ([torch.zeros(L, device="cuda") for _ in range(world)],
            [torch.zeros(L, device="cuda") for _ in range(world)])
    ranks = []
    for r in range(world):
        r0, r1 = part.range(r)
        ranks.append(dist.FusedIteratedSpMV(part, A.n, convert(sp, torch, A.row_slice(r0, r1)), x0, r,
                                            buffers=(*bufs, lambda: None)))
    for _ in range(K):
        for rk in ranks:
            rk.step(0.85, 0.15 / A.n)
    torch.cuda.synchronize()
    ref = oracle.pagerank(A.rowptr, A.colidx, A.values, 0.85, K, np.full(A.n, 1.0 / A.n))
    for rk in ranks:
        got = rk.x[: A.n].cpu().numpy().astype(np.float64)
        assert (np.abs(got - ref) / np.abs(ref)).max() <= TOL32


def test_concurrent_spmv_on_two_streams(sp, torch):
    """One handle with long block-rows (per-call scratch) driven from two streams
    at once: every result is bitwise the single-stream result (scratch sets are
    taken round robin per call)."""
    A = mid_cost_matrix(300, seed=4, lo_blocks=250, hi_blocks=400)
    M = convert(sp, torch, A)
    assert M.info.n_long > 0
    xs = [torch.from_numpy(W.vector(A.n, 100 + j)).cuda() for j in range(2)]
    refs = [M.spmv(x) for x in xs]
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream() for _ in range(2)]
    outs = [[torch.empty(A.m, device="cuda") for _ in range(20)] for _ in range(2)]
    for k in range(20):
        for j in range(2):
            M.spmv(xs[j], outs[j][k], stream=streams[j])
    torch.cuda.synchronize()
    for j in range(2):
        for o in outs[j]:
            assert torch.equal(o, refs[j])


def test_hybrid_empty_residual_chained_calls(sp, torch):
    """A hybrid handle whose residual is empty (every block holds > t entries)
    with beta = 1: the call launches no residual kernel, so the bitBSR kernels
    must not be programmatic-dependent launches; two chained calls y1 = A x,
    y2 = A y1 + y2 see the finished y1."""
    A = W.dense_block(72, 72, 2)                     # every block holds > 1 entry
    rp, ci, v = dev(torch, A)
    M = sp.convert(rp, ci, v, A.n, residual_max_popc=1)
    assert M.info.residual_max_popc == 1 and M.info.residual_nnz == 0
    x = torch.from_numpy(W.vector(A.n, 3)).cuda()
    y2_0 = torch.from_numpy(W.vector(A.m, 4)).cuda()
    for _ in range(5):
        y1 = M.spmv(x)
        y2 = y2_0.clone()
        M.spmv(y1, y2, beta=1.0)
        torch.cuda.synchronize()
        h1 = y1.cpu().numpy()
        ys, s = oracle.spmv(A.rowptr, A.colidx, A.values, h1)
        ref = ys + y2_0.cpu().numpy().astype(np.float64)
        assert oracle.componentwise_error(y2.cpu().numpy(), ref, s + np.abs(y2_0.cpu().numpy())) <= TOL32


# ------------------------------------------------- NEXT-4 tensor-core SpMM
def _spmm_tc_case(name):
    return {"fem": lambda: W.fem(7, 8, 9, seed=6), "hub": hub_matrix, "tiny": lambda: W.tiny(2),
            "h2": W.h2, "ragged": lambda: W.random_sparse(333, 517, 0.02, 5),
            "empty_rows": lambda: W.from_coo(90, 70, [0, 41, 89], [5, 69, 0], [1.5, -2.0, 3.0]),
            "dense64": lambda: W.dense_block(64, 64, 2)}[name]()


@pytest.mark.parametrize("k", [1, 64, 128, 200])
@pytest.mark.parametrize("name", ["fem", "hub", "tiny", "h2", "ragged", "empty_rows", "dense64"])
def test_spmm_tc_vs_oracle(sp, torch, name, k):
    """tcgen05 SpMM (UTCHMMA, TMEM accumulators) against the fp64 oracle on the
    stored fp16 values and fp16-rounded x (the paper's tensor-core input
    precision): every column componentwise <= 1e-5, alpha/beta honoured,
    rows of empty block-rows = beta*y."""
    A = _spmm_tc_case(name)
    M = convert(sp, torch, A, storage="fp16")
    rng = np.random.default_rng(k)
    X = rng.uniform(-1, 1, (k, A.n)).astype(np.float32)
    Y0 = rng.uniform(-1, 1, (k, A.m)).astype(np.float32)
    Xd = torch.from_numpy(X).cuda()
    Xb = M.pack_x_tc(Xd)
    Yd = torch.from_numpy(Y0).cuda()
    M.spmm_tc(Xb, k, Yd, alpha=0.5, beta=0.25)
    torch.cuda.synchronize()
    Y = Yd.cpu().numpy()
    vals = oracle.f32_to_f16(A.values)
    for j in range(k):
        xr = oracle.f32_to_f16(X[j]).astype(np.float64)
        ys, s = oracle.spmv(A.rowptr, A.colidx, vals, xr)
        ref = 0.5 * ys + 0.25 * Y0[j].astype(np.float64)
        sc = 0.5 * s + 0.25 * np.abs(Y0[j].astype(np.float64))
        err = oracle.componentwise_error(Y[j], ref, sc)
        assert err <= TOL32, (j, err)


def test_spmm_tc_deterministic_and_rejects(sp, torch):
    A = W.fem(6, 7, 8, seed=2)
    M = convert(sp, torch, A, storage="fp16")
    X = torch.from_numpy(np.random.default_rng(1).uniform(-1, 1, (96, A.n)).astype(np.float32)).cuda()
    Xb = M.pack_x_tc(X)
    y1 = M.spmm_tc(Xb, 96)
    y2 = M.spmm_tc(Xb, 96)
    torch.cuda.synchronize()
    assert torch.equal(y1, y2)
    M32 = convert(sp, torch, A, storage="fp32")
    with pytest.raises(sp.SpadenError):
        M32.spmm_tc(Xb, 96)
