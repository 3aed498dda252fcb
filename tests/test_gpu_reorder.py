"""Reordering before conversion through the C ABI:
spaden_degree_order and spaden_permute_csr bit-exact against the oracle's
definitions (oracle.degree_order / oracle.permute_csr), and SpMV on the reordered
matrix equal to the permuted oracle product within the usual tolerance."""
import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

TOL32 = 1e-5


@pytest.fixture(scope="module")
def sp():
    import paper_conf_icpp_cheny24_b200 as sp
    return sp


@pytest.fixture(scope="module")
def torch():
    import torch
    assert torch.cuda.is_available()
    return torch


def to_dev(torch, *arrays):
    return tuple(torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in arrays)


def matrices():
    yield "random", W.random_sparse(300, 300, 0.02, 1)
    yield "powerlaw12", W.powerlaw(12, 5, 0)
    yield "powerlaw12_relabel", W.powerlaw(12, 5, 1, relabel=True)
    eye = W.from_dense(np.eye(65, dtype=np.float32))
    yield "identity", eye
    yield "one", W.from_dense(np.ones((1, 1), np.float32))
    A = W.random_sparse(200, 200, 0.05, 3)
    rp = A.rowptr.copy()
    keep = np.ones(A.nnz, bool)
    for i in range(0, 200, 7):  # empty rows
        keep[rp[i]:rp[i + 1]] = False
    rows = np.repeat(np.arange(200), np.diff(rp))[keep]
    yield "empty_rows", W.from_coo(200, 200, rows, A.colidx[keep], A.values[keep])


@pytest.mark.parametrize("name,A", list(matrices()), ids=[n for n, _ in matrices()])
def test_degree_order_and_permute_bit_exact(sp, torch, name, A):
    rp, ci, v = to_dev(torch, A.rowptr, A.colidx, A.values)
    perm = sp.degree_order(rp)
    torch.cuda.synchronize()
    ref = oracle.degree_order(A.rowptr)
    assert np.array_equal(perm.cpu().numpy(), ref)
    for p in (ref, W.random_perm(A.m, 5).astype(np.int32)):
        (pd,) = to_dev(torch, p.astype(np.int32))
        brp, bci, bv = sp.permute_csr(rp, ci, v, pd)
        torch.cuda.synchronize()
        orp, oci, ov = oracle.permute_csr(A.rowptr, A.colidx, A.values, p)
        assert np.array_equal(brp.cpu().numpy(), orp)
        assert np.array_equal(bci.cpu().numpy(), oci)
        assert np.array_equal(bv.cpu().numpy().view(np.uint32), ov.view(np.uint32))


def test_permute_fp16_raw_bits(sp, torch):
    A = W.powerlaw(12, 5, 2, relabel=True)
    v16 = W.vector(A.nnz, 4).astype(np.float16)
    rp, ci, v = to_dev(torch, A.rowptr, A.colidx, v16)
    perm = sp.degree_order(rp)
    brp, bci, bv = sp.permute_csr(rp, ci, v, perm)
    torch.cuda.synchronize()
    orp, oci, ov = oracle.permute_csr(A.rowptr, A.colidx, v16, perm.cpu().numpy())
    assert np.array_equal(bci.cpu().numpy(), oci)
    assert np.array_equal(bv.cpu().numpy().view(np.uint16), ov.view(np.uint16))


@pytest.mark.parametrize("hybrid", [0, -1])
def test_spmv_on_reordered_matrix(sp, torch, hybrid):
    """y' = B x' with B = P A P^T, x' = P x equals P (A x) (componentwise 1e-5
    against the fp64 oracle on A)."""
    A = W.powerlaw(14, 5, 3, relabel=True)
    x = W.vector(A.n, 2)
    rp, ci, v = to_dev(torch, A.rowptr, A.colidx, A.values)
    perm = sp.degree_order(rp)
    brp, bci, bv = sp.permute_csr(rp, ci, v, perm)
    M = sp.convert(brp, bci, bv, A.n, residual_max_popc=hybrid)
    p = perm.cpu().numpy()
    (xd,) = to_dev(torch, x[p])
    y = torch.zeros(A.m, dtype=torch.float32, device="cuda")
    M.spmv(xd, y)
    torch.cuda.synchronize()
    ys, s = oracle.spmv(A.rowptr, A.colidx, A.values, x)
    err = oracle.componentwise_error(y.cpu().numpy(), ys[p], s[p])
    assert err <= TOL32
    M.free()


def test_reorder_raises_block_fill(sp, torch):
    """Degree ordering concentrates a relabelled power-law matrix's hubs: the
    block count drops (more nonzeros per 8x8 block)."""
    A = W.powerlaw(14, 5, 1, relabel=True)
    rp, ci, v = to_dev(torch, A.rowptr, A.colidx, A.values)
    perm = sp.degree_order(rp)
    brp, bci, bv = sp.permute_csr(rp, ci, v, perm)
    assert sp.count_blocks(brp, bci, A.n) < sp.count_blocks(rp, ci, A.n)


def test_permute_rejects_out_of_range(sp, torch):
    A = W.random_sparse(50, 50, 0.1, 1)
    ci_bad = A.colidx.copy()
    ci_bad[3] = 50
    rp, ci, v = to_dev(torch, A.rowptr, ci_bad, A.values)
    perm = torch.arange(50, dtype=torch.int32, device="cuda")
    with pytest.raises(sp.SpadenError) as ei:
        sp.permute_csr(rp, ci, v, perm)
    assert ei.value.status == 2  # SPADEN_ERR_INDEX_OUT_OF_RANGE


def test_empty_matrix(sp, torch):
    rp = torch.zeros(1, dtype=torch.int32, device="cuda")
    perm = sp.degree_order(rp)
    assert perm.numel() == 0
    brp, bci, bv = sp.permute_csr(rp, torch.zeros(0, dtype=torch.int32, device="cuda"),
                                  torch.zeros(0, dtype=torch.float32, device="cuda"), perm)
    torch.cuda.synchronize()
    assert brp.cpu().tolist() == [0]


def test_rmat25_reordered_hybrid_sampled(sp, torch):
    """The bench's `--workload rmat25 --reorder degree` path at full size (1.05B
    nnz): degree order and P A P^T on the GPU, automatic hybrid; the permutation is
    checked against the oracle's definition on the row degrees, and y' = B (P x)
    on 4096 sampled rows (incl. the hubs) against the fp64 oracle's P (A x) rows."""
    rp, ci, v, n, nnz = W.pagerank_slice_torch(25, 32, 0, 1 << 25, seed=0, device="cuda")
    perm = sp.degree_order(rp)
    torch.cuda.synchronize()
    rph = rp.cpu().numpy().astype(np.int64)
    assert np.array_equal(perm.cpu().numpy(), oracle.degree_order(rph))
    brp, bci, bv = sp.permute_csr(rp, ci, v, perm)
    M = sp.convert(brp, bci, bv, n, residual_max_popc=-1)
    torch.cuda.synchronize()
    assert M.info.nnz == nnz
    g = torch.Generator(device="cuda")
    g.manual_seed(7)
    x = torch.rand(n, generator=g, device="cuda")
    xp = x[perm.long()].contiguous()
    y = M.spmv(xp)
    torch.cuda.synchronize()
    p = perm.cpu().numpy()
    lens = np.diff(rph)
    rng = np.random.default_rng(5)
    krows = np.unique(np.concatenate([rng.choice(n, 4064, replace=False), np.arange(32)]))  # B's first rows = hubs
    orig = p[krows]  # row k of B is row perm[k] of A
    sub_rp = np.zeros(orig.size + 1, np.int64)
    sub_rp[1:] = np.cumsum(lens[orig])
    idx = torch.from_numpy(np.concatenate([np.arange(rph[r], rph[r + 1]) for r in orig])).cuda()
    ys, s = oracle.spmv(sub_rp, ci[idx].cpu().numpy(), v[idx].cpu().numpy(), x.cpu().numpy())
    err = oracle.componentwise_error(y[torch.from_numpy(krows).cuda()].cpu().numpy(), ys, s)
    assert err <= TOL32, err
    M.free()


@pytest.mark.parametrize("kind", ["range", "duplicate"])
def test_permute_rejects_bad_permutation(sp, torch, kind):
    A = W.random_sparse(40, 40, 0.1, 2)
    rp, ci, v = to_dev(torch, A.rowptr, A.colidx, A.values)
    p = np.arange(40, dtype=np.int32)
    if kind == "range":
        p[7] = 40
    else:
        p[7] = 3  # 3 twice, 7 missing
    (pd,) = to_dev(torch, p)
    with pytest.raises(sp.SpadenError) as ei:
        sp.permute_csr(rp, ci, v, pd)
    assert ei.value.status == 1  # SPADEN_ERR_INVALID_ARGUMENT
