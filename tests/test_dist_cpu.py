"""World-size-2 gloo tests (CPU) of the row-partitioned multi-GPU host logic
(paper_conf_icpp_cheny24_b200/dist.py): partition, per-rank slices, the
all-gather that rebuilds x, and the iterated (PageRank-style) SpMV.  The local
SpMV is the oracle here (no GPU); on GPUs it is the CUDA path."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import workloads as W


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def oracle_local_spmv(S):
    def f(x, y, alpha, beta):
        ys, _ = oracle.spmv(S.rowptr, S.colidx, S.values, x.numpy())
        out = alpha * ys + (beta * y.numpy().astype(np.float64) if beta != 0 else 0.0)
        y.copy_(torch.from_numpy(out.astype(np.float32)))
    return f


def _worker(rank, world, port, case, out_dir):
    from paper_conf_icpp_cheny24_b200.dist import IteratedSpMV, RowPartition
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        if case == "pagerank":
            src, dst = W.rmat_edges(9, 8, seed=5, relabel=True)
            A = W.pagerank_matrix(512, src, dst)
            x0 = torch.full((A.n,), 1.0 / A.n)
            alpha, c, K = 0.85, 0.15 / A.n, 15
        else:
            A = W.fem(5, 6, 7, seed=3)
            x0 = torch.from_numpy(W.vector(A.n, 4))
            csum = np.concatenate([[0.0], np.cumsum(np.abs(A.values.astype(np.float64)))])
            alpha, c, K = float(1.0 / (csum[A.rowptr[1:]] - csum[A.rowptr[:-1]]).max()), None, 6
        part = RowPartition(A.m, world)
        r0, r1 = part.range(rank)
        it = IteratedSpMV(part, A.n, oracle_local_spmv(A.row_slice(r0, r1)), x0, rank)
        for _ in range(K):
            x = it.step(alpha, c)
        np.save(os.path.join(out_dir, f"{case}_{rank}.npy"), x[: A.n].numpy())
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case", ["fem", "pagerank"])
def test_two_rank_iterated_spmv_matches_single_rank(tmp_path, case):
    mp.spawn(_worker, args=(2, free_port(), case, str(tmp_path)), nprocs=2, join=True)
    x0 = np.load(tmp_path / f"{case}_0.npy")
    x1 = np.load(tmp_path / f"{case}_1.npy")
    assert np.array_equal(x0, x1)                       # every rank holds the same x
    # single-process reference with the same per-row arithmetic
    from paper_conf_icpp_cheny24_b200.dist import RowPartition
    if case == "pagerank":
        src, dst = W.rmat_edges(9, 8, seed=5, relabel=True)
        A = W.pagerank_matrix(512, src, dst)
        x = np.full(A.n, 1.0 / A.n, np.float32)
        for _ in range(15):
            ys, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x)
            x = (0.85 * ys + np.float32(0.15 / A.n).astype(np.float64)).astype(np.float32)
        ref = oracle.pagerank(A.rowptr, A.colidx, A.values, 0.85, 15, np.full(A.n, 1.0 / A.n))
        assert np.abs(x0 - ref).max() <= 1e-6 * ref.max()
    else:
        A = W.fem(5, 6, 7, seed=3)
        csum = np.concatenate([[0.0], np.cumsum(np.abs(A.values.astype(np.float64)))])
        alpha = float(1.0 / (csum[A.rowptr[1:]] - csum[A.rowptr[:-1]]).max())
        x = W.vector(A.n, 4)
        for _ in range(6):
            ys, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x)
            x = (alpha * ys).astype(np.float32)
    assert np.array_equal(x0, x)


def test_partition_shapes():
    from paper_conf_icpp_cheny24_b200.dist import RowPartition
    for m in (0, 1, 7, 8, 9, 1000, 1_497_600):
        for P in (1, 2, 4, 8):
            p = RowPartition(m, P)
            assert p.slice_rows % 8 == 0 and p.padded >= m
            rs = [p.range(r) for r in range(P)]
            assert rs[0][0] == 0 and rs[-1][1] == m
            assert all(a[1] == b[0] for a, b in zip(rs[:-1], rs[1:]))


def test_single_process_without_process_group():
    """N=1 (no torch.distributed init): the driver degenerates to a local copy."""
    from paper_conf_icpp_cheny24_b200.dist import IteratedSpMV, RowPartition
    A = W.fem(4, 4, 5, seed=1)
    x0 = torch.from_numpy(W.vector(A.n, 3))
    it = IteratedSpMV(RowPartition(A.m, 1), A.n, oracle_local_spmv(A), x0, 0)
    x = it.step(0.01)
    ys, _ = oracle.spmv(A.rowptr, A.colidx, A.values, x0.numpy())
    assert np.array_equal(x[: A.n].numpy(), (0.01 * ys).astype(np.float32))


class _HostScatterSlice:
    """CPU stand-in for Matrix.spmv_scatter: the oracle computes the slice, the
    result is stored through raw host addresses like the kernel's peer stores."""

    def __init__(self, S):
        self.S = S

    def spmv_scatter(self, x, out_ptrs, out_offset, y=None, alpha=1.0, beta=0.0):
        import ctypes
        ys, _ = oracle.spmv(self.S.rowptr, self.S.colidx, self.S.values, x.numpy())
        out = alpha * ys + (beta * y.numpy().astype(np.float64) if beta != 0 else 0.0)
        out = np.ascontiguousarray(out.astype(np.float32))
        for p in out_ptrs:
            ctypes.memmove(p + 4 * out_offset, out.ctypes.data, out.nbytes)
        if y is not None:
            y.copy_(torch.from_numpy(out))


@pytest.mark.parametrize("world", [1, 2, 3, 5])
def test_fused_iterated_host_logic(world):
    """FusedIteratedSpMV's offsets, ping-pong and peer list (ranks emulated in one
    process, stepped in turn) reproduce the unfused single-rank iteration."""
    from paper_conf_icpp_cheny24_b200.dist import FusedIteratedSpMV, IteratedSpMV, RowPartition
    src, dst = W.rmat_edges(9, 8, seed=5, relabel=True)
    A = W.pagerank_matrix(512, src, dst)
    x0 = torch.full((A.n,), 1.0 / A.n)
    ref = IteratedSpMV(RowPartition(A.m, 1), A.n, oracle_local_spmv(A), x0, 0)
    part = RowPartition(A.m, world)
    L = max(part.padded, A.n)
    bufs = ([torch.zeros(L) for _ in range(world)], [torch.zeros(L) for _ in range(world)])
    ranks = [FusedIteratedSpMV(part, A.n, _HostScatterSlice(A.row_slice(*part.range(r))), x0, r,
                               buffers=(*bufs, lambda: None)) for r in range(world)]
    for _ in range(5):
        xr = ref.step(0.85, 0.15 / A.n)
        for rk in ranks:
            rk.step(0.85, 0.15 / A.n)
        for rk in ranks:
            assert torch.equal(rk.x[: A.n], xr[: A.n])
