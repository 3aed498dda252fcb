"""Real process groups on GPUs: NCCL all-gather and the
torch symmetric-memory peer buffers of dist.FusedIteratedSpMV, checked against
the fp64 oracle and against the single-rank CUDA result (bitwise: y is partition
invariant).  The one-rank case runs everywhere (it executes the symmetric-memory
rendezvous, peer view and device barrier on one GPU); the two-rank case needs
two visible GPUs and is skipped otherwise."""
import os
import socket

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

ALPHA, K_STEPS = 0.85, 8


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _matrix():
    src, dst = W.rmat_edges(13, 8, seed=7, relabel=True)
    return W.pagerank_matrix(1 << 13, src, dst)


def _worker(rank, world, port, out_dir, modes):
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_cheny24_b200 as sp
    from paper_conf_icpp_cheny24_b200 import dist as D

    torch.cuda.set_device(rank)
    dev = torch.device("cuda", rank)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world,
                            device_id=dev)
    try:
        A = _matrix()
        part = D.RowPartition(A.m, world)
        r0, r1 = part.range(rank)
        S = A.row_slice(r0, r1)
        M = D.convert_slice(torch.from_numpy(S.rowptr).to(dev), torch.from_numpy(S.colidx).to(dev),
                            torch.from_numpy(S.values).to(dev), A.n)
        x0 = torch.full((A.n,), 1.0 / A.n, device=dev)
        c = 0.15 / A.n
        for mode in modes:
            if mode == "nccl":
                it = D.IteratedSpMV(part, A.n, lambda x, y, a, b: M.spmv(x, y, alpha=a, beta=b), x0, rank)
            else:
                L = max(part.padded, A.n)
                bufs = D._symmetric_buffers(L, world, rank, None, dev, force_symmetric=True)
                it = D.FusedIteratedSpMV(part, A.n, M, x0, rank, buffers=bufs)
            for _ in range(K_STEPS):
                x = it.step(ALPHA, c)
            torch.cuda.synchronize()
            np.save(os.path.join(out_dir, f"{mode}_{rank}.npy"), x[: A.n].cpu().numpy())
            dist.barrier()
    finally:
        dist.destroy_process_group()


def _single_rank_reference():
    import torch

    import paper_conf_icpp_cheny24_b200 as sp
    A = _matrix()
    M = sp.convert(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.colidx).cuda(),
                   torch.from_numpy(A.values).cuda(), A.n)
    x = torch.full((A.n,), 1.0 / A.n, device="cuda")
    for _ in range(K_STEPS):
        y = torch.full((A.m,), 0.15 / A.n, device="cuda")
        M.spmv(x, y, alpha=ALPHA, beta=1.0)
        x = y
    torch.cuda.synchronize()
    ref = oracle.pagerank(A.rowptr, A.colidx, A.values, ALPHA, K_STEPS, np.full(A.n, 1.0 / A.n))
    return x.cpu().numpy(), ref


def _run(world, modes, tmp_path):
    import torch.multiprocessing as mp
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path), modes), nprocs=world, join=True)
    single, ref = _single_rank_reference()
    for mode in modes:
        for r in range(world):
            got = np.load(tmp_path / f"{mode}_{r}.npy")
            assert np.array_equal(got, single), f"{mode} rank {r} differs from the single-rank CUDA result"
            g = got.astype(np.float64)
            assert (np.abs(g - ref) / np.abs(ref)).max() <= 1e-5


def test_symmetric_memory_fused_pagerank_one_rank(tmp_path):
    """The symmetric-memory path of FusedIteratedSpMV (rendezvous, peer view,
    handle barrier) on a one-rank NCCL group: x after K steps equals the plain
    CUDA iteration bitwise and the oracle's PageRank within 1e-5."""
    _run(1, ("fused",), tmp_path)


def test_two_ranks_nccl_and_symmetric_memory(tmp_path):
    import torch
    if torch.cuda.device_count() < 2:
        pytest.skip("needs two visible GPUs (gpurun provides one)")
    _run(2, ("nccl", "fused"), tmp_path)
