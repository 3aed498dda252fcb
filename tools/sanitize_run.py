"""Small end-to-end exercise of every kernel for compute-sanitizer
(memcheck / racecheck / synccheck): conversions in all dtype modes, the tiled
SpMV, the long-row chunk path (fused and separate fix-up), alpha/beta, the
hybrid format (binned residual, long residual rows, PDL chain), SpMM, the
batched host pipeline."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import paper_conf_icpp_cheny24_b200 as sp  # noqa: E402
import workloads as W  # noqa: E402
from test_gpu_parity import binned_rows_matrix, hub_matrix  # noqa: E402


def run(A, storage, t=0):
    rp = torch.from_numpy(A.rowptr).cuda()
    ci = torch.from_numpy(A.colidx).cuda()
    v = torch.from_numpy(A.values).cuda()
    M = sp.convert(rp, ci, v, A.n, storage=storage, residual_max_popc=t)
    x = torch.from_numpy(W.vector(A.n, 1)).cuda()
    y = torch.from_numpy(W.vector(A.m, 2)).cuda()
    M.spmv(x, y, alpha=1.0, beta=0.5)
    M.spmv(x, y)
    torch.cuda.synchronize()
    M.free()


for A in (W.h2(), W.tiny(0), W.fem(6, 7, 8, seed=2), hub_matrix(m=40, n=70_001, hub_rows=(3, 30), hub_nnz=40_000)):
    for st in ("fp32", "fp16"):
        run(A, st)
        run(A, st, t=2)
for fixup in ("8192", "0"):  # long-row fix-up fused into the chunk kernel / separate launch
    os.environ["SPADEN_FUSED_FIXUP_MAX"] = fixup
    run(binned_rows_matrix(), "fp32", t=64)
    run(hub_matrix(m=40, n=70_001, hub_rows=(3, 30), hub_nnz=40_000), "fp32")
os.environ.pop("SPADEN_FUSED_FIXUP_MAX")
os.environ["SPADEN_XSEG_COLS"] = "3000"  # residual column parts (normally x > 64 MB)
run(binned_rows_matrix(), "fp32", t=64)
run(binned_rows_matrix(), "fp16", t=-1)
os.environ.pop("SPADEN_XSEG_COLS")
B = hub_matrix()
MB = sp.convert(torch.from_numpy(B.rowptr).cuda(), torch.from_numpy(B.colidx).cuda(),
                torch.from_numpy(B.values).cuda(), B.n, residual_max_popc=2)
MB.spmm(torch.from_numpy(np.stack([W.vector(B.n, k) for k in range(4)])).cuda())
torch.cuda.synchronize()
A = W.fem(5, 5, 6, seed=1)
M = sp.convert(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.colidx).cuda(),
               torch.from_numpy(A.values).cuda(), A.n)
X = torch.from_numpy(np.stack([W.vector(A.n, k) for k in range(3)])).pin_memory()
Y = torch.zeros((3, A.m)).pin_memory()
M.spmv_host_batched(X, Y)
# round 2: count pass, fused peer-store epilogue, tensor-core SpMM (fp16, k = 70)
assert sp.count_blocks(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.colidx).cuda(), A.n) == M.info.Bnnz
xd = torch.from_numpy(W.vector(A.n, 5)).cuda()
peers = [torch.zeros(A.m + 8, device="cuda") for _ in range(3)]
M.spmv_scatter(xd, [t.data_ptr() for t in peers], 4)
for C in (A, B, W.h2()):
    Mh = sp.convert(torch.from_numpy(C.rowptr).cuda(), torch.from_numpy(C.colidx).cuda(),
                    torch.from_numpy(C.values).cuda(), C.n, storage="fp16")
    Xk = torch.from_numpy(np.stack([W.vector(C.n, k) for k in range(70)])).cuda()
    Xb = Mh.pack_x_tc(Xk)
    Yk = torch.zeros((70, C.m), device="cuda")
    Mh.spmm_tc(Xb, 70, Yk, alpha=0.5, beta=0.5)
    torch.cuda.synchronize()
    Mh.free()
# reordering (NEXT-1): degree order + P A P^T, then the hybrid SpMV on it
P = W.powerlaw(12, 5, 1, relabel=True)
rp, ci, v = (torch.from_numpy(a).cuda() for a in (P.rowptr, P.colidx, P.values))
perm = sp.degree_order(rp)
rp2, ci2, v2 = sp.permute_csr(rp, ci, v, perm)
MR = sp.convert(rp2, ci2, v2, P.n, residual_max_popc=-1)
MR.spmv(torch.from_numpy(W.vector(P.n, 3)).cuda())
torch.cuda.synchronize()
MR.free()
print("sanitize run ok")
