"""Per-role timeline of the tensor-core SpMM on CTA 0 (experiment build with
-DSPADEN_TC_TRACE: SPADEN_LIB=exp/libspaden_tctrace.so python tools/tc_trace.py)."""
import ctypes
import sys

import numpy as np
import torch

import paper_conf_icpp_cheny24_b200 as sp
import workloads as W

K = int(sys.argv[1]) if len(sys.argv) > 1 else 128
A = W.make("fem1p5m")
dev = torch.device("cuda:0")
M = sp.convert(torch.from_numpy(A.rowptr).to(dev), torch.from_numpy(A.colidx).to(dev),
               torch.from_numpy(A.values).to(dev), A.n, storage="fp16")
X = torch.rand((K, A.n), device=dev) * 2 - 1
Xb = M.pack_x_tc(X)
Y = torch.empty((K, A.m), device=dev)
buf = torch.zeros(4 * 512 * 8, dtype=torch.int64, device=dev)
lib = ctypes.CDLL(sp.LIB_PATH)
for _ in range(3):
    M.spmm_tc(Xb, K, Y)
torch.cuda.synchronize()
assert lib.spaden_debug_tc_trace(ctypes.c_void_p(buf.data_ptr())) == 0
M.spmm_tc(Xb, K, Y)
torch.cuda.synchronize()
t = buf.cpu().numpy().reshape(4, 512, 8).astype(np.int64)
names = {0: ["start", "afree", "issued"], 1: ["start", "arr", "sfree", "slab_issued", "mma_free", "tiles_done"],
         2: ["start", "arr", "tiles", "slab", "epi", "desc", "issued"], 3: ["start", "mma", "done"]}
roles = ["producer", "decode0", "mma", "epilogue"]
lo, hi = 100, 400
base = t[0, lo, 0]
print("chunk period (mma start to start):", np.mean(np.diff(t[2, lo:hi, 0])))
for r, nm in enumerate(roles):
    ev = names[r]
    d = [np.mean(t[r, lo:hi, e + 1] - t[r, lo:hi, e]) for e in range(len(ev) - 1)]
    print(f"{nm:9s}", " ".join(f"{ev[e]}->{ev[e+1]}: {d[e]:7.0f}" for e in range(len(d))))
print("sample chunks (cycles relative to producer start of chunk 100):")
for c in range(lo, lo + 6):
    print(c, {roles[r]: [int(v - base) for v in t[r, c, :len(names[r])]] for r in range(4)})
