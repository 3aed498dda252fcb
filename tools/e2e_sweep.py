"""Sweep of the slot count of spaden_spmv_host_batched (SPADEN_PIPE_SLOTS) on
the bench workload: e2e GFLOP/s through the C ABI with pinned host vectors,
timed exactly as bench.py's e2e leg.  One JSON line per slot count."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_icpp_cheny24_b200 as sp  # noqa: E402


def main(workload="fem1p5m", slots=(2, 3, 4, 5, 6, 8), reps=3):
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    wl = bench.Workload(workload, 0, 1, dev)
    stream = torch.cuda.current_stream(dev)
    K = int(max(2, min(2000, (512 << 20) // (4 * (wl.n + wl.m)))))
    X = torch.empty((K, wl.n), dtype=torch.float32).pin_memory()
    X.copy_(wl.x0.cpu().expand(K, wl.n))
    Y = torch.zeros((K, wl.m), dtype=torch.float32).pin_memory()
    for S in slots:
        os.environ["SPADEN_PIPE_SLOTS"] = str(S)  # read when the handle builds its pipeline
        M = sp.convert(*wl.local, wl.n, storage="fp32", residual_max_popc=-1)
        M.spmv_host_batched(X[:2], Y[:2], alpha=wl.alpha, beta=0.0, stream=stream)
        ms = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize(dev)
            e0.record(stream)
            M.spmv_host_batched(X, Y, alpha=wl.alpha, beta=0.0, stream=stream)
            e1.record(stream)
            torch.cuda.synchronize(dev)
            ms.append(e0.elapsed_time(e1) / K)
        M.free()
        best = min(ms)
        print(json.dumps({"slots": S, "K": K, "ms_per_step": ms, "gflops_best": 2.0 * wl.nnz / (best * 1e-3) / 1e9}),
              flush=True)


if __name__ == "__main__":
    main(*(sys.argv[1:2] or ["fem1p5m"]))
