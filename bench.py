#!/usr/bin/env python3
"""bench.py -- bitBSR SpMV throughput on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload fem1p5m]
                    [--dtype fp32|fp16] [--impl spaden|reference]

A step is one iterated SpMV over the whole matrix: x_{k+1} = alpha * A x_k with
alpha = 1/||A||_inf (bounded iterates).  With N > 1 (torchrun, NCCL) A is
row-partitioned in 8-row-aligned slices, each rank computes its slice of
x_{k+1} and an NCCL all-gather rebuilds the replicated x;
total work is fixed ("strong" scaling).  The timed region is K steps between
barrier + synchronize; the time is the max over ranks of CUDA-event time.

Inputs are synthetic (workloads/, seeded) and resident in HBM; the matrix
(480 MB for fem1p5m fp32) is larger than the 126 MB L2, so no L2 flush is
needed between steps (x, 6 MB, is L2-resident as in any iterative solver).
A matrix that fits L2 (fem62k) is measured flushed by default (--l2 auto): a
256 MB write before every step, the step timed by the SpMV's own events.

--impl reference times the CPU oracle (oracle/, fp64 CSR SpMV, Alg. 1, the row
loop on all host cores) on a bounded row sample per step -- this tier's reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = "SpMV GFLOP/s (2*nnz/t) on bitBSR; achieved HBM GB/s and bytes/nnz alongside"
UNIT = "GFLOP/s"


L2_BYTES = 126 * 1000 * 1000  # B200 L2 (126 MB)


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=2000)
    p.add_argument("--warmup", type=int, default=20)
    p.add_argument("--workload", default=None,
                   help="one of %s, or rmatNN (PageRank on R-MAT scale NN, e.g. rmat25); default fem1p5m "
                        "at --gpus 1 (the single-GPU HBM-roofline config) and rmat25 for --gpus > 1 (the "
                        "north_star multi-GPU config; take a scaling curve with an explicit --workload)"
                        % sorted(W.CONFIGS))
    p.add_argument("--dtype", default="fp32", choices=["fp32", "fp16"])
    p.add_argument("--impl", default="spaden", choices=["spaden", "reference"])
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-cusparse", action="store_true")
    p.add_argument("--no-variants", action="store_true", help="skip the other-precision kernel timing")
    p.add_argument("--spmm", default="4", help="comma list of right-hand-side counts for the SpMM extra ('' = skip)")
    p.add_argument("--spmm-tc", default="64,128", help="comma list of right-hand-side counts for the tensor-core "
                                                   "SpMM extra (fp16 storage, tcgen05; '' = skip)")
    p.add_argument("--hybrid", type=int, default=-1,
                   help="hybrid format: blocks with <= HYBRID entries go to a CSR residual (0 = pure bitBSR, "
                        "-1 = automatic by mean block fill)")
    p.add_argument("--reorder", default="none", choices=["none", "degree"],
                   help="degree: symmetric degree ordering P A P^T before conversion (spaden_degree_order + "
                        "spaden_permute_csr, SURVEY.md NEXT-1); the iteration runs in the permuted space "
                        "(with N ranks every rank permutes the whole matrix and keeps its row slice)")
    p.add_argument("--cpu-seconds", type=float, default=12.0)
    p.add_argument("--exchange", default="nccl", choices=["nccl", "fused"],
                   help="x rebuild for N>1: NCCL all-gather after the SpMV, or peer stores fused into the "
                        "SpMV epilogue (spaden_spmv_scatter over symmetric memory, NEXT-2)")
    p.add_argument("--l2", default="auto", choices=["auto", "flush", "warm"],
                   help="flush = write a 256 MB buffer before every timed step and take the step time from "
                        "the SpMV's own events; auto = flush when the matrix fits the 126 MB L2")
    a = p.parse_args()
    if a.workload is None:
        a.workload = "fem1p5m" if a.gpus <= 1 else "rmat25"
    return a


def spawn_ranks(args):
    """--gpus N > 1 without a torchrun environment: re-launch this script as N
    NCCL ranks (one process per GPU) with torch.distributed.run on 127.0.0.1."""
    import socket
    import subprocess

    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")  # communicator lines (rank count, NVLS) on stderr
    return subprocess.call(cmd, env=env)


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def alg_bytes(m, n, nnz, Bnrow, Bnnz, sv, beta_nonzero=False, res_nnz=0):
    """Algorithmic bytes of one SpMV: the bitBSR arrays once
    (blk_rowptr, blk_col, bitmap, blk_offset, values), x once, y written once;
    in hybrid mode also the residual CSR (rowptr, colidx, values) and y re-read
    and re-written by the residual pass."""
    b = 4 * (Bnrow + 1) + (4 + 8 + 4) * Bnnz + sv * (nnz - res_nnz) + 4 * n + 4 * m + (4 * m if beta_nonzero else 0)
    if res_nnz:
        b += 4 * (m + 1) + (4 + sv) * res_nnz + 8 * m
    return b


class Clocks:
    """NVML sampler of SM clock and throttle reasons during the timed region."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, index, period=0.02):
        self.index, self.period = index, period
        self.samples, self.reasons = [], set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.nv:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons - {"gpu_idle"}), "samples": len(self.samples)}


def cpu_oracle_gflops(A, x, seconds, all_cores=False):
    """The oracle (fp64 CSR SpMV, Alg. 1) on whole-matrix passes, bounded in time:
    one thread, or the row loop on all host cores (OpenMP static schedule)."""
    import oracle
    oracle.lib()
    rp = np.ascontiguousarray(A.rowptr, np.int64)
    v = np.ascontiguousarray(A.values.astype(np.float64))
    xx = np.ascontiguousarray(x.astype(np.float64))
    fn = (lambda: oracle.spmv_omp(rp, A.colidx, v, xx)[2]) if all_cores else (lambda: oracle.spmv(rp, A.colidx, v, xx) and 1)
    t0 = time.perf_counter()
    passes = 0
    threads = 1
    while True:
        threads = fn()
        passes += 1
        if time.perf_counter() - t0 >= seconds:
            break
    dt = time.perf_counter() - t0
    return {"value": 2.0 * A.nnz * passes / dt / 1e9, "unit": UNIT, "cores": int(threads), "kind": "oracle",
            "host_cpu": _cpu_model(), "os_cpu_count": os.cpu_count(),
            "sample": f"{passes} full passes over the {A.m}x{A.n} matrix ({A.nnz} nnz), fp64, "
                      f"{'OpenMP ' + str(threads) + ' threads' if all_cores else '1 thread'}, {dt:.1f} s wall"}


def _cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def reference_arm(args):
    """--impl reference: the CPU oracle as this tier's reference arm."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    if args.workload.startswith("rmat"):  # GPU-generated (same stream as the CUDA arm), host sample
        import torch
        scale = int(args.workload[4:])
        dev = "cuda" if torch.cuda.is_available() else "cpu"
        k = max(8, (1 << scale) // 64)
        rp, ci, v, n, _ = W.pagerank_slice_torch(scale, 32, 0, k, seed=0, device=dev)
        A = W.CSR(k, n, rp.cpu().numpy(), ci.cpu().numpy(), v.cpu().numpy())
        x = np.full(n, 1.0 / n, np.float32)
    else:
        A = W.make(args.workload)
        x = W.vector(A.n, 2)
    vals = A.values if args.dtype == "fp32" else oracle.f32_to_f16(A.values)
    oracle.lib()
    # per-step budget so that K+W steps take ~90 s in total (all host cores)
    t0 = time.perf_counter()
    oracle.spmv_omp(A.rowptr, A.colidx, vals, x)
    full = time.perf_counter() - t0
    frac = min(1.0, 90.0 / max(1, args.steps + args.warmup) / max(full, 1e-6))
    r1 = max(8, int(A.m * frac) // 8 * 8)
    S = A.row_slice(0, r1)
    sv = vals[: S.nnz]
    rp = np.ascontiguousarray(S.rowptr, np.int64)
    v = np.ascontiguousarray(sv.astype(np.float64))
    xx = np.ascontiguousarray(x.astype(np.float64))
    threads = 1
    for _ in range(args.warmup):
        threads = oracle.spmv_omp(rp, S.colidx, v, xx)[2]
    t0 = time.perf_counter()
    for _ in range(args.steps):
        threads = oracle.spmv_omp(rp, S.colidx, v, xx)[2]
    dt = time.perf_counter() - t0
    val = 2.0 * S.nnz * args.steps / dt / 1e9
    line = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": args.workload, "m": A.m, "n": A.n, "nnz": A.nnz, "values": args.dtype,
                       "sample_rows": r1, "sample_nnz": S.nnz},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "host_cpu": _cpu_model(), "os_cpu_count": os.cpu_count(),
                             "sample": f"rows [0,{r1}) of {args.workload} ({S.nnz} nnz) per step, "
                                       f"OpenMP {threads} threads"},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


class Workload:
    """This rank's slice of the benchmark matrix plus the iteration it runs."""

    def __init__(self, name, rank, world, dev, reorder="none"):
        import torch

        from paper_conf_icpp_cheny24_b200.dist import RowPartition

        self.name = name
        if name.startswith("rmat"):  # PageRank on R-MAT (generated on the GPU)
            scale = int(name[4:])
            self.m = self.n = 1 << scale
            self.part = RowPartition(self.m, world)
            r0, r1 = self.part.range(rank)
            rp, ci, v, _, self.nnz = W.pagerank_slice_torch(scale, 32, r0, r1, seed=0, device=dev)
            self.local = (rp, ci, v)
            self.local_nnz = int(ci.numel())
            self.alpha, self.c = 0.85, 0.15 / self.n
            self.x0 = torch.full((self.n,), 1.0 / self.n, dtype=torch.float32, device=dev)
            self.host = None
            self.step_desc = "PageRank x <- 0.85 A x + 0.15/n"
        else:
            A = W.make(name)
            self.host = A
            self.m, self.n, self.nnz = A.m, A.n, A.nnz
            self.part = RowPartition(A.m, world)
            r0, r1 = self.part.range(rank)
            S = A.row_slice(r0, r1)
            self.local = tuple(torch.from_numpy(a).to(dev) for a in (S.rowptr, S.colidx, S.values))
            self.local_nnz = S.nnz
            csum = np.concatenate([[0.0], np.cumsum(np.abs(A.values.astype(np.float64)))])
            a_inf = float((csum[A.rowptr[1:]] - csum[A.rowptr[:-1]]).max()) if A.m else 0.0
            self.alpha, self.c = (1.0 / a_inf if a_inf > 0 else 1.0), None
            self.x0 = torch.from_numpy(W.vector(A.n, 2)).to(dev)
            self.step_desc = "x <- A x / ||A||_inf"
        self.r0, self.r1 = self.part.range(rank)
        self.reorder_s = None
        if reorder == "degree":  # B = P A P^T; x kept in the permuted space (x'[k] = x[perm[k]])
            import paper_conf_icpp_cheny24_b200 as sp
            full = self.local
            if world > 1:  # every rank permutes the whole matrix (the same B) and keeps its rows
                if name.startswith("rmat"):
                    rp, ci, v, _, _ = W.pagerank_slice_torch(int(name[4:]), 32, 0, self.m, seed=0, device=dev)
                    full = (rp, ci, v)
                else:
                    full = tuple(torch.from_numpy(a).to(dev) for a in (A.rowptr, A.colidx, A.values))
            times = []
            for _ in range(3):  # first call loads the sort kernels; median of the 3
                torch.cuda.synchronize(dev)
                t0 = time.perf_counter()
                perm = sp.degree_order(full[0])
                B = sp.permute_csr(*full, perm)
                torch.cuda.synchronize(dev)
                times.append(time.perf_counter() - t0)
            self.reorder_s = statistics.median(times)
            if world > 1:  # rows [r0, r1) of B, local rowptr
                brp, bci, bv = B
                a, b = int(brp[self.r0].item()), int(brp[self.r1].item())
                B = ((brp[self.r0:self.r1 + 1] - a).contiguous(), bci[a:b].contiguous(), bv[a:b].contiguous())
                del brp, bci, bv
            del full
            self.local = B
            self.local_nnz = int(B[1].numel())
            self.x0 = self.x0[perm.long()].contiguous()
            self.host = None


def main():
    args = parse()
    if args.impl == "reference":
        return reference_arm(args)

    import torch
    import torch.distributed as dist

    import paper_conf_icpp_cheny24_b200 as sp
    from paper_conf_icpp_cheny24_b200.dist import FusedIteratedSpMV, IteratedSpMV, convert_slice

    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return spawn_ranks(args)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world} (launch one rank per GPU)")
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)

    # ---- workload (identical on every rank), this rank's 8-row-aligned slice
    wl = Workload(args.workload, rank, world, dev, args.reorder)
    sv = 2 if args.dtype == "fp16" else 4
    stream = torch.cuda.current_stream(dev)
    # warm-up conversion of the same matrix: loads every kernel the conversion
    # uses (lazy module loading) so the timed conversion below measures the
    # conversion only
    convert_slice(*wl.local, wl.n, storage=args.dtype, residual_max_popc=args.hybrid).free()
    torch.cuda.synchronize(dev)
    # conversion time: median of 5 warm repetitions (each includes the handle's
    # allocations and the converter's host synchronisations)
    conv_times = []
    for rep in range(5):
        t0 = time.perf_counter()
        M = convert_slice(*wl.local, wl.n, storage=args.dtype, residual_max_popc=args.hybrid)
        torch.cuda.synchronize(dev)
        conv_times.append(time.perf_counter() - t0)
        if rep < 4:
            M.free()
    convert_s = statistics.median(conv_times)
    info = M.info
    local_csr = wl.local
    wl.local = None

    ev_pair = [None]

    def local_spmv(x, y, alpha, beta):
        if ev_pair[0] is not None:
            ev_pair[0][0].record(stream)
        M.spmv(x, y, alpha=alpha, beta=beta, stream=stream)
        if ev_pair[0] is not None:
            ev_pair[0][1].record(stream)

    class _Timed:  # spmv_scatter with the per-launch events of the roofline
        def spmv_scatter(self, x, ptrs, off, y=None, alpha=1.0, beta=0.0):
            if ev_pair[0] is not None:
                ev_pair[0][0].record(stream)
            M.spmv_scatter(x, ptrs, off, y=y, alpha=alpha, beta=beta, stream=stream)
            if ev_pair[0] is not None:
                ev_pair[0][1].record(stream)

    if args.exchange == "fused":
        if info.residual_max_popc > 0:
            raise SystemExit("--exchange fused needs pure bitBSR (--hybrid 0)")
        it = FusedIteratedSpMV(wl.part, wl.n, _Timed(), wl.x0, rank)
    else:
        it = IteratedSpMV(wl.part, wl.n, local_spmv, wl.x0, rank)

    for _ in range(max(3, args.warmup)):
        it.step(wl.alpha, wl.c)
    torch.cuda.synchronize(dev)

    flush = args.l2 == "flush" or (args.l2 == "auto" and info.format_bytes <= L2_BYTES)
    flush_buf = torch.empty(2 * L2_BYTES // 4, dtype=torch.float32, device=dev) if flush else None
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    gevs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)] \
        if (world > 1 and args.exchange == "nccl") else None
    start = torch.cuda.Event(enable_timing=True)
    end = torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    with Clocks(local) as clk:
        torch.cuda.nvtx.range_push("bench_timed_region")  # ncu --nvtx --nvtx-include bench_timed_region/
        start.record(stream)
        for i in range(args.steps):
            if flush:  # evict A, x and y from L2 (outside the step's events)
                flush_buf.fill_(float(i))
            ev_pair[0] = evs[i]
            if gevs is not None:
                it.gather_events = gevs[i]
            it.step(wl.alpha, wl.c)
        ev_pair[0] = None
        if gevs is not None:
            it.gather_events = None
        end.record(stream)
        torch.cuda.synchronize(dev)
        torch.cuda.nvtx.range_pop()
    if world > 1:
        dist.barrier()
    kernel_ms = [a.elapsed_time(b) for a, b in evs]
    # flushed: a step is the SpMV's own events (the flush between steps is not
    # work of the method); otherwise the whole timed region
    elapsed_ms = float(np.sum(kernel_ms)) if flush else start.elapsed_time(end)
    t = torch.tensor([elapsed_ms], device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    elapsed_ms = float(t.item())
    ms_per_step = elapsed_ms / args.steps
    gflops = 2.0 * wl.nnz * args.steps / (elapsed_ms * 1e-3) / 1e9

    # per-iteration SpMV and all-gather times (max over ranks of each rank's mean)
    kavg_ms = float(np.mean(kernel_ms))
    split = None
    if world > 1:
        tt = torch.tensor([kavg_ms, float(np.mean([a.elapsed_time(b) for a, b in gevs])) if gevs else 0.0],
                          device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        nz = torch.tensor([float(wl.local_nnz)], device=dev)
        dist.all_reduce(nz, op=dist.ReduceOp.MAX)
        split = {"nnz_imbalance_max_over_mean": float(nz.item()) / (wl.nnz / world),
                 "t_spmv_ms": float(tt[0]), "t_allgather_ms": float(tt[1]) if gevs else None,
                 "t_iter_ms": ms_per_step,
                 "note": ("NCCL all_gather_into_tensor after the SpMV" if gevs else
                          "fused peer stores: the exchange runs inside the SpMV (+ one device barrier)")}

    # ---- roofline of the dominant kernel (the SpMV) on this rank
    abytes = alg_bytes(wl.r1 - wl.r0, wl.n, wl.local_nnz, info.Bnrow, info.Bnnz, sv, beta_nonzero=wl.c is not None,
                       res_nnz=info.residual_nnz)
    peak, peak_kind = peaks()
    achieved = abytes / (kavg_ms * 1e-3) / 1e9
    # roofline.traffic: dram__bytes_read.sum + dram__bytes_write.sum per launch from an
    # `ncu --set full` capture of this kernel (not measurable inside a timed run);
    # a STORED value, labelled with the capture it came from (profiles/ncu_traffic.json)
    traffic, traffic_src = None, None
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            tr = json.load(f)
        key = f"{args.workload}/{args.dtype}"
        if key in tr and world == 1 and args.hybrid in (-1, 0):
            traffic = tr[key]["dram_bytes_per_launch"]
            traffic_src = {k: v for k, v in tr[key].items() if k != "dram_bytes_per_launch"}
            traffic_src["kind"] = "stored: ncu --set full capture (see source), not measured in this run"
    except Exception:
        pass

    # ---- e2e through the C ABI with host buffers (H2D x (+y), SpMV, D2H y per step),
    # every rank on its row slice (x replicated from host memory, no collective);
    # time = max over ranks, value = all ranks' nonzeros / that time
    beta = 0.0 if wl.c is None else 1.0
    m_loc = wl.r1 - wl.r0
    # spaden_spmv_host_batched: per step H2D of x_k (+ y_k if beta != 0), SpMV, D2H of y_k,
    # pipelined across steps (copies of neighbouring steps overlap the SpMV)
    K = int(max(2, min(args.steps, (512 << 20) // (4 * (wl.n + m_loc)))))
    X = torch.empty((K, wl.n), dtype=torch.float32).pin_memory()
    X.copy_(wl.x0.cpu().expand(K, wl.n))
    Y = torch.full((K, m_loc), wl.c or 0.0, dtype=torch.float32).pin_memory()
    # warm-up over the whole batch: the first pass over freshly pinned
    # buffers runs ~20% slower (measured, tools/e2e_sweep.py)
    M.spmv_host_batched(X, Y, alpha=wl.alpha, beta=beta, stream=stream)
    # three timed passes of K steps each (PCIe throughput varies run to
    # run); the reported value is the median pass
    passes = []
    for _ in range(3):
        if beta:
            Y.fill_(wl.c)
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        e0.record(stream)
        M.spmv_host_batched(X, Y, alpha=wl.alpha, beta=beta, stream=stream)
        e1.record(stream)
        torch.cuda.synchronize(dev)
        tp = torch.tensor([e0.elapsed_time(e1) / K], device=dev)
        if world > 1:
            dist.all_reduce(tp, op=dist.ReduceOp.MAX)
        passes.append(float(tp.item()))
    e2e_ms = statistics.median(passes)
    e2e = {"value": 2.0 * wl.nnz / (e2e_ms * 1e-3) / 1e9, "unit": UNIT,
           "h2d_bytes_per_step": world * 4 * wl.n + (4 * wl.m if beta else 0), "d2h_bytes_per_step": 4 * wl.m,
           "ms_per_step": e2e_ms, "steps": K, "passes_ms_per_step": passes,
           "api": "spaden_spmv_host_batched (pinned host x_k/y_k, copies overlapped with SpMV; "
                  "per rank: full x_k in, its row slice of y_k out; max over ranks)"}
    del X, Y

    line = None
    if rank == 0:
        clocks = clk.summary()
        # ---- cuSPARSE CSR SpMV on the same matrix and GPU (north_star comparison)
        cus = None
        if not args.no_cusparse and world == 1:
            try:
                sys.path.insert(0, os.path.join(ROOT, "tools"))
                import cusparse_csr
                rp_d, ci_d, v_d = local_csr
                v32 = v_d.float().contiguous()  # the paper's baseline: fp32 CSR
                res = cusparse_csr.time_spmv(rp_d, ci_d, v32, wl.x0.contiguous(), wl.m, wl.n, stream,
                                             reps=max(20, min(args.steps, 500)))
                best = min(res, key=lambda k: res[k]["ms"])
                cus = {"impl": "cusparseSpMV fp32 CSR, int32 indices (ctypes, same stream)",
                       "algs": {k: {"ms": r["ms"], "buffer_bytes": r["buffer_bytes"],
                                    "footprint_bytes": r["footprint_bytes"]} for k, r in res.items()},
                       "best": best, "ms": res[best]["ms"],
                       "gflops": 2.0 * wl.nnz / (res[best]["ms"] * 1e-3) / 1e9,
                       "footprint_bytes": res[best]["footprint_bytes"],
                       "bytes_per_nnz": res[best]["footprint_bytes"] / wl.nnz,
                       "speedup_spaden_vs_cusparse": res[best]["ms"] / kavg_ms,
                       "footprint_saving": res[best]["footprint_bytes"] / info.format_bytes,
                       "note": ("back-to-back calls, no L2 flush" + (" (matrix fits L2: warm)"
                                                                      if info.format_bytes <= L2_BYTES else ""))}
                del res, v32
            except Exception as e:  # pragma: no cover
                cus = {"error": repr(e)[:300]}

        cpu = None
        if not args.no_cpu_baseline and world == 1:
            if wl.host is not None:
                S = wl.host
            else:  # bounded row sample of the GPU-generated matrix
                rp, ci, v = local_csr
                k = max(8, min(wl.m, wl.m // 64))
                hi = int(rp[k].item())
                S = W.CSR(k, wl.n, rp[:k + 1].cpu().numpy(), ci[:hi].cpu().numpy(), v[:hi].cpu().numpy())
            xs = wl.x0.cpu().numpy()
            cpu = cpu_oracle_gflops(S, xs, args.cpu_seconds / 2, all_cores=True)
            cpu["single_thread"] = cpu_oracle_gflops(S, xs, args.cpu_seconds / 2, all_cores=False)

        # ---- the other value precision on the same matrix (kernel time only)
        variants = {}
        if world == 1 and not args.no_variants:
            other = "fp16" if args.dtype == "fp32" else "fp32"
            M2 = sp.convert(*local_csr, wl.n, storage=other, residual_max_popc=args.hybrid)
            i2 = M2.info
            ys = torch.empty(wl.m, dtype=torch.float32, device=dev)
            for _ in range(5):
                M2.spmv(wl.x0, ys, alpha=wl.alpha, stream=stream)
            reps = max(20, min(args.steps, 500))
            v0e = torch.cuda.Event(enable_timing=True)
            v1e = torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize(dev)
            v0e.record(stream)
            for _ in range(reps):
                M2.spmv(wl.x0, ys, alpha=wl.alpha, stream=stream)
            v1e.record(stream)
            torch.cuda.synchronize(dev)
            vms = v0e.elapsed_time(v1e) / reps
            vb = alg_bytes(wl.m, wl.n, wl.local_nnz, i2.Bnrow, i2.Bnnz, 2 if other == "fp16" else 4,
                           res_nnz=i2.residual_nnz)
            variants[other] = {"kernel_ms": vms, "gflops": 2.0 * wl.nnz / (vms * 1e-3) / 1e9,
                               "hbm_gbs": vb / (vms * 1e-3) / 1e9, "frac": vb / (vms * 1e-3) / 1e9 / peak,
                               "bytes_per_nnz_stored": i2.format_bytes / max(1, i2.nnz),
                               "note": "back-to-back launches, no L2 flush" + (" (matrix > L2)" if i2.format_bytes > 126e6
                                                                                 else " (matrix fits L2)")}
            M2.free()
            del ys

        # tiled kernel [+ long-row chunks and fix-up] [+ hybrid residual pass]
        # ---- SpMM (NEXT-4): K right-hand sides per decoded block
        spmm = {}
        if world == 1 and args.spmm:
            for K in [int(v) for v in args.spmm.split(",") if v]:
                X = wl.x0.expand(K, wl.n).contiguous()
                Yk = torch.empty((K, wl.m), dtype=torch.float32, device=dev)
                for _ in range(3):
                    M.spmm(X, Yk, alpha=wl.alpha, stream=stream)
                reps = max(10, min(args.steps, 200))
                s0e = torch.cuda.Event(enable_timing=True)
                s1e = torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize(dev)
                s0e.record(stream)
                for _ in range(reps):
                    M.spmm(X, Yk, alpha=wl.alpha, stream=stream)
                s1e.record(stream)
                torch.cuda.synchronize(dev)
                sms = s0e.elapsed_time(s1e) / reps
                spmm[str(K)] = {"ms": sms, "gflops": 2.0 * wl.nnz * K / (sms * 1e-3) / 1e9,
                                "per_vector_speedup_vs_spmv": kavg_ms * K / sms}
                del X, Yk

        # ---- NEXT-4: tensor-core SpMM (tcgen05, fp16 storage and fp16 x slabs)
        spmm_tc = {}
        if world == 1 and args.spmm_tc and info.residual_max_popc == 0:
            Mh = M if args.dtype == "fp16" else sp.convert(*local_csr, wl.n, storage="fp16", residual_max_popc=0)
            # the same matrix's fp16 SpMV kernel time (per-vector reference)
            yv = torch.empty(wl.m, dtype=torch.float32, device=dev)
            for _ in range(5):
                Mh.spmv(wl.x0, yv, stream=stream)
            s0e, s1e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize(dev)
            s0e.record(stream)
            for _ in range(50):
                Mh.spmv(wl.x0, yv, stream=stream)
            s1e.record(stream)
            torch.cuda.synchronize(dev)
            spmv16_ms = s0e.elapsed_time(s1e) / 50
            for K in [int(v) for v in args.spmm_tc.split(",") if v]:
                gen = torch.Generator(device=dev).manual_seed(7)
                X = torch.rand((K, wl.n), generator=gen, device=dev, dtype=torch.float32) * 2 - 1
                Yk = torch.empty((K, wl.m), dtype=torch.float32, device=dev)
                Xb = Mh.pack_x_tc(X, stream=stream)
                for _ in range(3):
                    Mh.spmm_tc(Xb, K, Yk, alpha=wl.alpha, stream=stream)
                reps = max(5, min(args.steps, 50))
                p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s0e, s1e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize(dev)
                p0.record(stream)
                for _ in range(reps):
                    Mh.pack_x_tc(X, Xb, stream=stream)
                p1.record(stream)
                s0e.record(stream)
                for _ in range(reps):
                    Mh.spmm_tc(Xb, K, Yk, alpha=wl.alpha, stream=stream)
                s1e.record(stream)
                torch.cuda.synchronize(dev)
                tms = s0e.elapsed_time(s1e) / reps
                pms = p0.elapsed_time(p1) / reps
                spmm_tc[str(K)] = {"ms": tms, "pack_x_ms": pms,
                                   "gflops": 2.0 * wl.nnz * K / (tms * 1e-3) / 1e9,
                                   "gflops_incl_pack": 2.0 * wl.nnz * K / ((tms + pms) * 1e-3) / 1e9,
                                   "per_vector_speedup_vs_fp16_spmv": spmv16_ms * K / tms,
                                   "fp16_spmv_ms": spmv16_ms,
                                   "precision": "fp16 A (stored), fp16 x (RNE), fp32 accumulation in TMEM"}
                del X, Yk, Xb
            if Mh is not M:
                Mh.free()
            del yv

        n_launch = M.launch_count(1.0 if wl.c is not None else 0.0)  # kernels + memsets of one spaden_spmv
        line = {
            "metric": METRIC, "value": gflops, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": max(3, args.warmup), "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32" if args.dtype == "fp32" else "f16xf32->f32",
            "data": "synthetic",
            "config": {"workload": args.workload, "m": wl.m, "n": wl.n, "nnz": wl.nnz,
                       "Bnrow": int((wl.m + 7) // 8), "Bnnz_rank0": int(info.Bnnz),
                       "fill_rank0": wl.local_nnz / max(1, info.Bnnz),
                       "values": args.dtype, "hybrid_residual_max_popc": int(info.residual_max_popc), "residual_parts": int(info.residual_parts),
                       "residual_nnz_rank0": int(info.residual_nnz),
                       "parallelism": f"row-partition x{world}" + (
                           (" + NCCL all-gather" if args.exchange == "nccl" else " + fused peer-store all-gather")
                           if world > 1 else ""),
                       "l2": ("256 MB L2 flush before every step; step time = spaden_spmv's CUDA events"
                              if flush else "inputs larger than L2 (A > 126 MB), no flush"
                              if info.format_bytes > L2_BYTES else "matrix fits L2, no flush (--l2 warm): warm-L2 number"),
                       "step": wl.step_desc,
                       "reorder": args.reorder if args.reorder == "none" else {
                           "kind": args.reorder, "seconds": wl.reorder_s,
                           "what": "spaden_degree_order + spaden_permute_csr on the GPU (median of 3, wall clock); "
                                   "x and y stay in the permuted space"},
                       **({"exchange": args.exchange} if world > 1 else {})},
            "hbm_gbs": achieved,
            "bytes_per_nnz": {"stored": info.format_bytes / max(1, info.nnz),
                              "moved": abytes / max(1, wl.local_nnz)},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "traffic_source": traffic_src,
                         "frac_of_8tbps_spec": achieved / 8000.0,
                         "peak_kind": f"{peak_kind} copy bandwidth (MEASURED_PEAKS.json hbm_gbs)",
                         "kernel": "spaden_spmv (k_spmv_tiled [+ long-row chunks/fix-up])",
                         "kernel_ms": kavg_ms, "alg_bytes_per_launch": abytes,
                         "kernel_ms_p10_p50_p90": [float(np.percentile(kernel_ms, q)) for q in (10, 50, 90)]},
            "convert": {"seconds": convert_s, "ns_per_nnz": convert_s * 1e9 / max(1, wl.local_nnz),
                        "reps_seconds": conv_times,
                        "what": "median of 5 warm spaden_convert_csr_to_bitmap_ex calls (host wall clock incl. "
                                "allocation and the converter's host synchronisations)"},
            "multi_gpu": split,
            "cusparse_csr": cus,
            "variants": variants,
            "spmm": spmm,
            "spmm_tc": spmm_tc,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": args.steps * n_launch,
            "clocks": clocks,
        }
        print(json.dumps(line), flush=True)
    M.free()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
