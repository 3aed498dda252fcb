"""cuSPARSE CSR SpMV baseline for bench.py (the north_star comparison).

Calls libcusparse directly through ctypes -- cusparseCreateCsr / cusparseCreateDnVec /
cusparseSpMV_bufferSize / cusparseSpMV with CUSPARSE_SPMV_CSR_ALG1 and CSR_ALG2 --
on the same device CSR arrays the bitBSR converter reads, on the caller's stream.
Footprint = CSR arrays + the SpMV external buffer (the
paper's CSR baseline is cuSPARSE).  Comparison harness only: not product code.
"""
from __future__ import annotations

import ctypes
import glob
import os

CUSPARSE_INDEX_32I = 2
CUSPARSE_INDEX_BASE_ZERO = 0
CUDA_R_32F = 0
CUSPARSE_OPERATION_NON_TRANSPOSE = 0
ALGS = {"CSR_ALG1": 2, "CSR_ALG2": 3}

_lib = None


def _load():
    global _lib
    if _lib is not None:
        return _lib
    cands = []
    try:
        import nvidia.cusparse  # torch's bundled copy (the one torch.sparse uses)
        cands += glob.glob(os.path.join(list(nvidia.cusparse.__path__)[0], "lib", "libcusparse.so*"))
    except Exception:
        pass
    cands += ["libcusparse.so.12", "/usr/local/cuda/lib64/libcusparse.so.12"]
    err = None
    for c in cands:
        try:
            _lib = ctypes.CDLL(c)
            break
        except OSError as e:
            err = e
    if _lib is None:
        raise OSError(f"libcusparse not found: {err}")
    P, VP = ctypes.POINTER(ctypes.c_void_p), ctypes.c_void_p
    I64 = ctypes.c_int64
    _lib.cusparseCreate.argtypes = [P]
    _lib.cusparseSetStream.argtypes = [VP, VP]
    _lib.cusparseCreateCsr.argtypes = [P, I64, I64, I64, VP, VP, VP, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                       ctypes.c_int]
    _lib.cusparseCreateDnVec.argtypes = [P, I64, VP, ctypes.c_int]
    _lib.cusparseSpMV_bufferSize.argtypes = [VP, ctypes.c_int, VP, VP, VP, VP, VP, ctypes.c_int, ctypes.c_int,
                                             ctypes.POINTER(ctypes.c_size_t)]
    _lib.cusparseSpMV.argtypes = [VP, ctypes.c_int, VP, VP, VP, VP, VP, ctypes.c_int, ctypes.c_int, VP]
    _lib.cusparseDestroySpMat.argtypes = [VP]
    _lib.cusparseDestroyDnVec.argtypes = [VP]
    _lib.cusparseDestroy.argtypes = [VP]
    return _lib


def _ok(st, what):
    if st != 0:
        raise RuntimeError(f"{what} failed: cusparse status {st}")


def time_spmv(rowptr, colidx, values, x, m, n, stream, reps=200, warmup=5):
    """Time cusparseSpMV (fp32 CSR, int32 indices) for CSR_ALG1 and CSR_ALG2.

    rowptr/colidx/values/x: device torch tensors (int32, int32, float32, float32).
    Returns {alg: {"ms", "buffer_bytes", "footprint_bytes", "y"}}; time = CUDA
    events around `reps` back-to-back calls on `stream` divided by reps.
    """
    import torch

    lib = _load()
    h = ctypes.c_void_p()
    _ok(lib.cusparseCreate(ctypes.byref(h)), "cusparseCreate")
    _ok(lib.cusparseSetStream(h, ctypes.c_void_p(stream.cuda_stream)), "cusparseSetStream")
    nnz = int(colidx.numel())
    A = ctypes.c_void_p()
    _ok(lib.cusparseCreateCsr(ctypes.byref(A), m, n, nnz, rowptr.data_ptr(), colidx.data_ptr(), values.data_ptr(),
                              CUSPARSE_INDEX_32I, CUSPARSE_INDEX_32I, CUSPARSE_INDEX_BASE_ZERO, CUDA_R_32F),
        "cusparseCreateCsr")
    y = torch.zeros(m, dtype=torch.float32, device=x.device)
    vx, vy = ctypes.c_void_p(), ctypes.c_void_p()
    _ok(lib.cusparseCreateDnVec(ctypes.byref(vx), n, x.data_ptr(), CUDA_R_32F), "cusparseCreateDnVec")
    _ok(lib.cusparseCreateDnVec(ctypes.byref(vy), m, y.data_ptr(), CUDA_R_32F), "cusparseCreateDnVec")
    alpha, beta = ctypes.c_float(1.0), ctypes.c_float(0.0)
    out = {}
    csr_bytes = 4 * (m + 1) + 8 * nnz
    try:
        for name, alg in ALGS.items():
            sz = ctypes.c_size_t(0)
            _ok(lib.cusparseSpMV_bufferSize(h, CUSPARSE_OPERATION_NON_TRANSPOSE, ctypes.byref(alpha), A, vx,
                                            ctypes.byref(beta), vy, CUDA_R_32F, alg, ctypes.byref(sz)),
                "cusparseSpMV_bufferSize")
            buf = torch.empty(max(1, sz.value), dtype=torch.uint8, device=x.device)

            def call():
                _ok(lib.cusparseSpMV(h, CUSPARSE_OPERATION_NON_TRANSPOSE, ctypes.byref(alpha), A, vx,
                                     ctypes.byref(beta), vy, CUDA_R_32F, alg, ctypes.c_void_p(buf.data_ptr())),
                    "cusparseSpMV")

            for _ in range(warmup):
                call()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize(x.device)
            e0.record(stream)
            for _ in range(reps):
                call()
            e1.record(stream)
            torch.cuda.synchronize(x.device)
            out[name] = {"ms": e0.elapsed_time(e1) / reps, "buffer_bytes": int(sz.value),
                         "footprint_bytes": csr_bytes + int(sz.value), "y": y.clone()}
            del buf
    finally:
        lib.cusparseDestroyDnVec(vx)
        lib.cusparseDestroyDnVec(vy)
        lib.cusparseDestroySpMat(A)
        lib.cusparseDestroy(h)
    return out
