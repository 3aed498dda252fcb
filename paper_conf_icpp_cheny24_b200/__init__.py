"""Thin Python binding (ctypes) over libspaden.so -- the C ABI in include/spaden.h.

Argument marshalling only: every step of CSR->bitBSR conversion and SpMV runs
in the library's CUDA kernels.  PyTorch supplies device memory and streams.
There is no CPU fallback: importing this package on a machine without the
built library raises ImportError, and every call on a missing device fails.

Raw entry points keep the C names (spaden_convert_csr_to_bitmap, spaden_count_blocks, spaden_spmv,
spaden_spmv_host, spaden_free, spaden_get_info, spaden_get_arrays, spaden_spmv_launch_count,
spaden_status_string, spaden_last_error_message, spaden_version); `convert`
and `Matrix` wrap them for torch tensors.
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SPADEN_LIB") or os.path.join(_PKG, "libspaden.so")  # override: A/B experiments

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_icpp_cheny24_b200.build` "
                      "(or __graft_entry__.build()); there is no fallback implementation")

_lib = ctypes.CDLL(LIB_PATH)

SPADEN_OK = 0
SPADEN_ERR_INVALID_ARGUMENT = 1
SPADEN_ERR_INDEX_OUT_OF_RANGE = 2
SPADEN_ERR_UNSORTED_OR_DUPLICATE = 3
SPADEN_ERR_UNSUPPORTED = 4
SPADEN_ERR_OUT_OF_MEMORY = 5
SPADEN_ERR_CUDA = 6
SPADEN_R_32F = 0
SPADEN_R_16F = 1


class spaden_info_t(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int64), ("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("Bnrow", ctypes.c_int64), ("Bnnz", ctypes.c_int64),
                ("storage_dtype", ctypes.c_int32), ("device", ctypes.c_int32),
                ("format_bytes", ctypes.c_int64), ("aux_bytes", ctypes.c_int64),
                ("n_tiles", ctypes.c_int64), ("n_long", ctypes.c_int64), ("residual_nnz", ctypes.c_int64),
                ("residual_max_popc", ctypes.c_int32), ("residual_parts", ctypes.c_int32)]


class spaden_arrays_t(ctypes.Structure):
    _fields_ = [("blk_rowptr", ctypes.c_void_p), ("blk_col", ctypes.c_void_p),
                ("bitmap", ctypes.c_void_p), ("blk_offset", ctypes.c_void_p),
                ("values", ctypes.c_void_p), ("res_rowptr", ctypes.c_void_p),
                ("res_colidx", ctypes.c_void_p), ("res_values", ctypes.c_void_p)]


class spaden_convert_opts_t(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_int32), ("residual_max_popc", ctypes.c_int32),
                ("auto_mean_fill", ctypes.c_float), ("reserved", ctypes.c_int32 * 5)]


_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_ST = ctypes.c_int
_F = ctypes.c_float

spaden_convert_csr_to_bitmap = _lib.spaden_convert_csr_to_bitmap
spaden_convert_csr_to_bitmap.argtypes = [_I64, _I64, _I64, _P, _P, _P, ctypes.c_int, ctypes.c_int, _P,
                                         ctypes.POINTER(_P)]
spaden_convert_csr_to_bitmap.restype = _ST
spaden_convert_csr_to_bitmap_ex = _lib.spaden_convert_csr_to_bitmap_ex
spaden_convert_csr_to_bitmap_ex.argtypes = [_I64, _I64, _I64, _P, _P, _P, ctypes.c_int, ctypes.c_int,
                                            ctypes.POINTER(spaden_convert_opts_t), _P, ctypes.POINTER(_P)]
spaden_convert_csr_to_bitmap_ex.restype = _ST
spaden_count_blocks = _lib.spaden_count_blocks
spaden_count_blocks.argtypes = [_I64, _I64, _I64, _P, _P, _P, ctypes.POINTER(_I64)]
spaden_count_blocks.restype = _ST
spaden_degree_order = _lib.spaden_degree_order
spaden_degree_order.argtypes = [_I64, _P, _P, _P]
spaden_degree_order.restype = _ST
spaden_permute_csr = _lib.spaden_permute_csr
spaden_permute_csr.argtypes = [_I64, _I64, _P, _P, _P, ctypes.c_int, _P, _P, _P, _P, _P]
spaden_permute_csr.restype = _ST
spaden_spmv = _lib.spaden_spmv
spaden_spmv.argtypes = [_P, _F, _P, _F, _P, _P]
spaden_spmv.restype = _ST
spaden_spmv_scatter = _lib.spaden_spmv_scatter
spaden_spmv_scatter.argtypes = [_P, _F, _P, _F, _P, ctypes.POINTER(_P), ctypes.c_int32, _I64, _P]
spaden_spmv_scatter.restype = _ST
spaden_spmm = _lib.spaden_spmm
spaden_spmm.argtypes = [_P, _F, _P, _I64, ctypes.c_int32, _F, _P, _I64, _P]
spaden_spmm.restype = _ST
spaden_spmm_tc_pack_x = _lib.spaden_spmm_tc_pack_x
spaden_spmm_tc_pack_x.argtypes = [_I64, ctypes.c_int32, _P, _I64, _P, _P]
spaden_spmm_tc_pack_x.restype = _ST
spaden_spmm_tc_xb_bytes = _lib.spaden_spmm_tc_xb_bytes
spaden_spmm_tc_xb_bytes.argtypes = [_I64, ctypes.c_int32]
spaden_spmm_tc_xb_bytes.restype = _I64
spaden_spmm_tc = _lib.spaden_spmm_tc
spaden_spmm_tc.argtypes = [_P, _F, _P, ctypes.c_int32, _F, _P, _I64, _P]
spaden_spmm_tc.restype = _ST
spaden_spmv_host = _lib.spaden_spmv_host
spaden_spmv_host.argtypes = [_P, _F, _P, _F, _P, _P]
spaden_spmv_host.restype = _ST
spaden_spmv_host_batched = _lib.spaden_spmv_host_batched
spaden_spmv_host_batched.argtypes = [_P, _F, _P, _I64, _F, _P, _I64, _I64, _P]
spaden_spmv_host_batched.restype = _ST
spaden_free = _lib.spaden_free
spaden_free.argtypes = [_P]
spaden_free.restype = _ST
spaden_get_info = _lib.spaden_get_info
spaden_get_info.argtypes = [_P, ctypes.POINTER(spaden_info_t)]
spaden_get_info.restype = _ST
spaden_spmv_launch_count = _lib.spaden_spmv_launch_count
spaden_spmv_launch_count.argtypes = [_P, _F, ctypes.POINTER(ctypes.c_int32)]
spaden_spmv_launch_count.restype = _ST
spaden_get_arrays = _lib.spaden_get_arrays
spaden_get_arrays.argtypes = [_P, ctypes.POINTER(spaden_arrays_t)]
spaden_get_arrays.restype = _ST
spaden_status_string = _lib.spaden_status_string
spaden_status_string.argtypes = [_ST]
spaden_status_string.restype = ctypes.c_char_p
spaden_last_error_message = _lib.spaden_last_error_message
spaden_last_error_message.argtypes = []
spaden_last_error_message.restype = ctypes.c_char_p
spaden_version = _lib.spaden_version
spaden_version.argtypes = []
spaden_version.restype = ctypes.c_char_p

EXPORTED = ["spaden_convert_csr_to_bitmap", "spaden_convert_csr_to_bitmap_ex", "spaden_count_blocks",
            "spaden_degree_order", "spaden_permute_csr", "spaden_spmv", "spaden_spmm",
            "spaden_spmv_scatter", "spaden_spmm_tc_pack_x", "spaden_spmm_tc_xb_bytes", "spaden_spmm_tc", "spaden_spmv_host", "spaden_spmv_host_batched",
            "spaden_free",
            "spaden_get_info", "spaden_get_arrays", "spaden_spmv_launch_count", "spaden_status_string",
            "spaden_last_error_message", "spaden_version"]


class SpadenError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = spaden_last_error_message().decode(errors="replace")
        super().__init__(f"{where}: {spaden_status_string(status).decode()} ({msg})")


def _check(status: int, where: str):
    if status != SPADEN_OK:
        raise SpadenError(status, where)


def _torch():
    import torch
    return torch


def _stream_ptr(stream):
    torch = _torch()
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _dtype_code(dt) -> int:
    torch = _torch()
    if dt in (torch.float32, "fp32", "f32", "float32", SPADEN_R_32F):
        return SPADEN_R_32F
    if dt in (torch.float16, "fp16", "f16", "float16", SPADEN_R_16F):
        return SPADEN_R_16F
    raise ValueError(f"unsupported dtype {dt!r}")


class _CudaArray:
    """__cuda_array_interface__ shim to view a library-owned device array."""

    def __init__(self, ptr: int, shape, typestr: str, owner):
        self.__cuda_array_interface__ = {"data": (ptr or 0, False), "shape": tuple(shape),
                                         "typestr": typestr, "version": 3, "strides": None}
        self._owner = owner


class Matrix:
    """Owning wrapper of a spaden_matrix_t (bitBSR on one device)."""

    def __init__(self, handle: ctypes.c_void_p, device):
        self._h = handle
        self.device = device
        self.info = self.get_info()

    @property
    def handle(self):
        return self._h

    def get_info(self) -> spaden_info_t:
        inf = spaden_info_t()
        _check(spaden_get_info(self._h, ctypes.byref(inf)), "spaden_get_info")
        return inf

    @property
    def m(self):
        return self.info.m

    @property
    def n(self):
        return self.info.n

    @property
    def nnz(self):
        return self.info.nnz

    def arrays(self):
        """Borrowed torch views (on device) of blk_rowptr, blk_col, bitmap, blk_offset, values."""
        torch = _torch()
        a = spaden_arrays_t()
        _check(spaden_get_arrays(self._h, ctypes.byref(a)), "spaden_get_arrays")
        i = self.info
        vt = "<f2" if i.storage_dtype == SPADEN_R_16F else "<f4"
        tdt = {"<i4": torch.int32, "<i8": torch.int64, "<f2": torch.float16, "<f4": torch.float32}

        def mk(p, n, t):
            if n == 0 or not p:
                return torch.empty(0, dtype=tdt[t], device=self.device)
            return torch.as_tensor(_CudaArray(p, (n,), t, self), device=self.device)
        out = {"blk_rowptr": mk(a.blk_rowptr, i.Bnrow + 1, "<i4"),
               "blk_col": mk(a.blk_col, i.Bnnz, "<i4"),
               "bitmap": mk(a.bitmap, i.Bnnz, "<i8"),       # uint64 bits viewed as int64
               "blk_offset": mk(a.blk_offset, i.Bnnz + 1, "<i4"),
               "values": mk(a.values, i.nnz - i.residual_nnz, vt)}
        if a.res_rowptr:
            out["res_rowptr"] = mk(a.res_rowptr, i.m + 1, "<i4")
            out["res_colidx"] = mk(a.res_colidx, i.residual_nnz, "<i4")
            out["res_values"] = mk(a.res_values, i.residual_nnz, vt)
        return out

    def launch_count(self, beta: float = 0.0) -> int:
        """Kernel launches (and memsets) one spmv(..., beta) call issues (bench accounting)."""
        c = ctypes.c_int32()
        _check(spaden_spmv_launch_count(self._h, beta, ctypes.byref(c)), "spaden_spmv_launch_count")
        return c.value

    def spmv(self, x, y=None, alpha: float = 1.0, beta: float = 0.0, stream=None):
        """y = alpha * A x + beta * y on the device (x, y float32 CUDA tensors)."""
        torch = _torch()
        if y is None:
            y = torch.empty(self.m, dtype=torch.float32, device=x.device)
        assert x.dtype == torch.float32 and y.dtype == torch.float32
        assert x.is_cuda and y.is_cuda and x.is_contiguous() and y.is_contiguous()
        assert x.numel() == self.n and y.numel() == self.m
        _check(spaden_spmv(self._h, alpha, ctypes.c_void_p(x.data_ptr()), beta,
                           ctypes.c_void_p(y.data_ptr()), _stream_ptr(stream)), "spaden_spmv")
        return y

    def spmv_scatter(self, x, out_ptrs, out_offset: int, y=None, alpha: float = 1.0, beta: float = 0.0,
                     stream=None):
        """Fused SpMV + all-gather store: y values written to every out_ptrs[p] + out_offset
        (device addresses as ints, e.g. symmetric-memory peer buffers)."""
        torch = _torch()
        assert x.dtype == torch.float32 and x.is_cuda and x.is_contiguous() and x.numel() == self.n
        if y is not None:
            assert y.dtype == torch.float32 and y.is_cuda and y.is_contiguous() and y.numel() == self.m
        arr = (ctypes.c_void_p * len(out_ptrs))(*[ctypes.c_void_p(int(p)) for p in out_ptrs])
        _check(spaden_spmv_scatter(self._h, alpha, ctypes.c_void_p(x.data_ptr()), beta,
                                   ctypes.c_void_p(y.data_ptr()) if y is not None else None,
                                   ctypes.cast(arr, ctypes.POINTER(ctypes.c_void_p)), len(out_ptrs),
                                   int(out_offset), _stream_ptr(stream)), "spaden_spmv_scatter")

    def spmm(self, X, Y=None, alpha: float = 1.0, beta: float = 0.0, stream=None):
        """Y[j] = alpha * A X[j] + beta * Y[j] for the rows j of X (k x n, CUDA float32,
        rows contiguous) -> Y (k x m)."""
        torch = _torch()
        k = X.shape[0]
        if Y is None:
            Y = torch.empty((k, self.m), dtype=torch.float32, device=X.device)
        assert X.dtype == torch.float32 and Y.dtype == torch.float32 and X.is_cuda and Y.is_cuda
        assert X.shape[1] == self.n and Y.shape == (k, self.m) and X.stride(1) == 1 and Y.stride(1) == 1
        _check(spaden_spmm(self._h, alpha, ctypes.c_void_p(X.data_ptr()), X.stride(0), k, beta,
                           ctypes.c_void_p(Y.data_ptr()), Y.stride(0), _stream_ptr(stream)), "spaden_spmm")
        return Y

    def pack_x_tc(self, X, Xb=None, stream=None):
        """fp16 x slabs for spmm_tc (spaden_spmm_tc_pack_x): X is k x n (CUDA float32, rows
        contiguous); returns a uint8 CUDA tensor of 2048 * ceil(n/8) * ceil(k/128) bytes."""
        torch = _torch()
        k = X.shape[0]
        assert X.dtype == torch.float32 and X.is_cuda and X.shape[1] == self.n and X.stride(1) == 1
        nbytes = int(spaden_spmm_tc_xb_bytes(self.n, k))
        if Xb is None:
            Xb = torch.empty(max(16, nbytes), dtype=torch.uint8, device=X.device)
        assert Xb.numel() >= nbytes and Xb.is_cuda
        _check(spaden_spmm_tc_pack_x(self.n, k, ctypes.c_void_p(X.data_ptr()), X.stride(0),
                                     ctypes.c_void_p(Xb.data_ptr()), _stream_ptr(stream)), "spaden_spmm_tc_pack_x")
        return Xb

    def spmm_tc(self, Xb, k: int, Y=None, alpha: float = 1.0, beta: float = 0.0, stream=None):
        """Y[j] = alpha * A x_j + beta * Y[j] on the tensor cores (spaden_spmm_tc) from the
        fp16 slabs of pack_x_tc; Y is k x m (CUDA float32, rows contiguous)."""
        torch = _torch()
        if Y is None:
            Y = torch.empty((k, self.m), dtype=torch.float32, device=Xb.device)
        assert Y.dtype == torch.float32 and Y.is_cuda and Y.shape == (k, self.m) and Y.stride(1) == 1
        _check(spaden_spmm_tc(self._h, alpha, ctypes.c_void_p(Xb.data_ptr()), k, beta,
                              ctypes.c_void_p(Y.data_ptr()), Y.stride(0), _stream_ptr(stream)), "spaden_spmm_tc")
        return Y

    def spmv_host(self, x_host, y_host, alpha: float = 1.0, beta: float = 0.0, stream=None):
        """Host-buffer variant (H2D x, SpMV, D2H y, stream sync) through the C ABI."""
        _check(spaden_spmv_host(self._h, alpha, ctypes.c_void_p(x_host.data_ptr()), beta,
                                ctypes.c_void_p(y_host.data_ptr()), _stream_ptr(stream)), "spaden_spmv_host")
        return y_host

    def spmv_host_batched(self, X_host, Y_host, alpha: float = 1.0, beta: float = 0.0, stream=None):
        """Rows of X_host (k x n, pinned) -> rows of Y_host (k x m); copies overlap the SpMVs."""
        k = X_host.shape[0]
        assert Y_host.shape[0] == k and X_host.stride(1) == 1 and Y_host.stride(1) == 1
        _check(spaden_spmv_host_batched(self._h, alpha, ctypes.c_void_p(X_host.data_ptr()), X_host.stride(0), beta,
                                        ctypes.c_void_p(Y_host.data_ptr()), Y_host.stride(0), k,
                                        _stream_ptr(stream)), "spaden_spmv_host_batched")
        return Y_host

    def free(self):
        if self._h:
            _check(spaden_free(self._h), "spaden_free")
            self._h = None

    def __del__(self):
        try:
            if self._h:
                spaden_free(self._h)
                self._h = None
        except Exception:
            pass


def count_blocks(rowptr, colidx, n: int, stream=None) -> int:
    """Non-empty 8x8 blocks (Bnnz) of a CSR matrix: the converter's validation and
    count pass only (spaden_count_blocks)."""
    torch = _torch()
    assert rowptr.dtype == torch.int32 and colidx.dtype == torch.int32 and rowptr.is_cuda and colidx.is_cuda
    out = ctypes.c_int64()
    _check(spaden_count_blocks(rowptr.numel() - 1, n, colidx.numel(), ctypes.c_void_p(rowptr.data_ptr()),
                               ctypes.c_void_p(colidx.data_ptr()), _stream_ptr(stream), ctypes.byref(out)),
           "spaden_count_blocks")
    return out.value


def degree_order(rowptr, stream=None):
    """perm (int32 CUDA tensor): rows by descending degree, ties by ascending index
    (spaden_degree_order; SURVEY.md §8(f) NEXT-1 reordering)."""
    torch = _torch()
    assert rowptr.dtype == torch.int32 and rowptr.is_cuda
    m = rowptr.numel() - 1
    perm = torch.empty(max(m, 0), dtype=torch.int32, device=rowptr.device)
    _check(spaden_degree_order(m, ctypes.c_void_p(rowptr.data_ptr()), ctypes.c_void_p(perm.data_ptr()),
                               _stream_ptr(stream)), "spaden_degree_order")
    return perm


def permute_csr(rowptr, colidx, values, perm, stream=None):
    """B = P A P^T of a square CSR matrix (spaden_permute_csr): row k of B is row
    perm[k] of A, columns renamed by the inverse permutation and sorted.  Returns
    (rowptr, colidx, values) CUDA tensors."""
    torch = _torch()
    assert rowptr.dtype == torch.int32 and colidx.dtype == torch.int32 and perm.dtype == torch.int32
    m = rowptr.numel() - 1
    nnz = colidx.numel()
    rp = torch.empty(m + 1, dtype=torch.int32, device=rowptr.device)
    ci = torch.empty(nnz, dtype=torch.int32, device=rowptr.device)
    v = torch.empty(nnz, dtype=values.dtype, device=rowptr.device)
    _check(spaden_permute_csr(m, nnz, ctypes.c_void_p(rowptr.data_ptr()), ctypes.c_void_p(colidx.data_ptr()),
                              ctypes.c_void_p(values.data_ptr()), _dtype_code(values.dtype),
                              ctypes.c_void_p(perm.data_ptr()), ctypes.c_void_p(rp.data_ptr()),
                              ctypes.c_void_p(ci.data_ptr()), ctypes.c_void_p(v.data_ptr()), _stream_ptr(stream)),
           "spaden_permute_csr")
    return rp, ci, v


def convert(rowptr, colidx, values, n: int, storage=None, stream=None, residual_max_popc: int = 0,
            auto_mean_fill: float = 0.0) -> Matrix:
    """CSR (int32 CUDA tensors + fp32/fp16 values) -> bitBSR Matrix (hybrid with a CSR
    residual for blocks of <= residual_max_popc entries when that is > 0; -1 = automatic:
    4 when the mean block fill is below 8, else pure bitBSR; the fill used is
    auto_mean_fill when > 0 -- a row slice passes the whole matrix's)."""
    torch = _torch()
    assert rowptr.dtype == torch.int32 and colidx.dtype == torch.int32
    assert rowptr.is_cuda and colidx.is_cuda and values.is_cuda
    vdt = _dtype_code(values.dtype)
    sdt = vdt if storage is None else _dtype_code(storage)
    m = rowptr.numel() - 1
    h = ctypes.c_void_p()
    opts = spaden_convert_opts_t(ctypes.sizeof(spaden_convert_opts_t), int(residual_max_popc),
                                 float(auto_mean_fill))
    st = spaden_convert_csr_to_bitmap_ex(m, n, colidx.numel(), ctypes.c_void_p(rowptr.data_ptr()),
                                         ctypes.c_void_p(colidx.data_ptr()),
                                         ctypes.c_void_p(values.data_ptr()), vdt, sdt, ctypes.byref(opts),
                                         _stream_ptr(stream), ctypes.byref(h))
    _check(st, "spaden_convert_csr_to_bitmap")
    return Matrix(h, rowptr.device)
