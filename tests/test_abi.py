"""CPU-only checks of the C-ABI boundary: libspaden.so loads, exports every
symbol include/spaden.h declares, and rejects bad arguments before touching a
GPU.  No compute calls."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "spaden.h")


@pytest.fixture(scope="module")
def sp():
    from paper_conf_icpp_cheny24_b200 import build
    build.build()
    import paper_conf_icpp_cheny24_b200 as sp
    return sp


def declared_functions():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"SPADEN_API\s+[\w\s\*]+?\b(spaden_\w+)\s*\(", src)))


def test_header_declares_the_boundary():
    fns = declared_functions()
    for f in ["spaden_convert_csr_to_bitmap", "spaden_spmv", "spaden_free"]:
        assert f in fns
    assert len(fns) >= 9


def test_library_exports_every_declared_symbol(sp):
    out = subprocess.check_output(["nm", "-D", "--defined-only", sp.LIB_PATH], text=True)
    exported = {l.split()[-1] for l in out.splitlines() if " T " in l}
    for f in declared_functions():
        assert f in exported, f
        assert hasattr(sp._lib, f)
    assert set(sp.EXPORTED) == set(declared_functions())


def test_library_is_sm100a(sp):
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", sp.LIB_PATH], text=True)
    assert "sm_100a" in out


def test_status_strings_and_version(sp):
    for code, name in [(0, "SPADEN_OK"), (1, "SPADEN_ERR_INVALID_ARGUMENT"), (2, "SPADEN_ERR_INDEX_OUT_OF_RANGE"),
                       (3, "SPADEN_ERR_UNSORTED_OR_DUPLICATE"), (4, "SPADEN_ERR_UNSUPPORTED"),
                       (5, "SPADEN_ERR_OUT_OF_MEMORY"), (6, "SPADEN_ERR_CUDA")]:
        assert sp.spaden_status_string(code).decode() == name
    assert b"sm_100a" in sp.spaden_version()


def test_rejects_bad_arguments_without_gpu(sp):
    h = ctypes.c_void_p(1234)
    dummy = ctypes.c_void_p(8)
    st = sp.spaden_convert_csr_to_bitmap(-1, 4, 0, dummy, None, None, 0, 0, None, ctypes.byref(h))
    assert st == sp.SPADEN_ERR_INVALID_ARGUMENT and h.value is None
    assert b"must be >= 0" in sp.spaden_last_error_message()
    st = sp.spaden_convert_csr_to_bitmap(4, 4, 0, dummy, None, None, 0, 7, None, ctypes.byref(h))
    assert st == sp.SPADEN_ERR_UNSUPPORTED
    st = sp.spaden_convert_csr_to_bitmap(4, 4, 3, dummy, None, None, 0, 0, None, ctypes.byref(h))
    assert st == sp.SPADEN_ERR_INVALID_ARGUMENT
    st = sp.spaden_convert_csr_to_bitmap(1 << 31, 4, 0, dummy, None, None, 0, 0, None, ctypes.byref(h))
    assert st == sp.SPADEN_ERR_UNSUPPORTED
    st = sp.spaden_convert_csr_to_bitmap(4, 4, 0, dummy, None, None, 0, 0, None, None)
    assert st == sp.SPADEN_ERR_INVALID_ARGUMENT
    assert sp.spaden_spmv(None, 1.0, dummy, 0.0, dummy, None) == sp.SPADEN_ERR_INVALID_ARGUMENT
    assert sp.spaden_spmv_host(None, 1.0, dummy, 0.0, dummy, None) == sp.SPADEN_ERR_INVALID_ARGUMENT
    assert sp.spaden_free(None) == sp.SPADEN_OK
    assert sp.spaden_get_info(None, None) == sp.SPADEN_ERR_INVALID_ARGUMENT
    assert sp.spaden_get_arrays(None, None) == sp.SPADEN_ERR_INVALID_ARGUMENT


def test_product_does_not_touch_oracle():
    """The product package never imports or links the oracle (and vice versa)."""
    pkg = os.path.join(ROOT, "paper_conf_icpp_cheny24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                bad = re.search(r"\bimport oracle\b|\bfrom oracle\b|liboracle|#include[^\n]*oracle", txt)
                assert bad is None, os.path.join(dirpath, f)
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c", ".h")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            assert "paper_conf_icpp_cheny24_b200" not in txt.replace("paper_conf_icpp_cheny24_b200/csrc", "")
            assert re.search(r"#include[^\n]*spaden", txt) is None
