"""CPU-side checks of the C-ABI boundary: the library loads and exports every symbol
include/spmv.h declares; status strings; no device => SPMV_ERR_UNSUPPORTED (no
compute call is made without a GPU)."""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "spmv.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = set(re.findall(r"\b(spmv_[a-z_0-9]+)\s*\(", src))
    return sorted(n for n in names if not n.endswith("_t"))


@pytest.fixture(scope="module")
def L():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_ipps_nisassvs18_b200 import spmv
    return spmv.lib()


def test_every_declared_symbol_is_exported(L):
    names = declared_functions()
    assert len(names) >= 18, names
    for n in names:
        assert hasattr(L, n), f"libspmv.so does not export {n}"


def test_abi_version_and_status_strings(L):
    assert L.spmv_abi_version() == 3
    for code, name in [(0, b"SPMV_OK"), (2, b"SPMV_ERR_NOT_CANONICAL"), (3, b"SPMV_ERR_SIZE"),
                       (6, b"SPMV_ERR_UNSUPPORTED")]:
        assert L.spmv_status_str(code) == name


def test_init_without_device_is_unsupported(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    p = C.c_void_p()
    st = L.spmv_init(0, None, C.byref(p))
    assert st == 6 and not p.value
    assert b"no CUDA device" in L.spmv_last_error()


def test_product_does_not_import_oracle():
    """The product package must not reference the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_nisassvs18_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", txt, re.M), f
                assert "oracle.h" not in txt and "liboracle" not in txt, f


def test_sm100a_only_build_flags():
    from paper_conf_ipps_nisassvs18_b200 import build_lib
    flags = " ".join(build_lib.NVCC_FLAGS)
    assert "arch=compute_100a,code=sm_100a" in flags and "-lineinfo" in flags
