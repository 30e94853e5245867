"""A realistic CPU SpMV baseline for bench.py: fp64 CSR loop with
OpenMP on all host cores.  Not the oracle and not the product -- a reported denominator."""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "libcpuspmv.so")
_SRC = os.path.join(_HERE, "cpu_spmv.c")
_lib = None


def build(force: bool = False) -> str:
    if not force and os.path.exists(_LIB) and os.path.getmtime(_LIB) >= os.path.getmtime(_SRC):
        return _LIB
    tmp = _LIB + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", "-O3", "-fopenmp", "-fPIC", "-shared", "-o", tmp, _SRC])
    os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        L.cpu_spmv_f64.restype = None
        L.cpu_spmv_f64.argtypes = [C.c_int64] + [C.c_void_p] * 4 + [C.c_double, C.c_double, C.c_void_p]
        L.cpu_threads.restype = C.c_int
        _lib = L
    return _lib


def spmv_f64(m, row_ptr, col, val, x, alpha, beta, y):
    """y[:m] = alpha*A[:m]*x + beta*y[:m] (in place), all host cores."""
    rp = np.ascontiguousarray(row_ptr, np.int64)
    c = np.ascontiguousarray(col, np.int32)
    v = np.ascontiguousarray(val, np.float64)
    xx = np.ascontiguousarray(x, np.float64)
    assert y.dtype == np.float64 and y.flags.c_contiguous
    lib().cpu_spmv_f64(int(m), rp.ctypes.data, c.ctypes.data, v.ctypes.data, xx.ctypes.data, float(alpha),
                       float(beta), y.ctypes.data)
    return y


def threads() -> int:
    return int(lib().cpu_threads())
