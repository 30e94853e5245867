"""Seeded synthetic sparse-matrix generators (input generation only).

Shared by the oracle tests and the CUDA path; contains none of the method's
arithmetic.  Heavy loops live in ``matgen/matgen.c`` (counter-based hashing, so
every output is a pure function of its seed and parameters).  Recipes and seeds
are listed in DESIGN.md §5 (workload shapes of BASELINE.json ``configs``).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libmatgen.so")

VALUE_KINDS = {"f64": 0, "f32": 1, "int": 2, "ones": 3}

SEEDS = {"u2048": 0x5EED0001, "lap4096": 0x5EED0002, "rmat24": 0x5EED0003,
         "sweep": 0x5EED1000, "rmat27": 0x5EED0005}


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "matgen.c")
    if not force and os.path.exists(_LIB_PATH) and os.path.getmtime(_LIB_PATH) >= os.path.getmtime(src):
        return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-fopenmp", "-fPIC", "-shared",
                           "-Wall", "-o", tmp, src])
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


_lib = None
_p = C.c_void_p
_i64 = C.c_int64
_u64 = C.c_uint64


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB_PATH)
        sig = {
            "mg_hash3": (_u64, [_u64, _u64, _u64]),
            "mg_vector": (None, [_u64, _u64, _i64, C.c_int, _p]),
            "mg_matrix_values": (None, [_u64, _i64, _p, _p, C.c_int, _p]),
            "mg_fill_random_rows": (C.c_int, [_u64, _i64, _i64, _p, _p]),
            "mg_laplacian5": (_i64, [_i64, _p, _p, _p]),
            "mg_rmat_keys": (None, [_u64, C.c_int, _i64, C.c_uint32, C.c_uint32, C.c_uint32, _p]),
            "mg_sort_unique": (_i64, [_p, _p, _i64, C.c_int]),
            "mg_keys_to_csr": (None, [_p, _i64, C.c_int, _i64, _p, _p]),
            "mg_window_rows": (None, [_u64, C.c_int, _i64, _i64, _i64, C.c_uint32, _p, _p, _p]),
            "mg_num_threads": (C.c_int, []),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _ptr(a):
    return a.ctypes.data if a is not None else None


@dataclass
class HostCSR:
    """Canonical host CSR: int64 row_ptr, int32 col (sorted, unique per row), fp64 val."""
    row_ptr: np.ndarray
    col: np.ndarray
    val: np.ndarray
    n_rows: int
    n_cols: int
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1]) if self.row_ptr.size else 0

    @property
    def shape(self):
        return (self.n_rows, self.n_cols)

    def lengths(self):
        return np.diff(self.row_ptr)


def vector(n, seed, stream=1, kind="f64"):
    out = np.empty(int(n), dtype=np.float64)
    if n > 0:
        lib().mg_vector(int(seed), int(stream), int(n), VALUE_KINDS[kind], _ptr(out))
    return out


def set_values(A: HostCSR, seed, kind="f64") -> HostCSR:
    """Position-keyed values: val(i,j) = f(hash(seed, i, j)) (A18)."""
    val = np.empty(A.nnz, dtype=np.float64)
    if A.nnz:
        lib().mg_matrix_values(int(seed), A.n_rows, _ptr(A.row_ptr), _ptr(A.col), VALUE_KINDS[kind], _ptr(val))
    return HostCSR(A.row_ptr, A.col, val, A.n_rows, A.n_cols, A.name)


def from_lengths(lengths, n_cols, seed, kind="f64", name="") -> HostCSR:
    """Rows with the given lengths, columns uniform without replacement, sorted."""
    lengths = np.asarray(lengths, dtype=np.int64)
    n_rows = lengths.size
    if np.any(lengths > n_cols) or np.any(lengths < 0):
        raise ValueError("row length out of range")
    row_ptr = np.zeros(n_rows + 1, dtype=np.int64)
    np.cumsum(lengths, out=row_ptr[1:])
    col = np.empty(int(row_ptr[-1]), dtype=np.int32)
    if n_rows:
        rc = lib().mg_fill_random_rows(int(seed), n_rows, int(n_cols), _ptr(row_ptr), _ptr(col))
        assert rc == 0
    A = HostCSR(row_ptr, col, np.empty(0), n_rows, int(n_cols), name)
    return set_values(A, seed + 7, kind)


def uniform_fixed(n_rows, n_cols, d, seed=SEEDS["u2048"], kind="f64") -> HostCSR:
    """cfg1: each row exactly d distinct uniform columns."""
    return from_lengths(np.full(n_rows, d, dtype=np.int64), n_cols, seed, kind,
                        name=f"uniform{n_rows}x{n_cols}d{d}")


def laplacian5(g, kind=None, seed=SEEDS["lap4096"]) -> HostCSR:
    """cfg2: 5-point Laplacian on a g x g grid (diag 4, off -1), natural ordering.
    kind=None keeps the exact stencil values; otherwise values are re-drawn."""
    n = g * g
    row_ptr = np.empty(n + 1, dtype=np.int64)
    nnz_cap = 5 * n
    col = np.empty(nnz_cap, dtype=np.int32)
    val = np.empty(nnz_cap, dtype=np.float64)
    nnz = lib().mg_laplacian5(int(g), _ptr(row_ptr), _ptr(col), _ptr(val))
    A = HostCSR(row_ptr, col[:nnz].copy(), val[:nnz].copy(), n, n, f"lap{g}")
    if kind is not None:
        A = set_values(A, seed, kind)
    return A


def rmat(scale, edge_factor=16, seed=SEEDS["rmat24"], abc=(0.57, 0.19, 0.19), kind="f64") -> HostCSR:
    """cfg3/cfg5: R-MAT (Graph500 parameters), duplicates coalesced, self loops kept,
    no vertex permutation (A18)."""
    n = 1 << scale
    E = edge_factor * n
    a, b, c = abc
    ta = min(int(round(a * 2 ** 32)), 2 ** 32 - 1)
    tab = min(int(round((a + b) * 2 ** 32)), 2 ** 32 - 1)
    tabc = min(int(round((a + b + c) * 2 ** 32)), 2 ** 32 - 1)
    keys = np.empty(E, dtype=np.uint64)
    lib().mg_rmat_keys(int(seed), int(scale), int(E), ta, tab, tabc, _ptr(keys))
    tmp = np.empty(E, dtype=np.uint64)
    m = lib().mg_sort_unique(_ptr(keys), _ptr(tmp), int(E), 2 * scale)
    del tmp
    row_ptr = np.empty(n + 1, dtype=np.int64)
    col = np.empty(m, dtype=np.int32)
    lib().mg_keys_to_csr(_ptr(keys), int(m), int(scale), int(n), _ptr(row_ptr), _ptr(col))
    del keys
    A = HostCSR(row_ptr, col, np.empty(0), n, n, f"rmat{scale}")
    return set_values(A, seed + 11, kind)


def window(n_rows, n_cols, w, p, seed, mode, kind="f64", name="") -> HostCSR:
    """Banded (mode 0, half-width w) or block-diagonal (mode 1, block w) with fill p."""
    thr = 0xFFFFFFFF if p >= 1.0 else int(p * 2 ** 32)
    lens = np.empty(n_rows, dtype=np.int64)
    lib().mg_window_rows(int(seed), int(mode), int(n_rows), int(n_cols), int(w), thr, _ptr(lens), None, None)
    row_ptr = np.zeros(n_rows + 1, dtype=np.int64)
    np.cumsum(lens, out=row_ptr[1:])
    col = np.empty(int(row_ptr[-1]), dtype=np.int32)
    lib().mg_window_rows(int(seed), int(mode), int(n_rows), int(n_cols), int(w), thr, None, _ptr(row_ptr), _ptr(col))
    A = HostCSR(row_ptr, col, np.empty(0), int(n_rows), int(n_cols), name)
    return set_values(A, seed + 13, kind)


def from_dense(D) -> HostCSR:
    """Small helper for tests: dense -> canonical CSR (exact zeros dropped)."""
    D = np.asarray(D, dtype=np.float64)
    n, m = D.shape
    rows, cols = np.nonzero(D)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(row_ptr, rows + 1, 1)
    np.cumsum(row_ptr, out=row_ptr)
    return HostCSR(row_ptr, cols.astype(np.int32), D[rows, cols].copy(), n, m, "dense")


def from_rows(rows, n_cols) -> HostCSR:
    """rows: list of lists of (col, val) -> canonical CSR (caller keeps cols sorted)."""
    row_ptr = [0]
    col, val = [], []
    for r in rows:
        for c, v in r:
            col.append(c)
            val.append(v)
        row_ptr.append(len(col))
    return HostCSR(np.array(row_ptr, dtype=np.int64), np.array(col, dtype=np.int32),
                   np.array(val, dtype=np.float64), len(rows), int(n_cols), "rows")
