"""GPU twins of the host generators (INPUT GENERATION ONLY; matgen/matgen_gpu.cu).

SURVEY §2.2 G15 / §8(d) d1 cfg5: R-MAT generated on the GPU (counter-based RNG ->
radix sort -> unique), bit-identical to ``matgen.rmat`` (same hash, same keys, same
position-keyed values), so a rank can build the matrix -- or only its rows' values --
without a host copy (R-MAT 27: 2.1e9 nonzeros, ~80 GB of host RAM through the host
generator).  torch only allocates device memory and supplies the stream.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import torch

from . import SEEDS, VALUE_KINDS

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libmatgen_gpu.so")
_SRC = os.path.join(_HERE, "matgen_gpu.cu")


def build(force: bool = False) -> str:
    if not force and os.path.exists(_LIB_PATH) and os.path.getmtime(_LIB_PATH) >= os.path.getmtime(_SRC):
        return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17",
                           "-Xcompiler", "-fPIC", "-shared", "-o", tmp, _SRC, "-lcudart_static", "-lrt", "-ldl",
                           "-lpthread"])
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
            "mgg_rmat_keys": (C.c_int, [_u64, C.c_int, _i64, C.c_uint32, C.c_uint32, C.c_uint32, _p, _p]),
            "mgg_sort_unique_temp_bytes": (_i64, [_i64, C.c_int]),
            "mgg_sort_unique": (_i64, [_p, _p, _i64, C.c_int, _p, _i64, _p, _p]),
            "mgg_keys_row_ptr": (C.c_int, [_p, _i64, C.c_int, _i64, _p, _p]),
            "mgg_keys_col": (C.c_int, [_p, _i64, _i64, C.c_int, _p, _p]),
            "mgg_keys_values": (C.c_int, [_u64, _p, _i64, _i64, C.c_int, C.c_int, C.c_int, _p, _p]),
            "mgg_vector": (C.c_int, [_u64, _u64, _i64, _i64, C.c_int, C.c_int, _p, _p]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _stream():
    return torch.cuda.current_stream().cuda_stream or None


def _chk(rc, what):
    if rc < 0:
        raise RuntimeError(f"{what}: CUDA error {-rc}")
    return rc


def vector(n, seed, stream=1, kind="f64", dtype=torch.float64, i0=0, device=None) -> torch.Tensor:
    """Entries [i0, i0+n) of matgen.vector(N, seed, stream, kind), on the GPU."""
    out = torch.empty(int(n), dtype=dtype, device=device or "cuda")
    _chk(lib().mgg_vector(int(seed), int(stream), int(i0), int(n), VALUE_KINDS[kind], int(dtype == torch.float32),
                          out.data_ptr() if n else None, _stream()), "mgg_vector")
    return out


class DeviceRMAT:
    """R-MAT (Graph500 parameters, duplicates coalesced, self loops kept, no vertex
    permutation; A18) built on the current GPU, identical to ``matgen.rmat``.

    After construction: ``row_ptr`` (int64 [n+1]) and ``nnz``; the sorted unique keys
    stay resident until ``release()`` so that ``values(k0, k1)`` / ``col(k0, k1)`` can
    materialise any nonzero range (a rank's own rows only)."""

    def __init__(self, scale, edge_factor=16, seed=SEEDS["rmat24"], abc=(0.57, 0.19, 0.19), device=None):
        L = lib()
        self.scale, self.seed = int(scale), int(seed)
        self.n = 1 << self.scale
        E = int(edge_factor) * self.n
        a, b, c = abc
        ta = min(int(round(a * 2 ** 32)), 2 ** 32 - 1)
        tab = min(int(round((a + b) * 2 ** 32)), 2 ** 32 - 1)
        tabc = min(int(round((a + b + c) * 2 ** 32)), 2 ** 32 - 1)
        dev = torch.device(device or "cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        s = _stream()
        keys = torch.empty(E, dtype=torch.int64, device=dev)
        _chk(L.mgg_rmat_keys(self.seed, self.scale, E, ta, tab, tabc, keys.data_ptr(), s), "mgg_rmat_keys")
        tb = L.mgg_sort_unique_temp_bytes(E, 2 * self.scale)
        tmp = torch.empty(E, dtype=torch.int64, device=dev)
        temp = torch.empty(max(int(tb), 16), dtype=torch.uint8, device=dev)
        cnt = torch.empty(1, dtype=torch.int64, device=dev)
        m = _chk(L.mgg_sort_unique(keys.data_ptr(), tmp.data_ptr(), E, 2 * self.scale, temp.data_ptr(), int(tb),
                                   cnt.data_ptr(), s), "mgg_sort_unique")
        del tmp, temp
        self._keys = keys[:m]
        self.nnz = int(m)
        self.row_ptr = torch.empty(self.n + 1, dtype=torch.int64, device=dev)
        _chk(L.mgg_keys_row_ptr(self._keys.data_ptr(), m, self.scale, self.n, self.row_ptr.data_ptr(), s),
             "mgg_keys_row_ptr")

    def col(self, k0=0, k1=None) -> torch.Tensor:
        k1 = self.nnz if k1 is None else int(k1)
        out = torch.empty(max(k1 - k0, 0), dtype=torch.int32, device=self.row_ptr.device)
        _chk(lib().mgg_keys_col(self._keys.data_ptr(), int(k0), k1, self.scale, out.data_ptr() if k1 > k0 else None,
                                _stream()), "mgg_keys_col")
        return out

    def values(self, k0=0, k1=None, kind="f64", dtype=torch.float64) -> torch.Tensor:
        """Values of nonzeros [k0, k1): matgen.rmat's set_values(A, seed + 11, kind)."""
        k1 = self.nnz if k1 is None else int(k1)
        out = torch.empty(max(k1 - k0, 0), dtype=dtype, device=self.row_ptr.device)
        _chk(lib().mgg_keys_values(self.seed + 11, self._keys.data_ptr(), int(k0), k1, self.scale,
                                   VALUE_KINDS[kind], int(dtype == torch.float32),
                                   out.data_ptr() if k1 > k0 else None, _stream()), "mgg_keys_values")
        return out

    def release(self):
        """Drop the keys (col/values can no longer be materialised)."""
        self._keys = None


def rmat(scale, edge_factor=16, seed=SEEDS["rmat24"], abc=(0.57, 0.19, 0.19), kind="f64", dtype=torch.float64):
    """The whole matrix on the GPU: (row_ptr int64, col int32, val) tensors, == matgen.rmat."""
    g = DeviceRMAT(scale, edge_factor, seed, abc)
    col = g.col()
    val = g.values(kind=kind, dtype=dtype)
    rp = g.row_ptr
    g.release()
    return rp, col, val
