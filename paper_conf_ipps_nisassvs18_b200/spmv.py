"""Thin ctypes binding of libspmv (include/spmv.h).  Argument marshalling only:
every step of the path runs in the library's CUDA kernels; there is no CPU
fallback.  Functions keep the C names (``spmv_features``, ``spmv_convert``,
``spmv_run`` ...) plus a small object layer (``CSR``, ``Handle``) on top.

PyTorch provides device memory (its caching allocator is passed to the library
as the ``spmv_allocator``), streams (``torch.cuda.current_stream()``) and, in
``dist.py``, process groups.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import Dict, Optional

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libspmv.so")

FORMATS = {"coo": 0, "ell": 1, "csr": 2, "hyb": 3, "merge": 4, "csr5": 5, "csr_scalar": 6}
FORMAT_NAMES = {v: k for k, v in FORMATS.items()}
#: the six formats of the study in the paper's Fig. 3 order
PAPER_FORMATS = ("coo", "ell", "csr", "hyb", "merge", "csr5")
STATUS = {0: "SPMV_OK", 1: "SPMV_ERR_INVALID_ARG", 2: "SPMV_ERR_NOT_CANONICAL", 3: "SPMV_ERR_SIZE",
          4: "SPMV_ERR_NO_MEMORY", 5: "SPMV_ERR_CUDA", 6: "SPMV_ERR_UNSUPPORTED"}
ARRAYS = {"row_ptr": 0, "col": 1, "val": 2, "coo_row": 3, "ell_col": 4, "ell_val": 5, "hyb_coo_col": 6,
          "hyb_coo_val": 7, "merge_coord_row": 8, "merge_coord_nz": 9, "csr5_tile_ptr": 10,
          "csr5_row_lo": 11, "csr5_tile_desc": 12, "csr5_map_off": 13, "csr5_seg_map": 14,
          "csr_chunk_row": 15, "csr_chunk_lo": 16, "merge_tile_class": 17,
          "merge_tile_order": 18, "hot_cols": 19}


class SpmvError(RuntimeError):
    def __init__(self, status: int, detail: str):
        self.status = status
        self.name = STATUS.get(status, str(status))
        super().__init__(f"{self.name}: {detail}")


# ----------------------------------------------------------------- C types

class spmv_csr(C.Structure):
    _fields_ = [("n_rows", C.c_int64), ("n_cols", C.c_int64), ("nnz", C.c_int64),
                ("ptr_type", C.c_int), ("row_ptr", C.c_void_p), ("col_idx", C.c_void_p),
                ("vals", C.c_void_p), ("dtype", C.c_int)]


class spmv_features_t(C.Structure):
    _fields_ = [
        ("n_rows", C.c_int64), ("n_cols", C.c_int64), ("nnz_tot", C.c_int64),
        ("nnz_mu", C.c_double), ("nnz_frac", C.c_double),
        ("nnz_max", C.c_int64), ("nnz_sigma", C.c_double),
        ("nnzb_mu", C.c_double), ("nnzb_sigma", C.c_double),
        ("snzb_mu", C.c_double), ("snzb_sigma", C.c_double),
        ("nnzb_tot", C.c_int64), ("nnzb_min", C.c_int64), ("nnzb_max", C.c_int64),
        ("snzb_min", C.c_int64), ("snzb_max", C.c_int64), ("nnz_min", C.c_int64),
        ("ell_width", C.c_int64), ("ell_slots", C.c_int64), ("ell_pad_frac", C.c_double),
        ("hyb_width", C.c_int64), ("hyb_coo_nnz", C.c_int64),
        ("hyb_width_floor", C.c_int64), ("hyb_width_cusp", C.c_int64),
        ("n_empty_rows", C.c_int64),
        ("sum_len2", C.c_uint64), ("sum_nnzb2", C.c_uint64), ("sum_snzb2", C.c_uint64),
    ]


#: the 17 features of Table II under the names of Figs 4-5
PAPER_FEATURES = ("n_rows", "n_cols", "nnz_tot", "nnz_mu", "nnz_frac",                 # set 1
                  "nnz_max", "nnz_sigma", "nnzb_mu", "nnzb_sigma", "snzb_mu", "snzb_sigma",  # set 2
                  "nnzb_tot", "nnzb_min", "nnzb_max", "snzb_min", "snzb_max", "nnz_min")    # set 3


class spmv_convert_opts(C.Structure):
    _fields_ = [("hyb_rule", C.c_int), ("hyb_width", C.c_int64), ("csr5_sigma", C.c_int),
                ("merge_items", C.c_int), ("vector_width", C.c_int), ("max_bytes", C.c_size_t),
                ("alias_input", C.c_int), ("index64", C.c_int), ("csr_chunk", C.c_int64),
                ("hot_x", C.c_int64), ("features", C.POINTER(spmv_features_t))]


class spmv_handle_info(C.Structure):
    _fields_ = [("format", C.c_int), ("dtype", C.c_int), ("ptr_type", C.c_int),
                ("n_rows", C.c_int64), ("n_cols", C.c_int64), ("nnz", C.c_int64),
                ("ell_width", C.c_int64), ("ell_ld", C.c_int64), ("hyb_coo_nnz", C.c_int64),
                ("csr5_sigma", C.c_int64), ("csr5_tiles", C.c_int64), ("csr5_map_len", C.c_int64),
                ("merge_items", C.c_int64), ("merge_tiles", C.c_int64), ("vector_width", C.c_int64),
                ("csr_chunks", C.c_int64), ("hot_cols", C.c_int64), ("device_bytes", C.c_size_t),
                ("bytes_per_run", C.c_size_t),
                ("bytes_per_run_beta0", C.c_size_t)]


_ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_int, C.c_void_p, C.c_void_p)
_FREE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_size_t, C.c_int, C.c_void_p, C.c_void_p)


class spmv_allocator(C.Structure):
    _fields_ = [("alloc", _ALLOC_FN), ("free", _FREE_FN), ("user", C.c_void_p)]


_lib = None
_P = C.c_void_p


def lib():
    """Load libspmv.so; fails loudly if it was not built (no fallback)."""
    global _lib
    if _lib is None:
        path = os.environ.get("SPMV_LIB_PATH", LIB_PATH)   # A/B experiments (tools/): another build
        if not os.path.exists(path):
            raise RuntimeError(f"{path} is missing: build it with __graft_entry__.build() "
                               "(there is no CPU fallback)")
        L = C.CDLL(path)
        sig = {
            "spmv_abi_version": (C.c_int, []),
            "spmv_init": (C.c_int, [C.c_int, C.POINTER(spmv_allocator), C.POINTER(_P)]),
            "spmv_finalize": (C.c_int, [_P]),
            "spmv_device_info": (C.c_int, [_P, C.POINTER(C.c_int), C.POINTER(C.c_int64)]),
            "spmv_features": (C.c_int, [_P, C.POINTER(spmv_csr), _P, C.POINTER(spmv_features_t)]),
            "spmv_convert_opts_default": (None, [C.POINTER(spmv_convert_opts)]),
            "spmv_convert": (C.c_int, [_P, C.c_int, C.POINTER(spmv_csr), C.POINTER(spmv_convert_opts), _P,
                                       C.POINTER(_P)]),
            "spmv_run": (C.c_int, [_P, _P, _P, _P, _P, _P]),
            "spmv_run_host": (C.c_int, [_P, _P, _P, _P, _P, _P]),
            "spmv_run_host_multi": (C.c_int, [C.POINTER(_P), C.c_int, _P, _P, _P, _P, C.POINTER(_P), _P]),
            "spmv_run_launches": (C.c_int, [_P, C.POINTER(C.c_int)]),
            "spmv_info": (C.c_int, [_P, C.POINTER(spmv_handle_info)]),
            "spmv_export": (C.c_int, [_P, C.c_int, _P, C.c_size_t, C.POINTER(C.c_size_t), _P]),
            "spmv_destroy": (C.c_int, [_P, _P]),
            "spmv_partition": (C.c_int, [_P, C.POINTER(spmv_csr), C.c_int, _P, C.POINTER(C.c_int64)]),
            "spmv_slice_size": (C.c_int, [_P, C.POINTER(spmv_csr), C.POINTER(C.c_int64), C.c_int, C.c_int, _P,
                                          C.POINTER(C.c_int64), C.POINTER(C.c_int64), C.POINTER(C.c_int64)]),
            "spmv_slice_remap": (C.c_int, [_P, C.POINTER(spmv_csr), C.POINTER(C.c_int64), C.c_int, C.c_int, _P,
                                           _P, _P, _P]),
            "spmv_partition_colmap": (C.c_int, [_P, C.POINTER(spmv_csr), C.POINTER(C.c_int64), C.c_int, _P, _P,
                                                C.POINTER(C.c_int64)]),
            "spmv_slice_remap_colmap": (C.c_int, [_P, C.POINTER(spmv_csr), C.POINTER(C.c_int64), C.c_int, C.c_int,
                                                  _P, _P, _P, _P, _P]),
            "spmv_colmap_pack_index": (C.c_int, [_P, _P, C.POINTER(C.c_int64), C.c_int, C.c_int, C.c_int64, _P, _P,
                                                 C.POINTER(C.c_int64)]),
            "spmv_gather": (C.c_int, [_P, C.c_int, _P, _P, C.c_int64, _P, _P]),
            "spmv_scatter": (C.c_int, [_P, C.c_int, _P, _P, C.c_int64, _P, _P]),
            "spmv_compress_rows": (C.c_int, [_P, C.POINTER(spmv_csr), _P, _P, _P, C.POINTER(C.c_int64)]),
            "spmv_halo_colmap": (C.c_int, [_P, C.POINTER(spmv_csr), C.POINTER(C.c_int64), C.c_int, C.c_int, _P, _P,
                                           C.POINTER(C.c_int64), C.POINTER(C.c_int64)]),
            "spmv_slice_split": (C.c_int, [_P, C.POINTER(spmv_csr), C.POINTER(C.c_int64), C.c_int, C.c_int, _P,
                                           C.c_int, _P, _P, _P, _P, C.POINTER(C.c_int64)]),
            "spmv_status_str": (C.c_char_p, [C.c_int]),
            "spmv_last_error": (C.c_char_p, []),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _check(status: int):
    if status != 0:
        raise SpmvError(status, (lib().spmv_last_error() or b"").decode())


def _stream_ptr(stream=None) -> Optional[int]:
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream or None


# ----------------------------------------------------------------- context

class Context:
    """One spmv_ctx per device; allocations go through torch's caching allocator."""

    def __init__(self, device: int = 0):
        self.device = device
        L = lib()

        def _alloc(nbytes, dev, stream, user):
            with torch.cuda.device(dev):
                return torch.cuda.caching_allocator_alloc(int(nbytes), dev, stream or 0)

        def _free(ptr, nbytes, dev, stream, user):
            with torch.cuda.device(dev):
                torch.cuda.caching_allocator_delete(ptr)

        self._cb = (_ALLOC_FN(_alloc), _FREE_FN(_free))
        self._alloc = spmv_allocator(self._cb[0], self._cb[1], None)
        p = _P()
        torch.cuda.init()
        _check(L.spmv_init(device, C.byref(self._alloc), C.byref(p)))
        self.ptr = p
        sm = C.c_int()
        l2 = C.c_int64()
        _check(L.spmv_device_info(p, C.byref(sm), C.byref(l2)))
        self.sm_count, self.l2_bytes = sm.value, l2.value

    def __del__(self):
        try:
            if getattr(self, "ptr", None):
                lib().spmv_finalize(self.ptr)
        except Exception:
            pass


_ctxs: Dict[int, Context] = {}


def context(device: Optional[int] = None) -> Context:
    dev = torch.cuda.current_device() if device is None else int(device)
    if dev not in _ctxs:
        _ctxs[dev] = Context(dev)
    return _ctxs[dev]


# ----------------------------------------------------------------- matrices

class CSR:
    """Canonical CSR on the GPU: row_ptr int32/int64, col int32, val fp32/fp64 (torch CUDA tensors)."""

    def __init__(self, row_ptr: torch.Tensor, col: torch.Tensor, val: torch.Tensor, shape):
        assert row_ptr.is_cuda and col.is_cuda and val.is_cuda, "CSR tensors must live on the GPU"
        assert row_ptr.dtype in (torch.int32, torch.int64) and col.dtype == torch.int32
        assert val.dtype in (torch.float32, torch.float64)
        self.row_ptr, self.col, self.val = row_ptr.contiguous(), col.contiguous(), val.contiguous()
        self.n_rows, self.n_cols = int(shape[0]), int(shape[1])
        self.nnz = int(col.numel())
        assert self.row_ptr.numel() == self.n_rows + 1

    @classmethod
    def from_host(cls, A, dtype=torch.float64, device=None, ptr_dtype=None):
        """From a host CSR (row_ptr/col/val numpy arrays, n_rows/n_cols) -- copy to the GPU."""
        dev = torch.device("cuda", torch.cuda.current_device() if device is None else device)
        nnz = int(A.row_ptr[-1]) if len(A.row_ptr) else 0
        if ptr_dtype is None:
            ptr_dtype = torch.int32 if nnz <= 2 ** 31 - 1 else torch.int64
        rp = torch.from_numpy(np.ascontiguousarray(A.row_ptr)).to(dev).to(ptr_dtype)
        col = torch.from_numpy(np.ascontiguousarray(A.col, dtype=np.int32)).to(dev)
        val = torch.from_numpy(np.ascontiguousarray(A.val)).to(dev).to(dtype)
        return cls(rp, col, val, (A.n_rows, A.n_cols))

    @property
    def dtype(self):
        return self.val.dtype

    def as_c(self) -> spmv_csr:
        return spmv_csr(self.n_rows, self.n_cols, self.nnz, 0 if self.row_ptr.dtype == torch.int32 else 1,
                        self.row_ptr.data_ptr(), self.col.data_ptr() if self.nnz else None,
                        self.val.data_ptr() if self.nnz else None, 1 if self.val.dtype == torch.float64 else 0)

    def bytes(self) -> int:
        return self.row_ptr.numel() * self.row_ptr.element_size() + self.nnz * (4 + self.val.element_size())


# ----------------------------------------------------------------- C-named entry points

def spmv_features(A: CSR, stream=None) -> dict:
    """Table II features + extras, computed on the GPU (blocking)."""
    ctx = context(A.row_ptr.device.index)
    f = spmv_features_t()
    a = A.as_c()
    _check(lib().spmv_features(ctx.ptr, C.byref(a), _stream_ptr(stream), C.byref(f)))
    return {name: getattr(f, name) for name, _ in spmv_features_t._fields_}


features = spmv_features


def convert_opts(**kw) -> spmv_convert_opts:
    o = spmv_convert_opts()
    lib().spmv_convert_opts_default(C.byref(o))
    rules = {"ceil": 0, "floor": 1, "cusp": 2}
    for k, v in kw.items():
        if k == "hyb_rule" and isinstance(v, str):
            v = rules[v]
        if k == "features":
            if v is None:
                continue
            ft = spmv_features_t(**{name: v[name] for name, _ in spmv_features_t._fields_})
            o._features_keep = ft                      # alive as long as the opts struct
            v = C.pointer(ft)
        setattr(o, k, v)
    return o


def spmv_convert(A: CSR, fmt, stream=None, **opts) -> "Handle":
    """CSR -> fmt on the GPU.  Raises SpmvError(SPMV_ERR_SIZE) for an
    infeasible ELL/HYB (A4), SpmvError(SPMV_ERR_NOT_CANONICAL) for bad input (A15)."""
    ctx = context(A.row_ptr.device.index)
    f = FORMATS[fmt] if isinstance(fmt, str) else int(fmt)
    o = convert_opts(**opts)
    a = A.as_c()
    h = _P()
    _check(lib().spmv_convert(ctx.ptr, f, C.byref(a), C.byref(o), _stream_ptr(stream), C.byref(h)))
    return Handle(h, ctx, A)


convert = spmv_convert


def run_host_multi(handles, alpha, x: np.ndarray, beta, y_in: Optional[np.ndarray], y_outs, stream=None):
    """spmv_run_host_multi: k handles of one matrix on the same host x / y_in (copied to the
    device once), result i copied back into y_outs[i] (host arrays of n_rows)."""
    hs = list(handles)
    if not hs or len(y_outs) != len(hs):
        raise ValueError("one output array per handle")
    h0 = hs[0]
    a, b = h0._scalar(alpha), h0._scalar(beta)
    arr = (_P * len(hs))(*[h.ptr for h in hs])
    outs = (_P * len(hs))(*[(y.ctypes.data if y.size else None) for y in y_outs])
    yin = y_in.ctypes.data if (y_in is not None and y_in.size) else None
    _check(lib().spmv_run_host_multi(arr, len(hs), C.byref(a), x.ctypes.data if x.size else None, C.byref(b),
                                     yin, outs, _stream_ptr(stream)))
    return y_outs


def spmv_partition(A: CSR, nparts: int, stream=None) -> np.ndarray:
    ctx = context(A.row_ptr.device.index)
    out = (C.c_int64 * (nparts + 1))()
    a = A.as_c()
    _check(lib().spmv_partition(ctx.ptr, C.byref(a), int(nparts), _stream_ptr(stream), out))
    return np.array(out[:], dtype=np.int64)


partition = spmv_partition


def spmv_slice_remap(A: CSR, splits, part: int, stream=None):
    """Shard `part` with columns remapped to gathered-x slots.  Returns (CSR shard, slot S)."""
    ctx = context(A.row_ptr.device.index)
    sp = np.ascontiguousarray(splits, dtype=np.int64)
    P = sp.size - 1
    csp = (C.c_int64 * sp.size)(*sp.tolist())
    a = A.as_c()
    rows, nnz, slot = C.c_int64(), C.c_int64(), C.c_int64()
    st = _stream_ptr(stream)
    _check(lib().spmv_slice_size(ctx.ptr, C.byref(a), csp, P, int(part), st, C.byref(rows), C.byref(nnz),
                                 C.byref(slot)))
    dev = A.row_ptr.device
    rp = torch.empty(rows.value + 1, dtype=torch.int32, device=dev)
    col = torch.empty(nnz.value, dtype=torch.int32, device=dev)
    val = torch.empty(nnz.value, dtype=A.val.dtype, device=dev)
    _check(lib().spmv_slice_remap(ctx.ptr, C.byref(a), csp, P, int(part), st, rp.data_ptr(),
                                  col.data_ptr() if nnz.value else None, val.data_ptr() if nnz.value else None))
    return CSR(rp, col, val, (rows.value, P * slot.value)), slot.value


slice_remap = spmv_slice_remap


def _splits_c(splits):
    sp = np.ascontiguousarray(splits, dtype=np.int64)
    return sp, (C.c_int64 * sp.size)(*sp.tolist())


def spmv_partition_colmap(A: CSR, splits, stream=None):
    """Compressed exchange map: int32 device colmap[n_cols] and slot S'."""
    ctx = context(A.row_ptr.device.index)
    sp, csp = _splits_c(splits)
    colmap = torch.empty(A.n_cols, dtype=torch.int32, device=A.row_ptr.device)
    slot = C.c_int64()
    a = A.as_c()
    _check(lib().spmv_partition_colmap(ctx.ptr, C.byref(a), csp, sp.size - 1, _stream_ptr(stream),
                                       colmap.data_ptr() if A.n_cols else None, C.byref(slot)))
    return colmap, slot.value


def spmv_slice_remap_colmap(A: CSR, splits, part: int, colmap: torch.Tensor, slot: int, stream=None) -> CSR:
    """Shard `part` with columns mapped through the compressed colmap."""
    ctx = context(A.row_ptr.device.index)
    sp, csp = _splits_c(splits)
    P = sp.size - 1
    a = A.as_c()
    rows, nnz, dslot = C.c_int64(), C.c_int64(), C.c_int64()
    st = _stream_ptr(stream)
    _check(lib().spmv_slice_size(ctx.ptr, C.byref(a), csp, P, int(part), st, C.byref(rows), C.byref(nnz),
                                 C.byref(dslot)))
    dev = A.row_ptr.device
    rp = torch.empty(rows.value + 1, dtype=torch.int32, device=dev)
    col = torch.empty(nnz.value, dtype=torch.int32, device=dev)
    val = torch.empty(nnz.value, dtype=A.val.dtype, device=dev)
    _check(lib().spmv_slice_remap_colmap(ctx.ptr, C.byref(a), csp, P, int(part), colmap.data_ptr(), st,
                                         rp.data_ptr(), col.data_ptr() if nnz.value else None,
                                         val.data_ptr() if nnz.value else None))
    return CSR(rp, col, val, (rows.value, P * slot))


def spmv_colmap_pack_index(colmap: torch.Tensor, splits, part: int, slot: int, stream=None) -> torch.Tensor:
    """Local positions (int32 device) of part `part`'s exchanged columns, in slot order."""
    ctx = context(colmap.device.index)
    sp, csp = _splits_c(splits)
    rows = int(sp[part + 1] - sp[part])
    idx = torch.empty(max(rows, 1), dtype=torch.int32, device=colmap.device)
    cnt = C.c_int64()
    _check(lib().spmv_colmap_pack_index(ctx.ptr, colmap.data_ptr(), csp, sp.size - 1, int(part), int(slot),
                                        _stream_ptr(stream), idx.data_ptr(), C.byref(cnt)))
    return idx[: cnt.value]


def spmv_halo_colmap(A: CSR, splits, part: int, stream=None):
    """Halo map of receiver `part`: (int32 device colmap[n_cols], per-owner
    counts (numpy int64), slot S)."""
    ctx = context(A.row_ptr.device.index)
    sp, csp = _splits_c(splits)
    P = sp.size - 1
    colmap = torch.empty(max(A.n_cols, 1), dtype=torch.int32, device=A.row_ptr.device)
    counts = np.zeros(P, dtype=np.int64)
    slot = C.c_int64()
    a = A.as_c()
    _check(lib().spmv_halo_colmap(ctx.ptr, C.byref(a), csp, P, int(part), _stream_ptr(stream), colmap.data_ptr(),
                                  counts.ctypes.data_as(C.POINTER(C.c_int64)), C.byref(slot)))
    return colmap[: A.n_cols], counts, slot.value


def spmv_slice_split(A: CSR, splits, part: int, which: int, colmap: Optional[torch.Tensor] = None,
                     slot: Optional[int] = None, stream=None) -> CSR:
    """Own (which=0, columns index the rank's x slice) or foreign (which=1, columns index the
    gathered x) block of shard `part`."""
    ctx = context(A.row_ptr.device.index)
    sp, csp = _splits_c(splits)
    P = sp.size - 1
    a = A.as_c()
    rows = int(sp[part + 1] - sp[part])
    dev = A.row_ptr.device
    rp = torch.empty(rows + 1, dtype=torch.int32, device=dev)
    nnz = C.c_int64()
    st = _stream_ptr(stream)
    cm = colmap.data_ptr() if colmap is not None else None
    _check(lib().spmv_slice_split(ctx.ptr, C.byref(a), csp, P, int(part), cm, int(which), st, rp.data_ptr(), None,
                                  None, C.byref(nnz)))
    col = torch.empty(nnz.value, dtype=torch.int32, device=dev)
    val = torch.empty(nnz.value, dtype=A.val.dtype, device=dev)
    _check(lib().spmv_slice_split(ctx.ptr, C.byref(a), csp, P, int(part), cm, int(which), st, rp.data_ptr(),
                                  col.data_ptr() if nnz.value else None, val.data_ptr() if nnz.value else None,
                                  C.byref(nnz)))
    if which == 0:
        n_cols = rows
    else:
        S = slot if slot is not None else int(np.max(np.diff(sp)))
        n_cols = P * S
    return CSR(rp, col, val, (rows, n_cols))


def spmv_gather(src: torch.Tensor, idx: torch.Tensor, dst: torch.Tensor, stream=None):
    """dst[q] = src[idx[q]] on the GPU (the per-step compressed-slot packing)."""
    ctx = context(src.device.index)
    n = idx.numel()
    dt = 1 if src.dtype == torch.float64 else 0
    _check(lib().spmv_gather(ctx.ptr, dt, src.data_ptr() if src.numel() else None,
                             idx.data_ptr() if n else None, n, dst.data_ptr() if dst.numel() else None,
                             _stream_ptr(stream)))
    return dst


def spmv_scatter(src: torch.Tensor, idx: torch.Tensor, dst: torch.Tensor, stream=None):
    """dst[idx[q]] = src[q] on the GPU (idx distinct; the inverse of spmv_gather, A33)."""
    ctx = context(src.device.index)
    n = idx.numel()
    dt = 1 if src.dtype == torch.float64 else 0
    _check(lib().spmv_scatter(ctx.ptr, dt, src.data_ptr() if src.numel() else None,
                              idx.data_ptr() if n else None, n, dst.data_ptr() if dst.numel() else None,
                              _stream_ptr(stream)))
    return dst


def spmv_compress_rows(A: CSR, stream=None):
    """A's non-empty rows (int32 [count]) and their row starts followed by nnz ([count + 1],
    A's index type): (rows, rp) with CSR(rp, A.col, A.val) the compressed-row block (A33)."""
    ctx = context(A.row_ptr.device.index)
    n = A.n_rows
    dev = A.row_ptr.device
    rows = torch.empty(max(n, 1), dtype=torch.int32, device=dev)
    rp = torch.empty(n + 1, dtype=A.row_ptr.dtype, device=dev)
    cnt = C.c_int64()
    a = A.as_c()
    _check(lib().spmv_compress_rows(ctx.ptr, C.byref(a), _stream_ptr(stream), rows.data_ptr(), rp.data_ptr(),
                                    C.byref(cnt)))
    k = cnt.value
    return rows[:k], rp[:k + 1]


# ----------------------------------------------------------------- handle

class Handle:
    """An spmv_handle: A in one format, owned device arrays, run() on the current stream."""

    def __init__(self, ptr, ctx: Context, A: CSR):
        self.ptr = ptr
        self.ctx = ctx
        self.dtype = A.val.dtype
        self._src = A  # keeps aliased inputs alive
        info = self.info()
        self.format = FORMAT_NAMES[info["format"]]
        self.n_rows, self.n_cols, self.nnz = info["n_rows"], info["n_cols"], info["nnz"]

    def _scalar(self, v):
        return C.c_double(v) if self.dtype == torch.float64 else C.c_float(v)

    def run(self, alpha, x: torch.Tensor, beta, y: torch.Tensor, stream=None):
        """y <- alpha*A*x + beta*y on the GPU (spmv_run; asynchronous)."""
        assert x.dtype == self.dtype and y.dtype == self.dtype and x.is_cuda and y.is_cuda
        assert x.is_contiguous() and y.is_contiguous()
        assert x.numel() == self.n_cols and y.numel() == self.n_rows
        a, b = self._scalar(alpha), self._scalar(beta)
        _check(lib().spmv_run(self.ptr, C.byref(a), x.data_ptr() if x.numel() else None, C.byref(b),
                              y.data_ptr() if y.numel() else None, _stream_ptr(stream)))
        return y

    def run_host(self, alpha, x: np.ndarray, beta, y: np.ndarray, stream=None):
        """End-to-end: host x/y (pinned or pageable numpy), H2D + run + D2H (spmv_run_host)."""
        a, b = self._scalar(alpha), self._scalar(beta)
        _check(lib().spmv_run_host(self.ptr, C.byref(a), x.ctypes.data if x.size else None, C.byref(b),
                                   y.ctypes.data if y.size else None, _stream_ptr(stream)))
        return y

    def launches(self) -> int:
        n = C.c_int()
        _check(lib().spmv_run_launches(self.ptr, C.byref(n)))
        return n.value

    def info(self) -> dict:
        i = spmv_handle_info()
        _check(lib().spmv_info(self.ptr, C.byref(i)))
        return {name: getattr(i, name) for name, _ in spmv_handle_info._fields_}

    def export(self, name: str, stream=None) -> np.ndarray:
        """Copy one of the handle's device arrays to host (bit-exact test access)."""
        aid = ARRAYS[name]
        written = C.c_size_t()
        st = _stream_ptr(stream)
        lib().spmv_export(self.ptr, aid, None, 0, C.byref(written), st)
        nbytes = written.value
        buf = np.empty(nbytes, dtype=np.uint8)
        _check(lib().spmv_export(self.ptr, aid, buf.ctypes.data if nbytes else None, nbytes,
                                 C.byref(written), st))
        vb = 8 if self.dtype == torch.float64 else 4
        itype = np.int32 if self.info()["ptr_type"] == 0 else np.int64
        dt = {"row_ptr": itype, "col": np.int32, "val": np.float64 if vb == 8 else np.float32,
              "coo_row": np.int32, "ell_col": np.int32, "ell_val": np.float64 if vb == 8 else np.float32,
              "hyb_coo_col": np.int32, "hyb_coo_val": np.float64 if vb == 8 else np.float32,
              "merge_coord_row": np.int64, "merge_coord_nz": np.int64, "csr5_tile_ptr": np.int64,
              "csr5_row_lo": np.int64, "csr5_tile_desc": np.uint32, "csr5_map_off": np.int64,
              "csr5_seg_map": np.int64, "csr_chunk_row": np.int64, "csr_chunk_lo": np.int64,
              "merge_tile_class": np.uint8, "merge_tile_order": np.int32, "hot_cols": np.int32}[name]
        return buf.view(dt)

    def destroy(self, stream=None):
        if getattr(self, "ptr", None):
            lib().spmv_destroy(self.ptr, _stream_ptr(stream))
            self.ptr = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


def spmv_run(h: Handle, alpha, x, beta, y, stream=None):
    return h.run(alpha, x, beta, y, stream)


def spmv_info(h: Handle) -> dict:
    return h.info()


def spmv_export(h: Handle, name: str) -> np.ndarray:
    return h.export(name)


def spmv_destroy(h: Handle):
    h.destroy()
