"""CPU ORACLE (test infrastructure only).

Thin ctypes wrapper over ``oracle/liboracle.so`` (plain C, ``oracle/oracle.c``).
Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
``paper_conf_ipps_nisassvs18_b200`` never imports it and shares no code with it.

Every function follows a passage of /root/reference/PAPER.md (cited in
oracle.c); the readings of ambiguous passages are SURVEY.md §8(c) A1..A22,
restated in DESIGN.md §3.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")

CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
          "-Wall", "-Wextra", "-Wno-unused-parameter"]


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so with gcc (idempotent)."""
    src = os.path.join(_HERE, "oracle.c")
    hdr = os.path.join(_HERE, "oracle.h")
    if (not force and os.path.exists(_LIB_PATH)
            and os.path.getmtime(_LIB_PATH) >= max(os.path.getmtime(src), os.path.getmtime(hdr))):
        return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, src, "-lm"])
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


_lib = None

_i64 = C.c_int64
_p = C.c_void_p


class Features(C.Structure):
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


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB_PATH)
        sig = {
            "ora_spmv_csr": (C.c_int, [_i64, _p, _p, _p, _p, C.c_double, C.c_double, _p, _p, _p]),
            "ora_spmv_coo": (C.c_int, [_i64, _i64, _p, _p, _p, _p, C.c_double, C.c_double, _p, _p]),
            "ora_is_canonical": (C.c_int, [_i64, _i64, _i64, _p, _p]),
            "ora_csr2coo": (C.c_int, [_i64, _p, _p]),
            "ora_ell_width": (_i64, [_i64, _p]),
            "ora_ell_ld": (_i64, [_i64]),
            "ora_csr2ell": (C.c_int, [_i64, _p, _p, _p, _i64, _i64, _p, _p]),
            "ora_hyb_width": (_i64, [_i64, _p, C.c_int]),
            "ora_hyb_coo_nnz": (_i64, [_i64, _p, _i64]),
            "ora_csr2hyb": (C.c_int, [_i64, _p, _p, _p, _i64, _i64, _p, _p, _p, _p, _p]),
            "ora_merge_ntiles": (_i64, [_i64, _i64, _i64]),
            "ora_csr_chunks": (_i64, [_i64, _p, _i64, _p, _p]),
            "ora_compress_rows": (_i64, [_i64, _p, _p, _p]),
            "ora_merge_coords": (C.c_int, [_i64, _p, _i64, _p, _p]),
            "ora_merge_class": (C.c_int, [_i64, _p, _i64, _i64, _i64, _p]),
            "ora_csr5_sigma": (_i64, [_i64, _i64]),
            "ora_csr5_map_len": (_i64, [_i64, _p, _i64]),
            "ora_csr5_encode": (C.c_int, [_i64, _p, _p, _p, _i64, C.c_int,
                                          _p, _p, _p, _p, _p, _p, _p]),
            "ora_csr5_decode": (C.c_int, [_i64, _i64, _p, _i64, C.c_int, _p, _p, _p, _p, _p,
                                          _p, _p, _p, _p, _p]),
            "ora_features": (C.c_int, [_i64, _i64, _p, _p, C.POINTER(Features)]),
            "ora_partition": (C.c_int, [_i64, _p, C.c_int, _p]),
            "ora_partition_slot": (_i64, [_p, C.c_int]),
            "ora_slice_remap": (C.c_int, [_i64, _p, _p, _p, _p, C.c_int, C.c_int, _p, _p, _p]),
            "ora_partition_colmap": (_i64, [_i64, _p, _p, _p, C.c_int, _p]),
            "ora_halo_colmap": (_i64, [_i64, _p, _p, _p, C.c_int, C.c_int, _p, _p]),
            "ora_hot_columns": (_i64, [_i64, _i64, _p, _i64, _p]),
            "ora_slice_remap_colmap": (C.c_int, [_i64, _p, _p, _p, _p, C.c_int, _p, _p, _p, _p]),
            "ora_slice_split": (_i64, [_i64, _p, _p, _p, _p, C.c_int, C.c_int, _p, C.c_int, _p, _p, _p]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


# ----------------------------------------------------------------- helpers

def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def _ptr(a):
    return a.ctypes.data if a is not None and a.size > 0 else (
        a.ctypes.data if a is not None else None)


class CSR:
    """Host CSR as the oracle sees it: int64 row_ptr, int32 col, fp64 val."""

    def __init__(self, row_ptr, col, val, shape):
        self.row_ptr = _c(row_ptr, np.int64)
        self.col = _c(col, np.int32)
        self.val = _c(val, np.float64)
        self.n_rows, self.n_cols = int(shape[0]), int(shape[1])
        self.nnz = int(self.row_ptr[-1]) if self.row_ptr.size else 0
        assert self.row_ptr.size == self.n_rows + 1

    @classmethod
    def of(cls, A):
        if isinstance(A, CSR):
            return A
        return cls(A.row_ptr, A.col, A.val, (A.n_rows, A.n_cols))


def _buf(n, dtype):
    return np.empty(max(int(n), 0), dtype=dtype)


# ----------------------------------------------------------------- SpMV

def spmv_csr(A, x, alpha=1.0, beta=0.0, y=None, with_bound=False):
    """y_ref (fp64) and optionally bound_i = |alpha| sum|a||x| + |beta||y_i| (c2.1)."""
    A = CSR.of(A)
    x = _c(x, np.float64)
    yin = _c(y, np.float64) if y is not None else None
    if beta != 0.0 and yin is None:
        raise ValueError("beta != 0 needs y")
    out = _buf(A.n_rows, np.float64)
    bnd = _buf(A.n_rows, np.float64)
    rc = lib().ora_spmv_csr(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(A.val), _ptr(x),
                            float(alpha), float(beta), _ptr(yin) if yin is not None else None,
                            _ptr(out), _ptr(bnd))
    assert rc == 0
    return (out, bnd) if with_bound else out


def spmv_coo(n_rows, row, col, val, x, alpha=1.0, beta=0.0, y=None):
    row, col, val, x = _c(row, np.int32), _c(col, np.int32), _c(val, np.float64), _c(x, np.float64)
    yin = _c(y, np.float64) if y is not None else None
    out = _buf(n_rows, np.float64)
    rc = lib().ora_spmv_coo(int(n_rows), row.size, _ptr(row), _ptr(col), _ptr(val), _ptr(x),
                            float(alpha), float(beta), _ptr(yin) if yin is not None else None,
                            _ptr(out))
    assert rc == 0
    return out


def is_canonical(A):
    A = CSR.of(A)
    return bool(lib().ora_is_canonical(A.n_rows, A.n_cols, A.nnz, _ptr(A.row_ptr), _ptr(A.col)))


# ----------------------------------------------------------------- converters

def csr2coo(A):
    A = CSR.of(A)
    row = _buf(A.nnz, np.int32)
    lib().ora_csr2coo(A.n_rows, _ptr(A.row_ptr), _ptr(row))
    return row


def ell_dims(A):
    A = CSR.of(A)
    return int(lib().ora_ell_width(A.n_rows, _ptr(A.row_ptr))), int(lib().ora_ell_ld(A.n_rows))


def csr2ell(A):
    A = CSR.of(A)
    K, ld = ell_dims(A)
    col = _buf(K * ld, np.int32)
    val = _buf(K * ld, np.float64)
    rc = lib().ora_csr2ell(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(A.val), K, ld,
                           _ptr(col), _ptr(val))
    assert rc == 0
    return dict(K=K, ld=ld, col=col, val=val)


HYB_RULES = {"ceil": 0, "floor": 1, "cusp": 2}


def hyb_width(A, rule="ceil"):
    A = CSR.of(A)
    return int(lib().ora_hyb_width(A.n_rows, _ptr(A.row_ptr), HYB_RULES[rule]))


def csr2hyb(A, rule="ceil", Kh=None):
    A = CSR.of(A)
    if Kh is None:
        Kh = hyb_width(A, rule)
    ld = int(lib().ora_ell_ld(A.n_rows))
    nc = int(lib().ora_hyb_coo_nnz(A.n_rows, _ptr(A.row_ptr), Kh))
    ec, ev = _buf(Kh * ld, np.int32), _buf(Kh * ld, np.float64)
    cr, cc, cv = _buf(nc, np.int32), _buf(nc, np.int32), _buf(nc, np.float64)
    rc = lib().ora_csr2hyb(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(A.val), Kh, ld,
                           _ptr(ec), _ptr(ev), _ptr(cr), _ptr(cc), _ptr(cv))
    assert rc == 0
    return dict(K=Kh, ld=ld, ell_col=ec, ell_val=ev, coo_row=cr, coo_col=cc, coo_val=cv)


def merge_coords(A, T):
    A = CSR.of(A)
    nt = int(lib().ora_merge_ntiles(A.n_rows, A.nnz, int(T)))
    cr, cn = _buf(nt + 1, np.int64), _buf(nt + 1, np.int64)
    rc = lib().ora_merge_coords(A.n_rows, _ptr(A.row_ptr), int(T), _ptr(cr), _ptr(cn))
    assert rc == 0
    return cr, cn


def merge_class(A, T, max_rows=64, max_len=32):
    """Merge tile class (A28): uint8 per tile, 1 = row-sum tile."""
    A = CSR.of(A)
    nt = int(lib().ora_merge_ntiles(A.n_rows, A.nnz, int(T)))
    cls = _buf(nt, np.uint8)
    rc = lib().ora_merge_class(A.n_rows, _ptr(A.row_ptr), int(T), int(max_rows), int(max_len), _ptr(cls))
    assert rc == 0
    return cls


def csr_chunks(A, C):
    """CSR long-row chunks (A25): (chunk_row, chunk_lo) int64 arrays."""
    A = CSR.of(A)
    m = int(lib().ora_csr_chunks(A.n_rows, _ptr(A.row_ptr), int(C), None, None))
    assert m >= 0
    cr, cl = _buf(max(m, 1), np.int64), _buf(max(m, 1), np.int64)
    lib().ora_csr_chunks(A.n_rows, _ptr(A.row_ptr), int(C), _ptr(cr), _ptr(cl))
    return cr[:m], cl[:m]


def compress_rows(A):
    """Compressed rows (A33): (rows, rp) int64 arrays -- A's non-empty rows and their row
    starts followed by nnz."""
    A = CSR.of(A)
    m = int(lib().ora_compress_rows(A.n_rows, _ptr(A.row_ptr), None, None))
    assert m >= 0
    rows, rp = _buf(max(m, 1), np.int64), _buf(m + 1, np.int64)
    lib().ora_compress_rows(A.n_rows, _ptr(A.row_ptr), _ptr(rows), _ptr(rp))
    return rows[:m], rp


def csr5_sigma(A):
    A = CSR.of(A)
    return int(lib().ora_csr5_sigma(A.n_rows, A.nnz))


def csr5_encode(A, val_bytes=8, sigma=None):
    A = CSR.of(A)
    if sigma is None:
        sigma = csr5_sigma(A)
    W = 32 * sigma
    nt = A.nnz // W
    mlen = int(lib().ora_csr5_map_len(A.n_rows, _ptr(A.row_ptr), sigma))
    out = dict(sigma=sigma, n_tiles=nt,
               tile_ptr=_buf(nt + 1, np.int64), row_lo=_buf(nt + 1, np.int64),
               tile_desc=_buf(nt * 32, np.uint32), map_off=_buf(nt, np.int64),
               seg_map=_buf(mlen, np.int64), col_perm=_buf(A.nnz, np.int32),
               val_perm=_buf(A.nnz, np.float64))
    rc = lib().ora_csr5_encode(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(A.val), sigma,
                               int(val_bytes), _ptr(out["tile_ptr"]), _ptr(out["row_lo"]),
                               _ptr(out["tile_desc"]), _ptr(out["map_off"]), _ptr(out["seg_map"]),
                               _ptr(out["col_perm"]), _ptr(out["val_perm"]))
    assert rc == 0, rc
    return out


def csr5_decode(A_shape_nnz, enc, row_ptr_tail, val_bytes=8):
    """Rebuild (row_ptr, col, val) from the CSR5 arrays; returns (rc, row_ptr, col, val)."""
    n_rows, nnz = A_shape_nnz
    rp = _buf(n_rows + 1, np.int64)
    col = _buf(nnz, np.int32)
    val = _buf(nnz, np.float64)
    tail = _c(row_ptr_tail, np.int64)
    rc = lib().ora_csr5_decode(int(n_rows), int(nnz), _ptr(tail), enc["sigma"], int(val_bytes),
                               _ptr(_c(enc["tile_ptr"], np.int64)), _ptr(_c(enc["row_lo"], np.int64)),
                               _ptr(_c(enc["tile_desc"], np.uint32)), _ptr(_c(enc["map_off"], np.int64)),
                               _ptr(_c(enc["seg_map"], np.int64)), _ptr(_c(enc["col_perm"], np.int32)),
                               _ptr(_c(enc["val_perm"], np.float64)), _ptr(rp), _ptr(col), _ptr(val))
    return rc, rp, col, val


# ----------------------------------------------------------------- features

FEATURE_NAMES = [f for f, _ in Features._fields_]


def features(A):
    A = CSR.of(A)
    f = Features()
    rc = lib().ora_features(A.n_rows, A.n_cols, _ptr(A.row_ptr), _ptr(A.col), C.byref(f))
    assert rc == 0
    return {name: getattr(f, name) for name in FEATURE_NAMES}


# ----------------------------------------------------------------- partition

def partition(A, nparts):
    A = CSR.of(A)
    s = _buf(nparts + 1, np.int64)
    rc = lib().ora_partition(A.n_rows, _ptr(A.row_ptr), int(nparts), _ptr(s))
    assert rc == 0
    return s


def partition_slot(splits):
    s = _c(splits, np.int64)
    return int(lib().ora_partition_slot(_ptr(s), s.size - 1))


def slice_remap(A, splits, part):
    A = CSR.of(A)
    s = _c(splits, np.int64)
    P = s.size - 1
    r0, r1 = int(s[part]), int(s[part + 1])
    nnz_p = int(A.row_ptr[r1] - A.row_ptr[r0])
    rp, col, val = _buf(r1 - r0 + 1, np.int64), _buf(nnz_p, np.int32), _buf(nnz_p, np.float64)
    rc = lib().ora_slice_remap(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(A.val), _ptr(s), P,
                               int(part), _ptr(rp), _ptr(col), _ptr(val))
    assert rc == 0, rc
    return rp, col, val


def partition_colmap(A, splits):
    """Compressed-exchange column map and slot size S'."""
    A = CSR.of(A)
    s = _c(splits, np.int64)
    cm = _buf(A.n_rows, np.int32)
    S = lib().ora_partition_colmap(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(s), s.size - 1, _ptr(cm))
    assert S >= 0
    return cm, int(S)


def hot_columns(A, kmax):
    """A30: the hot x columns of A for a budget of kmax columns (ascending int32)."""
    A = CSR.of(A)
    K = lib().ora_hot_columns(A.n_cols, A.nnz, _ptr(A.col), int(kmax), None)
    assert K >= 0
    out = _buf(K, np.int32)
    lib().ora_hot_columns(A.n_cols, A.nnz, _ptr(A.col), int(kmax), _ptr(out))
    return out


def halo_colmap(A, splits, part):
    """Halo map of receiver `part`: (colmap int32[n], counts int64[P], S)."""
    A = CSR.of(A)
    s = _c(splits, np.int64)
    cm = _buf(A.n_rows, np.int32)
    cnt = _buf(s.size - 1, np.int64)
    S = lib().ora_halo_colmap(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(s), s.size - 1, int(part), _ptr(cm),
                              _ptr(cnt))
    assert S >= 1
    return cm, cnt, int(S)


def halo_pack_index(colmap, splits, sender, S):
    """Sender's pack list for the receiver of `colmap`: local indices j - splits[sender] of
    the sender's columns the receiver references, in slot order (plain loop)."""
    s = np.asarray(splits, np.int64)
    out = [j - int(s[sender]) for j in range(int(s[sender]), int(s[sender + 1])) if colmap[j] >= 0]
    return np.asarray(out, dtype=np.int32)


def slice_remap_colmap(A, splits, part, colmap):
    A = CSR.of(A)
    s = _c(splits, np.int64)
    cm = _c(colmap, np.int32)
    r0, r1 = int(s[part]), int(s[part + 1])
    nnz_p = int(A.row_ptr[r1] - A.row_ptr[r0])
    rp, col, val = _buf(r1 - r0 + 1, np.int64), _buf(nnz_p, np.int32), _buf(nnz_p, np.float64)
    rc = lib().ora_slice_remap_colmap(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(A.val), _ptr(s), int(part),
                                      _ptr(cm), _ptr(rp), _ptr(col), _ptr(val))
    assert rc == 0
    return rp, col, val


def slice_split(A, splits, part, which, colmap=None):
    """Own (which=0) / foreign (which=1) block of shard `part`."""
    A = CSR.of(A)
    s = _c(splits, np.int64)
    cm = _c(colmap, np.int32) if colmap is not None else None
    r0, r1 = int(s[part]), int(s[part + 1])
    n = lib().ora_slice_split(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(A.val), _ptr(s), s.size - 1, int(part),
                              _ptr(cm) if cm is not None else None, int(which), None, None, None)
    rp, col, val = _buf(r1 - r0 + 1, np.int64), _buf(n, np.int32), _buf(n, np.float64)
    lib().ora_slice_split(A.n_rows, _ptr(A.row_ptr), _ptr(A.col), _ptr(A.val), _ptr(s), s.size - 1, int(part),
                          _ptr(cm) if cm is not None else None, int(which), _ptr(rp), _ptr(col), _ptr(val))
    return rp, col, val


# ----------------------------------------------------------------- pass rule

def check_tolerance(y_gpu, y_ref, bound, tol):
    """c2.3: |y_gpu - y_ref| <= tol * bound per row, evaluated in long double;
    bound == 0 => exact; any NaN fails.  Returns (ok, max_ratio, n_bad)."""
    yg = np.asarray(y_gpu, dtype=np.longdouble)
    yr = np.asarray(y_ref, dtype=np.longdouble)
    b = np.asarray(bound, dtype=np.longdouble)
    d = np.abs(yg - yr)
    # the oracle's own final rounding to double contributes <= 2^-53 |y_ref|
    lim = tol * b + np.abs(yr) * np.longdouble(2.0 ** -53)
    bad = ~(d <= lim) | np.isnan(yg)
    with np.errstate(divide="ignore", invalid="ignore"):
        ratio = np.where(b > 0, d / np.where(b > 0, b, 1), np.where(d > 0, np.inf, 0))
    mr = float(np.max(ratio)) if ratio.size else 0.0
    return (not bool(bad.any())), mr, int(bad.sum())
