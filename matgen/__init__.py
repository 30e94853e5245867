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
         "sweep": 0x5EED1000, "rmat27": 0x5EED0005, "rgg19": 0x5EED0019}


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


def rgg(scale, seed=SEEDS["rgg19"], kind="f64", r_coef=0.55) -> HostCSR:
    """Random geometric graph by the recipe of DIMACS10 rgg_n_2_{scale}_s0 (SuiteSparse;
    the matrix PAPER.md:131 quotes CSR5 / merge GFLOP/s on): n = 2^scale points uniform in
    the unit square, an edge between two distinct points closer than r = r_coef*sqrt(ln n/n)
    (symmetric pattern, no self loops); points numbered in grid-cell order (cells of side
    >= r, row-major; by x inside a cell), so neighbours get nearby indices.  A synthetic
    stand-in -- the SuiteSparse file is not reachable here -- with the same size and degree
    law (scale 19: 524,288 rows; rgg_n_2_19_s0 has 6,539,532 nonzeros).  Values
    position-keyed (A18)."""
    n = 1 << int(scale)
    rng = np.random.default_rng(seed)
    pts = rng.random((n, 2))
    r = r_coef * np.sqrt(np.log(n) / n)
    nc = max(1, int(1.0 / r))                              # cells per side, side 1/nc >= r
    cxy = np.minimum((pts * nc).astype(np.int64), nc - 1)
    cell = cxy[:, 1] * nc + cxy[:, 0]
    order = np.lexsort((pts[:, 0], cell))
    pts, cell, cxy = pts[order], cell[order], cxy[order]
    starts = np.searchsorted(cell, np.arange(nc * nc + 1))
    ii, jj = [], []
    idx = np.arange(n, dtype=np.int64)
    for dy in (-1, 0, 1):
        for dx in (-1, 0, 1):
            ny, nx = cxy[:, 1] + dy, cxy[:, 0] + dx
            ok = (ny >= 0) & (ny < nc) & (nx >= 0) & (nx < nc)
            c2 = np.where(ok, ny * nc + nx, 0)
            lo = starts[c2]
            cnt = np.where(ok, starts[c2 + 1] - lo, 0)
            tot = int(cnt.sum())
            i = np.repeat(idx, cnt)
            j = np.repeat(lo, cnt) + (np.arange(tot, dtype=np.int64) - np.repeat(np.cumsum(cnt) - cnt, cnt))
            d = pts[i] - pts[j]
            keep = (i != j) & ((d * d).sum(axis=1) < r * r)
            ii.append(i[keep])
            jj.append(j[keep])
    i = np.concatenate(ii)
    j = np.concatenate(jj)
    o = np.lexsort((j, i))
    i, j = i[o], j[o]
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(i, minlength=n), out=row_ptr[1:])
    A = HostCSR(row_ptr, j.astype(np.int32), np.empty(0), n, n, f"rgg{scale}")
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


# ----------------------------------------------------------------------------- cfg4 sweep

#: Table I nnz buckets: (lo, hi, count of 2299); upper bound 96M
NNZ_BUCKETS = [(3, 10_000, 747), (10_000, 50_000, 508), (50_000, 100_000, 209), (100_000, 500_000, 362),
               (500_000, 1_000_000, 147), (1_000_000, 5_000_000, 208), (5_000_000, 50_000_000, 109),
               (50_000_000, 96_000_000, 9)]
FAMILIES = ("uniform", "banded", "blockdiag", "powerlaw", "mixed")


def _loguniform(rng, lo, hi):
    return float(np.exp(rng.uniform(np.log(lo), np.log(hi))))


def nnz_bucket(nnz):
    """Index of the Table I bucket holding nnz (-1: outside all)."""
    for k, (lo, hi, _) in enumerate(NNZ_BUCKETS):
        if lo <= nnz < hi or (k == len(NNZ_BUCKETS) - 1 and nnz == hi):
            return k
    return -1


def sweep_params(i, max_nnz=None):
    """Parameters of sweep matrix i: family = i mod 5,
    nnz bucket drawn with Table I frequencies, log-uniform within it (cap 96M);
    mu log-uniform in [1, 256]; n_rows = max(8, nnz/mu); 80% square, else aspect
    log-uniform in [1/4, 4]; the shape is widened where n_rows x n_cols could not hold
    1.25 x the target (tiny matrices with long rows)."""
    rng = np.random.default_rng(SEEDS["sweep"] + i)
    fam = FAMILIES[i % 5]
    w = np.array([b[2] for b in NNZ_BUCKETS], dtype=float)
    bk = int(rng.choice(len(NNZ_BUCKETS), p=w / w.sum()))
    b = NNZ_BUCKETS[bk]
    nnz = int(_loguniform(rng, b[0], b[1]))
    if max_nnz:
        nnz = min(nnz, int(max_nnz))
    mu = _loguniform(rng, 1.0, 256.0)
    n_rows = max(8, int(nnz / mu))
    square = rng.random() < 0.8
    aspect = 1.0 if square else _loguniform(rng, 0.25, 4.0)
    n_cols = max(8, int(n_rows * aspect))
    if n_rows * n_cols < 1.25 * nnz:
        if square:
            n_rows = n_cols = int(np.ceil(np.sqrt(1.25 * nnz)))
        else:
            n_cols = int(np.ceil(1.25 * nnz / n_rows))
    p = dict(i=i, family=fam, nnz_target=nnz, bucket=bk, mu=mu, n_rows=n_rows, n_cols=n_cols,
             seed=SEEDS["sweep"] + i)
    if fam == "banded":
        p["fill"] = float(rng.uniform(0.3, 1.0))
    elif fam == "blockdiag":
        p["block"] = int(_loguniform(rng, 4, 256))
        p["fill"] = float(rng.uniform(0.3, 1.0))
        p["noise"] = float(rng.uniform(0.0, 0.05))
        # rows of a block hold ~block*fill entries: size the matrix to the nnz target
        p["n_rows"] = max(8, int(nnz / (p["block"] * p["fill"])))
        p["n_cols"] = max(8, int(p["n_rows"] * aspect))
    elif fam == "powerlaw":
        p["gamma"] = float(rng.uniform(1.5, 3.0))
    elif fam == "mixed":
        p["q"] = float(_loguniform(rng, 0.005, 0.10))
        p["long"] = float(rng.uniform(10.0, 100.0))
    return p


def fit_lengths(lens, target, m):
    """Row lengths rescaled to sum exactly to `target` with each <= m (water-filling over
    the rows below the cap, then largest-remainder rounding): the family's length
    distribution kept, its total pinned to the nnz target."""
    lens = np.asarray(lens, dtype=np.float64)
    n = lens.size
    target = int(min(target, n * m))
    if n == 0 or target == 0:
        return np.zeros(n, dtype=np.int64)
    s = lens if lens.sum() > 0 else np.ones(n)
    s = s / s.sum() * target
    for _ in range(64):
        s = np.minimum(s, m)
        short = target - s.sum()
        free = s < m
        if short <= 1e-9 or not free.any():
            break
        base = s[free].sum()
        s[free] = s[free] * (1.0 + short / base) if base > 0 else s[free] + short / free.sum()
    s = np.minimum(s, m)
    out = np.floor(s).astype(np.int64)
    rem = int(target - out.sum())
    if rem > 0:
        frac = np.where(out < m, s - out, -1.0)
        out[np.argsort(-frac, kind="stable")[:rem]] += 1
    return np.minimum(out, m)


def _union_rows(A: HostCSR, B: HostCSR) -> HostCSR:
    """Row-wise union of two structures (duplicates coalesced; A's values kept)."""
    ra = np.repeat(np.arange(A.n_rows, dtype=np.int64), np.diff(A.row_ptr))
    rb = np.repeat(np.arange(B.n_rows, dtype=np.int64), np.diff(B.row_ptr))
    keys = np.concatenate([ra * A.n_cols + A.col, rb * A.n_cols + B.col])
    keys = np.unique(keys)
    rows = keys // A.n_cols
    row_ptr = np.zeros(A.n_rows + 1, dtype=np.int64)
    np.add.at(row_ptr, rows + 1, 1)
    np.cumsum(row_ptr, out=row_ptr)
    return HostCSR(row_ptr, (keys % A.n_cols).astype(np.int32), np.empty(0), A.n_rows, A.n_cols, A.name)


def sweep_matrix(i, kind="f64", max_nnz=None):
    """Build sweep matrix i (canonical CSR, seeded values).  Returns (HostCSR, params).
    Length-drawn families (uniform, power-law, mixed) have their row lengths pinned to
    the nnz target (fit_lengths); window families (banded, block-diagonal) are resized
    (rows scaled by target / realized, up to 4 tries) until the realized nnz falls in the
    target's Table I bucket.  params["nnz"] records the realized count."""
    p = sweep_params(i, max_nnz)
    n, m, mu, seed = p["n_rows"], p["n_cols"], p["mu"], p["seed"]
    fam = p["family"]
    target = p["nnz_target"]
    if fam in ("uniform", "powerlaw", "mixed"):
        rng = np.random.default_rng(p["seed"] + 1)
        if fam == "uniform":
            lens = rng.poisson(mu, n)
        elif fam == "powerlaw":
            lens = rng.pareto(p["gamma"] - 1.0, n) + 1.0
        else:  # mixed: a fraction q of long rows at 10..long x mu
            lens = rng.poisson(mu, n).astype(np.float64)
            long = rng.random(n) < p["q"]
            lens[long] = mu * rng.uniform(10.0, p["long"], long.sum())
        A = from_lengths(fit_lengths(lens, target, m), m, seed, kind)
    else:
        for _ in range(4):
            rng = np.random.default_rng(p["seed"] + 1)
            if fam == "banded":
                half = max(0, int(round(mu / (2 * p["fill"]) - 0.5)))
                A = window(n, m, half, p["fill"], seed, 0, kind)
            else:
                bsz = min(p["block"], n)
                base = window(n, m, bsz, p["fill"], seed, 1, "ones")
                nl = np.minimum(rng.poisson(p["noise"] * max(1.0, base.nnz / n), n), m)
                noise = from_lengths(nl, m, seed + 3, "ones")
                A = set_values(_union_rows(base, noise), seed + 5, kind)
            if nnz_bucket(A.nnz) == nnz_bucket(target) or A.nnz == 0:
                break
            f = target / max(A.nnz, 1)
            n = max(8, int(round(n * f)))
            m = max(8, int(round(m * f)))
        p["n_rows"], p["n_cols"] = n, m
    p["nnz"] = A.nnz
    A.name = f"sweep{i}-{fam}"
    return A, p
