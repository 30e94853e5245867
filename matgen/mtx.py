"""Matrix Market ingestion: read a SuiteSparse ``.mtx`` file into the
canonical host CSR the path takes (sorted, duplicate-free columns, A15).

The paper's corpus is SuiteSparse, distributed as Matrix Market
coordinate files.  There is no network here, so only the reader is built; a file
placed on disk goes through ``read_mtx`` -> ``CSR.from_host`` -> ``features`` /
``convert`` like any generated matrix.  Input handling only: no SpMV arithmetic.

Supported headers: ``%%MatrixMarket matrix coordinate {real|integer|pattern}
{general|symmetric|skew-symmetric}`` (complex and array formats are rejected).
Conventions (NIST Matrix Market spec): 1-based indices; symmetric files store the
lower triangle and the mirror (j, i) is added for i != j; skew-symmetric mirrors with
the sign flipped; pattern entries get the value 1.0.  Duplicate (i, j) entries are
summed (how SuiteSparse's own readers assemble them).
"""
from __future__ import annotations

import io

import numpy as np

from . import HostCSR

_FIELDS = ("real", "integer", "pattern", "double")
_SYMM = ("general", "symmetric", "skew-symmetric")


def _open(path):
    if str(path).endswith(".gz"):
        import gzip
        return gzip.open(path, "rt")
    return open(path, "r")


def read_mtx(path, name: str = "") -> HostCSR:
    with _open(path) as fh:
        return parse_mtx(fh, name or str(path))


def parse_mtx(fh, name: str = "") -> HostCSR:
    header = fh.readline().split()
    if len(header) < 5 or header[0].lower() != "%%matrixmarket" or header[1].lower() != "matrix":
        raise ValueError("not a Matrix Market matrix file")
    fmt, field, symm = (h.lower() for h in header[2:5])
    if fmt != "coordinate":
        raise ValueError(f"unsupported format {fmt!r} (coordinate only)")
    if field not in _FIELDS:
        raise ValueError(f"unsupported field {field!r}")
    if symm not in _SYMM:
        raise ValueError(f"unsupported symmetry {symm!r}")
    line = fh.readline()
    while line and (line.startswith("%") or not line.strip()):
        line = fh.readline()
    m, n, nz = (int(t) for t in line.split()[:3])
    body = fh.read()
    ncols = 2 if field == "pattern" else 3
    data = np.loadtxt(io.StringIO(body), ndmin=2, dtype=np.float64, comments="%") if nz else np.zeros((0, ncols))
    if data.shape[0] != nz or (nz and data.shape[1] < ncols):
        raise ValueError(f"expected {nz} entries with {ncols} columns, got {data.shape}")
    i = data[:, 0].astype(np.int64) - 1
    j = data[:, 1].astype(np.int64) - 1
    v = np.ones(nz) if field == "pattern" else data[:, 2].astype(np.float64)
    if nz and (i.min() < 0 or j.min() < 0 or i.max() >= m or j.max() >= n):
        raise ValueError("index out of range")
    if symm != "general":
        off = i != j
        sign = -1.0 if symm == "skew-symmetric" else 1.0
        i, j, v = np.concatenate([i, j[off]]), np.concatenate([j, i[off]]), np.concatenate([v, sign * v[off]])
    return coo_to_csr(i, j, v, m, n, name)


def coo_to_csr(i, j, v, m: int, n: int, name: str = "") -> HostCSR:
    """Canonical CSR from unsorted triplets: sort by (row, col), sum duplicates."""
    i = np.asarray(i, np.int64)
    j = np.asarray(j, np.int64)
    v = np.asarray(v, np.float64)
    order = np.lexsort((j, i))
    i, j, v = i[order], j[order], v[order]
    if i.size:
        first = np.ones(i.size, bool)
        first[1:] = (i[1:] != i[:-1]) | (j[1:] != j[:-1])
        starts = np.flatnonzero(first)
        v = np.add.reduceat(v, starts)
        i, j = i[starts], j[starts]
    row_ptr = np.zeros(m + 1, np.int64)
    np.add.at(row_ptr, i + 1, 1)
    np.cumsum(row_ptr, out=row_ptr)
    return HostCSR(row_ptr, j.astype(np.int32), v, int(m), int(n), name)


def write_mtx(A: HostCSR, path_or_fh, field: str = "real") -> None:
    """Write A as a general coordinate file (1-based), %.17g values (round-trips fp64)."""
    rows = np.repeat(np.arange(A.n_rows, dtype=np.int64), np.diff(A.row_ptr))
    lines = [f"%%MatrixMarket matrix coordinate {field} general", f"{A.n_rows} {A.n_cols} {A.nnz}"]
    if field == "pattern":
        lines += [f"{r + 1} {c + 1}" for r, c in zip(rows, A.col)]
    else:
        lines += [f"{r + 1} {c + 1} {x:.17g}" for r, c, x in zip(rows, A.col, A.val)]
    text = "\n".join(lines) + "\n"
    if hasattr(path_or_fh, "write"):
        path_or_fh.write(text)
    else:
        with open(path_or_fh, "w") as fh:
            fh.write(text)
