"""GPU features (§8(a) a1/a2) against the oracle on shapes that cross the fused
feature kernel's work boundaries (csrc/features.cu): warp ranges of the rows +
nonzeros merge path, 8192-item sub-spans, 512-position chunks, blocks and rows open
across any of them, row-heavy and nonzero-heavy stretches, and the canonical-CSR
check (A15) with the defect placed anywhere in the matrix.  Bar: bit-exact
(north_star: integer features bit-exact; the fp64 finals follow A9 on both sides).
"""
import numpy as np
import pytest
import torch

import matgen
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sp():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_nisassvs18_b200 as pkg
    return pkg


def _rows(lens, cols_fn, n_cols):
    """Host CSR from row lengths and a per-row column generator (sorted, distinct)."""
    lens = np.asarray(lens, np.int64)
    rp = np.zeros(len(lens) + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    col = np.empty(int(rp[-1]), np.int32)
    for r, L in enumerate(lens):
        if L:
            col[rp[r]:rp[r + 1]] = cols_fn(r, int(L))
    return matgen.HostCSR(rp, col, np.ones(len(col)), len(lens), n_cols)


def _blocky(n_rows, n_cols, mean_len, mean_block, seed):
    """Rows made of runs of consecutive columns (blocks of geometric length)."""
    rng = np.random.default_rng(seed)
    lens = rng.poisson(mean_len, n_rows)
    rps = np.zeros(n_rows + 1, np.int64)
    cols = []
    for r in range(n_rows):
        out = []
        c = int(rng.integers(0, 50))
        while len(out) < lens[r] and c < n_cols:
            b = int(rng.geometric(1.0 / mean_block))
            out.extend(range(c, min(c + b, n_cols)))
            c = c + b + 1 + int(rng.integers(0, 40))
        out = out[:lens[r]]
        cols.append(np.asarray(out, np.int32))
        rps[r + 1] = rps[r] + len(out)
    col = np.concatenate(cols) if cols else np.zeros(0, np.int32)
    return matgen.HostCSR(rps, col, np.ones(len(col)), n_rows, n_cols)


def feature_cases():
    rng = np.random.default_rng(2024)
    c = {}
    # one block of 300K consecutive columns: a single row and block across many warps
    c["one_long_block"] = _rows([3, 300000, 2], lambda r, L: np.arange(L) + (5 if r != 1 else 0), 400000)
    # long rows of random sorted columns amid short rows (rows open across warps)
    lens = rng.integers(0, 7, 200000)
    lens[[10, 50000, 50001, 123456, 199999]] = [150000, 90000, 40000, 250000, 70000]
    c["long_rows"] = matgen.from_lengths(lens, 1 << 20, seed=5)
    # two million rows, almost all empty: the row walk dominates the warp ranges
    lens = np.zeros(2_000_000, np.int64)
    idx = rng.choice(2_000_000, 3000, replace=False)
    lens[idx] = rng.integers(1, 30, 3000)
    c["row_heavy"] = matgen.from_lengths(lens, 2_000_000, seed=6)
    # all rows empty except the last one
    lens = np.zeros(700000, np.int64)
    lens[-1] = 9000
    c["last_row_only"] = matgen.from_lengths(lens, 20000, seed=7)
    # blocks of varied length in every row
    c["blocky"] = _blocky(40000, 60000, 40, 6, seed=8)
    # every row one block of consecutive columns (blocks == rows)
    c["row_blocks"] = _rows(rng.integers(1, 200, 30000), lambda r, L: np.arange(L) + (r % 7), 300)
    # banded / Laplacian around sub-span sizes
    c["lap700"] = matgen.laplacian5(700)
    c["banded"] = matgen.window(300000, 300000, 7, 0.7, seed=9, mode=0)
    c["rmat18"] = matgen.rmat(18, seed=18)
    for i, n in enumerate([1, 31, 33, 511, 513, 8191, 8193, 65537]):
        c[f"rand_{n}"] = matgen.from_lengths(rng.integers(0, 9, n), 1000, seed=100 + i)
    return c


_CASES = {}


def fcase(name):
    if not _CASES:
        _CASES.update(feature_cases())
    return _CASES[name]


NAMES = ["one_long_block", "long_rows", "row_heavy", "last_row_only", "blocky", "row_blocks", "lap700",
         "banded", "rmat18", "rand_1", "rand_31", "rand_33", "rand_511", "rand_513", "rand_8191",
         "rand_8193", "rand_65537"]


@pytest.mark.parametrize("name", NAMES)
def test_features_boundaries_bit_exact(sp, name):
    A = fcase(name)
    fo = oracle.features(A)
    for ptr in (torch.int32, torch.int64):
        f = sp.features(sp.CSR.from_host(A, ptr_dtype=ptr))
        for k, v in fo.items():
            assert f[k] == v, (name, ptr, k, f[k], v)


def test_features_repeat_and_interleave(sp):
    """The kernel resets its own device state: repeated and interleaved calls agree."""
    A, B = fcase("rmat18"), fcase("blocky")
    dA, dB = sp.CSR.from_host(A), sp.CSR.from_host(B)
    fa, fb = sp.features(dA), sp.features(dB)
    for _ in range(3):
        assert sp.features(dB) == fb
        assert sp.features(dA) == fa


def test_features_unaligned_col(sp):
    """col_idx at an odd element offset (no 16-byte vector loads there)."""
    A = fcase("blocky")
    fo = oracle.features(A)
    dA = sp.CSR.from_host(A)
    big = torch.zeros(A.nnz + 3, dtype=torch.int32, device="cuda")
    big[3:] = dA.col
    B = sp.CSR(dA.row_ptr, big[3:], dA.val, (A.n_rows, A.n_cols))
    f = sp.features(B)
    for k, v in fo.items():
        assert f[k] == v, k


@pytest.mark.parametrize("where", [0.0, 0.37, 0.5, 0.999])
def test_not_canonical_anywhere(sp, where):
    """Each defect class is caught wherever it sits (A15)."""
    A = fcase("long_rows")
    nnz = A.nnz
    k = min(int(where * nnz), nnz - 2)
    r = int(np.searchsorted(A.row_ptr, k, side="right") - 1)
    bad = []
    c = A.col.copy()
    c[k] = A.n_cols                                      # column out of range
    bad.append(("range", A.row_ptr, c))
    c = A.col.copy()
    c[k] = -1
    bad.append(("negative", A.row_ptr, c))
    # duplicate / unsorted inside a row of >= 2 nonzeros near k
    rr = r
    while A.row_ptr[rr + 1] - A.row_ptr[rr] < 2:
        rr = (rr + 1) % A.n_rows
    a = int(A.row_ptr[rr])
    c = A.col.copy()
    c[a + 1] = c[a]
    bad.append(("duplicate", A.row_ptr, c))
    c = A.col.copy()
    c[a], c[a + 1] = c[a + 1], c[a]
    bad.append(("unsorted", A.row_ptr, c))
    rp = A.row_ptr.copy()
    j = max(1, min(int(where * A.n_rows), A.n_rows - 1))
    while rp[j + 1] == rp[j] and j + 1 < A.n_rows:
        j += 1
    rp[j] = rp[j + 1] + 1 if rp[j + 1] + 1 <= nnz else rp[j - 1] - 1
    bad.append(("row_ptr", rp, A.col))
    rp = A.row_ptr.copy()
    rp[-1] = nnz - 1
    bad.append(("row_ptr_end", rp, A.col))
    for label, rp_, col_ in bad:
        B = matgen.HostCSR(rp_, col_, A.val, A.n_rows, A.n_cols)
        if label != "row_ptr_end":            # the oracle reads nnz from row_ptr[-1]
            assert not oracle.is_canonical(B), label
        with pytest.raises(sp.SpmvError) as e:
            sp.features(sp.CSR.from_host(B, ptr_dtype=torch.int64))
        assert e.value.status == 2, label
    # and the untouched matrix still passes after the failures (state reset)
    f = sp.features(sp.CSR.from_host(A))
    assert f["nnzb_tot"] == oracle.features(A)["nnzb_tot"]


@pytest.mark.parametrize("fmt", ["coo", "csr", "hyb", "merge", "csr5"])
def test_convert_reuses_features(sp, fmt):
    """spmv_convert_opts.features: the conversion reuses the caller's feature pass and
    yields the same handle arrays and the same SpMV bits as a self-validating convert."""
    A = fcase("rmat18")
    dA = sp.CSR.from_host(A)
    f = sp.features(dA)
    h1 = sp.convert(dA, fmt)
    h2 = sp.convert(dA, fmt, features=f)
    for arr in ("col", "val", "coo_row", "ell_col", "merge_coord_row", "csr5_tile_desc"):
        try:
            a1 = h1.export(arr)
        except sp.SpmvError:
            continue
        assert np.array_equal(a1, h2.export(arr)), arr
    x = torch.from_numpy(matgen.vector(A.n_cols, 5, 1)).cuda()
    y1 = torch.from_numpy(matgen.vector(A.n_rows, 5, 2)).cuda()
    y2 = y1.clone()
    h1.run(1.5, x, -0.5, y1)
    h2.run(1.5, x, -0.5, y2)
    torch.cuda.synchronize()
    assert torch.equal(y1, y2)
    g = dict(f)
    g["nnz_tot"] += 1                                    # features of another matrix
    with pytest.raises(sp.SpmvError) as e:
        sp.convert(dA, fmt, features=g)
    assert e.value.status == 1
