"""Matrix Market ingestion: hand-written fixtures under tests/golden
against the CSR they spell out (Matrix Market spec conventions: 1-based, symmetric
files hold one triangle, pattern entries are 1, duplicates summed)."""
import io
import json
import os

import numpy as np
import pytest

import matgen
import oracle
from matgen.mtx import coo_to_csr, parse_mtx, read_mtx, write_mtx

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_app_a_fixture_matches_golden_csr():
    A = read_mtx(os.path.join(GOLD, "app_a_4x4.mtx"))
    g = json.load(open(os.path.join(GOLD, "app_a_4x4.json")))
    assert A.row_ptr.tolist() == g["row_ptr"] and A.col.tolist() == g["col"] and A.val.tolist() == g["val"]
    assert oracle.is_canonical(A)


def test_symmetric_fixture():
    A = read_mtx(os.path.join(GOLD, "sym_3x3.mtx"))
    dense = np.zeros((3, 3))
    for r in range(3):
        for k in range(A.row_ptr[r], A.row_ptr[r + 1]):
            dense[r, A.col[k]] = A.val[k]
    assert np.array_equal(dense, [[2, -1, 0], [-1, 0, 4], [0, 4, 1]])


def test_skew_and_pattern():
    skew = parse_mtx(io.StringIO("%%MatrixMarket matrix coordinate real skew-symmetric\n2 2 1\n2 1 3\n"))
    assert skew.row_ptr.tolist() == [0, 1, 2] and skew.col.tolist() == [1, 0] and skew.val.tolist() == [-3.0, 3.0]
    pat = parse_mtx(io.StringIO("%%MatrixMarket matrix coordinate pattern general\n2 3 3\n1 2\n2 3\n2 1\n"))
    assert pat.row_ptr.tolist() == [0, 1, 3] and pat.col.tolist() == [1, 0, 2] and pat.val.tolist() == [1, 1, 1]
    empty = parse_mtx(io.StringIO("%%MatrixMarket matrix coordinate real general\n5 7 0\n"))
    assert empty.n_rows == 5 and empty.n_cols == 7 and empty.nnz == 0


@pytest.mark.parametrize("bad", [
    "%%MatrixMarket matrix array real general\n2 2\n1\n2\n3\n4\n",
    "%%MatrixMarket matrix coordinate complex general\n1 1 1\n1 1 1 0\n",
    "%%MatrixMarket matrix coordinate real general\n2 2 1\n3 1 1\n",
    "%%MatrixMarket matrix coordinate real general\n2 2 2\n1 1 1\n",
])
def test_rejects(bad):
    with pytest.raises(ValueError):
        parse_mtx(io.StringIO(bad))


def test_round_trip_generated():
    for A in (matgen.rmat(8, seed=3), matgen.laplacian5(9)):
        buf = io.StringIO()
        write_mtx(A, buf)
        buf.seek(0)
        B = parse_mtx(buf)
        assert np.array_equal(A.row_ptr, B.row_ptr) and np.array_equal(A.col, B.col) and np.array_equal(A.val, B.val)


def test_coo_to_csr_sums_duplicates_any_order():
    rng = np.random.default_rng(0)
    i, j = rng.integers(0, 50, 2000), rng.integers(0, 40, 2000)
    v = rng.integers(-3, 4, 2000).astype(float)
    A = coo_to_csr(i, j, v, 50, 40)
    dense = np.zeros((50, 40))
    np.add.at(dense, (i, j), v)
    got = np.zeros((50, 40))
    for r in range(50):
        got[r, A.col[A.row_ptr[r]:A.row_ptr[r + 1]]] = A.val[A.row_ptr[r]:A.row_ptr[r + 1]]
    assert np.array_equal(dense, got) and oracle.is_canonical(A)
