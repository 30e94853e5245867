"""Pins for the oracle's SpMV, CPU only.

Each test checks the oracle against something other than itself: hand-worked
examples (tests/golden/), closed forms, dense brute force, scipy.sparse, exact
integer arithmetic and exact rational arithmetic.
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import matgen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def csr_of(g):
    return matgen.HostCSR(np.array(g["row_ptr"], np.int64), np.array(g["col"], np.int32),
                          np.array(g["val"], np.float64), g["n_rows"], g["n_cols"])


@pytest.mark.parametrize("name", ["app_a_4x4.json", "app_a_5x5.json"])
def test_golden_spmv(name):
    """P1/P2: hand-worked 4x4 and 5x5, exact."""
    g = load(name)
    A = csr_of(g)
    s = g["spmv"]
    Ax = oracle.spmv_csr(A, s["x"], 1.0, 0.0)
    assert Ax.tolist() == s["Ax"]
    y = oracle.spmv_csr(A, s["x"], s["alpha"], s["beta"], np.array(s["y_in"], float))
    assert y.tolist() == s["y"]


def _rand_vec(n, rng):
    return rng.uniform(-1, 1, n)


def test_identity_diagonal_permutation_closed_forms():
    """P3: I -> alpha x + beta y; D -> alpha d_i x_i + beta y_i; P -> alpha x_pi(i) + beta y_i."""
    rng = np.random.default_rng(1)
    n = 257
    x, y = _rand_vec(n, rng), _rand_vec(n, rng)
    alpha, beta = 1.5, -0.75
    rp = np.arange(n + 1, dtype=np.int64)
    ident = matgen.HostCSR(rp, np.arange(n, dtype=np.int32), np.ones(n), n, n)
    d = _rand_vec(n, rng)
    diag = matgen.HostCSR(rp, np.arange(n, dtype=np.int32), d, n, n)
    pi = rng.permutation(n).astype(np.int32)
    perm = matgen.HostCSR(rp, pi, np.ones(n), n, n)
    L = np.longdouble
    def fin(ax):  # alpha*ax + beta*y with one rounding, as the closed form states
        return (L(alpha) * ax.astype(L) + L(beta) * y.astype(L)).astype(np.float64)
    assert np.array_equal(oracle.spmv_csr(ident, x, alpha, beta, y), fin(x))
    assert np.array_equal(oracle.spmv_csr(diag, x, alpha, beta, y), fin(d.astype(L) * x.astype(L)))
    assert np.array_equal(oracle.spmv_csr(perm, x, alpha, beta, y), fin(x[pi]))


@pytest.mark.parametrize("g", [3, 4, 5, 8, 64])
def test_laplacian_closed_forms(g):
    """P4 (App. B): x = 1 => 0 interior, 1 on edges, 2 at corners; x_i = i => 0 interior."""
    A = matgen.laplacian5(g)
    y = oracle.spmv_csr(A, np.ones(A.n_cols), 1.0, 0.0).reshape(g, g)
    exp = np.zeros((g, g))
    exp[0, :] += 1; exp[-1, :] += 1; exp[:, 0] += 1; exp[:, -1] += 1
    assert np.array_equal(y, exp)
    y2 = oracle.spmv_csr(A, np.arange(A.n_cols, dtype=float), 1.0, 0.0).reshape(g, g)
    assert np.all(y2[1:-1, 1:-1] == 0)


@pytest.mark.parametrize("seed", range(6))
def test_integer_exact_regime(seed):
    """P5: a, x in {+-1, +-2}, y small ints, alpha, beta in {-2..2}: result is an exact
    integer; compare with Python-int arithmetic."""
    rng = np.random.default_rng(seed)
    n, m = int(rng.integers(1, 300)), int(rng.integers(1, 300))
    lens = rng.integers(0, min(m, 40) + 1, n)
    A = matgen.from_lengths(lens, m, seed=100 + seed, kind="int")
    x = matgen.vector(m, 100 + seed, 1, "int")
    y = rng.integers(-5, 6, n).astype(float)
    alpha, beta = [float(v) for v in rng.integers(-2, 3, 2)]
    got = oracle.spmv_csr(A, x, alpha, beta, y)
    for i in range(n):
        s = sum(int(A.val[k]) * int(x[A.col[k]]) for k in range(A.row_ptr[i], A.row_ptr[i + 1]))
        assert got[i] == int(alpha) * s + int(beta) * int(y[i])


@pytest.mark.parametrize("seed", range(4))
def test_dense_brute_force_bit_exact(seed):
    """P6: dense long-double brute force, j ascending (exact zeros add nothing)."""
    rng = np.random.default_rng(seed)
    n, m = int(rng.integers(1, 65)), int(rng.integers(1, 65))
    D = rng.uniform(-1, 1, (n, m)) * (rng.random((n, m)) < 0.3)
    A = matgen.from_dense(D)
    x, y = rng.uniform(-1, 1, m), rng.uniform(-1, 1, n)
    alpha, beta = 0.7, 1.3
    L = np.longdouble
    exp = np.empty(n)
    for i in range(n):
        acc = L(0)
        for j in range(m):
            if D[i, j] != 0:
                acc += L(D[i, j]) * L(x[j])
        exp[i] = np.float64(L(alpha) * acc + L(beta) * L(y[i]))
    assert np.array_equal(oracle.spmv_csr(A, x, alpha, beta, y), exp)


def test_scipy_library_pin():
    """P7: scipy.sparse CSR @ x (fp64 library) agrees within the fp64 tolerance."""
    sp = pytest.importorskip("scipy.sparse")
    A = matgen.rmat(12, seed=3)
    x = matgen.vector(A.n_cols, 3, 1)
    y = matgen.vector(A.n_rows, 3, 2)
    M = sp.csr_matrix((A.val, A.col, A.row_ptr), shape=A.shape)
    ref = 2.0 * (M @ x) - 0.5 * y
    got, bound = oracle.spmv_csr(A, x, 2.0, -0.5, y, with_bound=True)
    ok, ratio, _ = oracle.check_tolerance(ref, got, bound, 1e-12)
    assert ok, ratio


@pytest.mark.parametrize("seed", range(3))
def test_csr_equals_coo_bit_exact(seed):
    """P8: CSR oracle == COO oracle (independent loop) bit-for-bit."""
    A = matgen.rmat(10, seed=seed)
    row = oracle.csr2coo(A)
    x = matgen.vector(A.n_cols, seed, 1)
    y = matgen.vector(A.n_rows, seed, 2)
    a = oracle.spmv_csr(A, x, -1.25, 0.5, y)
    b = oracle.spmv_coo(A.n_rows, row, A.col, A.val, x, -1.25, 0.5, y)
    assert np.array_equal(a, b)


def test_long_row_accuracy_vs_exact_rational():
    """P9 (oracle side): a row of 20000 copies of 0.1 times x = 1; the oracle's long-double
    sum is within 20000 * 2^-64 (relative) of the exact rational sum."""
    k = 20000
    A = matgen.HostCSR(np.array([0, k], np.int64), np.arange(k, dtype=np.int32), np.full(k, 0.1), 1, k)
    got = oracle.spmv_csr(A, np.ones(k), 1.0, 0.0)[0]
    exact = Fraction(0.1) * k
    assert abs(Fraction(got) - exact) <= exact * Fraction(k + 1, 2 ** 64) + Fraction(abs(got)) / 2 ** 53


def test_alpha_zero_and_beta_zero_semantics():
    """A14: beta == 0 => y not read (NaN must not propagate); alpha == 0 => A not read."""
    A = matgen.from_rows([[(0, np.inf)], [(1, 2.0)]], 2)
    y = np.array([np.nan, np.nan])
    out = oracle.spmv_csr(matgen.from_rows([[(0, 1.0)], [(1, 2.0)]], 2), [3.0, 4.0], 1.0, 0.0, y)
    assert out.tolist() == [3.0, 8.0]
    out2 = oracle.spmv_csr(A, [1.0, 1.0], 0.0, 2.0, np.array([1.0, -3.0]))
    assert out2.tolist() == [2.0, -6.0]


def test_empty_and_degenerate():
    A = matgen.HostCSR(np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0), 0, 0)
    assert oracle.spmv_csr(A, np.zeros(0), 1.0, 0.0).size == 0
    B = matgen.HostCSR(np.zeros(4, np.int64), np.zeros(0, np.int32), np.zeros(0), 3, 5)
    assert oracle.spmv_csr(B, np.ones(5), 1.0, 3.0, np.array([1.0, 2.0, 3.0])).tolist() == [3.0, 6.0, 9.0]


def test_check_tolerance_rule():
    ok, _, _ = oracle.check_tolerance([1.0 + 1e-13], [1.0], [1.0], 1e-12)
    assert ok
    ok, _, n = oracle.check_tolerance([1.0 + 1e-11], [1.0], [1.0], 1e-12)
    assert not ok and n == 1
    ok, _, _ = oracle.check_tolerance([np.nan], [1.0], [1.0], 1e-12)
    assert not ok
    ok, _, _ = oracle.check_tolerance([1e-300], [0.0], [0.0], 1e-12)
    assert not ok


def test_canonical_check():
    A = matgen.from_rows([[(0, 1.0), (2, 1.0)], [(1, 1.0)]], 3)
    assert oracle.is_canonical(A)
    bad_sorted = matgen.HostCSR(A.row_ptr, np.array([2, 0, 1], np.int32), A.val, 2, 3)
    bad_range = matgen.HostCSR(A.row_ptr, np.array([0, 3, 1], np.int32), A.val, 2, 3)
    bad_dup = matgen.HostCSR(A.row_ptr, np.array([0, 0, 1], np.int32), A.val, 2, 3)
    bad_ptr = matgen.HostCSR(np.array([0, 2, 1], np.int64), A.col, A.val, 2, 3)
    for B in (bad_sorted, bad_range, bad_dup, bad_ptr):
        assert not oracle.is_canonical(B)
