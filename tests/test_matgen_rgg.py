"""The random-geometric-graph generator (matgen.rgg) against its definition: the recipe of
DIMACS10 rgg_n_2_k_s0, the matrix PAPER.md:131 quotes its CSR5 / merge GFLOP/s on."""
import numpy as np

import matgen


def test_rgg_matches_definition_brute_force():
    """scale 10: the edges are exactly the pairs of distinct points closer than
    r = 0.55 sqrt(ln n / n) (all n^2 pairs checked), the pattern is symmetric, rows are
    sorted, and the generator is deterministic."""
    A = matgen.rgg(10, seed=7)
    n = A.n_rows
    rng = np.random.default_rng(7)                   # the generator's points, in its numbering
    pts = rng.random((n, 2))
    r = 0.55 * np.sqrt(np.log(n) / n)
    nc = int(1.0 / r)
    cxy = np.minimum((pts * nc).astype(np.int64), nc - 1)
    order = np.lexsort((pts[:, 0], cxy[:, 1] * nc + cxy[:, 0]))
    pts = pts[order]
    d2 = ((pts[:, None, :] - pts[None, :, :]) ** 2).sum(axis=2)
    want = (d2 < r * r) & ~np.eye(n, dtype=bool)
    got = np.zeros((n, n), dtype=bool)
    rows = np.repeat(np.arange(n), np.diff(A.row_ptr))
    got[rows, A.col] = True
    assert np.array_equal(got, want)
    assert np.array_equal(got, got.T)
    for i in range(n):
        c = A.col[A.row_ptr[i]:A.row_ptr[i + 1]]
        assert np.all(np.diff(c) > 0)
    B = matgen.rgg(10, seed=7)
    assert np.array_equal(A.row_ptr, B.row_ptr) and np.array_equal(A.col, B.col) and np.array_equal(A.val, B.val)


def test_rgg19_size_of_the_papers_matrix():
    """scale 19 has rgg_n_2_19_s0's size: 524,288 rows and 6,539,532 nonzeros within 0.5%
    (SuiteSparse; the expected degree n*pi*r^2 = 0.3025*pi*ln n = 12.5)."""
    A = matgen.rgg(19)
    assert A.n_rows == A.n_cols == 524288
    assert abs(A.nnz - 6539532) / 6539532 < 0.005
    assert abs(A.nnz / A.n_rows - 0.3025 * np.pi * np.log(A.n_rows)) < 0.1
