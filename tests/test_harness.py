"""Host logic of the timing/label harness (a16) and the sweep recipe (configs[3])."""
import numpy as np

import matgen
import oracle
from paper_conf_ipps_nisassvs18_b200.harness import LABEL_SETS, labels


def test_label_rules():
    """A12: argmin time; label5 drops COO; label3 = ELL/CSR/HYB
    (PAPER.md:239); N/A excluded (A4); exact ties in Fig. 3 order."""
    t = {"coo": 1.0, "ell": None, "csr": 3.0, "hyb": 2.5, "merge": 2.0, "csr5": 2.0}
    lab = labels(t)
    assert lab["label6"] == "coo" and lab["label5"] == "merge" and lab["label3"] == "hyb"
    assert abs(lab["margin"] - 1.0) < 1e-12
    tie = labels({"coo": 5, "ell": 2, "csr": 2, "hyb": 2, "merge": 2, "csr5": 2})
    assert tie["label6"] == "ell" and tie["label3"] == "ell"
    none = labels({f: None for f in LABEL_SETS["label6"]})
    assert none["label6"] is None
    assert "label7" not in lab                       # CSR-scalar not timed -> no label7


def test_label7_scalar_class():
    """CSR-scalar as a seventh class; ties go to the paper's six first."""
    t = {"coo": 3.0, "ell": None, "csr": 2.0, "hyb": 2.5, "merge": 2.2, "csr5": 2.4, "csr_scalar": 1.5}
    lab = labels(t)
    assert lab["label7"] == "csr_scalar" and lab["label6"] == "csr"
    lab = labels({**t, "csr_scalar": 2.0})
    assert lab["label7"] == "csr"


def test_sweep_recipe_deterministic_and_canonical():
    for i in range(0, 25):
        A, p = matgen.sweep_matrix(i, max_nnz=300_000)
        B, q = matgen.sweep_matrix(i, max_nnz=300_000)
        assert p == q and np.array_equal(A.col, B.col) and np.array_equal(A.val, B.val)
        assert oracle.is_canonical(A)
        assert p["family"] == matgen.FAMILIES[i % 5]


def test_sweep_bucket_frequencies():
    """Table I bucket frequencies drive the nnz targets."""
    counts = np.zeros(len(matgen.NNZ_BUCKETS))
    for i in range(2000):
        nnz = matgen.sweep_params(i)["nnz_target"]
        for k, (lo, hi, _) in enumerate(matgen.NNZ_BUCKETS):
            if lo <= nnz < hi or (k == len(matgen.NNZ_BUCKETS) - 1 and nnz == hi):
                counts[k] += 1
                break
    expect = np.array([b[2] for b in matgen.NNZ_BUCKETS], float)
    expect = expect / expect.sum() * 2000
    assert np.all(np.abs(counts - expect) < 5 * np.sqrt(expect) + 5)


def test_sweep_realized_nnz_in_bucket():
    """configs[3] fidelity: the REALIZED nnz of every family lands in its target's Table I
    bucket (cap 96M) -- checked on every third matrix
    whose target is below 400K nonzeros (the CPU-cheap part of the sweep)."""
    seen = set()
    for i in range(0, 2000, 3):
        p = matgen.sweep_params(i)
        if p["nnz_target"] > 400_000:
            continue
        A, q = matgen.sweep_matrix(i)
        seen.add(q["family"])
        assert q["nnz"] == A.nnz
        assert matgen.nnz_bucket(A.nnz) == q["bucket"], (i, q["family"], q["nnz_target"], A.nnz)
    assert seen == set(matgen.FAMILIES)
    assert max(matgen.sweep_params(i)["nnz_target"] for i in range(2000)) <= 96_000_000


def test_fit_lengths():
    """Row lengths pinned to the target sum with the cap respected and the shape kept."""
    rng = np.random.default_rng(4)
    lens = rng.pareto(0.8, 5000) + 1.0
    out = matgen.fit_lengths(lens, 123_457, 300)
    assert out.sum() == 123_457 and out.max() <= 300 and out.min() >= 0
    o = out[np.argsort(lens, kind="stable")]
    assert np.all(np.diff(o) >= -1)                  # order of the drawn lengths kept (up to rounding)
    assert matgen.fit_lengths(np.ones(10), 1000, 7).sum() == 70           # capped by n x m
