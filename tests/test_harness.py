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
