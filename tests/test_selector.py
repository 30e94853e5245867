"""N1/N2 format selection and performance modelling (selector.py), on small synthetic
sweep records: the label, slowdown and RME definitions against hand values, and the
models on a separable rule.  CPU only."""
import math

import numpy as np
import pytest

from paper_conf_ipps_nisassvs18_b200 import selector as S


def rec(feats, t):
    """A sweep record with the given feature values and per-format times (None = N/A)."""
    return {"features": dict(feats), "formats": {f: ({"t_mean_ms": v} if v is not None else {"status": "N/A"})
                                                 for f, v in t.items()}}


F17 = S.FEATURE_SETS["set123"]


def test_rme_definition():
    """RME = (1/n) sum |pred - meas| / meas."""
    assert S.rme([1.1, 0.5, 3.0], [1.0, 1.0, 3.0]) == pytest.approx((0.1 + 0.5 + 0.0) / 3)


def test_best_ties_and_na():
    t = {"coo": 2.0, "ell": None, "csr": 1.0, "hyb": 1.0, "merge": 3.0, "csr5": 1.5}
    assert S.best(t, S.FORMATS6) == "csr"           # tie csr/hyb -> paper order (A12)
    assert S.best({"ell": None, "csr": None, "hyb": None}, S.FORMATS3) is None


def test_dataset_drops_coo_best_for_three_formats():
    f = {k: 1.0 for k in F17}
    recs = [rec(f, {"coo": 0.5, "ell": 1.0, "csr": 2.0, "hyb": 3.0, "merge": 4.0, "csr5": 5.0}),   # COO best
            rec(f, {"coo": 9.0, "ell": None, "csr": 2.0, "hyb": 1.0, "merge": 4.0, "csr5": 5.0})]  # ELL N/A
    X3, y3, T3 = S.dataset(recs, S.SET1, S.FORMATS3)
    assert len(y3) == 1 and S.FORMATS3[y3[0]] == "hyb" and math.isnan(T3[0, 0])
    X6, y6, _ = S.dataset(recs, S.SET1, S.FORMATS6)
    assert [S.FORMATS6[i] for i in y6] == ["coo", "hyb"]


def test_slowdowns_and_histogram():
    T = np.array([[1.0, 2.0, 4.0], [1.0, 1.1, np.nan], [3.0, 1.0, 1.5]])
    sd = S.slowdowns(T, np.array([0, 0, 1]), np.array([0, 2, 2]))
    assert sd[0] == 1.0 and math.isinf(sd[1]) and sd[2] == 1.5
    h = S.slowdown_histogram(np.array([1.0, 1.1, 1.3, 1.5, 1.9, 2.5, np.inf]))
    assert h == {"none": 1, "(1,1.2]": 1, "(1.2,1.5]": 2, "(1.5,2]": 1, ">2": 2}


def synthetic(n=240, seed=3):
    """ELL wins when the row-length spread is small, CSR otherwise (a separable rule)."""
    rng = np.random.default_rng(seed)
    recs = []
    for _ in range(n):
        f = {k: float(rng.integers(1, 1000)) for k in F17}
        f["nnz_sigma"] = float(rng.choice([0.1, 50.0]))
        ell_fast = f["nnz_sigma"] < 1
        t = {"coo": 3.0, "ell": 1.0 if ell_fast else 2.0, "csr": 2.0 if ell_fast else 1.0, "hyb": 1.5,
             "merge": 2.5, "csr5": 2.5}
        recs.append(rec(f, t))
    return recs


@pytest.mark.parametrize("model", ["dtree", "gbt"])
def test_models_learn_a_separable_rule(model):
    X, y, T = S.dataset(synthetic(), S.FEATURE_SETS["set12"], S.FORMATS3)
    r = S.evaluate(X, y, T, model, grid=False)
    assert r["test_acc"] >= 0.95 and r["cv_acc_mean"] >= 0.95
    assert r["slowdown_hist"]["none"] >= 0.95 * r["test_n"]


def test_importance_finds_the_rule():
    X, y, _ = S.dataset(synthetic(), F17, S.FORMATS6)
    imp = S.importance(X, y, F17)
    assert imp[0][0] == "nnz_sigma"


def test_regression_rme_and_indirect_choice():
    """N2: log-time MLP regressors recover t = nnz * c_f (c_f per format) closely, and the
    argmin of the predicted times picks the format that is fastest by construction."""
    rng = np.random.default_rng(5)
    c = {"coo": 3e-6, "ell": 2e-6, "csr": 1e-6, "hyb": 2.5e-6, "merge": 1.5e-6, "csr5": 1.2e-6}
    recs = []
    for _ in range(200):
        f = {k: float(rng.integers(1, 1000)) for k in F17}
        f["nnz_tot"] = float(10 ** rng.uniform(3, 7))
        recs.append(rec(f, {k: f["nnz_tot"] * v for k, v in c.items()}))
    r = S.regress(recs, ensemble=2)
    assert all(v["rme_mlp_ensemble"] < 0.35 for v in r["formats"].values()), r["formats"]
    assert r["indirect_mlp_ensemble"]["acc"] >= 0.9
