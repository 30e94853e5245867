"""Format selection and performance modelling from the regenerated B200 ground truth
(SURVEY §8(f) N1, N2 -- the paper's method step after the labels; CPU, scikit-learn).

Input: the sweep records of `harness.sweep` (BASELINE configs[3]; one JSON line per
matrix with the 17 Table II features, per-format mean times and labels).

N1 -- classification (§IV-D, §V, Tables IV-X):
  * feature sets: set 1 (5 features, O(1), Table IV), sets 1+2 (11, Sedaghati et al.,
    Table V), sets 1+2+3 (17, Table VI), and the top-7 by gradient-boosting importance
    ("imp.", Table X);
  * label sets: 3 formats ELL/CSR/HYB (Tables IV-VI) and the 6 formats (Tables VII-X);
    as in §V-A the 3-format study drops matrices whose best of the six is COO
    ("we remove the cases where COO format is the best format");
  * models: decision tree, SVM (RBF; GridSearchCV over C {100, 1000, 10000} x gamma
    {.1, .01, .001}), MLP (hidden 96-48-16, mini-batch 16)
    and gradient-boosted trees (GridSearchCV over n_estimators {50, 100, 200, 500} x
    max_depth {32, 64, 128} x learning_rate {.1, .01}).  XGBoost is not
    in this image: scikit-learn's HistGradientBoostingClassifier stands in (max_iter =
    n_estimators);
  * protocol: 5-fold cross-validation and an 80/20 train/test split;
    accuracy, and the slowdown of mispredictions t(predicted) / t(best)
    (Tables XI-XIII).

N2 -- performance modelling (§VI): per-format regression of the execution
time from the 17 features with an MLP and an MLP ensemble (mean of 5 seeds), scored by
RME = (1/n) sum |pred - meas| / meas; indirect classification = argmin of the
predicted times.

Readings (A27): features enter the models as log1p(value) then
standardised (they span 1 to 1e8); times are regressed as log(ms) and exponentiated;
infeasible formats (A4, N/A) are never labels and never predicted as best.
"""
from __future__ import annotations

import json
import math
from typing import Dict, List, Optional, Sequence

import numpy as np

FORMATS6 = ("coo", "ell", "csr", "hyb", "merge", "csr5")
FORMATS3 = ("ell", "csr", "hyb")
SET1 = ("n_rows", "n_cols", "nnz_tot", "nnz_mu", "nnz_frac")
SET2 = ("nnz_max", "nnz_sigma", "nnzb_mu", "nnzb_sigma", "snzb_mu", "snzb_sigma")
SET3 = ("nnzb_tot", "nnzb_min", "nnzb_max", "snzb_min", "snzb_max", "nnz_min")
FEATURE_SETS = {"set1": SET1, "set12": SET1 + SET2, "set123": SET1 + SET2 + SET3}
SVM_GRID = {"svc__C": [100, 1000, 10000], "svc__gamma": [0.1, 0.01, 0.001]}
GBT_GRID = {"max_iter": [50, 100, 200, 500], "max_depth": [32, 64, 128], "learning_rate": [0.1, 0.01]}


# ---------------------------------------------------------------------- data

def load_records(path: str) -> List[dict]:
    with open(path) as fh:
        return [json.loads(line) for line in fh if line.strip()]


def times(rec: dict, formats: Sequence[str]) -> Dict[str, Optional[float]]:
    out = {}
    for f in formats:
        r = rec.get("formats", {}).get(f, {})
        t = r.get("t_mean_ms") if isinstance(r, dict) else None
        out[f] = float(t) if t is not None and r.get("status", "ok") != "N/A" else None
    return out


def best(ts: Dict[str, Optional[float]], formats: Sequence[str]) -> Optional[str]:
    """argmin over the feasible formats; exact ties in the paper's order (A12)."""
    feas = [(ts[f], FORMATS6.index(f), f) for f in formats if ts.get(f) is not None]
    return min(feas)[2] if feas else None


def dataset(recs: List[dict], features: Sequence[str], formats: Sequence[str]):
    """X (raw features), y (label index into `formats`), T (times, NaN = N/A).
    For the 3-format study the matrices whose best of the six is COO are dropped
    (PAPER.md:235)."""
    X, y, T = [], [], []
    for r in recs:
        t6 = times(r, FORMATS6)
        if tuple(formats) == FORMATS3 and best(t6, FORMATS6) == "coo":
            continue
        lab = best(t6, formats)
        if lab is None:
            continue
        X.append([float(r["features"][k]) for k in features])
        y.append(formats.index(lab))
        T.append([t6[f] if t6[f] is not None else math.nan for f in formats])
    return np.asarray(X, np.float64), np.asarray(y, np.int64), np.asarray(T, np.float64)


def transform(X: np.ndarray) -> np.ndarray:
    """log1p of the (non-negative) features; the models standardise after this."""
    return np.log1p(np.maximum(X, 0.0))


# ---------------------------------------------------------------------- models

def make_model(name: str, seed: int = 0, grid: bool = True):
    from sklearn.ensemble import HistGradientBoostingClassifier
    from sklearn.model_selection import GridSearchCV
    from sklearn.neural_network import MLPClassifier
    from sklearn.pipeline import make_pipeline
    from sklearn.preprocessing import StandardScaler
    from sklearn.svm import SVC
    from sklearn.tree import DecisionTreeClassifier
    if name == "dtree":
        return DecisionTreeClassifier(random_state=seed)
    if name == "svm":
        m = make_pipeline(StandardScaler(), SVC(kernel="rbf"))
        return GridSearchCV(m, SVM_GRID, cv=3, n_jobs=-1) if grid else m.set_params(svc__C=1000, svc__gamma=0.01)
    if name == "mlp":
        return make_pipeline(StandardScaler(), MLPClassifier(hidden_layer_sizes=(96, 48, 16), batch_size=16,
                                                             max_iter=300, random_state=seed))
    if name == "gbt":
        m = HistGradientBoostingClassifier(random_state=seed)
        return GridSearchCV(m, GBT_GRID, cv=3, n_jobs=-1) if grid else m.set_params(max_iter=200, max_depth=32)
    raise ValueError(name)


MODELS = ("dtree", "svm", "mlp", "gbt")


def slowdowns(T: np.ndarray, y_true: np.ndarray, y_pred: np.ndarray) -> np.ndarray:
    """t(predicted format) / t(best format) per matrix (1.0 when correct; a predicted
    infeasible format counts as +inf)."""
    tb = T[np.arange(len(y_true)), y_true]
    tp = T[np.arange(len(y_pred)), y_pred]
    tp = np.where(np.isnan(tp), np.inf, tp)
    return tp / tb


def slowdown_histogram(sd: np.ndarray) -> Dict[str, int]:
    """Tables XI-XIII style buckets of the mispredictions' slowdown."""
    edges = [(1.0, 1.0, "none"), (1.0, 1.2, "(1,1.2]"), (1.2, 1.5, "(1.2,1.5]"), (1.5, 2.0, "(1.5,2]"),
             (2.0, math.inf, ">2")]
    out = {}
    for lo, hi, name in edges:
        if name == "none":
            out[name] = int(np.sum(sd <= 1.0))
        else:
            out[name] = int(np.sum((sd > lo) & (sd <= hi)))
    return out


def evaluate(X: np.ndarray, y: np.ndarray, T: np.ndarray, model: str, seed: int = 0, grid: bool = True,
             folds: int = 5) -> dict:
    """80/20 split (GridSearchCV, when on, picks the hyper-parameters on the 80%): test
    accuracy and the slowdown of mispredictions; then 5-fold cross-validation accuracy
    of the chosen configuration over all matrices."""
    from sklearn.base import clone
    from sklearn.model_selection import StratifiedKFold, cross_val_score, train_test_split
    Xt = transform(X)
    counts = np.bincount(y)
    strat = y if counts[counts > 0].min() >= folds else None
    idx = np.arange(len(y))
    tr, te = train_test_split(idx, test_size=0.2, random_state=seed, stratify=strat)
    m = make_model(model, seed, grid).fit(Xt[tr], y[tr])
    pred = m.predict(Xt[te])
    est = getattr(m, "best_estimator_", m)
    params = {k: v for k, v in getattr(m, "best_params_", {}).items()}
    cv = StratifiedKFold(n_splits=folds, shuffle=True, random_state=seed) if strat is not None else folds
    cv_acc = cross_val_score(clone(est), Xt, y, cv=cv)
    sd = slowdowns(T[te], y[te], pred)
    wrong = sd[pred != y[te]]
    # labels decided by >= 2% (the second-best format at least 2% slower): model error
    # separated from near-ties that re-running the sweep flips (tools/label_stability.py)
    Tte = np.where(np.isnan(T[te]), np.inf, T[te])
    srt = np.sort(Tte, axis=1)
    clear = (srt[:, 1] / srt[:, 0] - 1.0) >= 0.02 if Tte.shape[1] > 1 else np.ones(len(te), bool)
    return {"model": model, "n": int(len(y)), "params": params,
            "test_acc_clear_labels": float(np.mean(pred[clear] == y[te][clear])) if clear.any() else None,
            "test_n_clear_labels": int(clear.sum()),
            "cv_acc_mean": float(cv_acc.mean()), "cv_acc_std": float(cv_acc.std()),
            "test_acc": float(np.mean(pred == y[te])), "test_n": int(len(te)),
            "test_acc_within_2pct": float(np.mean(sd <= 1.02)), "test_acc_within_5pct": float(np.mean(sd <= 1.05)),
            "slowdown_hist": slowdown_histogram(sd),
            "mean_slowdown_mispredicted": float(np.mean(wrong)) if len(wrong) else 1.0,
            "geo_mean_slowdown_all": float(np.exp(np.mean(np.log(np.minimum(sd, 1e6)))))}


def importance(X: np.ndarray, y: np.ndarray, names: Sequence[str], seed: int = 0) -> List[tuple]:
    """Gradient-boosting feature importance (permutation importance on held-out data --
    HistGradientBoosting has no split-gain importances), descending (Figs. 4-5)."""
    from sklearn.inspection import permutation_importance
    from sklearn.model_selection import train_test_split
    Xt = transform(X)
    tr, te = train_test_split(np.arange(len(y)), test_size=0.2, random_state=seed)
    m = make_model("gbt", seed, grid=False).fit(Xt[tr], y[tr])
    r = permutation_importance(m, Xt[te], y[te], n_repeats=10, random_state=seed)
    return sorted(((names[i], float(r.importances_mean[i])) for i in range(len(names))), key=lambda t: -t[1])


# ---------------------------------------------------------------------- N2

def rme(pred: np.ndarray, meas: np.ndarray) -> float:
    """Relative mean error: (1/n) sum |pred - meas| / meas."""
    pred, meas = np.asarray(pred, np.float64), np.asarray(meas, np.float64)
    return float(np.mean(np.abs(pred - meas) / meas))


def regress(recs: List[dict], formats: Sequence[str] = FORMATS6, ensemble: int = 5, seed: int = 0) -> dict:
    """Per-format MLP and MLP-ensemble regressors of log(time) on the 17 features (80/20
    split); RME per format; indirect classification = argmin of the predicted times."""
    from sklearn.model_selection import train_test_split
    from sklearn.neural_network import MLPRegressor
    from sklearn.pipeline import make_pipeline
    from sklearn.preprocessing import StandardScaler
    feats = FEATURE_SETS["set123"]
    X = transform(np.asarray([[float(r["features"][k]) for k in feats] for r in recs], np.float64))
    T = np.asarray([[times(r, formats)[f] if times(r, formats)[f] is not None else math.nan for f in formats]
                    for r in recs], np.float64)
    tr, te = train_test_split(np.arange(len(recs)), test_size=0.2, random_state=seed)
    out = {"n_train": int(len(tr)), "n_test": int(len(te)), "formats": {}}
    P1 = np.full((len(te), len(formats)), np.nan)
    PE = np.full((len(te), len(formats)), np.nan)
    for j, f in enumerate(formats):
        ok_tr = tr[~np.isnan(T[tr, j])]
        ok_te = te[~np.isnan(T[te, j])]
        if len(ok_tr) < 10 or len(ok_te) == 0:
            continue
        preds = []
        for k in range(ensemble):
            m = make_pipeline(StandardScaler(), MLPRegressor(hidden_layer_sizes=(96, 48, 16), batch_size=16,
                                                             max_iter=500, random_state=seed + k))
            m.fit(X[ok_tr], np.log(T[ok_tr, j]))
            preds.append(np.exp(m.predict(X[te])))
        single, ens = preds[0], np.mean(preds, axis=0)
        mask = ~np.isnan(T[te, j])
        P1[:, j], PE[:, j] = np.where(mask, single, np.nan), np.where(mask, ens, np.nan)
        out["formats"][f] = {"rme_mlp": rme(single[mask], T[te, j][mask]),
                             "rme_mlp_ensemble": rme(ens[mask], T[te, j][mask]), "n_test": int(mask.sum())}
    # indirect classification: argmin predicted time over the feasible formats
    Tt = T[te]
    truth = np.nanargmin(Tt, axis=1)
    for name, P in (("mlp", P1), ("mlp_ensemble", PE)):
        Pm = np.where(np.isnan(Tt), np.inf, np.where(np.isnan(P), np.inf, P))
        pred = np.argmin(Pm, axis=1)
        sd = slowdowns(Tt, truth, pred)
        out[f"indirect_{name}"] = {"acc": float(np.mean(pred == truth)),
                                   "acc_within_5pct": float(np.mean(sd <= 1.05)),
                                   "slowdown_hist": slowdown_histogram(sd)}
    return out


# ---------------------------------------------------------------------- driver

def run_study(path: str, grid: bool = True, seed: int = 0, models: Sequence[str] = MODELS) -> dict:
    recs = load_records(path)
    res = {"source": path, "n_records": len(recs), "xgboost_stand_in": "sklearn HistGradientBoostingClassifier",
           "classification": {}}
    X17, y6, _ = dataset(recs, FEATURE_SETS["set123"], FORMATS6)
    imp = importance(X17, y6, FEATURE_SETS["set123"], seed)
    res["importance_6fmt"] = imp
    sets = dict(FEATURE_SETS)
    sets["imp7"] = tuple(n for n, _ in imp[:7])
    for lname, fmts in (("3fmt", FORMATS3), ("6fmt", FORMATS6)):
        for sname, feats in sets.items():
            X, y, T = dataset(recs, feats, fmts)
            for m in models:
                res["classification"][f"{lname}/{sname}/{m}"] = evaluate(X, y, T, m, seed, grid)
    res["regression"] = regress(recs, FORMATS6, seed=seed)
    return res


def _main():
    import argparse
    ap = argparse.ArgumentParser(description="format selection (N1) and performance modelling (N2)")
    ap.add_argument("records")
    ap.add_argument("--out", default="")
    ap.add_argument("--no-grid", action="store_true", help="fixed hyper-parameters instead of GridSearchCV")
    ap.add_argument("--seed", type=int, default=0)
    a = ap.parse_args()
    res = run_study(a.records, grid=not a.no_grid, seed=a.seed)
    txt = json.dumps(res, indent=1)
    if a.out:
        with open(a.out, "w") as fh:
            fh.write(txt + "\n")
    for k, v in res["classification"].items():
        print(f"{k:28s} cv {v['cv_acc_mean']:.3f}  test {v['test_acc']:.3f}  (<=2%: {v['test_acc_within_2pct']:.3f})  "
              f"slowdown {v['slowdown_hist']}")
    for f, v in res["regression"]["formats"].items():
        print(f"RME {f:6s} mlp {v['rme_mlp']:.3f}  ensemble {v['rme_mlp_ensemble']:.3f}")
    print("indirect", res["regression"]["indirect_mlp_ensemble"])


if __name__ == "__main__":
    _main()
