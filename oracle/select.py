"""oracle.select — the variant-select path of Nitro, step by step (CPU).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Follows PAPER.md §III-A L177-179 in the paper's order:
  1. exhaustive search labels each training input with its best variant
     (L177; "constraints ... force the variant to return an infinity value
     during the offline training phase", L134);
  2. features are scaled to [-1, 1] (L179);
  3. a cross-validation based parameter search picks the RBF kernel
     parameters (L179);
  4. an RBF C-SVC is fitted with libSVM (L61-62) — here sklearn.svm.SVC, which
     wraps libSVM, is the library step;
  5. at run time the model predicts a label; a label whose constraint fails
     reverts to the default variant (L134, L94).
Readings where the paper is silent (grid, folds, tie-breaks, statistic):
SURVEY.md §8(c) C10-C13, restated in DESIGN.md "Readings".
"""
from __future__ import annotations

import math

import numpy as np

FEATURE_NAMES = ("nnz", "rows", "mean", "sd", "max_dev", "dia_fill", "ell_fill")
LOG2C = tuple(range(-5, 16, 2))        # -5, -3, ..., 15   (libSVM grid.py default)
LOG2G = tuple(range(3, -16, -2))       # 3, 1, ..., -15
_M64 = (1 << 64) - 1


def splitmix64(z: int) -> int:
    z = (z + 0x9E3779B97F4A7C15) & _M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


# ---------------------------------------------------------------- C10 / C13
def exhaustive_best(costs) -> list:
    """Label = argmin over variants of the cost (disallowed = +inf); ties ->
    lowest variant id (reading C10)."""
    out = []
    for row in costs:
        best, bi = math.inf, -1
        for v, c in enumerate(row):
            if c < best:
                best, bi = c, v
        out.append(bi)
    return out


def nitro_percent(costs, selected) -> dict:
    """Per-matrix ratio t[best]/t[selected]; mean, share >= 0.7, share >= 0.9
    (reading C13: arithmetic mean of per-matrix ratios)."""
    best = exhaustive_best(costs)
    ratios = []
    for row, b, s in zip(costs, best, selected):
        ratios.append(row[b] / row[s] if math.isfinite(row[s]) else 0.0)
    n = len(ratios)
    return {"mean": sum(ratios) / n, "ge70": sum(r >= 0.7 for r in ratios) / n,
            "ge90": sum(r >= 0.9 for r in ratios) / n, "ratios": ratios}


# ---------------------------------------------------------------- C11 scaling
def scale_fit(X):
    X = np.asarray(X, dtype=np.float64)
    return X.min(axis=0), X.max(axis=0)


def scale_apply(X, lo, hi):
    """x' = -1 + 2 (x - lo) / (hi - lo); a constant feature maps to 0; no clipping."""
    X = np.asarray(X, dtype=np.float64)
    out = np.zeros_like(X)
    for j in range(X.shape[1]):
        if hi[j] == lo[j]:
            out[:, j] = 0.0
        else:
            out[:, j] = -1.0 + 2.0 * (X[:, j] - lo[j]) / (hi[j] - lo[j])
    return out


# ---------------------------------------------------------------- C12 SVM + CV
def fold_assign(y, k: int, seed: int = 0) -> np.ndarray:
    """Stratified deterministic folds: inside each class (ascending label), the
    members (input order) are ordered by key = splitmix64(splitmix64(seed) ^ j)
    (j = sample index, ties by j) and dealt round-robin to folds 0..k-1."""
    y = list(y)
    fold = np.empty(len(y), dtype=np.int64)
    s = splitmix64(seed & _M64)
    for c in sorted(set(y)):
        members = [j for j, lab in enumerate(y) if lab == c]
        members.sort(key=lambda j: (splitmix64(s ^ j), j))
        for t, j in enumerate(members):
            fold[j] = t % k
    return fold


class Model:
    """Scaled-feature RBF C-SVC (one-vs-one), or a constant if one class."""

    def __init__(self, lo, hi, C, gamma, svc=None, const_label=None):
        self.lo, self.hi, self.C, self.gamma = lo, hi, C, gamma
        self.svc, self.const_label = svc, const_label

    def predict_scaled(self, Xs):
        Xs = np.asarray(Xs, dtype=np.float64)
        if self.const_label is not None:
            return np.full(Xs.shape[0], self.const_label, dtype=np.int64)
        return self.svc.predict(Xs).astype(np.int64)

    def predict(self, X):
        return self.predict_scaled(scale_apply(X, self.lo, self.hi))


def svc_fit(Xs, y, C: float, gamma: float, tol: float = 1e-6):
    """libSVM C-SVC, RBF K(u,v) = exp(-gamma |u-v|^2), OvO."""
    from sklearn.svm import SVC
    y = np.asarray(y)
    if len(set(y.tolist())) == 1:
        return None, int(y[0])
    svc = SVC(kernel="rbf", C=C, gamma=gamma, tol=tol, decision_function_shape="ovo", cache_size=200)
    svc.fit(np.asarray(Xs, dtype=np.float64), y)
    return svc, None


def cv_accuracy(Xs, y, C, gamma, folds: int = 5, seed: int = 0, tol: float = 1e-6) -> float:
    y = np.asarray(y)
    fa = fold_assign(y.tolist(), folds, seed)
    correct = 0
    for f in range(folds):
        te = fa == f
        tr = ~te
        if te.sum() == 0:
            continue
        svc, const = svc_fit(Xs[tr], y[tr], C, gamma, tol)
        pred = np.full(te.sum(), const) if svc is None else svc.predict(Xs[te])
        correct += int((pred == y[te]).sum())
    return correct / len(y)


def grid_search(Xs, y, folds: int = 5, seed: int = 0, tol: float = 1e-6, log2c=LOG2C, log2g=LOG2G):
    """Max CV accuracy; ties -> smaller C, then larger gamma (reading C12)."""
    best = None
    table = {}
    for lc in sorted(log2c):
        for lg in sorted(log2g, reverse=True):
            acc = cv_accuracy(Xs, y, 2.0 ** lc, 2.0 ** lg, folds, seed, tol)
            table[(lc, lg)] = acc
            if best is None or acc > best[0]:
                best = (acc, lc, lg)
    return best, table


def train(F, labels, folds: int = 5, seed: int = 0, tol: float = 1e-6, log2c=LOG2C, log2g=LOG2G) -> Model:
    """Scale -> CV grid -> refit on all data."""
    F = np.asarray(F, dtype=np.float64)
    lo, hi = scale_fit(F)
    Xs = scale_apply(F, lo, hi)
    (acc, lc, lg), _ = grid_search(Xs, labels, folds, seed, tol, log2c, log2g)
    svc, const = svc_fit(Xs, labels, 2.0 ** lc, 2.0 ** lg, tol)
    m = Model(lo, hi, 2.0 ** lc, 2.0 ** lg, svc, const)
    m.cv_accuracy = acc
    return m


def select(model: Model, feat_vec, allowed, default: int = 1) -> int:
    """Predict; a disallowed prediction reverts to the default."""
    lab = int(model.predict(np.asarray([feat_vec], dtype=np.float64))[0])
    return lab if allowed[lab] else default
