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
# The paper's reading ("features are scaled to the range [-1, 1]"):
# libSVM svm-scale min-max with the training min/max, test inputs not clipped.
# That is the default of every function below (log_mask = 0, clip = False).
#
# EXTENSION (not from the paper; R11x): the SpMV features are >= 0 and
# heavy-tailed, so a variant of the model sees log1p(x) before the min-max
# scaling and clips scaled inputs to [-1, 1].  It is reported next to the
# paper-faithful model, never instead of it.
R11X_LOG_MASK, R11X_CLIP = 0x7F, True


def feature_transform(X, log_mask: int = 0):
    """log1p of the columns j with bit j of log_mask set (values must be >= 0).
    log_mask = 0 (the paper's reading) is the identity."""
    X = np.array(X, dtype=np.float64, copy=True)
    for j in range(X.shape[1]):
        if (log_mask >> j) & 1:
            X[:, j] = np.log1p(X[:, j])
    return X


def scale_fit(X):
    X = np.asarray(X, dtype=np.float64)
    return X.min(axis=0), X.max(axis=0)


def scale_apply(X, lo, hi, clip: bool = False):
    """x' = -1 + 2 (x - lo) / (hi - lo); a constant feature maps to 0; clipped
    to [-1, 1] only if clip."""
    X = np.asarray(X, dtype=np.float64)
    out = np.zeros_like(X)
    for j in range(X.shape[1]):
        if hi[j] == lo[j]:
            out[:, j] = 0.0
        else:
            out[:, j] = -1.0 + 2.0 * (X[:, j] - lo[j]) / (hi[j] - lo[j])
    return np.clip(out, -1.0, 1.0) if clip else out


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

    def __init__(self, lo, hi, C, gamma, svc=None, const_label=None, log_mask=0, clip=False):
        self.lo, self.hi, self.C, self.gamma = lo, hi, C, gamma
        self.svc, self.const_label = svc, const_label
        self.log_mask, self.clip = log_mask, clip

    def predict_scaled(self, Xs):
        Xs = np.asarray(Xs, dtype=np.float64)
        if self.const_label is not None:
            return np.full(Xs.shape[0], self.const_label, dtype=np.int64)
        return self.svc.predict(Xs).astype(np.int64)

    def predict(self, X):
        return self.predict_scaled(scale_apply(feature_transform(X, self.log_mask), self.lo, self.hi, self.clip))


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


def train(F, labels, folds: int = 5, seed: int = 0, tol: float = 1e-6, log2c=LOG2C, log2g=LOG2G,
          log_mask: int = 0, clip: bool = False) -> Model:
    """(Transform ->) scale -> CV grid -> refit on all data."""
    F = feature_transform(F, log_mask)
    lo, hi = scale_fit(F)
    Xs = scale_apply(F, lo, hi)
    (acc, lc, lg), _ = grid_search(Xs, labels, folds, seed, tol, log2c, log2g)
    svc, const = svc_fit(Xs, labels, 2.0 ** lc, 2.0 ** lg, tol)
    m = Model(lo, hi, 2.0 ** lc, 2.0 ** lg, svc, const, log_mask, clip)
    m.cv_accuracy = acc
    return m


def decisions(model: Model, X):
    """One-vs-one decision values [n, n_pairs] of raw feature rows (after the
    model's transform and scaling); None for a single-class model."""
    if model.svc is None:
        return None
    Xs = scale_apply(feature_transform(X, model.log_mask), model.lo, model.hi, model.clip)
    D = model.svc.decision_function(Xs)
    return D[:, None] if D.ndim == 1 else D


def decided(model: Model, X, eps: float = 1e-6):
    """Reading C12: two solvers of the same convex QP (to tolerance) may flip
    the sign of an OvO decision value within eps of 0, so a prediction is only
    required to agree where it is decided by the firm signs: every assignment
    of signs to the pairs with |decision| <= eps gives the same OvO vote
    winner (votes: dec > 0 -> the pair's first class, else the second; vote
    ties -> lowest label, as libSVM).  Boolean mask over the rows of X."""
    D = decisions(model, X)
    if D is None:
        return np.ones(len(X), dtype=bool)
    cls = list(model.svc.classes_)
    k = len(cls)
    pairs = [(a, b) for a in range(k) for b in range(a + 1, k)]
    out = np.zeros(len(X), dtype=bool)
    for i, row in enumerate(D):
        soft = [p for p in range(len(pairs)) if abs(row[p]) <= eps]
        if len(soft) > 12:
            continue
        winners = set()
        for mask in range(1 << len(soft)):
            sign = [row[p] > 0 for p in range(len(pairs))]
            for t, p in enumerate(soft):
                sign[p] = bool((mask >> t) & 1)
            votes = [0] * k
            for p, (a, b) in enumerate(pairs):
                votes[a if sign[p] else b] += 1
            winners.add(max(range(k), key=lambda c: (votes[c], -c)))
        out[i] = len(winners) == 1
    return out


def select(model: Model, feat_vec, allowed, default: int = 1) -> int:
    """Predict; a disallowed prediction reverts to the default."""
    lab = int(model.predict(np.asarray([feat_vec], dtype=np.float64))[0])
    return lab if allowed[lab] else default


# ---------------------------------------------------------------- probabilities + BvSB (NEXT f1)
def sigmoid_predict(f, A, B):
    fApB = f * A + B
    return math.exp(-fApB) / (1.0 + math.exp(-fApB)) if fApB >= 0 else 1.0 / (1.0 + math.exp(fApB))


def sigmoid_train(dec, y):
    """Platt's sigmoid P(+1|f) = 1/(1+exp(A f + B)), Newton with backtracking as
    written in Lin, Lin & Weng (2007), Algorithm 1 (the method libSVM uses)."""
    dec = [float(v) for v in dec]
    prior1 = sum(1 for v in y if v > 0)
    prior0 = len(y) - prior1
    hi, lo = (prior1 + 1.0) / (prior1 + 2.0), 1.0 / (prior0 + 2.0)
    t = [hi if v > 0 else lo for v in y]
    A, B = 0.0, math.log((prior0 + 1.0) / (prior1 + 1.0))

    def F(a, b):
        s = 0.0
        for f, ti in zip(dec, t):
            z = f * a + b
            s += ti * z + math.log1p(math.exp(-z)) if z >= 0 else (ti - 1) * z + math.log1p(math.exp(z))
        return s

    fval = F(A, B)
    for _ in range(100):
        h11 = h22 = 1e-12
        h21 = g1 = g2 = 0.0
        for f, ti in zip(dec, t):
            z = f * A + B
            if z >= 0:
                p, q = math.exp(-z) / (1 + math.exp(-z)), 1 / (1 + math.exp(-z))
            else:
                p, q = 1 / (1 + math.exp(z)), math.exp(z) / (1 + math.exp(z))
            d2 = p * q
            h11 += f * f * d2
            h22 += d2
            h21 += f * d2
            d1 = ti - p
            g1 += f * d1
            g2 += d1
        if abs(g1) < 1e-5 and abs(g2) < 1e-5:
            break
        det = h11 * h22 - h21 * h21
        dA, dB = -(h22 * g1 - h21 * g2) / det, -(-h21 * g1 + h11 * g2) / det
        gd = g1 * dA + g2 * dB
        step = 1.0
        while step >= 1e-10:
            nA, nB = A + step * dA, B + step * dB
            nf = F(nA, nB)
            if nf < fval + 0.0001 * step * gd:
                A, B, fval = nA, nB, nf
                break
            step /= 2.0
        if step < 1e-10:
            break
    return A, B


def pair_cv_decisions(Xp, ypm, C, gamma, folds, seed, tol=1e-6):
    """Decision values of a binary (+1/-1) problem by internal CV (libSVM
    svm_binary_svc_probability; folds stratified as fold_assign)."""
    from sklearn.svm import SVC
    Xp = np.asarray(Xp, dtype=np.float64)
    ypm = np.asarray(ypm)
    fa = fold_assign([0 if v > 0 else 1 for v in ypm], folds, seed)
    dec = np.zeros(len(ypm))
    for f in range(folds):
        te, tr = fa == f, fa != f
        if not te.any():
            continue
        pc, nc = int((ypm[tr] > 0).sum()), int((ypm[tr] < 0).sum())
        if pc == 0 or nc == 0:
            dec[te] = 1.0 if pc > 0 else (-1.0 if nc > 0 else 0.0)
            continue
        svc = SVC(kernel="rbf", C=C, gamma=gamma, tol=tol).fit(Xp[tr], ypm[tr])
        dec[te] = svc.decision_function(Xp[te])      # > 0 <=> +1 (sorted classes [-1, +1])
    return dec


def couple(r):
    """Wu, Lin & Weng (2004) method 2: p = argmin p'Qp, sum p = 1, solved as the
    KKT linear system (numpy)."""
    k = r.shape[0]
    Q = np.zeros((k, k))
    for t in range(k):
        for j in range(k):
            if j != t:
                Q[t, t] += r[j, t] ** 2
                Q[t, j] = -r[j, t] * r[t, j]
    Mx = np.zeros((k + 1, k + 1))
    Mx[:k, :k] = Q
    Mx[:k, k] = 1.0
    Mx[k, :k] = 1.0
    rhs = np.zeros(k + 1)
    rhs[k] = 1.0
    return np.linalg.solve(Mx, rhs)[:k]


class ProbModel:
    """OvO SVC + per-pair Platt sigmoids + coupling (libSVM's probability model)."""

    def __init__(self, Xs, y, C, gamma, folds=5, seed=0, tol=1e-6):
        Xs = np.asarray(Xs, dtype=np.float64)
        y = np.asarray(y)
        self.classes = sorted(set(y.tolist()))
        self.svc, _ = svc_fit(Xs, y, C, gamma, tol)
        self.sig = {}
        for a in range(len(self.classes)):
            for b in range(a + 1, len(self.classes)):
                m = (y == self.classes[a]) | (y == self.classes[b])
                ypm = np.where(y[m] == self.classes[a], 1, -1)
                dec = pair_cv_decisions(Xs[m], ypm, C, gamma, folds, seed, tol)
                self.sig[(a, b)] = sigmoid_train(dec, ypm)

    def proba(self, Xs):
        Xs = np.asarray(Xs, dtype=np.float64)
        k = len(self.classes)
        if k == 1:
            return np.ones((Xs.shape[0], 1))
        D = self.svc.decision_function(Xs)           # ovo columns: pairs (a<b), > 0 votes a
        if D.ndim == 1:                               # 2 classes: sklearn flips the sign
            D = -D[:, None]
        out = np.zeros((Xs.shape[0], k))
        for i in range(Xs.shape[0]):
            r = np.zeros((k, k))
            q = 0
            for a in range(k):
                for b in range(a + 1, k):
                    A, B = self.sig[(a, b)]
                    v = min(max(sigmoid_predict(D[i, q], A, B), 1e-7), 1 - 1e-7)
                    r[a, b], r[b, a] = v, 1 - v
                    q += 1
            out[i] = couple(r)
        return out


def bvsb_pick(P, candidates):
    """Best-vs-Second-Best: the candidate with the smallest gap between its two
    largest class probabilities (ties -> first candidate)."""
    best, pick = math.inf, None
    for row, c in zip(P, candidates):
        s = sorted(row, reverse=True)
        gap = s[0] - (s[1] if len(s) > 1 else 0.0)
        if gap < best:
            best, pick = gap, c
    return pick
