"""oracle.itune — incremental tuning (active learning) of Nitro, step by step.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

PAPER.md §III-B: compute feature vectors for ALL inputs (cheap, L185),
label only a subset by exhaustive search: an initial set (L188: "at least one
input that has the label of each variant" — reading R15: `init` inputs in a
seeded order, extended until two labels are present, since labels are unknown
before labelling), then iteratively add the pool input picked by the
Best-vs-Second-Best heuristic [20] on the current model's class probabilities,
updating the model each iteration; stop after `iters` picks or when accuracy
on a labelled test set reaches `acc` (L190).  Scaling uses the whole pool's
features (all known, L185); each refit runs the same CV grid as full training.
"""
from __future__ import annotations

import math

import numpy as np

from .select import (ProbModel, bvsb_pick, exhaustive_best, feature_transform, grid_search, scale_apply, scale_fit,
                     splitmix64, svc_fit, LOG2C, LOG2G)


def itune(F_pool, label_fn, n_var, init=0, iters=0, acc=0.0, seed=0, prob_folds=5, test_feat=None,
          test_cost=None, folds=5, tol=1e-6, log2c=LOG2C, log2g=LOG2G, default=1, log_mask=0, clip=False):
    F_pool = feature_transform(F_pool, log_mask)
    n = F_pool.shape[0]
    lo, hi = scale_fit(F_pool)
    Xall = scale_apply(F_pool, lo, hi)
    s = splitmix64(seed & ((1 << 64) - 1))
    order = sorted(range(n), key=lambda i: (splitmix64(s ^ i), i))
    labelled, lab = [], {}

    def label(i):
        costs = label_fn(i)
        lab[i] = exhaustive_best([costs])[0]
        labelled.append(i)

    init = init if init > 0 else n_var
    pos = 0
    while pos < n and (len(labelled) < init or len({lab[i] for i in labelled if lab[i] >= 0}) < 2):
        label(order[pos])
        pos += 1
    tlab = exhaustive_best(test_cost) if test_feat is not None else []
    hist = {"n_labelled": [], "picked": [], "test_acc": [], "test_perf": []}
    picks = 0
    while True:
        rows = [i for i in labelled if lab[i] >= 0]
        y = [lab[i] for i in rows]
        X = Xall[rows]
        k = max(2, min(folds, len(rows)))
        (cvacc, lc, lg), _ = grid_search(X, y, k, 0, tol, log2c, log2g)
        C, g = 2.0 ** lc, 2.0 ** lg
        svc, const = svc_fit(X, y, C, g, tol)
        a = p = float("nan")
        if test_feat is not None:
            Xt = scale_apply(feature_transform(test_feat, log_mask), lo, hi, clip)
            pred = np.full(len(Xt), const) if svc is None else svc.predict(Xt)
            ok, ps, cnt = 0, 0.0, 0
            for t, v in enumerate(pred):
                if tlab[t] < 0:
                    continue
                v = int(v)
                if not math.isfinite(test_cost[t][v]):
                    v = default
                cnt += 1
                ok += v == tlab[t]
                ps += test_cost[t][tlab[t]] / test_cost[t][v] if math.isfinite(test_cost[t][v]) else 0.0
            a, p = ok / cnt, ps / cnt
        hist["n_labelled"].append(len(labelled))
        hist["picked"].append(-1)
        hist["test_acc"].append(a)
        hist["test_perf"].append(p)
        if acc > 0 and a >= acc:
            break
        if iters > 0 and picks >= iters:
            break
        pool = [i for i in range(n) if i not in lab]
        if not pool:
            break
        if svc is None:
            pick = next(i for i in order if i not in lab)
        else:
            pm = ProbModel(X, y, C, g, max(2, prob_folds), seed, tol)
            pick = bvsb_pick(pm.proba(Xall[pool]), pool)
        hist["picked"][-1] = pick
        label(pick)
        picks += 1
    hist["final"] = {"C": C, "gamma": g, "cv_accuracy": cvacc, "labelled": list(labelled)}
    return hist
