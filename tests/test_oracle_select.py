"""Pins of the select-path oracle (oracle/select.py), CPU only."""
import math

import numpy as np
import pytest

from oracle import select as S


def test_exhaustive_best_hand_table():
    inf = math.inf
    costs = [[3.0, 2.0, inf, 1.0, 5.0],
             [1.0, 1.0, 1.0, inf, 2.0],       # tie -> lowest id
             [inf, 4.0, inf, inf, 4.0]]
    assert S.exhaustive_best(costs) == [3, 0, 1]


def test_nitro_percent_hand_table():
    costs = [[2.0, 1.0], [1.0, 4.0], [3.0, 3.0], [1.0, 10.0]]
    r = S.nitro_percent(costs, [1, 1, 0, 1])
    assert r["ratios"] == [1.0, 0.25, 1.0, 0.1]
    assert r["mean"] == pytest.approx(2.35 / 4)
    assert r["ge70"] == 0.5 and r["ge90"] == 0.5


def test_scaling_matches_minmaxscaler():
    from sklearn.preprocessing import MinMaxScaler
    rng = np.random.default_rng(0)
    X = np.exp(rng.normal(0, 3, (60, 7)))
    X[:, 3] = 5.0                                   # constant feature -> 0
    lo, hi = S.scale_fit(X)
    Xs = S.scale_apply(X, lo, hi)
    ref = MinMaxScaler(feature_range=(-1, 1)).fit(X).transform(X)
    ref[:, 3] = 0.0
    assert np.max(np.abs(Xs - ref)) <= 1e-12
    assert np.all(Xs[np.argmin(X[:, 0]), 0] == -1.0) and np.all(Xs[np.argmax(X[:, 0]), 0] == 1.0)
    T = np.exp(rng.normal(0, 4, (10, 7)))             # test points are not clipped
    assert np.max(np.abs(S.scale_apply(T, lo, hi)[:, [0, 1, 2, 4, 5, 6]]
                         - MinMaxScaler((-1, 1)).fit(X).transform(T)[:, [0, 1, 2, 4, 5, 6]])) <= 1e-9 * \
        np.max(np.abs(S.scale_apply(T, lo, hi)))


def test_fold_assign_stratified_deterministic():
    y = [0] * 13 + [1] * 7 + [2] * 3 + [4] * 21
    f = S.fold_assign(y, 5, seed=0)
    assert np.array_equal(f, S.fold_assign(y, 5, seed=0))
    for c in set(y):
        counts = np.bincount(f[np.array(y) == c], minlength=5)
        n = y.count(c)
        assert counts.max() - counts.min() <= 1 and counts.sum() == n
    assert not np.array_equal(f, S.fold_assign(y, 5, seed=1))


def test_two_point_closed_form():
    """Two points, labels -1/+1: alpha = min(C, 1/(1 - exp(-gamma d^2))), b = 0."""
    from sklearn.svm import SVC
    for gamma, C in [(0.7, 100.0), (0.7, 1.0), (3.0, 10.0)]:
        X = np.array([[0.2, -0.1], [-0.5, 0.6]])
        d2 = float(((X[0] - X[1]) ** 2).sum())
        svc, _ = S.svc_fit(X, [0, 1], C, gamma)
        alpha = min(C, 1.0 / (1.0 - math.exp(-gamma * d2)))
        assert np.allclose(np.abs(svc.dual_coef_), alpha, rtol=1e-6)
        assert abs(svc.intercept_[0]) < 1e-8


def test_separable_clusters_cv_one_and_select_default():
    rng = np.random.default_rng(5)
    centers = np.array([[1, 1, 0], [10, 1, 0], [1, 10, 5], [10, 10, 5]], float)
    F = np.concatenate([c + rng.normal(0, 0.3, (12, 3)) for c in centers])
    y = np.repeat(np.arange(4), 12)
    m = S.train(F, y, log2c=(1, 5), log2g=(1, -1))
    assert m.cv_accuracy == 1.0
    assert list(m.predict(centers)) == [0, 1, 2, 3]
    # a disallowed prediction reverts to the default
    assert S.select(m, centers[2], [True, True, False, True], default=1) == 1
    assert S.select(m, centers[3], [True] * 4, default=1) == 3


def test_single_class_is_constant():
    m = S.train(np.random.default_rng(1).normal(size=(6, 3)), [2] * 6, log2c=(1,), log2g=(1,))
    assert list(m.predict(np.zeros((3, 3)))) == [2, 2, 2]


def test_grid_tie_break_smaller_C_larger_gamma():
    rng = np.random.default_rng(2)
    F = np.concatenate([rng.normal(0, 0.1, (10, 2)), rng.normal(5, 0.1, (10, 2))])
    y = [0] * 10 + [1] * 10
    Xs = S.scale_apply(F, *S.scale_fit(F))
    (acc, lc, lg), table = S.grid_search(Xs, y, log2c=(-1, 3), log2g=(1, -3))
    assert acc == 1.0
    assert lc == -1 and lg == 1


def test_decided_marks_only_near_boundary_points():
    """C12 helper: with two mirror-symmetric classes the decision value on the
    mirror plane is 0 (within solver tolerance): not decided; points near the
    class centres are decided.  A 3-class problem: a point whose only
    near-zero pair cannot change the vote winner stays decided."""
    import numpy as np
    from oracle import select as S
    F = np.array([[-1.0, 0.0], [-0.8, 0.1], [-0.9, -0.1], [1.0, 0.0], [0.8, -0.1], [0.9, 0.1]])
    m = S.train(F, [0, 0, 0, 1, 1, 1], log2c=(1,), log2g=(1,))
    assert list(S.decided(m, np.array([[0.0, 0.0], [-0.9, 0.0], [0.9, 0.0]]))) == [False, True, True]
    # three classes on a line: a point deep inside class 0 is decided even if
    # the (1, 2) pair is exactly balanced there
    F3 = np.array([[-2.0, 0], [-2.1, 0.1], [0.0, 1.0], [0.1, 1.1], [0.0, -1.0], [0.1, -1.1]])
    m3 = S.train(F3, [0, 0, 1, 1, 2, 2], log2c=(1,), log2g=(-1,))
    assert bool(S.decided(m3, np.array([[-2.05, 0.0]]))[0])
