"""Incremental tuning (NEXT f1): probability model, BvSB, itune loop.

Oracle pins (math, not the oracle's own formulas): two-class coupling returns
the pairwise probability; the Platt fit is a stationary point of its objective;
BvSB hand case.  Library vs oracle: probabilities, sigmoids, and the whole
itune history on a host-table problem."""
import math

import numpy as np
import pytest

from oracle import select as S
from oracle.itune import itune as oracle_itune


def nitro():
    import paper_conf_ipps_muralidharanshgc14_b200 as n
    return n


def _blobs(seed, n_per=12, k=3, d=3, spread=0.8):
    rng = np.random.default_rng(seed)
    C = rng.uniform(-1, 1, (k, d)) * 2.5
    X = np.concatenate([c + rng.normal(0, spread, (n_per, d)) for c in C])
    return X, np.repeat(np.arange(k), n_per)


# ------------------------------------------------------------------ oracle pins
def test_couple_two_classes_closed_form():
    for r01 in (0.1, 0.5, 0.93):
        r = np.array([[0.0, r01], [1 - r01, 0.0]])
        assert np.allclose(S.couple(r), [r01, 1 - r01], atol=1e-12)


def test_couple_consistent_pairwise_recovers_p():
    """If r_ij = p_i / (p_i + p_j) exactly, the minimiser is p itself (Q p = 0)."""
    p = np.array([0.5, 0.3, 0.15, 0.05])
    k = len(p)
    r = np.array([[p[i] / (p[i] + p[j]) if i != j else 0 for j in range(k)] for i in range(k)])
    assert np.allclose(S.couple(r), p, atol=1e-12)


def test_sigmoid_train_is_stationary_point():
    rng = np.random.default_rng(3)
    f = np.concatenate([rng.normal(1.2, 1.0, 40), rng.normal(-1.0, 1.0, 30)])
    y = np.array([1] * 40 + [-1] * 30)
    A, B = S.sigmoid_train(f, y)
    prior1, prior0 = 40, 30
    t = np.where(y > 0, (prior1 + 1) / (prior1 + 2), 1 / (prior0 + 2))

    def obj(a, b):  # regularised negative log likelihood, written from its definition
        z = f * a + b
        pp = 1 / (1 + np.exp(z))
        return -np.sum(t * np.log(pp) + (1 - t) * np.log(1 - pp))

    h = 1e-6
    ga = (obj(A + h, B) - obj(A - h, B)) / (2 * h)
    gb = (obj(A, B + h) - obj(A, B - h)) / (2 * h)
    assert abs(ga) < 1e-4 and abs(gb) < 1e-4
    assert A < 0                       # larger decision value -> more likely +1


def test_bvsb_hand_case():
    P = [[0.9, 0.05, 0.05], [0.45, 0.40, 0.15], [0.5, 0.2, 0.3]]
    assert S.bvsb_pick(P, [7, 8, 9]) == 8


def test_splitmix64_published_vector():
    """The seeded orders (fold deal, R12; initial labelling order, R15) hash
    with SplitMix64: the published output stream of seed 1234567 (state
    advanced by the golden gamma before each output)."""
    g, st = 0x9E3779B97F4A7C15, 1234567
    want = [6457827717110365317, 3203168211198807973, 9817491932198370423, 4593380528125082431,
            16408922859458223821]
    assert [S.splitmix64((st + i * g) % (1 << 64)) for i in range(5)] == want


def _seeded_order(n, seed):
    s = S.splitmix64(seed)
    return sorted(range(n), key=lambda i: (S.splitmix64(s ^ i), i))


def _geometric_pool(seed):
    """1-D pool (second feature constant): 16 points placed at the first 16
    positions of the seeded order (8 of class 0 on [-1, -0.3], 8 of class 1 on
    [0.3, 1]; label = sign of x via the costs), then 4 candidates."""
    base = list(np.linspace(-1, -0.3, 8)) + list(np.linspace(0.3, 1, 8))
    cands = [0.9, -0.25, 0.02, 0.15]
    n = len(base) + len(cands)
    xs = np.empty(n)
    for pos, i in enumerate(_seeded_order(n, seed)):
        xs[i] = (base + cands)[pos]
    F = np.stack([xs, np.zeros(n)], axis=1)
    cost = np.where(xs[:, None] < 0, [[1.0, 2.0]], [[2.0, 1.0]])
    return xs, F, cost


def test_itune_bvsb_picks_nearest_the_boundary():
    """P:L188 [20]: Best-vs-Second-Best labels the input whose two largest
    class probabilities are closest.  With well-separated symmetric classes
    and a monotone probability in the decision value, that is the candidate
    nearest the current boundary: first 0.02 (boundary ~0), then -0.25 (0.02
    joined class 1: boundary ~-0.14), then 0.15, then 0.9."""
    for seed, pf in ((3, 5), (11, 3)):
        xs, F, cost = _geometric_pool(seed)
        h = oracle_itune(F, lambda i: list(cost[i]), 2, init=16, iters=4, seed=seed, prob_folds=pf)
        assert h["n_labelled"] == [16, 17, 18, 19, 20]
        assert [float(xs[p]) for p in h["picked"][:4]] == [0.02, -0.25, 0.15, 0.9]
        assert h["picked"][4] == -1
        # the initial set is the seeded-order prefix (R15)
        assert h["final"]["labelled"][:16] == _seeded_order(len(xs), seed)[:16]


def test_itune_initial_set_extends_until_two_labels():
    """R15: `init` inputs in the seeded order, extended until two different
    labels are present (P:L188 wants every variant represented; labels are
    unknown before labelling)."""
    n, seed = 8, 0
    order = _seeded_order(n, seed)
    xs = np.empty(n)
    # the first four in seeded order share class 0, the fifth is class 1
    for pos, v in enumerate([-1.0, -0.9, -0.8, -0.7, 0.9, 0.8, -0.2, 0.3]):
        xs[order[pos]] = v
    F = np.stack([xs, np.zeros(n)], axis=1)
    cost = np.where(xs[:, None] < 0, [[1.0, 2.0]], [[2.0, 1.0]])
    for init in (1, 2, 4):
        h = oracle_itune(F, lambda i: list(cost[i]), 2, init=init, iters=0, seed=seed, log2c=(1,), log2g=(1,))
        assert h["n_labelled"][0] == 5                     # extended to the first class-1 input
        assert h["final"]["labelled"][:5] == order[:5]
    h = oracle_itune(F, lambda i: list(cost[i]), 2, init=6, iters=1, seed=seed, log2c=(1,), log2g=(1,))
    assert h["n_labelled"] == [6, 7] and h["final"]["labelled"][:6] == order[:6]


def test_itune_stopping_rules():
    """stop after `iter` picks, or once the accuracy on the labelled
    test set reaches `acc`, or when the pool is empty."""
    xs, F, cost = _geometric_pool(3)
    h = oracle_itune(F, lambda i: list(cost[i]), 2, init=16, iters=2, seed=3)
    assert h["n_labelled"] == [16, 17, 18] and h["picked"][-1] == -1 and len(h["picked"]) == 3
    h = oracle_itune(F, lambda i: list(cost[i]), 2, init=16, iters=0, seed=3)   # until the pool is empty
    assert h["n_labelled"][-1] == len(xs) and sorted(h["final"]["labelled"]) == list(range(len(xs)))
    # test set: boundary probes a model only gets right once it has labelled
    # 0.02 and -0.25 (test points at 0.0 -> class 1, -0.2 -> class 0)
    Ft = np.array([[-0.2, 0.0], [0.0, 0.0], [0.8, 0.0], [-0.8, 0.0]])
    Ct = [[1.0, 2.0], [2.0, 1.0], [2.0, 1.0], [1.0, 2.0]]
    h = oracle_itune(F, lambda i: list(cost[i]), 2, init=16, acc=1.0, seed=3, test_feat=Ft, test_cost=Ct)
    assert h["test_acc"][-1] == 1.0
    assert all(a < 1.0 for a in h["test_acc"][:-1])
    assert h["picked"][-1] == -1 and len(h["n_labelled"]) == len(h["test_acc"])
    assert all(0.0 <= p <= 1.0 for p in h["test_perf"])


def test_prob_model_separated_and_symmetric():
    """libSVM-style probabilities: two well-separated classes give p ~ 1 at one
    centre and ~ 0 at the other; mirror-symmetric classes give p = 1/2 on the
    mirror plane (the decision value is 0 there and the fitted sigmoid of
    symmetric data passes through 1/2).  Platt's regularised targets
    ((n+1)/(n+2), Lin, Lin & Weng 2007) keep the confident side below 1, so
    "~ 1" is checked as 0.95 < p < 1 with 40 points per class."""
    rng = np.random.default_rng(4)
    a = rng.normal(0, 0.1, (40, 2)) + [-0.7, 0.0]
    X = np.concatenate([a, a * [-1, 1]])            # class 1 = mirror image of class 0 in x
    y = np.array([0] * 40 + [1] * 40)
    pm = S.ProbModel(X, y, 4.0, 1.0, 5, 0)
    P = pm.proba(np.array([[-0.7, 0.0], [0.7, 0.0], [0.0, 0.0], [0.0, 0.3]]))
    assert 0.95 < P[0, 0] < 1.0 and 0.95 < P[1, 1] < 1.0
    assert np.allclose(P.sum(axis=1), 1.0)
    assert abs(P[2, 0] - 0.5) < 0.02 and abs(P[3, 0] - 0.5) < 0.02


# ------------------------------------------------------------------ library vs oracle
def test_probability_model_matches_oracle():
    n = nitro()
    X, y = _blobs(1)
    Xs = S.scale_apply(X, *S.scale_fit(X))
    for C, g in [(1.0, 1.0), (16.0, 0.25)]:
        lib = n.SVM(Xs, y, C, g, 1e-6, probability=True, prob_folds=5, seed=0)
        ref = S.ProbModel(Xs, y, C, g, 5, 0)
        T = np.random.default_rng(2).uniform(-1, 1, (50, 3))
        assert np.max(np.abs(lib.probability(T) - ref.proba(T))) < 2e-4
        A, B = lib.pair_sigmoid(0)
        Ar, Br = ref.sig[(0, 1)]
        assert abs(A - Ar) < 1e-3 * (1 + abs(Ar)) and abs(B - Br) < 1e-3 * (1 + abs(Br))
        assert np.allclose(lib.probability(T).sum(axis=1), 1.0, atol=1e-12)


def _table_problem(seed=5, n_pool=45, n_test=20):
    rng = np.random.default_rng(seed)
    centers = np.array([[0, 0], [3, 0], [0, 3]], float)

    def draw(m):
        lab = rng.integers(0, 3, m)
        F = centers[lab] + rng.normal(0, 0.9, (m, 2))
        cost = np.full((m, 3), 2.0) + rng.uniform(0, 0.1, (m, 3))
        cost[np.arange(m), lab] = 1.0
        return F, cost

    Fp, Cp = draw(n_pool)
    Ft, Ct = draw(n_test)
    return Fp, Cp, Ft, Ct


def test_itune_matches_oracle():
    n = nitro()
    Fp, Cp, Ft, Ct = _table_problem()
    grid = dict(log2c_lo=-1, log2c_hi=3, log2g_lo=-3, log2g_hi=1)
    ctx = n.Context()
    cv = n.CodeVariant(ctx, "toy")
    for v in range(3):
        cv.add_variant(f"v{v}", lambda i, v=v: Cp[i, v])
    cv.add_feature("f0", lambda i: Fp[i, 0])
    cv.add_feature("f1", lambda i: Fp[i, 1])
    cv.set_default(1)
    for i in range(len(Fp)):
        cv.add_training_input(i)
    h = cv.itune(init=3, iters=12, seed=4, test_feat=Ft, test_cost=Ct, **grid)
    ref = oracle_itune(Fp, lambda i: list(Cp[i]), 3, init=3, iters=12, seed=4, test_feat=Ft,
                       test_cost=Ct.tolist(), log2c=(-1, 1, 3), log2g=(1, -1, -3), default=1)
    assert h["n_labelled"] == ref["n_labelled"]
    assert h["picked"] == ref["picked"]
    assert np.allclose(h["test_acc"], ref["test_acc"]) and np.allclose(h["test_perf"], ref["test_perf"])
    assert h["n_labelled"][0] >= 3 and h["n_labelled"][-1] == h["n_labelled"][0] + 12


def test_itune_stops_at_accuracy():
    n = nitro()
    Fp, Cp, Ft, Ct = _table_problem(seed=9)
    ctx = n.Context()
    cv = n.CodeVariant(ctx, "toy")
    for v in range(3):
        cv.add_variant(f"v{v}", lambda i, v=v: Cp[i, v])
    cv.add_feature("f0", lambda i: Fp[i, 0])
    cv.add_feature("f1", lambda i: Fp[i, 1])
    for i in range(len(Fp)):
        cv.add_training_input(i)
    h = cv.itune(init=3, acc=0.8, seed=1, test_feat=Ft, test_cost=Ct, log2c_lo=-1, log2c_hi=3, log2g_lo=-3,
                 log2g_hi=1)
    assert h["test_acc"][-1] >= 0.8 or h["n_labelled"][-1] == len(Fp)
    assert all(a < 0.8 for a in h["test_acc"][:-1])
