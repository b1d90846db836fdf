"""C-ABI library checks that need no GPU: every symbol declared in
include/nitro.h is exported, and the host logic (SVM, folds, generic
code-variant training/selection, model I/O) behaves — checked against the
oracle's select path (sklearn/libSVM) and hand-built cases."""
import math
import os
import re
import subprocess

import numpy as np
import pytest

from oracle import select as S

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def nitro():
    import paper_conf_ipps_muralidharanshgc14_b200 as n
    return n


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "nitro.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(nitro_[a-z0-9_]+)\s*\(", src)) - {"nitro_variant_fn"})


def test_library_exports_every_declared_symbol():
    n = nitro()
    so = n.LIB_PATH
    out = subprocess.run(["nm", "-D", "--defined-only", so], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (nitro_\w+)", out))
    decl = declared_symbols()
    assert len(decl) > 50
    missing = [s for s in decl if s not in exported]
    assert not missing, missing
    assert set(decl) <= set(n.EXPORTED) | {"nitro_feature_fn", "nitro_constraint_fn"}
    assert n.version().startswith("nitro-b200")


def test_errors_without_gpu_are_reported_not_raised():
    n = nitro()
    import ctypes
    h = ctypes.c_void_p()
    rc = n._L.nitro_spmv_create(0, None, 4, 4, 0, ctypes.c_void_p(16), 0, None, None, 0, ctypes.byref(h))
    assert rc != 0 and n._L.nitro_last_error()
    rc = n._L.nitro_spmv_create(0, None, -1, 4, 0, None, 0, None, None, 0, ctypes.byref(h))
    assert rc == 1


def test_fold_assign_matches_oracle():
    n = nitro()
    rng = np.random.default_rng(0)
    for seed in (0, 1, 12345):
        y = rng.integers(0, 5, 97)
        assert np.array_equal(n.fold_assign(y, 5, seed), S.fold_assign(y.tolist(), 5, seed))


def _blobs(seed, n_per=15, k=4, d=3, spread=0.6):
    rng = np.random.default_rng(seed)
    C = rng.uniform(-1, 1, (k, d)) * 3
    X = np.concatenate([c + rng.normal(0, spread, (n_per, d)) for c in C])
    y = np.repeat(np.arange(k), n_per)
    return X, y


@pytest.mark.parametrize("C,gamma", [(1.0, 0.5), (32.0, 2.0), (0.125, 8.0), (1024.0, 0.03125)])
def test_svm_matches_libsvm(C, gamma):
    """Own SMO vs sklearn.svm.SVC (libSVM): same dual solution to tolerance,
    same predictions on points away from the decision boundaries."""
    from sklearn.svm import SVC
    n = nitro()
    X, y = _blobs(1)
    lo, hi = S.scale_fit(X)
    Xs = S.scale_apply(X, lo, hi)
    ours = n.SVM(Xs, y, C, gamma, 1e-6)
    ref = SVC(kernel="rbf", C=C, gamma=gamma, tol=1e-6, decision_function_shape="ovo").fit(Xs, y)
    T = np.random.default_rng(9).uniform(-1.2, 1.2, (400, 3))
    d_ours = ours.decision(T)
    d_ref = ref.decision_function(T)
    scale = 1.0 + np.abs(d_ref).max()
    assert np.max(np.abs(d_ours - d_ref)) <= 1e-3 * scale
    far = np.all(np.abs(d_ref) > 2e-3 * scale, axis=1)
    assert far.sum() >= 40
    assert np.array_equal(ours.predict(T)[far], ref.predict(T)[far])


def test_svm_two_point_closed_form():
    n = nitro()
    X = np.array([[0.2, -0.1], [-0.5, 0.6]])
    for gamma, C in [(0.7, 100.0), (0.7, 1.0), (3.0, 10.0)]:
        m = n.SVM(X, [0, 1], C, gamma)
        coef, rho = m.pair_dual(0)
        d2 = float(((X[0] - X[1]) ** 2).sum())
        alpha = min(C, 1.0 / (1.0 - math.exp(-gamma * d2)))
        assert np.allclose(np.abs(coef), alpha, rtol=1e-6)
        assert abs(rho) < 1e-8


def test_cv_accuracy_matches_oracle_on_separable_data():
    n = nitro()
    X, y = _blobs(2, spread=0.3)
    Xs = S.scale_apply(X, *S.scale_fit(X))
    for C, g in [(1.0, 1.0), (8.0, 0.25)]:
        assert n.cv_accuracy(Xs, y, C, g, 1e-6, 5, 0) == pytest.approx(S.cv_accuracy(Xs, y, C, g, 5, 0), abs=1e-12)


def _toy_cv(n):
    """Generic layer with host callbacks: the input is an int id into a table of
    (features, costs); variant v's cost = table cost; constraint on variant 2."""
    ctx = n.Context()
    cv = n.CodeVariant(ctx, "toy")
    rng = np.random.default_rng(4)
    F = np.concatenate([rng.normal(c, 0.2, (12, 2)) for c in ([0, 0], [4, 0], [0, 4])])
    lab = np.repeat([0, 1, 2], 12)
    costs = np.ones((36, 3)) * 2.0
    costs[np.arange(36), lab] = 1.0
    table = {"F": F, "costs": costs, "forbid2": {35}}
    for v in range(3):
        cv.add_variant(f"v{v}", lambda i, v=v: table["costs"][i, v])
    cv.add_feature("f0", lambda i: table["F"][i, 0])
    cv.add_feature("f1", lambda i: table["F"][i, 1])
    cv.add_constraint(2, lambda i: i not in table["forbid2"])
    cv.set_default(1)
    return ctx, cv, table


def test_generic_code_variant_train_select(tmp_path):
    n = nitro()
    ctx, cv, table = _toy_cv(n)
    for i in range(36):
        cv.add_training_input(i)
    cv.train(log2c_lo=-1, log2c_hi=3, log2g_lo=-3, log2g_hi=1)
    cost, feat, lab = cv.training_table()
    assert np.array_equal(feat, table["F"])
    assert np.isinf(cost[35, 2]) and np.isfinite(cost[:35]).all()  # constraint -> infinite cost
    assert list(lab) == S.exhaustive_best(cost.tolist())
    # the same table through the oracle: same scaling, grid choice and predictions
    m = S.train(feat, lab, log2c=range(-1, 4, 2), log2g=range(1, -4, -2))
    info = cv.model_info()
    assert (info["C"], info["gamma"]) == (m.C, m.gamma)
    assert info["cv_accuracy"] == pytest.approx(m.cv_accuracy)
    probe = np.array([[0.1, 0.0], [3.9, 0.1], [0.0, 4.2]])
    assert [cv.predict(p) for p in probe] == list(m.predict(probe))
    # deployment: a ruled-out prediction reverts to the default
    assert cv.select(24)[0] == 2
    table["forbid2"] = set(range(24, 36))
    assert cv.select(24)[0] == 1
    assert cv.select(0)[0] == 0
    v, c = cv.call(5)
    assert (v, c) == (0, 1.0)
    p = tmp_path / "toy.model"
    cv.save(p)
    _, cv2, _ = _toy_cv(n)
    cv2.load(p)
    assert [cv2.predict(p_) for p_ in probe] == [cv.predict(p_) for p_ in probe]
    with pytest.raises(n.NitroError) as e:
        cv.add_training_input(3)
    assert e.value.code == 3


def test_select_before_train_is_state_error():
    n = nitro()
    ctx, cv, _ = _toy_cv(n)
    with pytest.raises(n.NitroError) as e:
        cv.select(0)
    assert e.value.code == 3


@pytest.mark.parametrize("ext", [False, True], ids=["paper_scaling", "r11x_log_clip"])
def test_train_from_table_equals_oracle(ext):
    """nitro_cv_train_from_table = the oracle's select path on the same table:
    the paper's plain [-1, 1] scaling (default of nitro_spmv_register) and the
    opt-in R11x extension.  Predictions must agree wherever every OvO decision
    value of the oracle model has |decision| > 1e-6 (reading C12)."""
    n = nitro()
    rng = np.random.default_rng(8)
    F = np.abs(rng.normal(0, 1, (40, 7))) * np.array([1e6, 1e5, 10, 3, 50, 2, 2])
    costs = rng.uniform(1, 2, (40, 5))
    costs[F[:, 2] > 8, 3] = 0.5
    costs[rng.uniform(size=40) < 0.2, 2] = math.inf
    ctx = n.Context()
    cv = n.CodeVariant(ctx, "t")
    for v in range(5):
        cv.add_variant(f"v{v}", lambda inp: 0.0)
    for j in range(7):
        cv.add_feature(f"f{j}", lambda inp: 0.0)
    if ext:
        cv.set_feature_transform(S.R11X_LOG_MASK, S.R11X_CLIP)
        m = S.train(F, S.exhaustive_best(costs.tolist()), log_mask=S.R11X_LOG_MASK, clip=S.R11X_CLIP)
    else:
        m = S.train(F, S.exhaustive_best(costs.tolist()))
    cv.train_from_table(F, costs, log2c_lo=-5, log2c_hi=15, log2g_lo=-15, log2g_hi=3)
    info = cv.model_info()
    assert (info["C"], info["gamma"]) == (m.C, m.gamma)
    assert info["cv_accuracy"] == pytest.approx(m.cv_accuracy)
    # predictions agree, including inputs far outside the training range
    T = np.abs(rng.normal(0, 1, (30, 7))) * np.array([1e6, 1e5, 10, 3, 50, 2, 2])
    T[:10] *= 1e3
    ours = np.array([cv.predict(t) for t in T])
    ref = m.predict(T)
    firm = S.decided(m, T)
    assert firm.sum() >= len(T) // 2
    assert np.array_equal(ours[firm], ref[firm]), (ours, ref, firm)


def test_spmv_register_uses_paper_scaling(tmp_path):
    """nitro_spmv_register leaves the paper's plain [-1, 1] scaling in place
    (no log transform, no clipping): the saved model records transform 0 0."""
    n = nitro()
    ctx = n.Context()
    cv = n.CodeVariant(ctx, "spmv")
    cv.register_spmv()
    rng = np.random.default_rng(3)
    F = np.abs(rng.normal(0, 1, (12, 7))) + 1
    costs = rng.uniform(1, 2, (12, 5))
    cv.train_from_table(F, costs, log2c_lo=1, log2c_hi=1, log2g_lo=1, log2g_hi=1)
    p = tmp_path / "m.txt"
    cv.save(p)
    assert p.read_text().split("\n")[2].split() == ["0", "0"]


def test_feature_transform_clips_to_training_extremes():
    """With clipping, an input beyond the training range predicts like the
    training extreme it is clipped to; without it the RBF model extrapolates."""
    n = nitro()
    F = np.array([[1.0, 10.0], [2.0, 20.0], [3.0, 30.0], [4.0, 40.0], [5.0, 50.0], [6.0, 60.0]])
    costs = np.array([[1, 2], [1, 2], [1, 2], [2, 1], [2, 1], [2, 1]], float)
    for clip in (False, True):
        ctx = n.Context()
        cv = n.CodeVariant(ctx, f"clip{clip}")
        for v in range(2):
            cv.add_variant(f"v{v}", lambda inp: 0.0)
        for j in range(2):
            cv.add_feature(f"f{j}", lambda inp: 0.0)
        cv.set_feature_transform(0b11, clip)
        cv.train_from_table(F, costs, log2c_lo=1, log2c_hi=1, log2g_lo=1, log2g_hi=1)
        m = S.train(F, S.exhaustive_best(costs.tolist()), log2c=[1], log2g=[1], log_mask=0b11, clip=clip)
        far = np.array([[6.0e6, 6.0e7]])
        assert cv.predict(far[0]) == m.predict(far)[0]
        if clip:
            assert cv.predict(far[0]) == cv.predict(F[-1]) == 1
    with pytest.raises(n.NitroError):
        cv.set_feature_transform(0, False)   # after training: NITRO_E_STATE


def test_dist_partition_nnz_balanced():
    n = nitro()
    rp = np.concatenate([[0], np.cumsum(np.random.default_rng(1).integers(0, 30, 1000))]).astype(np.int64)
    for P in (1, 2, 3, 8):
        b = n.dist_partition(rp, P)
        assert b[0] == 0 and b[-1] == 1000 and np.all(np.diff(b) >= 0)
        Z = rp[-1]
        for r in range(1, P):
            target = -(-r * Z // P)
            assert rp[b[r]] >= target and (b[r] == 0 or rp[b[r] - 1] < target)


@pytest.mark.parametrize("corrupt", ["dim", "class", "sv", "pair", "nf"])
def test_load_model_validates_indices(tmp_path, corrupt):
    """A stale or corrupted model file is NITRO_E_IO at load, never an
    out-of-bounds read at predict time (dimension, class ids,
    support-vector ids and pair class indices are checked)."""
    n = nitro()
    ctx, cv, _ = _toy_cv(n)
    for i in range(36):
        cv.add_training_input(i)
    cv.train(log2c_lo=1, log2c_hi=1, log2g_lo=1, log2g_hi=1)
    p = tmp_path / "ok.model"
    cv.save(p)
    lines = p.read_text().split("\n")
    # layout (cv.cpp save): header, n_feat n_var default, transform, scaler lines, params, svm header, ...
    hdr_i = next(i for i, l in enumerate(lines) if len(l.split()) == 4 and i > 3)
    d, ntr, const, ncls = map(int, lines[hdr_i].split())
    if corrupt == "dim":
        lines[hdr_i] = f"{d + 1} {ntr} {const} {ncls}"
    elif corrupt == "nf":
        nf_line = lines[1].split()
        lines[1] = " ".join([str(int(nf_line[0]) + 5)] + nf_line[1:])
    elif corrupt == "class":
        lines[hdr_i + 1] = " ".join(["99"] * ncls)
    else:
        # first pair line "ca cb rho ns", then "sv coef" lines
        pi = next(i for i in range(hdr_i + 2, len(lines)) if len(lines[i].split()) == 4)
        if corrupt == "pair":
            ca, cb, rho, ns = lines[pi].split()
            lines[pi] = f"{ncls + 3} {cb} {rho} {ns}"
        else:
            sv, coef = lines[pi + 1].split()
            lines[pi + 1] = f"{ntr + 100} {coef}"
    q = tmp_path / "bad.model"
    q.write_text("\n".join(lines))
    _, cv2, _ = _toy_cv(n)
    with pytest.raises(n.NitroError) as e:
        cv2.load(q)
    assert e.value.code == 8
