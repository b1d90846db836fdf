"""Pins of the CPU oracle against things other than itself (not gpu).

Each test names what pins it: dense matvec, brute force over all 3x3
patterns, scipy, closed forms of Poisson stencils (tests/golden/), identity /
permutation special cases, round trips, hand-derived HYB-width cases, sklearn.
"""
import itertools
import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
import synth
from synth import Csr

GOLDEN = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "stencil_closed_forms.json")))


def from_dense(Ad, fp64=True):
    Ad = np.asarray(Ad)
    N, M = Ad.shape
    rp = [0]
    ci, v = [], []
    for i in range(N):
        for j in range(M):
            if Ad[i, j] != 0:
                ci.append(j)
                v.append(Ad[i, j])
        rp.append(len(ci))
    return Csr(N, M, np.array(rp, np.int64), np.array(ci, np.int32),
               np.array(v, np.float64 if fp64 else np.float32), fp64)


def rand_sparse(N, M, density, seed, fp64=True):
    rng = np.random.default_rng(seed)
    Ad = rng.uniform(-1, 1, (N, M)) * (rng.uniform(0, 1, (N, M)) < density)
    if not fp64:
        Ad = Ad.astype(np.float32)
    return Ad, from_dense(Ad, fp64)


# ------------------------------------------------------------------ SpMV (C1)
@pytest.mark.parametrize("seed", range(6))
def test_spmv_vs_dense(seed):
    N, M = [(1, 1), (7, 5), (33, 64), (64, 64), (64, 17), (40, 40)][seed]
    Ad, A = rand_sparse(N, M, 0.3, seed)
    x = np.random.default_rng(100 + seed).uniform(-1, 1, M)
    y, r = oracle.spmv(A, x)
    yd = Ad @ x
    rd = np.abs(Ad) @ np.abs(x)
    assert np.all(np.abs(y - yd) <= 1e-14 * rd + 1e-300)
    np.testing.assert_allclose(r, rd, rtol=1e-14, atol=0)


def test_spmv_all_3x3_patterns():
    """Brute force: every one of the 512 sparsity patterns of a 3x3 matrix."""
    rng = np.random.default_rng(7)
    for mask in range(512):
        P = np.array([(mask >> b) & 1 for b in range(9)]).reshape(3, 3)
        Ad = P * rng.uniform(0.5, 2.0, (3, 3)) * rng.choice([-1, 1], (3, 3))
        A = from_dense(Ad)
        x = rng.uniform(-1, 1, 3)
        y, _ = oracle.spmv(A, x)
        for i in range(3):  # explicit row sums in column order
            s = 0.0
            for j in range(3):
                if P[i, j]:
                    s = s + Ad[i, j] * x[j]
            assert y[i] == s
        assert oracle.is_canonical(A)


@pytest.mark.parametrize("seed", range(3))
def test_spmv_bit_identical_to_scipy(seed):
    """scipy's csr_matvec sums each row sequentially in storage order (fp64)."""
    S = sp.random(3000, 2500, density=0.01, random_state=seed, format="csr", dtype=np.float64)
    S.sort_indices()
    A = Csr(3000, 2500, S.indptr.astype(np.int64), S.indices.astype(np.int32), S.data, True)
    x = np.random.default_rng(seed).uniform(-1, 1, 2500)
    y, _ = oracle.spmv(A, x)
    assert np.array_equal(y, S @ x)


@pytest.mark.parametrize("threads", [1, 3, 8])
def test_spmv_threads_bit_identical(threads):
    """The all-core baseline loop (rows split over threads, bench.py only) is
    the same per-row sequential sum: y and r bit-identical to oracle.spmv."""
    A = synth.rmat(12, 8, seed=5, fp64=True)
    x = synth.vector(A.cols, seed=3, fp64=True)
    y, r = oracle.spmv(A, x)
    y2, r2, used = oracle.spmv_threads(A, x, threads)
    assert used == threads
    assert np.array_equal(y, y2) and np.array_equal(r, r2)
    fn = oracle.spmv_prepared(A, x, threads)
    assert fn() == threads
    assert np.array_equal(fn.y, y) and np.array_equal(fn.r, r)


def test_spmv_identity_and_permutation():
    N = 1000
    x = np.random.default_rng(1).uniform(-1, 1, N)
    I = Csr(N, N, np.arange(N + 1, dtype=np.int64), np.arange(N, dtype=np.int32), np.ones(N), True)
    assert np.array_equal(oracle.spmv(I, x)[0], x)
    pi = np.random.default_rng(2).permutation(N)
    P = Csr(N, N, np.arange(N + 1, dtype=np.int64), pi.astype(np.int32), np.ones(N), True)
    assert np.array_equal(oracle.spmv(P, x)[0], x[pi])


def test_spmv_empty_rows_and_nnz0():
    A = Csr(5, 4, np.zeros(6, np.int64), np.zeros(0, np.int32), np.zeros(0), True)
    y, r = oracle.spmv(A, np.ones(4))
    assert np.array_equal(y, np.zeros(5)) and np.array_equal(r, np.zeros(5))


@pytest.mark.parametrize("n", [64, 100])
def test_spmv_2d5_poisson_row_sums(n):
    A = synth.stencil("2d5", n)
    y, _ = oracle.spmv(A, np.ones(A.cols))
    assert set(np.unique(y).tolist()) == {0.0, 1.0, 2.0}
    assert y.sum() == 4 * n
    if n == 64:
        assert y.sum() == GOLDEN["2d5_n64"]["sum_y_x1"]


@pytest.mark.parametrize("n", [8, 20])
def test_spmv_3d27_poisson_row_sums(n):
    A = synth.stencil("3d27", n)
    y, _ = oracle.spmv(A, np.ones(A.cols))
    assert set(np.unique(y).tolist()) == {0.0, 9.0, 15.0, 19.0}
    assert y.sum() == 27 * n ** 3 - (3 * n - 2) ** 3


def test_spmv_integer_stencil_fp32_exact():
    """Integer stencil x integer x: every partial sum is an integer < 2^24, so
    a float32 evaluation equals the fp64 oracle exactly (C2 pin)."""
    A = synth.stencil("2d5", 64)
    x = synth.vector(A.cols, seed=1, mode=1)
    y, _ = oracle.spmv(A, x)
    Ad = np.zeros((A.rows, A.cols), np.float32)
    for i in range(A.rows):
        c, v = A.row(i)
        Ad[i, c] = v
    assert np.array_equal((Ad @ x.astype(np.float32)).astype(np.float64), y)


# ------------------------------------------------------------------ features (C4)
def exact_sd(N, S1, S2):
    return math.sqrt(Fraction(N * S2 - S1 * S1, N * N))


def ulp_close(a, b, k=2):
    return abs(a - b) <= k * math.ulp(max(abs(a), abs(b), 1e-300))


def test_features_2d5_n64_golden():
    g = GOLDEN["2d5_n64"]
    f = oracle.features(synth.stencil("2d5", 64))
    for key in ("rows", "nnz", "sum_len2", "max_row", "ndiag", "mean", "dia_fill", "ell_fill"):
        assert f[key] == g[key], key
    assert ulp_close(f["sd"], exact_sd(4096, 20224, 100104))
    assert f["max_dev"] == 5 - 4.9375
    assert f["canonical"] == 1


@pytest.mark.parametrize("n", [3, 8, 16, 40])
def test_features_3d27_closed_form(n):
    f, offs = oracle.features(synth.stencil("3d27", n), with_offsets=True)
    N = n ** 3
    assert f["nnz"] == (3 * n - 2) ** 3
    assert f["sum_len2"] == (9 * n - 10) ** 3
    assert f["max_row"] == 27 and f["ndiag"] == 27
    want = sorted(dz * n * n + dy * n + dx for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1))
    assert offs.tolist() == want
    assert ulp_close(f["sd"], exact_sd(N, (3 * n - 2) ** 3, (9 * n - 10) ** 3))
    assert f["ell_fill"] == 27 * N / (3 * n - 2) ** 3


def test_features_3d27_n128_golden():
    g = GOLDEN["3d27_n128"]
    f = oracle.features(synth.stencil("3d27", 128))
    for key in ("rows", "nnz", "sum_len2", "max_row", "ndiag"):
        assert f[key] == g[key]
    assert ulp_close(f["sd"], exact_sd(g["rows"], g["nnz"], g["sum_len2"]))


def test_finish_features_matches_full_pass_and_n512_closed_form():
    """The finishing step alone (used where the integers come from closed forms)
    equals the full pass on a computed matrix, and at 512^3 (BASELINE configs[4],
    whose CSR does not fit the host) gives the exact-rational sd within 2 ulp."""
    A = synth.stencil("3d27", 12, mode=1, seed=4)
    f = oracle.features(A)
    g = oracle.finish_features(f["rows"], f["cols"], f["nnz"], f["sum_len"], f["sum_len2"], f["max_row"], f["ndiag"])
    assert g == f
    c = GOLDEN["3d27_n512"]
    g = oracle.finish_features(c["rows"], c["rows"], c["nnz"], c["nnz"], c["sum_len2"], 27, 27)
    assert ulp_close(g["sd"], exact_sd(c["rows"], c["nnz"], c["sum_len2"]))
    assert g["mean"] == c["nnz"] / c["rows"] and g["max_dev"] == 27 - c["nnz"] / c["rows"]
    assert g["dia_fill"] == g["ell_fill"] == 27 * c["rows"] / c["nnz"]
    z = oracle.finish_features(0, 5, 0, 0, 0, 0, 0)
    assert z["mean"] == z["sd"] == z["dia_fill"] == 0.0


@pytest.mark.parametrize("n", [2, 5, 1000])
def test_features_1d3(n):
    f = oracle.features(synth.stencil("1d3", n))
    assert f["nnz"] == 3 * n - 2 and f["ndiag"] == 3 and f["max_row"] == min(3, n)


@pytest.mark.parametrize("N,b", [(100, 1), (500, 7), (300, 48)])
def test_features_banded_full(N, b):
    f = oracle.features(synth.banded(N, b, 1.0, seed=3))
    assert f["nnz"] == (2 * b + 1) * N - b * (b + 1)
    assert f["ndiag"] == 2 * b + 1


def test_features_identity_uniform_permutation():
    N = 777
    I = Csr(N, N, np.arange(N + 1, dtype=np.int64), np.arange(N, dtype=np.int32), np.ones(N), True)
    f = oracle.features(I)
    assert (f["nnz"], f["sd"], f["ndiag"], f["dia_fill"], f["ell_fill"], f["mean"]) == (N, 0.0, 1, 1.0, 1.0, 1.0)
    U = synth.uniform(2000, 13, seed=5)
    fu = oracle.features(U)
    assert fu["sd"] == 0.0 and fu["ell_fill"] == 1.0 and fu["max_dev"] == 0.0 and fu["mean"] == 13.0
    pi = np.random.default_rng(3).permutation(N)
    P = Csr(N, N, np.arange(N + 1, dtype=np.int64), pi.astype(np.int32), np.ones(N), True)
    fp, offs = oracle.features(P, with_offsets=True)
    assert fp["ndiag"] == len(set((pi - np.arange(N)).tolist()))
    assert offs.tolist() == sorted(set((pi - np.arange(N)).tolist()))


def test_features_rectangular_offsets_brute_force():
    for seed in range(20):
        rng = np.random.default_rng(seed)
        N, M = int(rng.integers(1, 9)), int(rng.integers(1, 9))
        Ad, A = rand_sparse(N, M, 0.4, seed)
        f, offs = oracle.features(A, with_offsets=True)
        want = sorted({j - i for i in range(N) for j in range(M) if Ad[i, j] != 0})
        assert offs.tolist() == want
        L = (Ad != 0).sum(axis=1)
        assert f["sum_len2"] == int((L * L).sum()) and f["max_row"] == int(L.max())


def test_features_n0_all_zero():
    A = Csr(0, 5, np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0), True)
    f = oracle.features(A)
    assert all(f[k] == 0 for k in ("mean", "sd", "max_dev", "dia_fill", "ell_fill", "ndiag"))


def test_canonical_detection():
    base = dict(rows=2, cols=3, fp64=True)
    ok = Csr(rowptr=np.array([0, 2, 3]), colidx=np.array([0, 2, 1], np.int32), vals=np.ones(3), **base)
    assert oracle.is_canonical(ok)
    for rp, ci in [([0, 2, 3], [2, 0, 1]), ([0, 2, 3], [1, 1, 1]), ([0, 2, 3], [0, 3, 1]),
                   ([0, 2, 1], [0, 1, 1]), ([1, 2, 3], [0, 1, 1]), ([0, 2, 3], [-1, 1, 1])]:
        bad = Csr(rowptr=np.array(rp), colidx=np.array(ci, np.int32), vals=np.ones(3), **base)
        assert not oracle.is_canonical(bad), (rp, ci)


# ------------------------------------------------------------------ conversions (C5-C7)
def _mats():
    yield synth.stencil("2d5", 17, mode=1, seed=4)
    yield synth.stencil("3d27", 6, mode=1, seed=5, fp64=True)
    yield synth.banded(300, 5, 0.5, seed=6)
    yield synth.uniform(500, 9, variable=True, seed=7, M=800)
    yield synth.rmat(10, 8, seed=8)
    yield Csr(7, 3, np.zeros(8, np.int64), np.zeros(0, np.int32), np.zeros(0), True)


def _same_csr(A, rp, ci, v):
    assert np.array_equal(np.asarray(A.rowptr, np.int64), rp)
    assert np.array_equal(np.asarray(A.colidx), ci)
    assert np.array_equal(np.asarray(A.vals, np.float64), v)


def test_ell_round_trip_and_layout():
    for A in _mats():
        K, ld, ecol, ev = oracle.csr_to_ell(A)
        assert ld % 32 == 0 and ld >= A.rows
        _same_csr(A, *oracle.ell_to_csr(A.rows, K, ld, ecol, ev))
        assert np.all(ecol.reshape(K, ld)[:, A.rows:] == -1)


def test_ell_dia_layout_brute_force_3x3():
    rng = np.random.default_rng(11)
    for mask in range(1, 512):
        P = np.array([(mask >> b) & 1 for b in range(9)]).reshape(3, 3)
        Ad = P * rng.uniform(0.5, 2.0, (3, 3))
        A = from_dense(Ad)
        K, ld, ecol, ev = oracle.csr_to_ell(A)
        E = ecol.reshape(K, ld)
        V = ev.reshape(K, ld)
        for i in range(3):
            nzc = [j for j in range(3) if P[i, j]]
            for k in range(K):
                if k < len(nzc):
                    assert E[k, i] == nzc[k] and V[k, i] == Ad[i, nzc[k]]
                else:
                    assert E[k, i] == -1 and V[k, i] == 0.0
        offs, ld2, dv = oracle.csr_to_dia(A)
        DV = dv.reshape(len(offs), ld2)
        assert offs.tolist() == sorted({j - i for i in range(3) for j in range(3) if P[i, j]})
        for d, o in enumerate(offs):
            for i in range(3):
                j = i + o
                want = Ad[i, j] if 0 <= j < 3 else 0.0
                assert DV[d, i] == want


def test_dia_round_trip():
    for A in _mats():
        if A.nnz == 0:
            continue
        offs, ld, dv = oracle.csr_to_dia(A)
        _same_csr(A, *oracle.dia_to_csr(A.rows, A.cols, offs, ld, dv))


def test_dia_inrange_slots_3d27():
    n = 12
    A = synth.stencil("3d27", n)
    offs, ld, dv = oracle.csr_to_dia(A)
    N = n ** 3
    inrange = sum(N - abs(o) for o in offs.tolist())
    assert inrange == sum(N - abs(dz * n * n + dy * n + dx)
                          for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1))


def test_hyb_round_trip():
    for A in _mats():
        K, ld, ecol, ev, tr, tc, tv = oracle.csr_to_hyb(A)
        _same_csr(A, *oracle.hyb_to_csr(A.rows, K, ld, ecol, ev, tr, tc, tv))
        # tail sorted by (row, col)
        if len(tr) > 1:
            key = tr.astype(np.int64) * (A.cols + 1) + tc
            assert np.all(np.diff(key) > 0)


def _lengths_matrix(lengths, M=None):
    lengths = np.asarray(lengths, np.int64)
    M = int(lengths.max()) + 1 if M is None else M
    rp = np.zeros(len(lengths) + 1, np.int64)
    rp[1:] = np.cumsum(lengths)
    ci = np.concatenate([np.arange(L, dtype=np.int32) for L in lengths]) if rp[-1] else np.zeros(0, np.int32)
    return Csr(len(lengths), M, rp, ci, np.ones(int(rp[-1])), True)


def test_hyb_width_hand_cases():
    """Hand-derived from the C7 rule (R_k = #rows longer than k)."""
    # 4096 rows of length 5 + 8192 of length 1: R_k = 4096 for k = 1..4, 3*R_k == N (not <),
    # R_k == 4096 (not <)  => never triggers => K = Lmax = 5
    assert oracle.hyb_width(_lengths_matrix([5] * 4096 + [1] * 8192)) == 5
    # one fewer long row: R_1 = 4095 < 4096 => K = 1
    assert oracle.hyb_width(_lengths_matrix([5] * 4095 + [1] * 8193)) == 1
    # fewer than 4096 rows at all: R_0 < 4096 => K = 0 (everything in the tail)
    assert oracle.hyb_width(_lengths_matrix([3] * 100)) == 0
    # uniform rows, N large: R_k = N for all k < k0 => K = Lmax
    assert oracle.hyb_width(synth.uniform(20000, 32, seed=1)) == 32
    # 3D 27-point stencil n = 32: interior rows (30^3 = 27000 >= N/3, >= 4096) keep R_k large
    assert oracle.hyb_width(synth.stencil("3d27", 32)) == 27
    # power law: most rows short => small K, most entries in the tail
    R = synth.rmat(14, 16, seed=3)
    K = oracle.hyb_width(R)
    assert K < int(np.diff(R.rowptr).max()) // 100


# ------------------------------------------------------------------ constraints (C9)
def test_constraints():
    big = 1e18
    f = oracle.features(synth.stencil("3d27", 10))
    assert oracle.allowed_mask(f, 1024, 4, big) == [True] * 5
    fu = oracle.features(synth.uniform(5000, 16, seed=2))
    assert oracle.allowed_mask(fu, 5024, 4, big) == [True, True, True, False, True]
    fr = oracle.features(synth.rmat(12, 16, seed=2))
    m = oracle.allowed_mask(fr, 4096, 8, big)
    assert m[2] is False and m[3] is False and m[1] and m[4]
    # memory budget alone rules a format out
    assert not oracle.dia_allowed(f, 1024, 4, 27 * 1024 * 4 - 1)
    assert oracle.dia_allowed(f, 1024, 4, 27 * 1024 * 4)
