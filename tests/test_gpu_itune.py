"""Incremental tuning (NEXT f1) on the GPU: nitro_cv_itune over
registered SpMV inputs whose labels come from LIVE exhaustive timing of the
five variants (the registered variant functions time the kernels), compared
with the oracle's itune fed the very costs the library measured: the same
initial set, the same BvSB pick sequence and the same history.  Also the
training timeout of the exhaustive search."""
import math

import numpy as np
import pytest

import synth
from oracle.itune import itune as oracle_itune
from oracle import select as S

pytestmark = pytest.mark.gpu


def nitro():
    import paper_conf_ipps_muralidharanshgc14_b200 as n
    return n


def _inputs(cuda):
    """12 mixed-class matrices (stencil / banded / uniform / power-law), small
    enough that a whole labelling takes seconds."""
    return [synth.stencil("3d27", 40, mode=1, seed=1), synth.stencil("2d5", 300, mode=1, seed=2),
            synth.stencil("1d3", 200_000, mode=1, seed=3), synth.stencil("3d7", 50, mode=1, seed=4),
            synth.banded(150_000, 8, 1.0, seed=5), synth.banded(120_000, 30, 0.1, seed=6),
            synth.uniform(150_000, 3, variable=True, seed=7), synth.uniform(100_000, 32, seed=8),
            synth.uniform(200_000, 12, variable=True, seed=9), synth.rmat(16, 16, seed=10, fp64=False),
            synth.rmat(17, 8, seed=11, fp64=False), synth.rmat(15, 32, seed=12, fp64=False)]


def test_itune_live_labels_match_oracle(cuda):
    import torch
    n = nitro()
    ctx = n.Context()
    cv = n.CodeVariant(ctx, "spmv")
    cv.register_spmv()
    keep = []
    for A in _inputs(cuda):
        Ad = synth.to_device(A, cuda)
        M = n.SpMV.from_csr(Ad)
        x = torch.from_numpy(synth.vector(A.cols, seed=3)).to(cuda)
        y = torch.empty(A.rows, dtype=torch.float32, device=cuda)
        rec = n.spmv_input(M, x, y, warmup=2, reps=7)
        keep.append((Ad, M, x, y, rec))
        cv.add_training_input(n.addr(rec))
    grid = dict(log2c_lo=1, log2c_hi=5, log2g_lo=-3, log2g_hi=1)
    h = cv.itune(init=3, iters=5, seed=2, **grid)
    cost, feat, lab = cv.training_table()
    n0 = h["n_labelled"][0]
    assert n0 >= 3 and len(h["n_labelled"]) == 6 and h["n_labelled"][-1] == n0 + 5
    assert len(set(lab.tolist())) >= 2                        # the initial set holds two labels (R15)
    # labels = exhaustive argmin of the live costs, disallowed = +inf
    assert list(lab) == S.exhaustive_best(cost.tolist())
    # input index of each table row: the seeded initial order, then the picks
    s = S.splitmix64(2)
    order = sorted(range(len(keep)), key=lambda i: (S.splitmix64(s ^ i), i))
    labelled = order[:n0] + [p for p in h["picked"] if p >= 0]
    assert len(labelled) == cost.shape[0] and len(set(labelled)) == len(labelled)
    by_input = {i: list(cost[r]) for r, i in enumerate(labelled)}
    # all features of the pool (the library computed them first)
    F = np.array([[M.features()[k] for k in n.FEATURE_NAMES] for _, M, _, _, _ in keep])
    np.testing.assert_array_equal(F[labelled], feat)

    def label_fn(i):
        assert i in by_input, f"oracle asked to label input {i}, which the library never labelled"
        return by_input[i]

    ref = oracle_itune(F, label_fn, n.NUM_VARIANTS, init=3, iters=5, seed=2, log2c=(1, 3, 5), log2g=(1, -1, -3))
    assert ref["n_labelled"] == h["n_labelled"]
    assert ref["picked"] == h["picked"]
    assert ref["final"]["labelled"] == labelled
    for _, M, _, _, _ in keep:
        M.close()


def test_training_timeout_stops_slow_variants(cuda):
    """With the default timeout factor (20), a variant far slower than the
    input's best so far is ranked after >= 3 reps: its cost still exceeds
    20x the best, the label is unchanged, and the whole labelling is faster
    than with the timeout off.  (The default, CSR-vector, is timed first, so
    CSR-scalar — variant 0 — already has a reference cost.)"""
    import time
    import torch
    n = nitro()
    # one 150K-entry row: CSR-scalar walks it with one thread (hundreds of x slower)
    rng = np.random.default_rng(1)
    N = 20000
    lens = rng.integers(0, 6, N)
    lens[7] = 150_000
    rp = np.zeros(N + 1, np.int64)
    rp[1:] = np.cumsum(lens)
    M_ = 160_000
    ci = np.concatenate([np.sort(rng.choice(M_, int(L), replace=False)) for L in lens]).astype(np.int32)
    A = synth.Csr(N, M_, rp, ci, np.ones(ci.size, np.float32), False)
    Ad = synth.to_device(A, cuda)
    res = {}
    M = n.SpMV.from_csr(Ad)                 # one handle: formats prepared once (by the warm-up run)
    x = torch.ones(M_, device=cuda)
    y = torch.empty(N, device=cuda)
    for factor in (0.0, 20.0, 0.0):
        ctx = n.Context()
        cv = n.CodeVariant(ctx, "spmv")
        cv.register_spmv()
        rec = n.spmv_input(M, x, y, warmup=1, reps=61)
        cv.add_training_input(n.addr(rec))
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        cv.train(log2c_lo=1, log2c_hi=1, log2g_lo=1, log2g_hi=1, timeout_factor=factor)
        res[factor] = (time.perf_counter() - t0, cv.training_table())
    M.close()
    (t_on, (c_on, _, l_on)), (t_off, (c_off, _, l_off)) = res[20.0], res[0.0]
    best = np.min(c_on[0])
    assert l_on[0] == l_off[0]
    assert c_on[0, n.CSR_SCALAR] > 20 * best and c_off[0, n.CSR_SCALAR] > 20 * best
    assert t_on < t_off
