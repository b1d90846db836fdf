"""BASELINE configs[4] at its full size on one B200: the 3D 27-point stencil on
a 512^3 grid (134,217,728 rows, 3,609,741,304 nnz > 2^31, so int64 rowptr and
64-bit entry offsets everywhere), fp32, random values.

* Feature pass: exact integers against the closed forms (tests/golden/,
  Z = (3n-2)^3, S2 = (9n-10)^3, Lmax = D = 27) and the doubles bit-exact against
  the oracle's finishing step on those integers (the CSR does not fit the host).
* Every variant (same launch configuration as bench / tools/c4_probe.py): y on
  sampled rows — both grid boundaries, the rows around the 2^31-th entry, and
  random rows — against the oracle on those rows (per-row tolerance of the
  north star).
* One rank of the 8-way nnz-balanced partition (halo exchange layout, SURVEY
  §8(f) f3) at the same size: run from the exchanged x, same sampled check.
"""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from synth import Csr

pytestmark = pytest.mark.gpu

N1 = 512
GOLDEN = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "stencil_closed_forms.json")))["3d27_n512"]


def nitro():
    import paper_conf_ipps_muralidharanshgc14_b200 as n
    return n


def sample_rows(rp_d, N, rng, lo=0, hi=None, k=3000):
    """Sorted unique rows: first / last two z-planes' corners and edges, the
    rows whose entries straddle entry 2^31, and k random rows in [lo, hi)."""
    import torch
    hi = N if hi is None else hi
    P = N1 * N1
    fixed = [0, 1, N1 - 1, N1, P - 1, P, P + N1 + 1, N - 1, N - P, N - P - 1, N - N1 - 1, lo, hi - 1]
    t = int(torch.searchsorted(rp_d, torch.tensor([2 ** 31], dtype=torch.int64, device=rp_d.device)).item())
    fixed += [t - 2, t - 1, t, t + 1]
    rows = np.concatenate([np.array(fixed, np.int64), rng.integers(lo, hi, k)])
    rows = rows[(rows >= lo) & (rows < hi)]
    return np.unique(rows)


def sub_csr(A, rows, M):
    """Host CSR of the given rows of a device CSR (global column ids)."""
    import torch
    rd = torch.from_numpy(rows).to(A.rowptr.device)
    st = A.rowptr[rd].cpu().numpy()
    en = A.rowptr[rd + 1].cpu().numpy()
    lens = en - st
    ix = np.concatenate([np.arange(s, e, dtype=np.int64) for s, e in zip(st, en)])
    ixd = torch.from_numpy(ix).to(A.rowptr.device)
    rp = np.zeros(len(rows) + 1, np.int64)
    rp[1:] = np.cumsum(lens)
    return Csr(len(rows), M, rp, A.colidx[ixd].cpu().numpy(), A.vals[ixd].cpu().numpy(), False)


def check_rows(y, y_ref, r, what):
    err = np.abs(np.asarray(y, np.float64) - y_ref)
    tol = 1e-5 * r + 1e-30
    bad = np.nonzero(err > tol)[0]
    assert bad.size == 0, f"{what}: {bad.size} sampled rows out of tolerance, first {bad[:5]}"


@pytest.fixture(scope="module")
def c4(cuda):
    import torch
    A = synth.stencil("3d27", N1, mode=1, seed=1, device=cuda)   # int64 rowptr (nnz > 2^31)
    assert A.rowptr.dtype == torch.int64 and A.nnz == GOLDEN["nnz"]
    x = synth.vector(A.cols, seed=2)                               # host, U(-1,1) \ {0}
    xd = torch.from_numpy(x).to(cuda)
    yield A, x, xd
    del A, xd
    torch.cuda.empty_cache()


def test_c4_features_closed_form(cuda, c4):
    n = nitro()
    A, _, _ = c4
    M = n.SpMV.from_csr(A)
    f = M.features()
    g = GOLDEN
    assert (f["rows"], f["nnz"], f["sum_len"], f["sum_len2"], f["max_row"], f["ndiag"]) == \
        (g["rows"], g["nnz"], g["nnz"], g["sum_len2"], 27, 27)
    want = oracle.finish_features(g["rows"], g["rows"], g["nnz"], g["nnz"], g["sum_len2"], 27, 27)
    for k in ("mean", "sd", "max_dev", "dia_fill", "ell_fill"):
        assert f[k] == want[k], k
    assert f["canonical"] == 1
    M.close()


def test_c4_all_variants_sampled(cuda, c4):
    import torch
    n = nitro()
    A, x, xd = c4
    rows = sample_rows(A.rowptr, A.rows, np.random.default_rng(5))
    S = sub_csr(A, rows, A.cols)
    y_ref, r = oracle.spmv(S, x)
    M = n.SpMV.from_csr(A)
    M.set_budget(1e12)
    rd = torch.from_numpy(rows).to(cuda)
    y = torch.empty(A.rows, dtype=torch.float32, device=cuda)
    for v in range(n.NUM_VARIANTS):
        assert M.allowed(v), v
        y.fill_(float("nan"))
        M.run(v, xd, y)
        torch.cuda.synchronize()
        check_rows(y[rd].cpu().numpy(), y_ref, r, n.VARIANT_NAMES[v])
        if v == n.DIA:
            assert M.format_info(v)["compulsory_bytes"] == GOLDEN["dia_inrange_slots"] * 4 + 27 * 4 + 2 * A.rows * 4
        M.release(v)
    M.close()


def test_c4_rank_of_8_halo_sampled(cuda, c4):
    import torch
    n = nitro()
    A, x, xd = c4
    P, q = 8, 3
    bounds = n.dist_partition(A.rowptr.cpu().numpy(), P)
    lo, hi = int(bounds[q]), int(bounds[q + 1])
    rows = sample_rows(A.rowptr, A.rows, np.random.default_rng(6), lo, hi, k=2000)
    S = sub_csr(A, rows, A.cols)
    y_ref, r = oracle.spmv(S, x)
    blk = synth.stencil("3d27", N1, mode=1, seed=1, device=cuda, row0=lo, nrows=hi - lo)
    D = n.Dist.local(q, P, 0)
    Mq = D.spmv(A.rows, bounds, blk.rowptr, blk.colidx, blk.vals, exchange=1)
    info = n.Dist.exchange_info(Mq)
    # the neighbouring plane on each side (+ one row and one point when the
    # nnz-balanced bound is not plane-aligned)
    assert info["mode"] == "halo" and 2 * N1 * N1 <= info["halo_len"] <= 2 * (N1 * N1 + N1 + 1)
    H = torch.from_numpy(n.Dist.halo_cols(Mq).astype(np.int64)).to(cuda)
    below = int((H < lo).sum())
    xe = torch.cat([xd[H[:below]], xd[lo:hi], xd[H[below:]]])
    rl = torch.from_numpy(rows - lo).to(cuda)
    for v in range(n.NUM_VARIANTS):
        yq = torch.full((hi - lo,), float("nan"), dtype=torch.float32, device=cuda)
        D.run_gathered(Mq, v, xe, yq)
        torch.cuda.synchronize()
        check_rows(yq[rl].cpu().numpy(), y_ref, r, f"rank {q}/{P} {n.VARIANT_NAMES[v]}")
        Mq.release(v)
    Mq.close()
    D.close()
