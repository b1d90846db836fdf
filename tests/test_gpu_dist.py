"""Multi-GPU row-partitioned SpMV (nitro_dist_*) on one B200.

* Every rank of a P-way partition (P = 2, 3, 4, 8) is built on the one GPU with
  a communicator-less handle and run from the gathered x: the concatenated y
  equals the single-GPU y bit for bit for the row-local CSR variants and is
  within tolerance of the oracle for all variants.
* P = 1 through a real NCCL communicator: run (copy + in-place all-gather +
  interior/boundary split) and global features equal the single-GPU path.
"""
import numpy as np
import pytest

import oracle
import synth
from synth import Csr

pytestmark = pytest.mark.gpu


def nitro():
    import paper_conf_ipps_muralidharanshgc14_b200 as n
    return n


def block(A, lo, hi):
    rp = np.asarray(A.rowptr, np.int64)
    a, b = rp[lo], rp[hi]
    return Csr(hi - lo, A.cols, rp[lo:hi + 1] - a, A.colidx[a:b], A.vals[a:b], A.fp64)


def mats():
    yield "3d27_n24", synth.stencil("3d27", 24, mode=1, seed=3)
    yield "banded", synth.banded(20011, 9, 0.5, seed=4)
    yield "uniform_var", synth.uniform(30000, 12, variable=True, seed=5)
    yield "rmat13", synth.rmat(13, 16, seed=6, fp64=False)
    yield "rmat12_fp64", synth.rmat(12, 8, seed=7, fp64=True)


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("name,A", list(mats()))
def test_emulated_ranks_match_single_gpu(cuda, name, A, P):
    import torch
    n = nitro()
    x = synth.vector(A.cols, seed=11, fp64=A.fp64)
    y_ref, r = oracle.spmv(A, x)
    Ad = synth.to_device(A, cuda)
    M1 = n.SpMV.from_csr(Ad)
    xd = torch.from_numpy(x).to(cuda)
    bounds = n.dist_partition(np.asarray(A.rowptr, np.int64), P)
    B = int(np.diff(bounds).max())
    xg = torch.zeros((P * B,), dtype=xd.dtype, device=cuda)  # padding: finite (DIA reads zero slots)
    for q in range(P):
        xg[q * B: q * B + bounds[q + 1] - bounds[q]] = xd[bounds[q]:bounds[q + 1]]
    ranks = []
    for q in range(P):
        D = n.Dist.local(q, P, 0)
        blk = synth.to_device(block(A, bounds[q], bounds[q + 1]), cuda)
        Mq = D.spmv(A.rows, bounds, blk.rowptr, blk.colidx, blk.vals, exchange=0)
        assert n.Dist.layout(Mq)[0] == B
        ranks.append((D, Mq, blk))
    tol = 1e-12 if A.fp64 else 1e-5
    for v in range(n.NUM_VARIANTS):
        if not M1.allowed(v) and v in (n.ELL, n.DIA):
            continue
        y1 = M1.run(v, xd)
        ys = []
        for D, Mq, blk in ranks:
            yq = torch.full((Mq.rows,), float("nan"), dtype=xd.dtype, device=cuda)
            D.run_gathered(Mq, v, xg, yq)
            ys.append(yq)
        yd = torch.cat(ys)
        torch.cuda.synchronize()
        yd, y1 = yd.cpu().numpy(), y1.cpu().numpy()
        err = np.abs(yd.astype(np.float64) - y_ref)
        assert np.all(err <= tol * r + 1e-30), (name, P, v)
        if v == n.CSR_SCALAR:
            # row-local summation order is partition independent for CSR-scalar.
            # (CSR-vector's is not: K6v's lanes take 16-byte-aligned chunks of
            # the arrays, so the association follows each row start's phase
            # modulo 4 within its part, and a part whose slices are misaligned
            # runs K6 — within the tolerance above, not bit-identical.)
            assert np.array_equal(yd, y1), (name, P, v)


def test_interior_run_of_stencil_slabs(cuda):
    """z-slab partition of a 3D stencil: the interior run is the block minus one
    boundary plane on each side."""
    n = nitro()
    nx = 16
    A = synth.stencil("3d27", (nx, nx, 4 * nx), mode=1, seed=1)
    bounds = np.array([q * nx * nx * nx for q in range(5)], np.int64)
    for q in range(4):
        D = n.Dist.local(q, 4, 0)
        blk = synth.to_device(block(A, bounds[q], bounds[q + 1]), cuda)
        Mq = D.spmv(A.rows, bounds, blk.rowptr, blk.colidx, blk.vals, exchange=0)
        B, i0, i1 = n.Dist.layout(Mq)
        assert B == nx ** 3
        assert i0 == (0 if q == 0 else nx * nx)
        assert i1 == nx ** 3 - (0 if q == 3 else nx * nx)


def test_nccl_single_rank(cuda):
    import torch
    n = nitro()
    A = synth.stencil("3d27", 32, mode=1, seed=2)
    x = synth.vector(A.cols, seed=3)
    Ad = synth.to_device(A, cuda)
    M1 = n.SpMV.from_csr(Ad)
    D = n.Dist(n.dist_unique_id(), 0, 1, 0)
    bounds = np.array([0, A.rows], np.int64)
    Md = D.spmv(A.rows, bounds, Ad.rowptr, Ad.colidx, Ad.vals)
    f1, fd = M1.features(), D.features(Md)
    assert f1 == fd
    xd = torch.from_numpy(x).to(cuda)
    for v in range(5):
        y1 = M1.run(v, xd)
        yd = torch.empty_like(y1)
        D.run(Md, v, xd, yd)
        torch.cuda.synchronize()
        assert torch.equal(y1, yd), v
    D.close()


@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("name,A", list(mats()))
def test_emulated_ranks_halo_layout(cuda, name, A, P):
    """Halo exchange: each rank's layout is [x_local | x[halo]],
    halo = the sorted remote columns its rows reference."""
    import torch
    n = nitro()
    x = synth.vector(A.cols, seed=12, fp64=A.fp64)
    y_ref, r = oracle.spmv(A, x)
    xd = torch.from_numpy(x).to(cuda)
    rp = np.asarray(A.rowptr, np.int64)
    bounds = n.dist_partition(rp, P)
    tol = 1e-12 if A.fp64 else 1e-5
    ranks = []
    for q in range(P):
        lo, hi = int(bounds[q]), int(bounds[q + 1])
        D = n.Dist.local(q, P, 0)
        blk = synth.to_device(block(A, lo, hi), cuda)
        Mq = D.spmv(A.rows, bounds, blk.rowptr, blk.colidx, blk.vals, exchange=1)
        info = n.Dist.exchange_info(Mq)
        H = n.Dist.halo_cols(Mq)
        a, b = rp[lo], rp[hi]
        cols = np.asarray(A.colidx[a:b], np.int64)
        want = np.unique(cols[(cols < lo) | (cols >= hi)])
        assert info["mode"] == "halo" and np.array_equal(H, want)
        assert info["layout_len"] == (hi - lo) + len(H)
        Hd = torch.from_numpy(H.astype(np.int64)).to(cuda)
        below = int((H < lo).sum())
        xe = torch.cat([xd[Hd[:below]], xd[lo:hi], xd[Hd[below:]]])   # [x[H_below] | x_local | x[H_above]]
        ranks.append((D, Mq, blk, xe))
    for v in range(n.NUM_VARIANTS):
        ys = []
        for D, Mq, blk, xe in ranks:
            yq = torch.full((Mq.rows,), float("nan"), dtype=xd.dtype, device=cuda)
            D.run_gathered(Mq, v, xe, yq)
            ys.append(yq)
        yd = torch.cat(ys)
        torch.cuda.synchronize()
        err = np.abs(yd.cpu().numpy().astype(np.float64) - y_ref)
        assert np.all(err <= tol * r + 1e-30), (name, P, v)


def test_halo_is_small_for_stencil_slabs(cuda):
    """3D 27-point z-slabs: the halo is the neighbouring plane(s), so auto mode picks it."""
    n = nitro()
    nx = 16
    A = synth.stencil("3d27", (nx, nx, 4 * nx), mode=1, seed=1)
    bounds = np.array([q * nx ** 3 for q in range(5)], np.int64)
    for q in range(4):
        D = n.Dist.local(q, 4, 0)
        blk = synth.to_device(block(A, bounds[q], bounds[q + 1]), cuda)
        Mq = D.spmv(A.rows, bounds, blk.rowptr, blk.colidx, blk.vals)   # auto
        info = n.Dist.exchange_info(Mq)
        assert info["mode"] == "halo"
        assert info["halo_len"] == nx * nx * (1 if q in (0, 3) else 2)


def test_nccl_single_rank_halo_in_place_x(cuda):
    import torch
    n = nitro()
    A = synth.stencil("3d27", 24, mode=1, seed=5)
    x = synth.vector(A.cols, seed=6)
    Ad = synth.to_device(A, cuda)
    M1 = n.SpMV.from_csr(Ad)
    D = n.Dist(n.dist_unique_id(), 0, 1, 0)
    Md = D.spmv(A.rows, np.array([0, A.rows], np.int64), Ad.rowptr, Ad.colidx, Ad.vals, exchange=1)
    xl = n.Dist.x_local(Md)             # write x straight into the exchange buffer: no copy per multiply
    xl.copy_(torch.from_numpy(x).to(cuda))
    for v in range(5):
        y1 = M1.run(v, xl)
        yd = torch.empty_like(y1)
        D.run(Md, v, xl, yd)
        torch.cuda.synchronize()
        assert torch.equal(y1, yd), v
    D.close()
