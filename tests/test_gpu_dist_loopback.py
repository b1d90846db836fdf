"""P-rank distributed SpMV through the LOOPBACK transport on one B200.

Every rank is a host thread with its own stream and its own nitro_dist handle
of one loopback group (nitro_dist_loopback_create), so the real P > 1 code of
nitro_dist_* runs: the exchange plan (need-matrix all-gather, send-list
send/recv, k_to_local), the per-multiply x exchange (in-place all-gather into
the padded layout, or k_pack + grouped send/recv into the halo layout at
halo_dest), the interior/boundary overlap, and the global features (sum / max
all-reduces, compacted-offset all-gather + union).  Checked against the CPU
oracle: y within the north-star tolerance for every variant
(exact for integer data), features bit-exact."""
import threading

import numpy as np
import pytest

import oracle
import synth
from synth import Csr

pytestmark = pytest.mark.gpu

FEAT_KEYS = ("rows", "cols", "nnz", "sum_len", "sum_len2", "max_row", "ndiag", "canonical",
             "mean", "sd", "max_dev", "dia_fill", "ell_fill")


def nitro():
    import paper_conf_ipps_muralidharanshgc14_b200 as n
    return n


def block(A, lo, hi):
    rp = np.asarray(A.rowptr, np.int64)
    a, b = rp[lo], rp[hi]
    return Csr(hi - lo, A.cols, rp[lo:hi + 1] - a, A.colidx[a:b], A.vals[a:b], A.fp64)


def run_group(A, x, P, exchange, variants, cuda, bounds=None):
    """Run the P ranks as threads; returns (y per variant (concatenated),
    features per rank, exchange info per rank)."""
    import torch
    n = nitro()
    if bounds is None:
        bounds = n.dist_partition(np.asarray(A.rowptr, np.int64), P)
    group = n.Loopback(P, 0)
    out = {"y": {}, "feat": [None] * P, "info": [None] * P, "err": []}
    ys = {v: [None] * P for v in variants}

    def rank(q):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                D = n.Dist.loopback(group, q)
                blk = synth.to_device(block(A, bounds[q], bounds[q + 1]), cuda)
                M = D.spmv(A.rows, bounds, blk.rowptr, blk.colidx, blk.vals, exchange=exchange)
                out["info"][q] = n.Dist.exchange_info(M)
                out["feat"][q] = D.features(M)
                xq = torch.from_numpy(x[bounds[q]:bounds[q + 1]].copy()).to(cuda)
                for v in variants:
                    yq = torch.full((M.rows,), float("nan"), dtype=xq.dtype, device=cuda)
                    D.run(M, v, xq, yq)
                    D.run(M, v, xq, yq)             # twice: the exchange buffers are reused
                    torch.cuda.current_stream().synchronize()
                    ys[v][q] = yq.cpu().numpy()
                M.close()
                D.close()
        except Exception as e:  # surfaced in the main thread
            out["err"].append((q, repr(e)))

    th = [threading.Thread(target=rank, args=(q,)) for q in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=300)
    assert not any(t.is_alive() for t in th), "loopback ranks hung"
    assert not out["err"], out["err"]
    group.close()
    out["y"] = {v: np.concatenate(ys[v]) for v in variants}
    return out


def mats():
    yield "3d27_n20_int", synth.stencil("3d27", 20), True
    yield "3d27_n24", synth.stencil("3d27", 24, mode=1, seed=3), False
    yield "banded_fp64", synth.banded(20011, 9, 0.5, seed=4, fp64=True), False
    yield "uniform_var", synth.uniform(30000, 12, variable=True, seed=5), False
    yield "rmat13", synth.rmat(13, 16, seed=6, fp64=False), False


@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("exchange", [0, 1], ids=["allgather", "halo"])
@pytest.mark.parametrize("name,A,exact", list(mats()))
def test_loopback_ranks_match_oracle(cuda, name, A, exact, exchange, P):
    n = nitro()
    x = synth.vector(A.cols, seed=11, fp64=A.fp64, mode=1 if exact else 0)
    y_ref, r = oracle.spmv(A, x)
    allowed = n.SpMV.from_csr(synth.to_device(A, cuda)).allowed_mask()
    variants = [v for v in range(n.NUM_VARIANTS) if allowed[v] or v not in (n.ELL, n.DIA)]
    res = run_group(A, x, P, exchange, variants, cuda)
    tol = 1e-12 if A.fp64 else 1e-5
    for v in variants:
        y = res["y"][v].astype(np.float64)
        if exact:
            assert np.array_equal(y, y_ref), (name, P, v)
        else:
            assert np.all(np.abs(y - y_ref) <= tol * r + 1e-30), (name, P, v)
    # the exchange really ran: every rank of a P > 1 partition received and sent entries
    for q, info in enumerate(res["info"]):
        assert info["mode"] == ("allgather", "halo")[exchange]
        if exchange == 1:
            assert info["halo_len"] > 0 and info["send_len"] > 0, (q, info)
        else:
            assert info["layout_len"] == P * int(np.diff(n.dist_partition(np.asarray(A.rowptr, np.int64), P)).max())
    f_ref = oracle.features(A)
    for f in res["feat"]:
        for k in FEAT_KEYS:
            assert f[k] == f_ref[k], (k, f[k], f_ref[k])


def test_loopback_halo_lists_are_the_referenced_remote_columns(cuda):
    """Halo mode: each rank's halo = the sorted distinct remote columns its rows
    reference (brute force), and what rank q sends to rank r is exactly r's
    halo entries owned by q (sum of send lengths = sum of halo lengths)."""
    n = nitro()
    A = synth.banded(9001, 40, 0.3, seed=9)
    P = 4
    bounds = n.dist_partition(np.asarray(A.rowptr, np.int64), P)
    x = synth.vector(A.cols, seed=2)
    res = run_group(A, x, P, 1, [n.CSR_SCALAR], cuda, bounds=bounds)
    rp = np.asarray(A.rowptr, np.int64)
    tot_h = tot_s = 0
    for q in range(P):
        cols = A.colidx[rp[bounds[q]]:rp[bounds[q + 1]]]
        remote = np.unique(cols[(cols < bounds[q]) | (cols >= bounds[q + 1])])
        assert res["info"][q]["halo_len"] == len(remote)
        tot_h += res["info"][q]["halo_len"]
        tot_s += res["info"][q]["send_len"]
    assert tot_h == tot_s


def test_loopback_empty_rank_and_uneven_blocks(cuda):
    """A rank that owns no rows (bounds repeat) and very uneven blocks: the
    padded all-gather layout and the empty send/recv lists still work."""
    n = nitro()
    A = synth.stencil("2d5", 40, mode=1, seed=4)
    bounds = np.array([0, 100, 100, 900, A.rows], np.int64)
    x = synth.vector(A.cols, seed=5)
    y_ref, r = oracle.spmv(A, x)
    for exchange in (0, 1):
        res = run_group(A, x, 4, exchange, [n.CSR_SCALAR, n.CSR_VECTOR, n.HYB], cuda, bounds=bounds)
        for v, y in res["y"].items():
            assert np.all(np.abs(y.astype(np.float64) - y_ref) <= 1e-5 * r + 1e-30), (exchange, v)


# ------------------------------------------------------------------ f3 (ii): fused y -> x epilogue (solver loop)
def _loop_ref(A, x0, steps):
    """x_{k+1} = A x_k with the oracle (fp64); integer data keeps it exact."""
    xs, x = [], np.asarray(x0, np.float64)
    for _ in range(steps):
        x, _ = oracle.spmv(A, x)
        xs.append(x)
    return xs


def run_loop_group(A, x0, P, variant, steps, cuda):
    import torch
    n = nitro()
    bounds = n.dist_partition(np.asarray(A.rowptr, np.int64), P)
    group = n.Loopback(P, 0)
    ys = [[None] * P for _ in range(steps)]
    xnext = [None] * P
    err = []

    def rank(q):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                D = n.Dist.loopback(group, q)
                blk = synth.to_device(block(A, bounds[q], bounds[q + 1]), cuda)
                M = D.spmv(A.rows, bounds, blk.rowptr, blk.colidx, blk.vals, exchange=0)
                L = D.loop(M)
                L.x().copy_(torch.from_numpy(np.ascontiguousarray(x0[bounds[q]:bounds[q + 1]])).to(cuda))
                L.start()
                for k in range(steps):
                    y = torch.full((M.rows,), float("nan"), dtype=M.dtype, device=cuda)
                    L.step(variant, y)
                    torch.cuda.current_stream().synchronize()
                    ys[k][q] = y.cpu().numpy()
                xnext[q] = L.x().cpu().numpy()           # the fused epilogue's copy of my block
                L.close()
                M.close()
                D.close()
        except Exception as e:
            err.append((q, repr(e)))

    th = [threading.Thread(target=rank, args=(q,)) for q in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=300)
    assert not any(t.is_alive() for t in th), "loop ranks hung"
    assert not err, err
    group.close()
    return [np.concatenate(ys[k]) for k in range(steps)], np.concatenate(xnext)


@pytest.mark.parametrize("P", [2, 4])
@pytest.mark.parametrize("variant", [0, 1, 2, 3, 4], ids=["csr_scalar", "csr_vector", "ell", "dia", "hyb"])
def test_solver_loop_fused_epilogue(cuda, variant, P):
    """Three multiplies x_{k+1} = A x_k on P loopback ranks: every rank's y
    block equals the oracle's (integer stencil, exact), and the next x each
    rank holds (written by the fused epilogue of every rank: CSR-scalar, ELL,
    DIA; the push fallback for CSR-vector, HYB) equals the last y."""
    A = synth.stencil("2d5", 48)                    # values 4, -1: |row sum| <= 8 -> exact after 3 steps
    x0 = synth.vector(A.cols, seed=3, mode=1)
    ref = _loop_ref(A, x0, 3)
    ys, xlast = run_loop_group(A, x0, P, variant, 3, cuda)
    for k in range(3):
        assert np.array_equal(ys[k].astype(np.float64), ref[k]), (variant, P, k)
    assert np.array_equal(xlast.astype(np.float64), ref[-1])


def test_solver_loop_nccl_single_rank(cuda):
    """The NCCL path of the loop (symmetric windows, device-API peer pointers,
    LSA barrier kernel) with one rank: same results as the oracle."""
    import torch
    n = nitro()
    A = synth.stencil("2d5", 40)
    x0 = synth.vector(A.cols, seed=5, mode=1)
    ref = _loop_ref(A, x0, 3)
    D = n.Dist(n.dist_unique_id(), 0, 1, 0)
    Ad = synth.to_device(A, cuda)
    M = D.spmv(A.rows, np.array([0, A.rows], np.int64), Ad.rowptr, Ad.colidx, Ad.vals, exchange=0)
    for v in (n.DIA, n.CSR_SCALAR, n.CSR_VECTOR):
        L = D.loop(M)
        L.x().copy_(torch.from_numpy(x0).to(cuda))
        L.start()
        for k in range(3):
            y = torch.full((A.rows,), float("nan"), device=cuda)
            L.step(v, y)
            torch.cuda.synchronize()
            assert np.array_equal(y.cpu().numpy().astype(np.float64), ref[k]), (v, k)
        L.close()
    M.close()
    D.close()


def test_dist_format_info_sums_the_rank_parts(cuda):
    """nitro_dist_format_info: a rank's compulsory bytes = its parts' matrix +
    y bytes + the exchanged x layout read once.  Summed over the ranks of a
    CSR-scalar multiply that is the single-GPU CSR bytes minus the single
    x read plus P layout reads (+ (#parts - 1) extra rowptr entries per rank)."""
    import torch
    n = nitro()
    A = synth.stencil("3d27", 24, mode=1, seed=8)
    P = 4
    bounds = n.dist_partition(np.asarray(A.rowptr, np.int64), P)
    group = n.Loopback(P, 0)
    got = [None] * P
    err = []

    def rank(q):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                D = n.Dist.loopback(group, q)
                blk = synth.to_device(block(A, bounds[q], bounds[q + 1]), cuda)
                M = D.spmv(A.rows, bounds, blk.rowptr, blk.colidx, blk.vals, exchange=0)
                got[q] = (n.Dist.format_info(M, n.CSR_SCALAR), n.Dist.exchange_info(M), n.Dist.layout(M))
                M.close()
                D.close()
        except Exception as e:
            err.append(repr(e))

    th = [threading.Thread(target=rank, args=(q,)) for q in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=300)
    assert not err, err
    group.close()
    N, Z = A.rows, A.nnz
    nparts = [sum(1 for lo, hi in ((0, l[1]), (l[1], l[2]), (l[2], hi_q - lo_q)) if hi > lo)
              for l, lo_q, hi_q in ((g[2], bounds[q], bounds[q + 1]) for q, g in enumerate(got))]
    want = Z * 8 + N * 4 + sum(p + 0 for p in nparts) * 4 + sum(g[1]["layout_len"] * 4 for g in got) + N * 4
    tot = sum(g[0]["compulsory_bytes"] for g in got)
    assert abs(tot - want) < 1e-6 * want, (tot, want, nparts)


def test_solver_loop_needs_the_allgather_layout(cuda):
    """nitro_dist_loop_create on a halo-exchange handle: NITRO_E_UNSUPPORTED (9)."""
    n = nitro()
    A = synth.stencil("2d5", 32)
    D = n.Dist(n.dist_unique_id(), 0, 1, 0)
    Ad = synth.to_device(A, cuda)
    M = D.spmv(A.rows, np.array([0, A.rows], np.int64), Ad.rowptr, Ad.colidx, Ad.vals, exchange=1)
    with pytest.raises(n.NitroError) as e:
        D.loop(M)
    assert e.value.code == 9
    M.close()
    D.close()
