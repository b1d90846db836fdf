"""world_size-2 CPU (gloo) check of the multi-GPU decomposition: the library's
nnz-balanced partition, x distributed like y and all-gathered, each rank
multiplying its row block (here with the oracle as the local compute), gives
the single-process y.  Also checks the global-feature reduction rule (sum of
moments, max of Lmax, union of diagonals) against the single-process features."""
import os
import socket

import numpy as np
import pytest


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch
    import torch.distributed as dist
    import oracle
    import synth
    from synth import Csr
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = synth.rmat(11, 8, seed=5, fp64=True)
        rp = np.asarray(A.rowptr, np.int64)
        bounds = nitro.dist_partition(rp, world)
        lo, hi = int(bounds[rank]), int(bounds[rank + 1])
        a, b = rp[lo], rp[hi]
        blk = Csr(hi - lo, A.cols, rp[lo:hi + 1] - a, A.colidx[a:b], A.vals[a:b], True)
        x_local = torch.from_numpy(synth.vector(hi - lo, seed=9, fp64=True, j0=lo))
        B = int(np.diff(bounds).max())
        pad = torch.zeros(B, dtype=torch.float64)
        pad[: hi - lo] = x_local
        parts = [torch.zeros(B, dtype=torch.float64) for _ in range(world)]
        dist.all_gather(parts, pad)
        x_full = torch.cat([parts[r][: bounds[r + 1] - bounds[r]] for r in range(world)]).numpy()
        y_local, _ = oracle.spmv(blk, x_full)
        ys = [torch.zeros(B, dtype=torch.float64) for _ in range(world)]
        yp = torch.zeros(B, dtype=torch.float64)
        yp[: hi - lo] = torch.from_numpy(y_local)
        dist.all_gather(ys, yp)
        y = torch.cat([ys[r][: bounds[r + 1] - bounds[r]] for r in range(world)]).numpy()
        # global features from per-rank integer moments + diagonal union
        f_loc, offs = oracle.features(Csr(hi - lo, A.cols, blk.rowptr, blk.colidx, blk.vals, True),
                                      with_offsets=True)
        glob_offs = set((offs - lo).tolist())       # local offsets are relative to local rows
        mom = torch.tensor([f_loc["sum_len"], f_loc["sum_len2"]], dtype=torch.float64)
        dist.all_reduce(mom)
        mx = torch.tensor([f_loc["max_row"]], dtype=torch.float64)
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        allo = [None] * world
        dist.all_gather_object(allo, glob_offs)
        if rank == 0:
            y_ref, _ = oracle.spmv(A, synth.vector(A.rows, seed=9, fp64=True))
            f = oracle.features(A)
            union = set().union(*allo)
            q.put((bool(np.array_equal(y, y_ref)), int(mom[0]) == f["sum_len"], int(mom[1]) == f["sum_len2"],
                   int(mx[0]) == f["max_row"], len(union) == f["ndiag"], list(bounds)))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_row_partition():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert res[:5] == (True, True, True, True, True), res
