#!/usr/bin/env python
"""Small end-to-end exercise of every kernel (features K1 / K1s, conversions,
five variants incl. the CSR-vector stream mode with and without hot-x staging,
timing/flush, dist parts, the 2-rank loopback exchange and the fused solver
loop, a malformed rowptr) for compute-sanitizer runs:

  NITRO_CSRV_HOT=2 compute-sanitizer --tool memcheck  python tools/sanitize_run.py
  NITRO_CSRV_HOT=2 compute-sanitizer --tool racecheck python tools/sanitize_run.py
(NITRO_CSRV_HOT=2 stages hot x values even for these small matrices.)
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import numpy as np
    import torch
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    import synth
    dev = torch.device("cuda:0")
    if os.environ.get("SANITIZE_PARTS", "all") == "loopback":
        mats = []
    else:
        mats = [synth.stencil("2d5", 64), synth.stencil("3d27", 12, mode=1, seed=2),
                synth.uniform(3000, 9, variable=True, seed=3, M=4000), synth.rmat(11, 8, seed=4, fp64=True),
                synth.banded(2000, 5, 0.5, seed=5), synth.uniform(1500, 90, seed=6, M=5000),   # K1s
                synth.stencil("3d27", (40, 12, 6), mode=1, seed=7), synth.stencil("2d9", 48)]  # K1 shifted-row paths
    for A in mats:
        Ad = synth.to_device(A, dev)
        M = nitro.SpMV.from_csr(Ad)
        M.set_budget(1e18)
        M.features()
        x = synth.vector(A.cols, seed=1, fp64=A.fp64, device=dev)
        for v in range(nitro.NUM_VARIANTS):
            if M.allowed(v):
                y = M.run(v, x)
                M.time(v, x, y, warmup=0, reps=1, flush_l2=False)
        M.set_csr_impl(nitro.CSR_IMPL_STREAM)       # K6s (+ hot-x for fp64 under NITRO_CSRV_HOT=2)
        M.run(nitro.CSR_VECTOR, x)
        torch.cuda.synchronize()
        M.close()
        if A.rows != A.cols:  # the dist path partitions x like y: square matrices only
            continue
        # a 3-way emulated dist partition of the same matrix
        rp = np.asarray(A.rowptr, np.int64)
        b = nitro.dist_partition(rp, 3)
        B = int(np.diff(b).max())
        xg = torch.zeros(3 * B, dtype=x.dtype, device=dev)
        for q in range(3):
            lo, hi = int(b[q]), int(b[q + 1])
            D = nitro.Dist.local(q, 3, 0)
            a0, a1 = rp[lo], rp[hi]
            blk = synth.Csr(hi - lo, A.cols, rp[lo:hi + 1] - a0, A.colidx[a0:a1], A.vals[a0:a1], A.fp64)
            bd = synth.to_device(blk, dev)
            Mq = D.spmv(A.rows, b, bd.rowptr, bd.colidx, bd.vals)
            yq = torch.empty(hi - lo, dtype=x.dtype, device=dev)
            for v in range(nitro.NUM_VARIANTS):
                D.run_gathered(Mq, v, xg, yq)
            torch.cuda.synchronize()
    if os.environ.get("SANITIZE_PARTS", "all") == "single":
        print("sanitize run complete (single-thread part)")
        return
    # 2 loopback ranks: the all-gather and halo exchanges, features, the fused solver loop
    import threading
    A = synth.stencil("2d5", 40)
    rp = np.asarray(A.rowptr, np.int64)
    b = nitro.dist_partition(rp, 2)
    x = synth.vector(A.cols, seed=3, mode=1)
    group = nitro.Loopback(2, 0)
    errs = []

    def rank(q):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                D = nitro.Dist.loopback(group, q)
                lo, hi = int(b[q]), int(b[q + 1])
                a0, a1 = rp[lo], rp[hi]
                bd = synth.to_device(synth.Csr(hi - lo, A.cols, rp[lo:hi + 1] - a0, A.colidx[a0:a1], A.vals[a0:a1],
                                               False), dev)
                for ex in (0, 1):
                    Mq = D.spmv(A.rows, b, bd.rowptr, bd.colidx, bd.vals, exchange=ex)
                    D.features(Mq)
                    xq = torch.from_numpy(x[lo:hi].copy()).to(dev)
                    yq = torch.empty(hi - lo, device=dev)
                    for v in range(nitro.NUM_VARIANTS):
                        D.run(Mq, v, xq, yq)
                    if ex == 0:
                        L = D.loop(Mq)
                        L.x().copy_(xq)
                        L.start()
                        for v in (nitro.DIA, nitro.CSR_SCALAR, nitro.ELL, nitro.CSR_VECTOR):
                            L.step(v, yq)
                        L.close()
                    torch.cuda.current_stream().synchronize()
                    Mq.close()
                D.close()
        except Exception as e:
            errs.append(repr(e))

    th = [threading.Thread(target=rank, args=(q,)) for q in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    group.close()
    assert not errs, errs
    # a malformed rowptr with long rows: rejected, no stray writes
    Z, N = 20000, 96
    rpb = np.zeros(N + 1, np.int64)
    rpb[1:33] = Z
    rpb[65:] = Z
    Bad = synth.Csr(N, Z, rpb, np.arange(Z, dtype=np.int32), np.ones(Z, np.float32), False)
    Mb = nitro.SpMV.from_csr(synth.to_device(Bad, dev))
    try:
        Mb.features()
    except nitro.NitroError:
        pass
    torch.cuda.synchronize()
    print("sanitize run complete")


if __name__ == "__main__":
    main()
