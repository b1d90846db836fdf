#!/usr/bin/env python
"""Small end-to-end exercise of every kernel (features, conversions, five
variants, timing/flush, dist parts) for compute-sanitizer runs:

  compute-sanitizer --tool memcheck  python tools/sanitize_run.py
  compute-sanitizer --tool racecheck python tools/sanitize_run.py
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
    mats = [synth.stencil("2d5", 64), synth.stencil("3d27", 12, mode=1, seed=2),
            synth.uniform(3000, 9, variable=True, seed=3, M=4000), synth.rmat(11, 8, seed=4, fp64=True),
            synth.banded(2000, 5, 0.5, seed=5)]
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
    print("sanitize run complete")


if __name__ == "__main__":
    main()
