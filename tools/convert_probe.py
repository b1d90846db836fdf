#!/usr/bin/env python
"""Conversion (prepare) cost per variant: release + prepare timed with events
and wall clock (median of 3), next to one multiply of the same variant."""
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))


def main():
    import torch
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    import synth
    from profile_variants import make
    dev = torch.device("cuda:0")
    cfgs = [a for a in sys.argv[1:] if not a.startswith("-")] or ["c1", "c2a", "c2b", "short"]
    reps = 1 if "--once" in sys.argv else 3
    for cfg in cfgs:
        A = make(cfg, dev)
        A.rowptr = A.rowptr.to(torch.int32)
        M = nitro.SpMV.from_csr(A)
        M.features()
        x = synth.vector(A.cols, seed=2, fp64=A.fp64, device=dev)
        y = torch.empty(A.rows, dtype=x.dtype, device=dev)
        out = {}
        for v in range(5):
            if not M.allowed(v):
                continue
            ev, wall = [], []
            for _ in range(reps):
                M.release(v)
                torch.cuda.synchronize()
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                t0 = time.perf_counter()
                s.record()
                M.prepare(v)
                e.record()
                torch.cuda.synchronize()
                wall.append((time.perf_counter() - t0) * 1e3)
                ev.append(s.elapsed_time(e))
            med, _ = M.time(v, x, y, warmup=2, reps=5)
            out[nitro.VARIANT_NAMES[v]] = (round(statistics.median(ev), 3), round(statistics.median(wall), 3),
                                           round(med * 1e3, 3))
        print(cfg, "prepare ms (events, wall) + spmv ms:", out, flush=True)
        M.close()
        del A, x, y
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
