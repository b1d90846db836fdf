#!/usr/bin/env python
"""Break down the host-buffer SpMV call on configs[1] (DIA): run_host vs the
same copies + multiply issued from torch, each timed with events (median)."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def timed(fn, reps=20, pre=None):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for r in range(reps + 3):
        if pre:
            pre()
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        if r >= 3:
            ts.append(s.elapsed_time(e))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    import synth
    dev = torch.device("cuda:0")
    A = synth.stencil("3d27", 128, mode=1, seed=1, device=dev)
    A.rowptr = A.rowptr.to(torch.int32)
    M = nitro.SpMV.from_csr(A)
    v = nitro.DIA
    M.prepare(v)
    N = A.rows
    hx = torch.ones(N, dtype=torch.float32).pin_memory()
    hy = torch.empty(N, dtype=torch.float32).pin_memory()
    dx = torch.ones(N, dtype=torch.float32, device=dev)
    dy = torch.empty(N, dtype=torch.float32, device=dev)
    hxn, hyn = hx.numpy(), hy.numpy()
    print("run_host          ", round(timed(lambda: M.run_host(v, hxn, hyn), pre=M.flush_l2), 3), "ms")
    print("H2D only          ", round(timed(lambda: dx.copy_(hx, non_blocking=True)), 3), "ms")
    print("D2H only          ", round(timed(lambda: hy.copy_(dy, non_blocking=True)), 3), "ms")
    print("SpMV only         ", round(timed(lambda: M.run(v, dx, dy), pre=M.flush_l2), 3), "ms")

    def serial():
        dx.copy_(hx, non_blocking=True)
        M.run(v, dx, dy)
        hy.copy_(dy, non_blocking=True)
    print("torch serial      ", round(timed(serial, pre=M.flush_l2), 3), "ms")
    import time

    def wall(fn, reps=50):
        for _ in range(5):
            fn()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(reps):
            fn()
            torch.cuda.synchronize()
        return (time.perf_counter() - t0) / reps * 1e3
    print("wall run_host     ", round(wall(lambda: M.run_host(v, hxn, hyn)), 3), "ms")
    print("wall torch serial ", round(wall(serial), 3), "ms")
    print("wall empty sync   ", round(wall(lambda: None), 3), "ms")


if __name__ == "__main__":
    main()
