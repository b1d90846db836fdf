#!/usr/bin/env python
"""Run every SpMV variant (and the feature pass) on one BASELINE config, for
ncu captures.  Usage: python tools/profile_variants.py c1|c2a|c2b [variants...]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def make(cfg, dev):
    import synth
    if cfg == "c1":
        return synth.stencil("3d27", 128, mode=1, seed=1, device=dev)
    if cfg == "c2a":
        return synth.uniform(1 << 23, 32, seed=5, device=dev)
    if cfg == "c2b":
        return synth.rmat(23, 16, seed=7, fp64=True, device=dev)
    raise SystemExit(f"unknown config {cfg}")


def main():
    import torch
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    import synth
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c1"
    want = [nitro.VARIANT_NAMES.index(v) for v in sys.argv[2:]] or list(range(5))
    dev = torch.device("cuda:0")
    A = make(cfg, dev)
    A.rowptr = A.rowptr.to(torch.int32)
    M = nitro.SpMV.from_csr(A)
    f = M.features()
    x = synth.vector(A.cols, seed=2, fp64=A.fp64, device=dev)
    y = torch.empty(A.rows, dtype=x.dtype, device=dev)
    for v in want:
        if not M.allowed(v):
            continue
        M.prepare(v)
        for _ in range(2):
            M.flush_l2()
            M.run(v, x, y)
        torch.cuda.synchronize()
        info = M.format_info(v)
        print(cfg, nitro.VARIANT_NAMES[v], "bytes", info["compulsory_bytes"], "launches", M.launches(v), flush=True)
    print(cfg, "features", f)


if __name__ == "__main__":
    main()
