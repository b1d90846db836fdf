#!/usr/bin/env python
"""Run (or time) every SpMV variant and the feature pass on BASELINE configs.

  python tools/profile_variants.py c1 [variants...]        # 2 runs each, for ncu
  python tools/profile_variants.py --time c1 c2a c2b       # JSON table (median of 20, L2 flushed)
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def make(cfg, dev):
    import synth
    if cfg == "c0":
        return synth.stencil("2d5", 64, device=dev)
    if cfg == "c1":
        return synth.stencil("3d27", 128, mode=1, seed=1, device=dev)
    if cfg == "c4":      # BASELINE configs[4]: 3D 27-pt 512^3 (int64 rowptr), the bench workload
        return synth.stencil("3d27", 512, mode=1, seed=1, device=dev)
    if cfg == "c1big":   # 3D 27-pt 256^3: the asymptotic (ramp-free) DIA/ELL rate
        return synth.stencil("3d27", 256, mode=1, seed=1, device=dev)
    if cfg == "c2a":
        return synth.uniform(1 << 23, 32, seed=5, device=dev)
    if cfg == "c2b":
        return synth.rmat(23, 16, seed=7, fp64=True, device=dev)
    if cfg == "short":   # very short rows (CSR-scalar class): 1D 3-pt, 2^23 rows
        return synth.stencil("1d3", 1 << 23, mode=1, seed=3, device=dev)
    if cfg == "band01":  # sparse band (b = 28, density 0.1): CSR-scalar wins these in configs[3]
        return synth.banded(1 << 23, 28, 0.1, seed=4, device=dev)
    if cfg == "uvar3":   # short random rows of variable length (k ~ U{1..4}): CSR-scalar class in configs[3]
        return synth.uniform(1 << 23, 3, variable=True, seed=6, device=dev)
    if cfg == "band48":  # dense band (b = 48): 97-entry local rows, the long-row CSR-vector class
        return synth.banded(1 << 21, 48, 1.0, seed=8, device=dev)
    if cfg == "band96h": # half-dense wide band (b = 96, density 0.5): ~97 local entries per row, uneven lengths
        return synth.banded(1 << 21, 96, 0.5, seed=9, device=dev)
    raise SystemExit(f"unknown config {cfg}")


def main():
    import torch
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    import synth
    args = sys.argv[1:]
    timing = "--time" in args
    csr_ab = "--csr-ab" in args   # also time the CSR variants with the direct kernels
    args = [a for a in args if a not in ("--time", "--csr-ab")]
    cfgs = [a for a in args if a in ("c0", "c1", "c1big", "c2a", "c2b", "c4", "short", "band01", "uvar3", "band48", "band96h")] or ["c1"]
    want = [] if "none" in args else ([nitro.VARIANT_NAMES.index(v) for v in args if v in nitro.VARIANT_NAMES] or list(range(5)))
    dev = torch.device("cuda:0")
    table = {}
    for cfg in cfgs:
        A = make(cfg, dev)
        if A.nnz < 2 ** 31:
            A.rowptr = A.rowptr.to(torch.int32)
        M = nitro.SpMV.from_csr(A)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        M.features()                    # allocates the feature buffers
        fts = []
        for _ in range(7 if timing else 1):   # then time warm feature passes (median)
            M.invalidate()
            M.flush_l2()
            torch.cuda.synchronize()
            s.record()
            f = M.features()
            e.record()
            torch.cuda.synchronize()
            fts.append(s.elapsed_time(e))
        feat_ms = sorted(fts)[len(fts) // 2]
        fgs = []
        for _ in range(7 if timing else 0):   # device time of the pass: async launches, events around them
            M.invalidate()
            M.flush_l2()
            torch.cuda.synchronize()
            s.record()
            M.features_async()
            e.record()
            torch.cuda.synchronize()
            M.features()
            fgs.append(s.elapsed_time(e))
        feat_gpu_ms = sorted(fgs)[len(fgs) // 2] if fgs else None
        x = synth.vector(A.cols, seed=2, fp64=A.fp64, device=dev)
        y = torch.empty(A.rows, dtype=x.dtype, device=dev)
        row = {"rows": A.rows, "nnz": A.nnz, "feature_ms": feat_ms, "feature_gpu_ms": feat_gpu_ms,
               "feature_GBps": ((A.rows + 1) * A.rowptr.element_size() + A.nnz * 4) / (feat_ms * 1e-3) / 1e9,
               "variants": {}}
        for v in want:
            if not M.allowed(v):
                continue
            M.prepare(v)
            info = M.format_info(v)
            if timing:
                med, allt = M.time(v, x, y, warmup=3, reps=20, flush_l2=True)
                row["variants"][nitro.VARIANT_NAMES[v]] = {
                    "ms": med * 1e3, "GBps": info["compulsory_bytes"] / med / 1e9,
                    "GFLOPs": 2 * A.nnz / med / 1e9, "bytes": info["compulsory_bytes"], "width": info["width"],
                    "tail": info["tail"], "launches": M.launches(v)}
                if csr_ab and v in (nitro.CSR_SCALAR, nitro.CSR_VECTOR):
                    M.set_csr_impl(nitro.CSR_IMPL_DIRECT)
                    med, _ = M.time(v, x, y, warmup=3, reps=20, flush_l2=True)
                    M.set_csr_impl(nitro.CSR_IMPL_AUTO)
                    row["variants"][nitro.VARIANT_NAMES[v] + "_direct"] = {
                        "ms": med * 1e3, "GBps": info["compulsory_bytes"] / med / 1e9}
            else:
                for _ in range(2):
                    M.flush_l2()
                    M.run(v, x, y)
                torch.cuda.synchronize()
                print(cfg, nitro.VARIANT_NAMES[v], "bytes", info["compulsory_bytes"], flush=True)
            M.release(v)
        table[cfg] = row
        del M, A, x, y
        torch.cuda.empty_cache()
    print(json.dumps(table, indent=1))


if __name__ == "__main__":
    main()
