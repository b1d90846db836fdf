#!/usr/bin/env python
"""BASELINE configs[4] on one B200: 3D 27-point stencil 512^3 (134,217,728
rows, 3,609,741,304 nnz, int64 rowptr), fp32, random values.

1. Single GPU: the feature pass, the Nitro-selected variant (model
   artifacts/spmv_model.txt) and every variant timed with the library's timing
   (median of R L2-flushed CUDA-event runs), GB/s of each format's compulsory
   bytes and the fraction of the measured HBM copy peak.
2. The P-way row partition (P = 2, 4, 8; nnz-balanced bounds, halo exchange
   layout) EMULATED on the one GPU: every rank's local multiply is built and
   timed in turn from its exchanged x (nitro_dist_* with a communicator-less
   handle).  T_P(compute) = max over ranks; the halo each rank receives is
   reported in bytes together with the time it needs at the NVLink 5 rate
   (900 GB/s per direction) — a projection, not a multi-GPU measurement (one
   GPU is reachable here).  Interior rows overlap the exchange, so the
   projected step is max(T_compute, T_halo) + the boundary rows' share.

usage: python tools/c4_probe.py [--reps 10] [--ranks 2,4,8] [--out artifacts/c4_probe.json]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

N1 = 512
NVLINK_GBS = 900.0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--ranks", default="2,4,8")
    ap.add_argument("--variants", default="csr_scalar,csr_vector,ell,dia,hyb")
    ap.add_argument("--out", default=os.path.join(ROOT, "artifacts", "c4_probe.json"))
    a = ap.parse_args()
    import numpy as np
    import torch
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    import synth
    dev = torch.device("cuda:0")
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))).get("hbm_gbs", 6650.0) \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    want = [nitro.VARIANT_NAMES.index(v) for v in a.variants.split(",")]
    t0 = time.time()
    A = synth.stencil("3d27", N1, mode=1, seed=1, device=dev)
    torch.cuda.synchronize()
    gen_s = time.time() - t0
    x = synth.vector(A.cols, seed=2, device=dev)
    y = torch.empty(A.rows, dtype=torch.float32, device=dev)
    M = nitro.SpMV.from_csr(A)
    M.set_budget(1e12)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    M.features()
    fts = []
    for _ in range(5):
        M.invalidate()
        M.flush_l2()
        torch.cuda.synchronize()
        s.record()
        f = M.features()
        e.record()
        torch.cuda.synchronize()
        fts.append(s.elapsed_time(e))
    ctx = nitro.Context()
    cv = nitro.CodeVariant(ctx, "spmv")
    cv.register_spmv()
    cv.load(os.path.join(ROOT, "artifacts", "spmv_model.txt"))
    sel = cv.predict([f[k] for k in ("nnz", "rows", "mean", "sd", "max_dev", "dia_fill", "ell_fill")],
                     [M.allowed(v) for v in range(nitro.NUM_VARIANTS)])
    one = {}
    for v in want:
        t1 = time.time()
        M.prepare(v)
        torch.cuda.synchronize()
        conv_ms = (time.time() - t1) * 1e3
        info = M.format_info(v)
        med, allt = M.time(v, x, y, warmup=3, reps=a.reps, flush_l2=True)
        one[nitro.VARIANT_NAMES[v]] = {"ms": med * 1e3, "GBps": info["compulsory_bytes"] / med / 1e9,
                                       "frac_of_peak": info["compulsory_bytes"] / med / 1e9 / peak,
                                       "GFLOPs": 2 * A.nnz / med / 1e9, "bytes": info["compulsory_bytes"],
                                       "conversion_ms": conv_ms}
        M.release(v)
        print(nitro.VARIANT_NAMES[v], {k: round(v2, 3) for k, v2 in one[nitro.VARIANT_NAMES[v]].items()}, flush=True)
    out = {"config": "BASELINE configs[4]: 3d27pt 512^3 fp32 (134,217,728 rows, 3,609,741,304 nnz)",
           "peak_hbm_gbs": peak, "generate_s": gen_s,
           "feature_ms": sorted(fts)[len(fts) // 2],
           "feature_GBps": ((A.rows + 1) * 8 + A.nnz * 4) / (sorted(fts)[len(fts) // 2] * 1e-3) / 1e9,
           "selected": nitro.VARIANT_NAMES[sel], "single_gpu": one, "emulated": {}}
    rp_h = A.rowptr.cpu().numpy()
    M.close()
    del M, A
    torch.cuda.empty_cache()
    # ---------------------------------------------------------------- emulated P-way partition
    for P in [int(p) for p in a.ranks.split(",") if p]:
        bounds = nitro.dist_partition(rp_h, P)
        per = {nitro.VARIANT_NAMES[v]: [] for v in want}
        halo = []
        for q in range(P):
            lo, hi = int(bounds[q]), int(bounds[q + 1])
            blk = synth.stencil("3d27", N1, mode=1, seed=1, device=dev, row0=lo, nrows=hi - lo)
            D = nitro.Dist.local(q, P, 0)
            Mq = D.spmv(N1 ** 3, bounds, blk.rowptr, blk.colidx, blk.vals, exchange=1)
            Mq.set_budget(1e12)
            info = nitro.Dist.exchange_info(Mq)
            halo.append(int(info["halo_len"]) * 4)
            xe = torch.zeros(int(info["layout_len"]), dtype=torch.float32, device=dev)
            xe.uniform_(-1, 1)
            yq = torch.empty(hi - lo, dtype=torch.float32, device=dev)
            for v in want:
                # the rank's multiply from its exchanged x (nitro_dist_spmv_run_gathered), L2 flushed, events
                for _ in range(3):
                    D.run_gathered(Mq, v, xe, yq)
                ts = []
                for _ in range(a.reps):
                    Mq.flush_l2()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    D.run_gathered(Mq, v, xe, yq)
                    e1.record()
                    torch.cuda.synchronize()
                    ts.append(e0.elapsed_time(e1))
                per[nitro.VARIANT_NAMES[v]].append(sorted(ts)[len(ts) // 2])
                Mq.release(v)
            Mq.close()
            D.close()
            del blk, xe, yq
            torch.cuda.empty_cache()
        hmax = max(halo)
        t_halo = hmax / (NVLINK_GBS * 1e9) * 1e3
        res = {"bounds": [int(b) for b in bounds], "halo_bytes_max": hmax, "halo_ms_at_nvlink": t_halo}
        for name, ts in per.items():
            tc = max(ts)
            t1 = one[name]["ms"]
            res[name] = {"rank_ms": ts, "t_compute_ms": tc, "projected_step_ms": max(tc, t_halo),
                         "projected_speedup": t1 / max(tc, t_halo)}
        out["emulated"][str(P)] = res
        print(P, {k: (round(v["projected_speedup"], 2) if isinstance(v, dict) else v) for k, v in res.items()
                  if k not in ("bounds",)}, flush=True)
    out["note"] = ("emulated ranks: every rank's local multiply timed on the one GPU from its exchanged x; "
                   "projected step = max(max-rank compute, largest halo / 900 GB/s NVLink 5): not a multi-GPU "
                   "measurement")
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump(out, open(a.out, "w"), indent=1)
    print(json.dumps({k: out[k] for k in ("feature_ms", "selected")}))


if __name__ == "__main__":
    main()
