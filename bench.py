#!/usr/bin/env python
"""bench.py — Nitro-selected SpMV throughput on B200 (BASELINE.json metric:
"selected-variant SpMV GB/s vs HBM peak; % of exhaustive-best variant").

Workload at N=1: BASELINE configs[1], the 3D 27-point stencil on a 128^3 grid
(2,097,152 rows, 55,742,968 nnz, fp32), synthetic (synth/), resident in HBM.
A step is one Nitro-selected multiply y = A.x.  Before the timed region the
hot path runs once end to end: GPU feature pass -> host SVM select (model in
artifacts/spmv_model.txt, trained by tools/train_select.py on the 60
synthetic training matrices of configs[3]) -> format conversion (cached,
P:L271) -> SpMV; every variant is also timed once for the exhaustive-best
reference.  L2 is flushed (read of 3x L2) between timed steps, outside the
per-step CUDA events.

N > 1 (torchrun): weak scaling — rank r owns z-planes [128 r, 128 (r+1)) of a
128 x 128 x (128 N) grid (the same per-rank block as N = 1) and every multiply
all-gathers x with NCCL (nitro_dist_*), as in an iterative solver.

--impl reference: the CPU oracle (oracle/, fp64, one thread) on the same
workload; rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOAD = "3d27pt_stencil_128^3_fp32 (BASELINE configs[1])"
MODEL = os.path.join(ROOT, "artifacts", "spmv_model.txt")
NCU_SUMMARY = os.path.join(ROOT, "profiles", "ncu_summary.json")


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback"


class Clocks:
    """nvidia-smi sampler during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index, self.rows, self.p = index, [], None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.p = None
        return self

    def _read(self):
        for line in self.p.stdout:
            self.rows.append([s.strip() for s in line.split(",")])

    def __exit__(self, *a):
        if self.p:
            time.sleep(0.25)
            self.p.terminate()
            try:
                self.p.wait(timeout=2)
            except Exception:
                self.p.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if len(r) > 2 + i and r[2 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def compulsory_csr_bytes(N, M, Z, sv=4, sp=4):
    return Z * (sv + 4) + (N + 1) * sp + (M + N) * sv


# ---------------------------------------------------------------------------- reference arm (CPU oracle)
def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import numpy as np
    import oracle
    import synth
    A = synth.stencil("3d27", 128, mode=1, seed=1)
    x = synth.vector(A.cols, seed=2)
    # bytes credited per step = what the Nitro arm credits for the same multiply:
    # the compulsory bytes of its selected format on this workload (DIA, the
    # committed model's pick = the exhaustive best; §8(d) DIA formula from the
    # oracle's own offsets), so the driver's value ratio is the time ratio
    _, offs = oracle.features(A, with_offsets=True)
    inrange = int(sum(max(0, min(A.rows, A.cols - int(o)) - max(0, -int(o))) for o in offs))
    nbytes = inrange * 4 + len(offs) * 4 + (A.rows + A.cols) * 4
    for _ in range(args.warmup):
        oracle.spmv(A, x)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.spmv(A, x)
        ts.append(time.perf_counter() - t0)
    t = sum(ts) / len(ts)
    val = nbytes / t / 1e9
    line = {"impl": "reference", "metric": "selected-variant SpMV GB/s vs HBM peak; % of exhaustive-best variant",
            "value": val, "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": t * 1e3, "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": WORKLOAD, "rows_per_gpu": A.rows, "nnz_per_gpu": A.nnz, "l2": "n/a (host)",
                       "parallelism": "one host thread (CPU oracle, fp64 CSR loop)",
                       "bytes_per_step": nbytes},
            "cpu_baseline": {"value": val, "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": f"full configs[1] matrix, {args.steps} multiplies"},
            "e2e": {"value": val, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))


# ---------------------------------------------------------------------------- CPU baseline (oracle) leg
def cpu_baseline(nbytes, seconds=12.0):
    """The oracle on the same matrix; nbytes = the bytes the GPU arm credits per
    multiply (the selected format's compulsory bytes), so value ratios are time ratios."""
    import oracle
    import synth
    A = synth.stencil("3d27", 128, mode=1, seed=1)
    x = synth.vector(A.cols, seed=2)
    oracle.spmv(A, x)
    n, t0 = 0, time.perf_counter()
    while time.perf_counter() - t0 < seconds:
        oracle.spmv(A, x)
        n += 1
    t = (time.perf_counter() - t0) / n
    return {"value": nbytes / t / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
            "sample": f"full configs[1] matrix (55.7M nnz), {n} multiplies in {seconds:.0f}s, single thread fp64"}


# ---------------------------------------------------------------------------- our arm
def run_nitro(args):
    import numpy as np
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    import synth

    rank, world, local = dist_env()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    stream = torch.cuda.current_stream(dev)

    n = 128
    row0 = rank * n * n * n
    # this rank's block: z-planes [n*rank, n*(rank+1)) of an n x n x (n*world) grid
    A = synth.stencil("3d27", (n, n, n * world), mode=1, seed=1, device=dev, row0=row0, nrows=n * n * n)
    A.rowptr = A.rowptr.to(torch.int32)
    N, Z = A.rows, A.nnz
    x_local = synth.vector(N, seed=2, device=dev, j0=row0)
    y = torch.empty(N, dtype=torch.float32, device=dev)

    use_dist = world > 1 or args.dist   # --dist: the multi-GPU code path even at N = 1
    if not use_dist:
        M = nitro.SpMV(A.rowptr, A.colidx, A.vals, N, A.cols)
        x = x_local
    else:
        D = _dist_setup(nitro, dist if world > 1 else None, rank, world, local)
        bounds = np.array([r * n * n * n for r in range(world + 1)], dtype=np.int64)
        M = D.spmv(A.cols, bounds, A.rowptr, A.colidx, A.vals, exchange=args.exchange)
        exch = nitro.Dist.exchange_info(M)
        x = nitro.Dist.x_local(M)      # x lives inside the exchange buffer: no per-multiply copy
        x.copy_(x_local)

    # --- one end-to-end pass of the hot path (features -> select -> prepare -> run)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    feats = M.features() if not use_dist else D.features(M)   # first call: allocates its buffers
    feature_first_ms = (time.perf_counter() - t0) * 1e3
    feature_ms = None
    if not use_dist:                                        # warm feature pass (+ host finishing)
        M.invalidate()
        ev0.record(stream)
        feats = M.features()
        ev1.record(stream)
        torch.cuda.synchronize()
        feature_ms = ev0.elapsed_time(ev1)
    fvec = [feats[k] for k in nitro.FEATURE_NAMES]
    allowed = M.allowed_mask() if not use_dist else [True] * 5   # dist parts check their own constraints
    ctx = nitro.Context()
    cv = nitro.CodeVariant(ctx, "spmv")
    cv.register_spmv()
    selection = "svm"
    if os.path.exists(MODEL):
        cv.load(MODEL)
        t0 = time.perf_counter()
        sel = cv.predict(fvec, allowed)
        select_us = (time.perf_counter() - t0) * 1e6
    else:
        sel, select_us, selection = None, None, "exhaustive (no model file)"

    # exhaustive reference: every allowed variant timed the same way (median of R, L2 flushed)
    exhaustive = {}
    if not use_dist:
        for v in range(5):
            if allowed[v]:
                med, _ = M.time(v, x, y, warmup=3, reps=20, flush_l2=True)
                info = M.format_info(v)
                exhaustive[nitro.VARIANT_NAMES[v]] = {"ms": med * 1e3, "GBps": info["compulsory_bytes"] / med / 1e9,
                                                      "bytes": info["compulsory_bytes"]}
        best = min(exhaustive, key=lambda k: exhaustive[k]["ms"])
        if sel is None:
            sel = nitro.VARIANT_NAMES.index(best)
    else:
        best = None
        if sel is None:
            sel = nitro.DIA
    vname = nitro.VARIANT_NAMES[sel]
    if not use_dist:
        M.prepare(sel)
        nbytes = M.format_info(sel)["compulsory_bytes"]
        launches = M.launches(sel)
    else:
        nbytes = D_bytes(M, nitro, sel)
        launches = 1

    def step():
        if not use_dist:
            M.run(sel, x, y)
        else:
            D.run(M, sel, x, y)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    with Clocks(local) as clk:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        for i in range(args.steps):
            M.flush_l2()
            starts[i].record(stream)
            step()
            ends[i].record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    times = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    ms = sum(times) / len(times)
    if world > 1:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    gbps = nbytes * world / (ms * 1e-3) / 1e9

    # --- size-matched ceiling: a device copy moving the same byte count (half read,
    # half write), timed the same way (L2 flushed, median of 20): at 242 MB the
    # DRAM ramp/drain is a visible share of a ~45 us kernel
    copy_gbps = None
    if world == 1:
        half = max(int(nbytes) // 8, 1)
        ca = torch.ones(half, dtype=torch.float32, device=dev)
        cb = torch.empty_like(ca)
        cts = []
        for i in range(23):
            M.flush_l2()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            cb.copy_(ca)
            b.record(stream)
            b.synchronize()
            if i >= 3:
                cts.append(a.elapsed_time(b))
        copy_gbps = 8 * half / (statistics.median(cts) * 1e-3) / 1e9
        del ca, cb

    # --- e2e through the C ABI with host buffers (pinned), copies inside the timed region
    e2e = None
    hx = torch.empty(N, dtype=torch.float32).pin_memory()
    hx.copy_(x.cpu())
    hy = torch.empty(N, dtype=torch.float32).pin_memory()
    if use_dist:   # no host-buffer entry in the dist API: pinned copies around nitro_dist_spmv_run
        xs = torch.empty_like(x)
        et = []
        for i in range(args.steps + 3):
            M.flush_l2()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            xs.copy_(hx, non_blocking=True)
            D.run(M, sel, xs, y)
            hy.copy_(y, non_blocking=True)
            b.record(stream)
            b.synchronize()
            if i >= 3:
                et.append(a.elapsed_time(b))
        e2e_ms = sum(et) / len(et)
        if world > 1:
            t = torch.tensor([e2e_ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_ms = float(t.item())
        e2e = {"value": nbytes * world / (e2e_ms * 1e-3) / 1e9, "unit": "GB/s", "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": N * 4 * world, "d2h_bytes_per_step": N * 4 * world}
    else:
        hx.copy_(x.cpu())
        hy = torch.empty(N, dtype=torch.float32).pin_memory()
        hxn, hyn = hx.numpy(), hy.numpy()
        for _ in range(3):
            M.run_host(sel, hxn, hyn)
        et = []
        for _ in range(args.steps):
            M.flush_l2()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            M.run_host(sel, hxn, hyn)
            b.record(stream)
            b.synchronize()
            et.append(a.elapsed_time(b))
        e2e_ms = sum(et) / len(et)
        e2e = {"value": nbytes / (e2e_ms * 1e-3) / 1e9, "unit": "GB/s", "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": N * 4, "d2h_bytes_per_step": N * 4}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return
    pk, pk_kind = peaks()
    peak = float(pk.get("hbm_gbs", 6650.0))
    traffic = None
    try:
        summ = json.load(open(NCU_SUMMARY))
        rec = summ.get("c1", {}).get(vname)
        if rec:
            traffic = rec.get("dram_bytes_per_launch")
    except Exception:
        pass
    per_gpu = nbytes / (ms * 1e-3) / 1e9
    line = {
        "metric": "selected-variant SpMV GB/s vs HBM peak; % of exhaustive-best variant",
        "value": gbps, "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic",
        "config": {"workload": WORKLOAD if world == 1 else f"3d27pt_stencil_128x128x{128 * world}_fp32 (128^3 rows/rank)",
                   "rows_per_gpu": N, "nnz_per_gpu": Z, "l2": "flushed between steps (read of 3x L2)",
                   "parallelism": "single GPU" if not use_dist else
                   f"row-partitioned x{world}, NCCL x {exch['mode']} ({exch['halo_len']} halo entries/rank)",
                   "selection": selection, "selected_variant": vname},
        "selected_variant": vname,
        "gflops": 2.0 * Z * world / (ms * 1e-3) / 1e9,
        "pct_of_hbm_peak": per_gpu / peak,
        "pct_of_exhaustive_best": (exhaustive[best]["ms"] / exhaustive[vname]["ms"]) if exhaustive else None,
        "exhaustive_best": best, "exhaustive": exhaustive,
        "feature_ms": feature_ms, "feature_first_call_ms": feature_first_ms, "select_us": select_us,
        "features_per_spmv": (feature_ms / ms) if feature_ms else None, "features": {k: feats[k] for k in nitro.FEATURE_NAMES},
        "roofline": {"bound": "hbm", "achieved": per_gpu, "peak": peak, "unit": "GB/s", "frac": per_gpu / peak,
                     "traffic": traffic, "peak_kind": f"{pk_kind} hbm_gbs (copy)",
                     "kernel": f"{vname} ({launches} launch/step)",
                     "size_matched_copy_gbs": copy_gbps,
                     "frac_of_size_matched_copy": (per_gpu / copy_gbps) if copy_gbps else None,
                     "bytes_per_launch": nbytes},
        "gpu_launches": args.steps * (launches + 1),
        "gpu_launches_note": f"{args.steps} x ({launches} SpMV + 1 L2-flush) kernels of libnitro",
        "clocks": clk.summary(),
        "e2e": e2e,
    }
    if world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(nbytes)
    print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()


def D_bytes(M, nitro, v):
    return M.format_info(v)["compulsory_bytes"]


def _dist_setup(nitro, dist, rank, world, local):
    import torch
    uid = nitro.dist_unique_id() if rank == 0 else bytes(128)
    if dist is not None:
        t = torch.tensor(list(uid), dtype=torch.uint8, device="cuda")
        dist.broadcast(t, 0)
        uid = bytes(t.cpu().tolist())
    return nitro.Dist(uid, rank, world, local)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="nitro", choices=["nitro", "reference"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--dist", action="store_true", help="use the multi-GPU (NCCL) code path even at N=1")
    ap.add_argument("--exchange", type=int, default=-1, help="multi-GPU x exchange: -1 auto, 0 all-gather, 1 halo")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_nitro(args)


if __name__ == "__main__":
    main()
