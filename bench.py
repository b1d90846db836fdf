#!/usr/bin/env python
"""bench.py — Nitro-selected SpMV throughput on B200 (BASELINE.json metric:
"selected-variant SpMV GB/s vs HBM peak; % of exhaustive-best variant").

Workload at every N (strong scaling): BASELINE configs[4], the 3D 27-point
stencil on a 512^3 grid (134,217,728 rows, 3,609,741,304 nnz, fp32), random
values, synthetic (synth/), generated in HBM.  At N = 1 it is the largest
single-GPU configuration of BASELINE (CSR 31 GB), so the SCALE N = 1 point and
the BENCH line are the same measurement.

A step is one Nitro-selected multiply y = A.x.  Before the timed region the
hot path runs once end to end: GPU feature pass -> host SVM select -> format
conversion (cached: the paper amortises features and conversion over the many
multiplies of a solver) -> SpMV; every allowed variant is timed the
same way for the exhaustive-best reference.  The matrix formats (>= 15 GB)
are far larger than L2; L2 is still flushed (streaming read of 3x L2) before
every timed step, outside the per-step CUDA events.

Selection: two models trained on configs[3] (tools/train_select.py):
artifacts/spmv_model.txt = the paper's plain [-1, 1] scaling and
artifacts/spmv_model_r11x.txt = the R11x extension (log1p + clip).
--model picks the deployed one (default paper: the configs[3] recipe spans
2^18-2^27.2 rows, so every bench matrix lies inside its training range); both
picks and their % of the exhaustive best are always reported.

N = 1 adds (unless --quick): the same measurement on configs[1], configs[2]
(uniform fp32 and R-MAT fp64) as extra keys, a selection leg that re-times
held-out configs[3] matrices on this box and re-derives Nitro % for both
models, and the CPU oracle baseline (one thread and all host cores).

N > 1: one process per GPU (torchrun; `python bench.py --gpus N` relaunches
itself under torch.distributed.run when WORLD_SIZE is unset).  Rank r owns the
contiguous nnz-balanced row block of configs[4] (nitro_dist_partition) and
every multiply all-gathers x with NCCL (A13, nitro_dist_* exchange 0), the
interior rows overlapping the exchange; the halo exchange (f3) is timed as
extra keys.  Max over ranks of CUDA-event times.

--impl reference: the CPU oracle (oracle/, fp64) on a bounded row sample of
the same workload, all host cores; rank 0 only.
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

METRIC = "selected-variant SpMV GB/s vs HBM peak; % of exhaustive-best variant"
MODELS = {"paper": os.path.join(ROOT, "artifacts", "spmv_model.txt"),
          "r11x": os.path.join(ROOT, "artifacts", "spmv_model_r11x.txt")}
MODEL_DOC = {"paper": "plain [-1,1] min-max scaling (P:L179)",
             "r11x": "EXTENSION R11x: log1p of the 7 features + clip (DESIGN.md; not from the paper)"}
NCU_SUMMARY = os.path.join(ROOT, "profiles", "ncu_summary.json")
GATHER_PROBE = os.path.join(ROOT, "profiles", "r02", "l2_gather_probe.jsonl")


def gather_rate():
    """Measured random-gather ceiling (gathers/s) of this part: the best
    'gathers only' case of tools/probes/l2_gather_probe.cu (profiles/r02)."""
    try:
        best = 0.0
        for line in open(GATHER_PROBE):
            d = json.loads(line)
            if str(d.get("case", "")).startswith("A_gather_only"):
                best = max(best, float(d["gathers_per_s"]))
        return best or None
    except Exception:
        return None

WORKLOADS = {
    "c4": ("3d27pt_stencil_512^3_fp32 (BASELINE configs[4])", "stencil", ("3d27", 512, False)),
    "c1": ("3d27pt_stencil_128^3_fp32 (BASELINE configs[1])", "stencil", ("3d27", 128, False)),
    "c2a": ("uniform_8M_rows_x32_fp32 (BASELINE configs[2], uniform)", "uniform", (1 << 23, 32, False)),
    "c2b": ("rmat_scale23_ef16_fp64 (BASELINE configs[2], power-law)", "rmat", (23, 16, True)),
}


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback (B200_PROFILING.md)"


class Clocks:
    """nvidia-smi sampler during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index, self.rows, self.p = index, [], None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "50"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            time.sleep(0.3)
        except Exception:
            self.p = None
        return self

    def _read(self):
        for line in self.p.stdout:
            self.rows.append([s.strip() for s in line.split(",")])

    def __exit__(self, *a):
        if self.p:
            time.sleep(0.2)
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


def make(cfg, dev=None, row0=0, nrows=None):
    """Synthetic BASELINE matrix (device when dev is given, else host)."""
    import synth
    _, cls, p = WORKLOADS[cfg]
    if cls == "stencil":
        return synth.stencil(p[0], p[1], mode=1, seed=1, device=dev, row0=row0, nrows=nrows)
    if cls == "uniform":
        return synth.uniform(p[0], p[1], seed=5, device=dev)
    return synth.rmat(p[0], p[1], seed=7, fp64=True, device=dev)


def stencil_rowptr_host(n):
    """Closed-form rowptr of the 3D 27-point stencil on an n^3 grid (row length
    = product over the 3 axes of the neighbours inside the grid), for the
    nnz-balanced partition without materialising the matrix on the host."""
    import numpy as np
    c = np.full(n, 3, dtype=np.int64)
    c[0] = c[-1] = 2
    lens = (c[:, None, None] * c[None, :, None] * c[None, None, :]).reshape(-1)   # z-major rows
    rp = np.zeros(n ** 3 + 1, dtype=np.int64)
    np.cumsum(lens, out=rp[1:])
    return rp


def load_models(nitro):
    out = {}
    for k, p in MODELS.items():
        if os.path.exists(p):
            ctx = nitro.Context()
            cv = nitro.CodeVariant(ctx, "spmv")
            cv.register_spmv()
            cv.load(p)
            out[k] = (ctx, cv)
    return out


def feature_gpu_times(M, stream, reps=3):
    """Device time of the feature pass (A1): the launches enqueued asynchronously
    (features_async), CUDA events on the launching stream around them."""
    import torch
    out = []
    for _ in range(reps):
        M.invalidate()
        M.flush_l2()
        a, b = ev_pair()
        a.record(stream) if stream is not None else a.record()
        M.features_async()
        b.record(stream) if stream is not None else b.record()
        torch.cuda.synchronize()
        M.features()
        out.append(a.elapsed_time(b))
    return out


def ev_pair():
    import torch
    return torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


# ---------------------------------------------------------------------------- CPU oracle legs
def cpu_sample(nrows_target=2 * 1024 * 1024):
    """Bounded host sample of configs[4]: the 8 z-planes in the middle of the
    512^3 grid (2,097,152 rows, interior stencil rows), generated on the host."""
    n = 512
    planes = max(1, nrows_target // (n * n))
    row0 = (n // 2 - planes // 2) * n * n
    A = make("c4", None, row0=row0, nrows=planes * n * n)
    import synth
    x = synth.vector(n ** 3, seed=2)
    return A, x, f"configs[4] rows [{row0}, {row0 + planes * n * n}) ({planes} middle z-planes of 512^3, " \
                 f"{A.nnz} nnz), fp64 oracle CSR loop"


def time_oracle(A, x, threads, seconds):
    """Seconds per multiply of the oracle loop (inputs converted to its fp64
    layout once, outside the timing), multiplies run, threads used."""
    import oracle
    fn = oracle.spmv_prepared(A, x, threads)
    used = fn()
    n, t0 = 0, time.perf_counter()
    while True:
        fn()
        n += 1
        if time.perf_counter() - t0 >= seconds:
            break
    return (time.perf_counter() - t0) / n, n, used


def cpu_baseline(bytes_per_row, seconds=6.0):
    """The oracle as it stands (one thread, and the same loop over all host
    cores), on a bounded sample of the workload; credited with the GPU arm's
    bytes per row of the selected format, so value ratios are time ratios."""
    A, x, desc = cpu_sample()
    cores = os.cpu_count() or 1
    t1, n1, _ = time_oracle(A, x, 1, seconds)
    tn, nn, used = time_oracle(A, x, cores, seconds)
    nb = bytes_per_row * A.rows
    return {"value": nb / tn / 1e9, "unit": "GB/s", "cores": used, "kind": "oracle",
            "sample": f"{desc}; {nn} multiplies on {used} threads in {tn * nn:.1f}s",
            "host_cpu_count": cores,
            "single_thread": {"value": nb / t1 / 1e9, "unit": "GB/s", "cores": 1,
                              "sample": f"{n1} multiplies in {t1 * n1:.1f}s"},
            "gflops": 2 * A.nnz / tn / 1e9, "ms_per_multiply": tn * 1e3}


def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import numpy as np
    A, x, desc = cpu_sample()
    # bytes credited per row: the compulsory DIA bytes per row of configs[4] (the
    # Nitro arm's selected format there), (in-range slots*4 + D*4 + 8 N) / N
    n = 512
    N = n ** 3
    inrange = 0
    for dz in (-1, 0, 1):
        for dy in (-1, 0, 1):
            for dx in (-1, 0, 1):
                inrange += N - abs(dz * n * n + dy * n + dx)
    bpr = (inrange * 4 + 27 * 4 + 8 * N) / N
    cores = os.cpu_count() or 1
    import oracle
    fn = oracle.spmv_prepared(A, x, cores)
    for _ in range(args.warmup):
        fn()
    ts, used = [], cores
    for _ in range(args.steps):
        t0 = time.perf_counter()
        used = fn()
        ts.append(time.perf_counter() - t0)
    t = sum(ts) / len(ts)
    val = bpr * A.rows / t / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": WORKLOADS["c4"][0], "sample_rows": A.rows, "sample_nnz": A.nnz,
                       "parallelism": f"CPU oracle (fp64 CSR loop), rows over {used} host threads",
                       "bytes_per_row_credited": bpr},
            "cpu_baseline": {"value": val, "unit": "GB/s", "cores": used, "kind": "oracle",
                             "sample": f"{desc}; one step = one multiply of the sample"},
            "e2e": {"value": val, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------- single-config measurement
def measure_config(nitro, cfg, dev, models, reps, log):
    """features -> both models' picks -> every allowed variant timed (median of
    reps, L2 flushed) -> selected GB/s, fraction of peak, % of exhaustive best."""
    import torch
    import synth
    t0 = time.time()
    A = make(cfg, dev)
    if A.nnz < 2 ** 31:
        A.rowptr = A.rowptr.to(torch.int32)
    torch.cuda.synchronize()
    gen_s = time.time() - t0
    M = nitro.SpMV.from_csr(A)
    x = synth.vector(A.cols, seed=2, fp64=A.fp64, device=dev)
    y = torch.empty(A.rows, dtype=A.vals.dtype, device=dev)
    f = M.features()
    fts = []
    for _ in range(3):
        M.invalidate()
        M.flush_l2()
        a, b = ev_pair()
        a.record()
        f = M.features()
        b.record()
        torch.cuda.synchronize()
        fts.append(a.elapsed_time(b))
    fgs = feature_gpu_times(M, None)
    allowed = M.allowed_mask()
    fvec = [f[k] for k in nitro.FEATURE_NAMES]
    picks = {k: nitro.VARIANT_NAMES[cv.predict(fvec, allowed)] for k, (_, cv) in models.items()}
    ex = {}
    for v in range(nitro.NUM_VARIANTS):
        if not allowed[v]:
            continue
        a, b = ev_pair()
        a.record()
        M.prepare(v)
        b.record()
        torch.cuda.synchronize()
        med, _ = M.time(v, x, y, warmup=2, reps=reps, flush_l2=True)
        info = M.format_info(v)
        ex[nitro.VARIANT_NAMES[v]] = {"ms": med * 1e3, "GBps": info["compulsory_bytes"] / med / 1e9,
                                      "bytes": info["compulsory_bytes"], "conversion_ms": a.elapsed_time(b)}
        M.release(v)
    best = min(ex, key=lambda k: ex[k]["ms"])
    A_nnz = A.nnz
    out = {"workload": WORKLOADS[cfg][0], "rows": A.rows, "nnz": A.nnz, "generate_s": gen_s,
           "feature_ms": statistics.median(fts), "feature_gpu_ms": statistics.median(fgs),
           "features": {k: f[k] for k in nitro.FEATURE_NAMES},
           "allowed": [nitro.VARIANT_NAMES[v] for v in range(nitro.NUM_VARIANTS) if allowed[v]],
           "picks": picks, "exhaustive_best": best, "exhaustive": ex}
    for k, name in picks.items():
        out[f"pct_of_exhaustive_best_{k}"] = ex[best]["ms"] / ex[name]["ms"]
    g = gather_rate()
    if g:  # random-column classes: one x gather per nonzero bounds the multiply
        out["gather_bound_ms"] = A_nnz / g * 1e3
        out["best_frac_of_gather_bound"] = out["gather_bound_ms"] / ex[best]["ms"]
    M.close()
    del A, x, y, M
    torch.cuda.empty_cache()
    log(f"{cfg}: best {best} picks {picks} ({time.time() - t0:.1f}s)")
    return out


def selection_leg(nitro, dev, models, per_class, reps, log):
    """Re-time held-out configs[3] matrices (tools/train_select.py recipe, seeds
    2000+i) on this box and re-derive Nitro % for both models."""
    sys.path.insert(0, os.path.join(ROOT, "tools"))
    import train_select as ts
    rows = []
    t0 = time.time()
    nclass = len(ts.CLASSES)
    for i in range(per_class * nclass):
        cls = ts.CLASSES[i % nclass]
        seed = 2000 + i
        rows.append(ts.measure(ts.params_for(cls, seed), seed, dev, reps))
    res = {"matrices": len(rows), "seeds": [2000 + i for i in range(len(rows))],
           "subset": f"the first {per_class} held-out matrices of each class (configs[3] seeds 2000+i)",
           "wall_s": time.time() - t0}
    for k, (_, cv) in models.items():
        ratios, sel = [], []
        for r in rows:
            v = cv.predict(r["features"], r["allowed"])
            c = r["cost"]
            sel.append(nitro.VARIANT_NAMES[v])
            ratios.append(min(c) / c[v] if math.isfinite(c[v]) else 0.0)
        res[k] = {"nitro_pct_mean": sum(ratios) / len(ratios), "share_ge_70": sum(q >= 0.7 for q in ratios) / len(ratios),
                  "share_ge_90": sum(q >= 0.9 for q in ratios) / len(ratios), "selected": sel, "ratios": ratios,
                  "model": MODEL_DOC[k]}
    res["exhaustive_best"] = [nitro.VARIANT_NAMES[min(range(len(r["cost"])), key=lambda j: r["cost"][j])] for r in rows]
    log(f"selection leg: {len(rows)} matrices in {res['wall_s']:.1f}s: " +
        ", ".join(f"{k} {res[k]['nitro_pct_mean']:.3f}" for k in models))
    return res


# ---------------------------------------------------------------------------- our arm
def run_nitro(args):
    import numpy as np
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    import synth

    rank, world, local = dist_env()
    log = (lambda m: print(f"[bench] {m}", file=sys.stderr, flush=True)) if rank == 0 else (lambda m: None)
    if world > 1 and torch.cuda.device_count() < world:
        # rank 0 reports and fails the job; the other ranks leave quietly (a
        # failing rank would make torchrun stop rank 0 before it prints)
        if rank == 0:
            print(json.dumps({"error": f"--gpus {world} needs {world} GPUs, this node has "
                                       f"{torch.cuda.device_count()}", "n_gpus": world}), flush=True)
            sys.exit(2)
        sys.exit(0)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    use_dist = world > 1 or args.dist   # --dist: the multi-rank code path with one rank (NCCL communicator of 1)
    if use_dist:
        if world == 1:
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            os.environ.setdefault("MASTER_PORT", str(_free_port()))
            dist.init_process_group("nccl", device_id=dev, rank=0, world_size=1)
        else:
            dist.init_process_group("nccl", device_id=dev)
    stream = torch.cuda.current_stream(dev)
    models = load_models(nitro)
    deployed = args.model if args.model in models else next(iter(models), None)
    cfg = args.workload
    n = WORKLOADS[cfg][2][1] if WORKLOADS[cfg][1] == "stencil" else None
    t_start = time.time()

    # ---- this rank's rows (N = 1: the whole matrix)
    if not use_dist:
        A = make(cfg, dev)
        bounds = None
    else:
        assert n is not None, "multi-GPU workloads are the stencils"
        rp = stencil_rowptr_host(n)
        bounds = nitro.dist_partition(rp, world)
        del rp
        lo, hi = int(bounds[rank]), int(bounds[rank + 1])
        A = make(cfg, dev, row0=lo, nrows=hi - lo)
    if A.nnz < 2 ** 31:
        A.rowptr = A.rowptr.to(torch.int32)
    torch.cuda.synchronize()
    log(f"generated {cfg} rows {A.rows} nnz {A.nnz} in {time.time() - t_start:.1f}s")
    Ng = A.cols                               # global rows = cols (square)
    row0 = int(bounds[rank]) if use_dist else 0
    xfull_seed = 2
    y = torch.empty(A.rows, dtype=A.vals.dtype, device=dev)

    if not use_dist:
        M = nitro.SpMV.from_csr(A)
        x = synth.vector(Ng, seed=xfull_seed, fp64=A.fp64, device=dev)
        D = None
    else:
        uid = nitro.dist_unique_id() if rank == 0 else bytes(128)
        t = torch.tensor(list(uid), dtype=torch.uint8, device=dev)
        dist.broadcast(t, 0)
        D = nitro.Dist(bytes(t.cpu().tolist()), rank, world, local)
        M = D.spmv(Ng, bounds, A.rowptr, A.colidx, A.vals, exchange=0)    # A13: NCCL x all-gather
        x = nitro.Dist.x_local(M)             # x lives inside the exchange buffer: no per-multiply copy
        x.copy_(synth.vector(A.rows, seed=xfull_seed, fp64=A.fp64, device=dev, j0=row0))

    # ---- one end-to-end pass of the hot path: features -> select -> conversion
    a, b = ev_pair()
    t0 = time.perf_counter()
    feats = M.features() if D is None else D.features(M)
    feature_first_ms = (time.perf_counter() - t0) * 1e3
    fts = []
    if D is None:
        for _ in range(3):
            M.invalidate()
            M.flush_l2()
            a.record(stream)
            feats = M.features()
            b.record(stream)
            torch.cuda.synchronize()
            fts.append(a.elapsed_time(b))
    fgs = feature_gpu_times(M, stream) if D is None else []
    fvec = [feats[k] for k in nitro.FEATURE_NAMES]
    allowed = M.allowed_mask() if D is None else [True] * nitro.NUM_VARIANTS   # dist parts check their own
    picks, select_us = {}, {}
    for k, (_, cv) in models.items():
        t0 = time.perf_counter()
        picks[k] = cv.predict(fvec, allowed)
        select_us[k] = (time.perf_counter() - t0) * 1e6
    sel = picks[deployed] if deployed else nitro.DIA
    vname = nitro.VARIANT_NAMES[sel]
    log(f"features {feature_first_ms:.1f} ms (first call); picks " +
        str({k: nitro.VARIANT_NAMES[v] for k, v in picks.items()}) + f", deployed {deployed}: {vname}")

    def fmt_info(v):
        return M.format_info(v) if D is None else nitro.Dist.format_info(M, v)

    def run(v, xx, yy):
        if D is None:
            M.run(v, xx, yy)
        else:
            D.run(M, v, xx, yy)

    def timed(v, reps, xx=None, yy=None, flush=True):
        """median / mean of per-multiply CUDA-event times, max over ranks"""
        xx = x if xx is None else xx
        yy = y if yy is None else yy
        for _ in range(2):
            run(v, xx, yy)
        torch.cuda.synchronize()
        if use_dist:
            dist.barrier()
        ts = []
        for _ in range(reps):
            if flush:
                M.flush_l2()
            e0, e1 = ev_pair()
            e0.record(stream)
            run(v, xx, yy)
            e1.record(stream)
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        med = statistics.median(ts)
        if use_dist:
            tt = torch.tensor([med], device=dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            med = float(tt.item())
        return med

    # ---- exhaustive reference: every allowed variant timed the same way (conversion timed too)
    exhaustive = {}
    for v in range(nitro.NUM_VARIANTS):
        if not allowed[v] or (args.quick and v not in (sel, nitro.CSR_VECTOR)):
            continue
        a.record(stream)
        if D is None:
            M.prepare(v)
        else:
            run(v, x, y)
        b.record(stream)
        torch.cuda.synchronize()
        conv = a.elapsed_time(b)
        info = fmt_info(v)
        ms = timed(v, args.ex_reps)
        nb = info["compulsory_bytes"]
        if use_dist:
            tb = torch.tensor([nb], dtype=torch.float64, device=dev)
            dist.all_reduce(tb)
            nb = float(tb.item())
        exhaustive[nitro.VARIANT_NAMES[v]] = {"ms": ms, "GBps": nb / (ms * 1e-3) / 1e9, "bytes_all_ranks": nb,
                                             "conversion_ms": conv}
        if v != sel and D is None:
            M.release(v)
        log(f"  {nitro.VARIANT_NAMES[v]}: {ms:.3f} ms {nb / (ms * 1e-3) / 1e9:.0f} GB/s (conversion {conv:.1f} ms)")
    best = min(exhaustive, key=lambda k: exhaustive[k]["ms"])

    # ---- the timed region: K selected multiplies
    info = fmt_info(sel)
    nbytes = info["compulsory_bytes"]                  # this rank's bytes per multiply
    launches = M.launches(sel) if D is None else 3
    for _ in range(args.warmup):
        run(sel, x, y)
    torch.cuda.synchronize()
    if use_dist:
        dist.barrier()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    with Clocks(local) as clk:
        torch.cuda.synchronize()
        if use_dist:
            dist.barrier()
        for i in range(args.steps):
            M.flush_l2()
            starts[i].record(stream)
            run(sel, x, y)
            ends[i].record(stream)
        torch.cuda.synchronize()
        if use_dist:
            dist.barrier()
    times = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    ms = sum(times) / len(times)
    tot_bytes = nbytes
    if use_dist:
        tt = torch.tensor([ms], device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())
        tb = torch.tensor([nbytes], dtype=torch.float64, device=dev)
        dist.all_reduce(tb)
        tot_bytes = float(tb.item())
    gbps = tot_bytes / (ms * 1e-3) / 1e9
    per_gpu = gbps / world
    log(f"timed: {vname} {ms:.4f} ms/step, {gbps:.0f} GB/s total")

    # ---- halo exchange (f3) on the same rows, extra keys
    halo = None
    if D is not None and not args.quick:
        Mh = D.spmv(Ng, bounds, A.rowptr, A.colidx, A.vals, exchange=1)
        xh = nitro.Dist.x_local(Mh)
        xh.copy_(x)
        hinfo = nitro.Dist.exchange_info(Mh)
        Msave = M
        M = Mh
        halo = {"exchange": hinfo}
        for v in sorted({sel, nitro.CSR_VECTOR}):
            msv = timed(v, args.ex_reps, xh, y)
            halo[nitro.VARIANT_NAMES[v]] = {"ms": msv}
        M = Msave
        Mh.close()
        del xh

    # ---- e2e through the public API with HOST buffers (pinned), copies inside the timed region
    hx = torch.empty(A.rows, dtype=A.vals.dtype).pin_memory()
    hx.copy_(x.cpu())
    hy = torch.empty(A.rows, dtype=A.vals.dtype).pin_memory()
    sv = 8 if A.fp64 else 4
    if D is None:
        hxn, hyn = hx.numpy(), hy.numpy()
        for _ in range(2):
            M.run_host(sel, hxn, hyn)
        et = []
        for _ in range(max(3, min(args.steps, 10))):
            M.flush_l2()
            e0, e1 = ev_pair()
            e0.record(stream)
            M.run_host(sel, hxn, hyn)
            e1.record(stream)
            e1.synchronize()
            et.append(e0.elapsed_time(e1))
    else:
        xs = torch.empty_like(x)
        et = []
        for i in range(max(3, min(args.steps, 10)) + 2):
            M.flush_l2()
            e0, e1 = ev_pair()
            e0.record(stream)
            xs.copy_(hx, non_blocking=True)
            D.run(M, sel, xs, y)
            hy.copy_(y, non_blocking=True)
            e1.record(stream)
            e1.synchronize()
            if i >= 2:
                et.append(e0.elapsed_time(e1))
    e2e_ms = sum(et) / len(et)
    if use_dist:
        tt = torch.tensor([e2e_ms], device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        e2e_ms = float(tt.item())
    e2e = {"value": tot_bytes / (e2e_ms * 1e-3) / 1e9, "unit": "GB/s", "ms_per_step": e2e_ms,
           "h2d_bytes_per_step": A.rows * sv * world, "d2h_bytes_per_step": A.rows * sv * world,
           "api": "nitro_spmv_run_host (pinned host x/y)" if D is None else
           "pinned H2D x + nitro_dist_spmv_run + D2H y"}

    # ---- free the big matrix before the extra legs (N = 1)
    bytes_per_row = nbytes / A.rows
    rows_local, nnz_local = A.rows, A.nnz
    M.close()
    del M, A, x, y, hx, hy
    torch.cuda.empty_cache()

    extra = {}
    selection = None
    if world == 1 and not args.quick:
        for c in ("c1", "c2a", "c2b"):
            if c != cfg:
                extra[c] = measure_config(nitro, c, dev, models, 10, log)
        selection = selection_leg(nitro, dev, models, args.selection_per_class, 10, log)

    if rank != 0:
        if use_dist:
            dist.destroy_process_group()
        return
    pk, pk_kind = peaks()
    peak = float(pk.get("hbm_gbs", 6650.0))
    traffic = None
    try:
        rec = json.load(open(NCU_SUMMARY)).get(cfg, {}).get(vname)
        if rec:
            traffic = rec.get("dram_bytes_per_launch")
    except Exception:
        pass
    par = "single GPU" if not use_dist else \
        f"row-partitioned x{world} (nnz-balanced blocks), NCCL in-place x all-gather per multiply (A13), " \
        f"interior rows overlap the exchange"
    line = {
        "metric": METRIC, "value": gbps, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64" if WORKLOADS[cfg][2][2] else "f32", "data": "synthetic",
        "config": {"workload": WORKLOADS[cfg][0], "rows": Ng, "rows_per_gpu_max": rows_local,
                   "nnz_rank0": nnz_local,
                   "l2": "inputs larger than L2 (>= 1.9 GB per rank) and L2 flushed between steps (read of 3x L2)",
                   "parallelism": par, "selection": f"{deployed}: {MODEL_DOC.get(deployed)}",
                   "selected_variant": vname},
        "selected_variant": vname,
        "selection": {"deployed_model": deployed,
                      "picks": {k: nitro.VARIANT_NAMES[v] for k, v in picks.items()},
                      "pct_of_exhaustive_best": {k: exhaustive[best]["ms"] / exhaustive[nitro.VARIANT_NAMES[v]]["ms"]
                                                 for k, v in picks.items()
                                                 if nitro.VARIANT_NAMES[v] in exhaustive},
                      "models": {k: MODEL_DOC[k] for k in picks}, "select_us": select_us},
        "pct_of_exhaustive_best": exhaustive[best]["ms"] / exhaustive[vname]["ms"],
        "exhaustive_best": best, "exhaustive": exhaustive,
        "gflops": 2.0 * (feats["nnz"]) / (ms * 1e-3) / 1e9,
        "pct_of_hbm_peak": per_gpu / peak,
        "feature_ms": statistics.median(fts) if fts else None,
        "feature_gpu_ms": statistics.median(fgs) if fgs else None,
        "feature_ms_note": "feature_ms: the blocking features() call (launches, device time, D2H of the sums, host "
                           "wake-up); feature_gpu_ms: the same launches enqueued asynchronously, stream events around "
                           "them (device time of the pass incl. its small launches and the D2H)",
        "feature_first_call_ms": feature_first_ms,
        "features": {k: feats[k] for k in nitro.FEATURE_NAMES},
        "roofline": {"bound": "hbm", "achieved": per_gpu, "peak": peak, "unit": "GB/s", "frac": per_gpu / peak,
                     "traffic": traffic, "peak_kind": f"{pk_kind} hbm_gbs (device copy, read+write)",
                     "kernel": f"{vname} ({launches} launch/step)", "bytes_per_launch": nbytes,
                     "algorithmic_bytes": "DESIGN.md §6 compulsory bytes of the selected format (x read once, y "
                                          "written once)"},
        "gpu_launches": args.steps * (launches + 1),
        "gpu_launches_note": f"{args.steps} x ({launches} SpMV + 1 L2-flush) kernels of libnitro"
                             + (" + NCCL all-gather" if world > 1 else ""),
        "clocks": clk.summary(),
        "e2e": e2e,
    }
    if halo:
        line["halo_exchange"] = halo
    if use_dist:
        line["nccl_all_gather_floor_ms"] = (world - 1) / world * Ng * sv / 900e9 * 1e3
    if extra:
        line["configs"] = extra
    if selection:
        line["selection_leg"] = selection
    if world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(bytes_per_row)
    line["bench_wall_s"] = time.time() - t_start
    print(json.dumps(line), flush=True)
    if use_dist:
        dist.destroy_process_group()


def _free_port():
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def relaunch(args):
    """--gpus N > 1 without torchrun: start N ranks with torch.distributed.run."""
    port = _free_port()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="nitro", choices=["nitro", "reference"])
    ap.add_argument("--workload", default="c4", choices=["c4", "c1"])
    ap.add_argument("--model", default="paper", choices=["paper", "r11x"], help="deployed selection model")
    ap.add_argument("--ex-reps", type=int, default=7, help="timed reps per variant in the exhaustive reference")
    ap.add_argument("--selection-per-class", type=int, default=10, help="held-out configs[3] matrices per class")
    ap.add_argument("--quick", action="store_true", help="primary workload only (no extra configs/selection leg)")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--dist", action="store_true",
                    help="the multi-rank (nitro_dist_*, NCCL) code path even with one rank")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch(args))
    if args.impl == "reference":
        run_reference(args)
    else:
        run_nitro(args)


if __name__ == "__main__":
    main()
