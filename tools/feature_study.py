#!/usr/bin/env python
"""Feature-evaluation overhead study (the Fig. 8 analogue,
P:L264-271) on the configs[3] matrices.

Part A (host, from artifacts/c3_table.json): the model retrained through the
library (nitro_cv_train_from_table) on cumulative feature sets ordered by
their evaluation cost, scored on the 40 held-out matrices (% of exhaustive
best):
  L0  nnz, rows                      known at nitro_spmv_create (no GPU work)
  L0m + mean                         O(1) from nnz / rows
  L1  + sd, max_dev, ell_fill        one pass over rowptr (nitro_spmv_row_features)
  L2  + dia_fill                     the full pass over rowptr + colidx (nitro_spmv_features)

Part B (GPU, --gpu): per held-out matrix, regenerated from its recorded seed:
the rowptr-only level, the full feature pass, the host select, the conversion
of the selected variant, and its multiply; the break-even count of multiplies
after which Nitro (features + select + conversion, once) beats running the
paper's default variant (CSR-vector) without any of it: overhead / (t_default -
t_selected) (the feature cost is amortised over many SpMVs).

Writes artifacts/feature_study.json.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

LEVELS = [("L0", ["nnz", "rows"]), ("L0m", ["nnz", "rows", "mean"]),
          ("L1", ["nnz", "rows", "mean", "sd", "max_dev", "ell_fill"]),
          ("L2", ["nnz", "rows", "mean", "sd", "max_dev", "dia_fill", "ell_fill"])]


def ablation(table, nitro, ext=False):
    names = list(nitro.FEATURE_NAMES)
    Ftr = np.array([r["features"] for r in table["train"]], np.float64)
    Ctr = np.array([r["cost"] for r in table["train"]], np.float64)
    out = {}
    for lev, feats in LEVELS:
        cols = [names.index(f) for f in feats]
        ctx = nitro.Context()
        cv = nitro.CodeVariant(ctx, f"spmv_{lev}")
        for v in nitro.VARIANT_NAMES:
            cv.add_variant(v, lambda i: 0.0)          # costs come from the table
        for f in feats:
            cv.add_feature(f, lambda i: 0.0)
        cv.set_default(nitro.CSR_VECTOR)
        if ext:
            cv.set_feature_transform((1 << len(cols)) - 1, True)   # R11x extension (log1p + clip)
        cv.train_from_table(Ftr[:, cols], Ctr)
        ratios = []
        for r in table["test"]:
            v = cv.predict(np.array(r["features"], np.float64)[cols], r["allowed"])
            c = r["cost"]
            ratios.append(min(c) / c[v] if math.isfinite(c[v]) else 0.0)
        out[lev] = {"features": feats, "nitro_pct_mean": sum(ratios) / len(ratios),
                    "share_ge_90": sum(q >= 0.9 for q in ratios) / len(ratios)}
        print(f"{lev:4s} {out[lev]['nitro_pct_mean']:.4f}  {feats}", flush=True)
    return out


def gpu_overheads(table, nitro, model_path):
    import torch
    import synth
    from train_select import generate
    dev = torch.device("cuda:0")
    ctx = nitro.Context()
    cv = nitro.CodeVariant(ctx, "spmv")
    cv.register_spmv()
    cv.load(model_path)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def ev_ms(fn, reps=5, pre=None):
        ts = []
        for _ in range(reps):
            if pre:
                pre()
            torch.cuda.synchronize()
            s.record()
            fn()
            e.record()
            torch.cuda.synchronize()
            ts.append(s.elapsed_time(e))
        return statistics.median(ts)

    rows = []
    for r in table["test"]:
        A = generate(r["params"], r["seed"], dev)
        if A.nnz < 2 ** 31:
            A.rowptr = A.rowptr.to(torch.int32)
        M = nitro.SpMV.from_csr(A)
        M.features()                                   # buffers allocated once
        t_row = ev_ms(M.row_features, pre=M.flush_l2)

        def full():
            M.invalidate()
            M.features()
        t_full = ev_ms(full, pre=M.flush_l2)
        f = M.features()
        fvec = [f[k] for k in nitro.FEATURE_NAMES]
        allowed = M.allowed_mask()
        t0 = time.perf_counter()
        for _ in range(20):
            v = cv.predict(fvec, allowed)
        t_sel_host = (time.perf_counter() - t0) / 20 * 1e3

        def conv():
            M.release(v)
            M.prepare(v)
        t_conv = ev_ms(conv, reps=3) if v != nitro.CSR_SCALAR else 0.0
        c = r["cost"]
        t_v, t_def = c[v] * 1e3, c[nitro.CSR_VECTOR] * 1e3
        overhead = t_full + t_sel_host + t_conv
        gain = t_def - t_v
        row = {"params": r["params"], "rows": r["rows"], "nnz": r["nnz"], "selected": nitro.VARIANT_NAMES[v],
               "row_features_ms": t_row, "features_ms": t_full, "select_ms": t_sel_host, "convert_ms": t_conv,
               "spmv_ms": t_v, "default_ms": t_def, "features_per_spmv": t_full / t_v,
               "break_even_spmvs": (overhead / gain) if gain > 0 else None}
        rows.append(row)
        print(f"{r['params']['class']:9s} N={r['rows']:9d} sel={row['selected']:10s} row {t_row:.3f} full {t_full:.3f} "
              f"sel {t_sel_host:.3f} conv {t_conv:.3f} spmv {t_v:.3f} def {t_def:.3f} "
              f"break-even {row['break_even_spmvs']}", flush=True)
        M.close()
        del A
        torch.cuda.empty_cache()
    fps = [q["features_per_spmv"] for q in rows]
    be = [q["break_even_spmvs"] for q in rows if q["break_even_spmvs"] is not None]
    summ = {"features_per_spmv_median": statistics.median(fps), "features_per_spmv_max": max(fps),
            "row_level_fraction_of_full_median": statistics.median(q["row_features_ms"] / q["features_ms"]
                                                                   for q in rows),
            "break_even_spmvs_median": statistics.median(be) if be else None,
            "break_even_spmvs_max": max(be) if be else None,
            "n_default_already_best": sum(1 for q in rows if q["break_even_spmvs"] is None)}
    return rows, summ


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpu", action="store_true", help="also measure the per-matrix overheads on the GPU")
    ap.add_argument("--table", default=os.path.join(ROOT, "artifacts", "c3_table.json"))
    ap.add_argument("--model", default=os.path.join(ROOT, "artifacts", "spmv_model.txt"))
    ap.add_argument("--out", default=os.path.join(ROOT, "artifacts", "feature_study.json"))
    args = ap.parse_args()
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    table = json.load(open(args.table))
    res = {"ablation": ablation(table, nitro), "scaling": "paper: [-1, 1] min-max (P:L179)",
           "ablation_r11x": ablation(table, nitro, ext=True)}
    if args.gpu:
        rows, summ = gpu_overheads(table, nitro, args.model)
        res["per_matrix"] = rows
        res["summary"] = summ
        print(json.dumps(summ, indent=1))
    elif os.path.exists(args.out):   # keep an earlier GPU part
        old = json.load(open(args.out))
        for k in ("per_matrix", "summary"):
            if k in old:
                res[k] = old[k]
    json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
