#!/usr/bin/env python
"""Incremental tuning on the configs[3] experiment (paper Fig. 7 analogue).

Replays artifacts/c3_table.json (GPU-measured costs of every variant on the 60
training matrices and 40 held-out matrices): the library's nitro_cv_itune
labels training matrices one at a time (labelling = the measured exhaustive
search of that matrix, returned by host callbacks), refitting after each, and
scores the held-out set after every refit.  Writes artifacts/c3_itune.json.
"""
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import numpy as np
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    t = json.load(open(os.path.join(ROOT, "artifacts", "c3_table.json")))
    rep = json.load(open(os.path.join(ROOT, "artifacts", "c3_report.json")))
    Fp = np.array([r["features"] for r in t["train"]])
    Cp = np.array([[math.inf if c is None else c for c in r["cost"]] for r in t["train"]])
    Ft = np.array([r["features"] for r in t["test"]])
    Ct = np.array([[math.inf if c is None else c for c in r["cost"]] for r in t["test"]])
    seeds = [0, 1, 2, 3, 4]
    out = {"note": "P:L266: ~25 iterations reach 90% of full-training performance, <= 50 match it (C2050, UFL)"}
    for mode in ("paper", "r11x"):
        out[mode] = replay(nitro, Fp, Cp, Ft, Ct, seeds, mode == "r11x",
                           rep["nitro_pct_mean"] if mode == "paper" else rep["extension_r11x"]["nitro_pct_mean"])
    json.dump(out, open(os.path.join(ROOT, "artifacts", "c3_itune.json"), "w"), indent=1)


def replay(nitro, Fp, Cp, Ft, Ct, seeds, ext, full):
    """nitro_cv_itune over the table, the paper's [-1, 1] scaling (ext False)
    or the R11x extension (log1p + clip)."""
    runs = []
    for sd in seeds:
        ctx_i = nitro.Context()
        cvi = nitro.CodeVariant(ctx_i, "spmv-replay")
        for v, name in enumerate(nitro.VARIANT_NAMES):
            cvi.add_variant(name, lambda i, v=v: Cp[i, v])
        for j, name in enumerate(nitro.FEATURE_NAMES):
            cvi.add_feature(name, lambda i, j=j: Fp[i, j])
        for v in (nitro.ELL, nitro.DIA):
            cvi.add_constraint(v, lambda i, v=v: math.isfinite(Cp[i, v]))
        cvi.set_default(nitro.CSR_VECTOR)
        if ext:
            cvi.set_feature_transform(0x7F, True)   # R11x extension
        for i in range(len(Fp)):
            cvi.add_training_input(i)
        h = cvi.itune(init=len(nitro.VARIANT_NAMES), iters=0, seed=sd, test_feat=Ft, test_cost=Ct)
        runs.append(h)
        print(f"{'r11x' if ext else 'paper'} seed {sd}: perf " + " ".join(f"{p:.3f}" for p in h["test_perf"]),
              flush=True)
    summary = []
    for sd, h in zip(seeds, runs):
        perf = h["test_perf"]
        it90 = next((k for k, p in enumerate(perf) if p >= 0.9 * full), None)
        itmatch = next((k for k, p in enumerate(perf) if p >= full - 1e-12), None)
        summary.append({"seed": sd, "init_labelled": h["n_labelled"][0],
                        "iters_to_90pct_of_full": it90, "iters_to_match_full": itmatch,
                        "labelled_at_90pct": h["n_labelled"][it90] if it90 is not None else None})
    print(json.dumps(summary, indent=1))
    return {"full_training_nitro_pct": full, "runs": runs, "summary": summary}


if __name__ == "__main__":
    main()
