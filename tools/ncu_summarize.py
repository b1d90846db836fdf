#!/usr/bin/env python
"""Summarise ncu --set full raw CSV exports (gpurun_out/prof_<cfg>_raw.csv) into
profiles/ncu_summary.json and a markdown table (profiles/ncu_<tag>.md).

Per kernel launch: duration, DRAM bytes read/write, DRAM throughput % of peak,
L2/L1 hit rates, achieved occupancy, registers.  Variant attribution follows
tools/profile_variants.py's launch order (features, then 2 runs per allowed
variant; HYB = k_ell + k_hyb_tail)."""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = {
    "dur_ns": "gpu__time_duration.sum",
    "dram_read": "dram__bytes_read.sum",
    "dram_write": "dram__bytes_write.sum",
    "dram_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "l2_hit": "lts__t_sector_hit_rate.pct",
    "l1_hit": "l1tex__t_sector_hit_rate.pct",
    "occupancy": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "regs": "launch__registers_per_thread",
    "issue_active": "sm__inst_issued.avg.pct_of_peak_sustained_active",
}
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
              "nsecond": 1, "usecond": 1e3, "msecond": 1e6, "ns": 1, "us": 1e3, "ms": 1e6}


def load(path):
    rows = list(csv.reader(open(path)))
    # the CSV may start with ==PROF== lines
    start = next(i for i, r in enumerate(rows) if r and r[0] in ("ID", '"ID"') or (r and "Kernel Name" in r))
    hdr, units, data = rows[start], rows[start + 1], rows[start + 2:]
    out = []
    for r in data:
        if len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        rec = {"kernel": d.get("Kernel Name", "?")}
        for k, m in METRICS.items():
            if m in d and d[m] not in ("", "n/a"):
                try:
                    v = float(d[m].replace(",", ""))
                except ValueError:
                    continue
                rec[k] = v * UNIT_SCALE.get(u.get(m, ""), 1)
        out.append(rec)
    return out


def short(name):
    for k in ("k_features_long", "k_features", "k_csr_scalar", "k_csr_vector", "k_csr_vec4", "k_csr_stream", "k_hyb_tail",
              "k_hyb_fixup", "k_ell", "k_dia"):
        if k in name:
            return k
    return name[:40]


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
    src = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "gpurun_out")
    summ_path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    summary = json.load(open(summ_path)) if os.path.exists(summ_path) else {}
    md = [f"# ncu --set full summary ({tag})", "",
          "Cold-cache replays (ncu default cache control), one row per captured launch.", ""]
    for cfg in ("c1", "c2a", "c2b", "c4"):
        p = os.path.join(src, f"prof_{cfg}_raw.csv")
        if not os.path.exists(p):
            continue
        recs = load(p)
        md += [f"## {cfg}", "", "| # | kernel | attributed | time us | DRAM MB (r+w) | DRAM % peak | L2 hit % | L1 hit % | occ % | regs |",
               "|---|---|---|---|---|---|---|---|---|---|"]
        seen_ell = 0
        cfgsum = {}
        for i, r in enumerate(recs):
            k = short(r["kernel"])
            var = {"k_features": "features", "k_features_long": "features_long", "k_csr_scalar": "csr_scalar",
                   "k_csr_vector": "csr_vector", "k_csr_vec4": "csr_vector", "k_csr_stream": "csr_vector", "k_dia": "dia", "k_hyb_tail": "hyb",
                   "k_hyb_fixup": "hyb_fixup"}.get(k)
            if k == "k_ell":
                var = "ell" if seen_ell < 2 and cfg != "c2b" else "hyb_ell"
                seen_ell += 1
            traffic = r.get("dram_read", 0) + r.get("dram_write", 0)
            md.append(f"| {i} | {k} | {var} | {r.get('dur_ns', 0) / 1e3:.1f} | {traffic / 1e6:.1f} | "
                      f"{r.get('dram_pct', 0):.1f} | {r.get('l2_hit', 0):.1f} | {r.get('l1_hit', 0):.1f} | "
                      f"{r.get('occupancy', 0):.1f} | {r.get('regs', 0):.0f} |")
            if var:
                cfgsum.setdefault(var, []).append({"dram_bytes": traffic, "dur_ns": r.get("dur_ns"),
                                                   "dram_pct": r.get("dram_pct")})
        summary[cfg] = {v: {"dram_bytes_per_launch": sum(x["dram_bytes"] for x in l) / len(l),
                            "ncu_dur_us": sum(x["dur_ns"] or 0 for x in l) / len(l) / 1e3,
                            "dram_pct": sum(x["dram_pct"] or 0 for x in l) / len(l), "launches": len(l),
                            "source": f"profiles/ncu_{tag}.md"} for v, l in cfgsum.items()}
        md.append("")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    open(os.path.join(ROOT, "profiles", f"ncu_{tag}.md"), "w").write("\n".join(md) + "\n")
    json.dump(summary, open(summ_path, "w"), indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    main()
