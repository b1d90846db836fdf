#!/usr/bin/env python
"""Summarise an ncu launch list (--metrics gpu__time_duration.sum[,dram__bytes_*] --csv)
into a per-kernel markdown table: launches, total / mean device time, DRAM bytes.

usage: python tools/launch_summary.py gpurun_out/launches_bench.csv profiles/launches_<tag>.md"""
import collections
import csv
import re
import sys


def main():
    src, dst = sys.argv[1], sys.argv[2]
    lines = [l for l in open(src) if l.startswith('"')]
    rows = list(csv.DictReader(lines))
    per = collections.defaultdict(lambda: {"n": set(), "t_ns": 0.0, "dram": 0.0})
    order = []
    for r in rows:
        name = re.sub(r"\(.*", "", r["Kernel Name"]).replace("<unnamed>::", "")
        name = re.sub(r"nitro::", "", name)
        k = per[name]
        if name not in order:
            order.append(name)
        k["n"].add(r["ID"])
        v = float(r["Metric Value"].replace(",", "")) if r["Metric Value"] else 0.0
        unit = r["Metric Unit"]
        if r["Metric Name"] == "gpu__time_duration.sum":
            k["t_ns"] += v * {"nsecond": 1, "usecond": 1e3, "msecond": 1e6, "ns": 1, "us": 1e3, "ms": 1e6}.get(unit, 1)
        elif r["Metric Name"].startswith("dram__bytes"):
            k["dram"] += v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
    tot = sum(k["t_ns"] for k in per.values())
    out = [f"# ncu launch list: `{src}`", "",
           "Cold-cache, serialised replays (compare shares, not absolutes).", "",
           "| kernel | launches | total us | mean us | share % | DRAM MB / launch |", "|---|---|---|---|---|---|"]
    for name in sorted(order, key=lambda n: -per[n]["t_ns"]):
        k = per[name]
        n = len(k["n"])
        out.append(f"| `{name}` | {n} | {k['t_ns'] / 1e3:.1f} | {k['t_ns'] / 1e3 / n:.2f} | {100 * k['t_ns'] / tot:.1f} | "
                   f"{k['dram'] / n / 1e6:.1f} |")
    open(dst, "w").write("\n".join(out) + "\n")
    print("\n".join(out))


if __name__ == "__main__":
    main()
