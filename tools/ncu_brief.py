#!/usr/bin/env python
"""Brief of an ncu --page details CSV (+ optional source CSVs): per kernel the
key throughput/occupancy/stall lines; per source CSV the stall-reason mix and
the hottest SASS lines."""
import collections
import csv
import sys

KEYS = ["Duration", "DRAM Throughput", "Memory Throughput", "L1/TEX Hit Rate", "L2 Hit Rate", "Achieved Occupancy",
        "Theoretical Occupancy", "Registers Per Thread", "Issued Warp Per Scheduler", "No Eligible",
        "Warp Cycles Per Issued Instruction", "L2 Cache Throughput", "L1/TEX Cache Throughput",
        "Compute (SM) Throughput", "Executed Ipc Active"]


def details(path):
    rows = list(csv.reader(open(path)))
    hdr = rows[0]
    seen = collections.OrderedDict()
    for r in rows[1:]:
        d = dict(zip(hdr, r))
        key = (d["ID"], d["Kernel Name"][:70])
        if d["Metric Name"] in KEYS:
            seen.setdefault(key, {})[d["Metric Name"]] = d["Metric Value"] + " " + d.get("Metric Unit", "")
    for (i, k), m in seen.items():
        print(f"[{i}] {k}")
        print("    " + "; ".join(f"{n}={m[n]}" for n in KEYS if n in m))


def source(path, top=12):
    rows = list(csv.reader(open(path)))
    ks = [i for i, r in enumerate(rows) if r and r[0] == "Kernel Name"]
    k0 = ks[0]
    hdr = rows[k0 + 1]
    data = rows[k0 + 2:(ks[1] if len(ks) > 1 else len(rows))]
    si = hdr.index("Warp Stall Sampling (All Samples)")
    tot = sum(float(r[si] or 0) for r in data if len(r) > si) or 1
    reasons = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
    agg = collections.Counter()
    for r in data:
        for h in reasons:
            try:
                agg[h] += float(r[hdr.index(h)] or 0)
            except ValueError:
                pass
    print(f"== {path}: {rows[k0][1][:70]}  samples {tot:.0f}")
    print("   stalls: " + ", ".join(f"{k[6:]} {100 * v / tot:.0f}%" for k, v in agg.most_common(8)))
    for i in sorted(range(len(data)), key=lambda i: -float(data[i][si] or 0))[:top]:
        print(f"   {100 * float(data[i][si]) / tot:5.1f}% [{i:4d}] {data[i][1][:100]}")


if __name__ == "__main__":
    for p in sys.argv[1:]:
        (source if "_src" in p else details)(p)
