#!/usr/bin/env python
"""Summarise the histogram-family ncu --set full capture (gpurun_out/prof_hist_raw.csv,
from tools/hist_probe.py: 6 variants x 2 runs) into profiles/ncu_hist_<tag>.md."""
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
from ncu_summarize import load  # noqa: E402

NAMES = ("sort_es", "sort_dynamic", "shared_atomic_es", "shared_atomic_dynamic", "global_atomic_es",
         "global_atomic_dynamic")


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
    recs = load(os.path.join(ROOT, "gpurun_out", "prof_hist_raw.csv"))
    md = [f"# ncu --set full: histogram family ({tag})", "",
          "`tools/hist_probe.py uniform`: 16 M uint32 samples (64 MB), 256 bins over 2^16 values; two runs per",
          "variant in id order; cold-cache replays (ncu default cache control).", "",
          "| # | variant | kernel | time us | DRAM MB (r+w) | DRAM % peak | L2 hit % | occ % | issue active % | regs |",
          "|---|---|---|---|---|---|---|---|---|---|"]
    for i, r in enumerate(recs):
        k = re.sub(r"\(.*", "", r["kernel"]).replace("nitro::", "").replace("<unnamed>::", "")
        v = NAMES[i // 2] if i // 2 < len(NAMES) else "?"
        dram = (r.get("dram_read", 0) + r.get("dram_write", 0)) / 1e6
        md.append(f"| {i} | {v} | `{k[:60]}` | {r.get('dur_ns', 0) / 1e3:.1f} | {dram:.1f} | {r.get('dram_pct', 0):.1f} | "
                  f"{r.get('l2_hit', 0):.1f} | {r.get('occupancy', 0):.1f} | {r.get('issue_active', 0):.1f} | "
                  f"{int(r.get('regs', 0))} |")
    out = os.path.join(ROOT, "profiles", f"ncu_hist_{tag}.md")
    open(out, "w").write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
