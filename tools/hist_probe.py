#!/usr/bin/env python
"""Histogram family on one large input (16 M uint32 samples, 256 bins over
2^16 values): every variant run twice (for ncu) or timed (--time: median of
20, L2 flushed), GB/s of the 64 MB sample read."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import paper_conf_ipps_muralidharanshgc14_b200 as nitro
    import synth
    timing = "--time" in sys.argv
    dist = next((a for a in sys.argv[1:] if a in synth.HIST_DISTS), "uniform")
    n, nbins, rng = 1 << 24, 256, 1 << 16
    s = synth.hist_samples(n, dist, rng, seed=11, param=0.01)
    dev = torch.device("cuda:0")
    H = nitro.Hist(torch.from_numpy(s.view(np.int32)).to(dev), nbins, rng)
    h = torch.empty(nbins, dtype=torch.int32, device=dev)
    for v in range(nitro.HIST_NUM_VARIANTS):
        if timing:
            t = H.time(v, h, warmup=3, reps=20, flush_l2=True)
            print(f"{dist} {nitro.HIST_VARIANT_NAMES[v]:22s} {t * 1e6:8.1f} us {4 * n / t / 1e9:7.1f} GB/s", flush=True)
        else:
            for _ in range(2):
                H.run(v, h)
            torch.cuda.synchronize()


if __name__ == "__main__":
    main()
