"""oracle.hist — plain CPU reference of the histogram code-variant family
(TEST INFRASTRUCTURE ONLY, like the rest of oracle/).

  histogram     P:L226 ("counts the number of observations that fall into one
                of a set of disjoint categories or bins"); the even binning
                h[b] = #{i : s_i < range, floor(s_i * nbins / range) = b} is
                this build's reading (R17), in exact integers.
  subsample_sd  P:L216 (feature "SubSampleSD"), P:L269 ("the standard deviation
                of a sub-sample of the input ... 25% of the size of the input
                sample, or 10,000 elements, whichever is lower"); reading R17:
                k = min(ceil(N/4), 10000) samples at indices floor(j*N/k),
                population SD from exact integer moments.
  features      P:L216: N, N/#bins, SubSampleSD.
"""
from __future__ import annotations

import math

import numpy as np


def bin_of(s: int, nbins: int, value_range: int):
    """Bin of one sample (None when s >= range): floor(s * nbins / range)."""
    return (s * nbins) // value_range if s < value_range else None


def histogram(samples, nbins: int, value_range: int) -> np.ndarray:
    """Counts per bin (uint32 wrap never occurs for n < 2^32)."""
    s = np.asarray(samples, dtype=np.uint64)
    s = s[s < np.uint64(value_range)]
    b = (s * np.uint64(nbins)) // np.uint64(value_range)        # exact: s * nbins < 2^48
    return np.bincount(b.astype(np.int64), minlength=nbins).astype(np.int64)


def histogram_loop(samples, nbins: int, value_range: int) -> list:
    """Brute-force definition, one sample at a time (small inputs)."""
    h = [0] * nbins
    for s in samples:
        b = bin_of(int(s), nbins, value_range)
        if b is not None:
            h[b] += 1
    return h


def subsample_indices(n: int) -> list:
    k = min((n + 3) // 4, 10000)
    return [j * n // k for j in range(k)]


def subsample_sd(samples) -> float:
    n = len(samples)
    idx = subsample_indices(n)
    k = len(idx)
    if k == 0:
        return 0.0
    v = [int(samples[i]) for i in idx]
    s1 = sum(v)
    s2 = sum(x * x for x in v)
    return math.sqrt(float(k * s2 - s1 * s1) / (float(k) * float(k)))


def features(samples, nbins: int) -> list:
    n = len(samples)
    return [float(n), float(n) / float(nbins), subsample_sd(samples)]
