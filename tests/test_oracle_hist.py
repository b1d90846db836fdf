"""Pins of the histogram oracle (oracle/hist.py) against what the definition
and the mathematics fix — not against itself (DESIGN R17)."""
import math

import numpy as np
import pytest

from oracle import hist as H
import synth


@pytest.mark.parametrize("nbins,rng_", [(1, 7), (3, 10), (7, 7), (16, 256), (5, 1 << 32)])
def test_histogram_equals_brute_force(nbins, rng_):
    r = np.random.default_rng(nbins)
    s = r.integers(0, min(rng_ + 5, 2**32), 500, dtype=np.uint64).astype(np.uint32)  # includes s >= range
    assert list(H.histogram(s, nbins, rng_)) == H.histogram_loop(s, nbins, rng_)


def test_counts_sum_to_in_range_samples():
    s = synth.hist_samples(100_003, "normal", 1000, seed=3, param=0.4)
    h = H.histogram(s, 37, 900)                   # 900 < max value: some samples dropped
    assert h.sum() == int((s < 900).sum()) and h.sum() < len(s)


def test_constant_input_single_bin():
    s = np.full(1234, 77, np.uint32)
    h = H.histogram(s, 10, 100)
    assert h[7] == 1234 and h.sum() == 1234


def test_full_sweep_is_uniform():
    # every value of [0, range) once, nbins | range: range / nbins per bin
    for nbins, rng_ in ((4, 64), (256, 65536), (1, 5), (5, 5)):
        h = H.histogram(np.arange(rng_, dtype=np.uint32), nbins, rng_)
        assert (h == rng_ // nbins).all()


def test_nbins_equal_range_is_value_count():
    s = np.array([0, 3, 3, 9, 9, 9, 2], np.uint32)
    assert list(H.histogram(s, 10, 10)) == [1, 0, 1, 2, 0, 0, 0, 0, 0, 3]


def test_bin_edges_floor():
    # range 10, 3 bins: edges at 10/3 and 20/3 -> values 0..3 | 4..6 | 7..9
    assert [H.bin_of(v, 3, 10) for v in range(11)] == [0, 0, 0, 0, 1, 1, 1, 2, 2, 2, None]


def test_top_of_32bit_range():
    s = np.array([0, 2**31 - 1, 2**31, 2**32 - 1], np.uint32)
    assert list(H.histogram(s, 2, 1 << 32)) == [2, 2]
    assert list(H.histogram(s, 65536, 1 << 32)[[0, 32767, 32768, 65535]]) == [1, 1, 1, 1]


def test_subsample_size_and_indices():
    assert len(H.subsample_indices(10)) == 3                   # ceil(10/4)
    assert len(H.subsample_indices(39_999)) == 10_000          # ceil(N/4) = 10000
    assert len(H.subsample_indices(10**7)) == 10_000           # cap
    assert H.subsample_indices(8) == [0, 4]
    assert H.subsample_indices(0) == []


def test_subsample_sd_closed_forms():
    assert H.subsample_sd(np.full(1000, 5, np.uint32)) == 0.0
    # N = 4k, s[i] = i: sub-sample 0, 4, ..., 4(k-1): sd = 4 sqrt((k^2 - 1) / 12)
    for k in (10, 2500, 10000):
        got = H.subsample_sd(np.arange(4 * k, dtype=np.uint32))
        assert got == pytest.approx(4 * math.sqrt((k * k - 1) / 12), rel=1e-15)
    # alternating 0 / v at the sampled positions: sd = v / 2
    s = np.zeros(4000, np.uint32)
    s[4::8] = 2**32 - 1                                        # sub-sample = every 4th: 0, v, 0, v, ...
    assert H.subsample_sd(s) == pytest.approx((2**32 - 1) / 2, rel=1e-15)


def test_features_vector():
    s = np.arange(100, dtype=np.uint32)
    f = H.features(s, 8)
    assert f[0] == 100.0 and f[1] == 12.5 and f[2] == pytest.approx(4 * math.sqrt((25 * 25 - 1) / 12))
