"""Histogram code-variant family through the C ABI vs the
oracle: counts bit-exact for all six variants (integer work), features
bit-exact (exact integer moments), constraint and selection plumbing."""
import numpy as np
import pytest

import synth
from oracle import hist as OH

pytestmark = pytest.mark.gpu


def nitro():
    import paper_conf_ipps_muralidharanshgc14_b200 as n
    return n


def dev_samples(s, cuda, shift=0):
    import torch
    t = torch.from_numpy(s.view(np.int32).copy())
    if shift:
        buf = torch.zeros(t.numel() + shift, dtype=torch.int32)
        buf[shift:] = t
        return buf.to(cuda)[shift:]                 # 4-byte misaligned view: scalar load path
    return t.to(cuda)


CASES = [
    # (n, dist, range, nbins, param) — several tiles + ragged tails, both sort tile (2048) and atomic tile (4096)
    (1, "uniform", 256, 16, 0.1),
    (2047, "uniform", 256, 256, 0.1),
    (4097, "normal", 1 << 16, 1000, 0.05),
    (100_003, "uniform", 1 << 20, 4096, 0.1),
    (100_003, "spike", 1 << 12, 64, 0.9),
    (65_537, "exponential", 1 << 16, 65536, 0.01),   # nbins > 49152: shared variants ruled out
    (70_001, "sorted", 1000, 7, 0.1),
    (50_000, "normal", 1 << 30, 1, 0.2),
    (33_333, "uniform", 1 << 32, 49152, 0.1),
    # power-of-two bin widths (the shift path), incl. width 2^32 (one bin) and width 1
    (123_457, "uniform", 1 << 32, 1024, 0.1),
    (9_999, "uniform", 1 << 32, 1, 0.1),
    (20_000, "exponential", 256, 256, 0.05),
    (77_777, "normal", 1 << 16, 4096, 0.2),
]


@pytest.mark.parametrize("n,dist,rng_,nbins,param", CASES)
@pytest.mark.parametrize("shift", [0, 1])
def test_all_variants_bit_exact(cuda, n, dist, rng_, nbins, param, shift):
    import torch
    nn = nitro()
    s = synth.hist_samples(n, dist, min(rng_ + rng_ // 8, 2**32), seed=n + nbins, param=param)  # some >= range
    want = OH.histogram(s, nbins, rng_)
    H = nn.Hist(dev_samples(s, cuda, shift), nbins, rng_)
    for v in range(nn.HIST_NUM_VARIANTS):
        if not H.allowed(v):
            assert v in (nn.HIST_SHARED_ES, nn.HIST_SHARED_DYN) and nbins > 49152
            with pytest.raises(nn.NitroError) as e:
                H.run(v)
            assert e.value.code == 4
            continue
        h = torch.full((nbins,), -1, dtype=torch.int32, device=cuda)
        H.run(v, h)
        h = H.run(v, h)                                  # twice: outputs are overwritten, queues re-armed
        torch.cuda.synchronize()
        got = h.cpu().numpy().view(np.uint32).astype(np.int64)
        assert np.array_equal(got, want), (nn.HIST_VARIANT_NAMES[v], np.nonzero(got != want)[0][:5])
    H.close()


def test_empty_input(cuda):
    import torch
    nn = nitro()
    H = nn.Hist(torch.zeros(0, dtype=torch.int32, device=cuda), 10, 100)
    for v in range(nn.HIST_NUM_VARIANTS):
        h = torch.full((10,), 5, dtype=torch.int32, device=cuda)
        H.run(v, h)
        torch.cuda.synchronize()
        assert (h.cpu() == 0).all()
    assert H.features() == {"n": 0.0, "n_per_bin": 0.0, "subsample_sd": 0.0}


@pytest.mark.parametrize("n,dist", [(1, "uniform"), (10, "uniform"), (39_999, "normal"), (1_000_003, "exponential"),
                                    (4_000_000, "spike")])
def test_features_bit_exact(cuda, n, dist):
    nn = nitro()
    s = synth.hist_samples(n, dist, 1 << 32, seed=7, param=0.3)
    H = nn.Hist(dev_samples(s, cuda), 333, 1 << 32)
    f = H.features()
    want = OH.features(s, 333)
    assert [f["n"], f["n_per_bin"], f["subsample_sd"]] == want


def test_bad_arguments(cuda):
    import torch
    nn = nitro()
    t = torch.zeros(4, dtype=torch.int32, device=cuda)
    for nb, r in ((0, 10), (65537, 10), (10, 0), (10, 2**32 + 1)):
        with pytest.raises(nn.NitroError) as e:
            nn.Hist(t, nb, r)
        assert e.value.code == 1


def test_register_train_select(cuda, tmp_path):
    """The generic layer with the histogram registration: exhaustive timing of
    the six variants on a few inputs, train, select (ruled-out -> default)."""
    import torch
    nn = nitro()
    ctx = nn.Context()
    cv = nn.CodeVariant(ctx, "hist")
    cv.register_hist()
    keep = []
    cfgs = [("uniform", 1 << 16, 256, 0.1), ("spike", 1 << 16, 256, 0.95), ("normal", 1 << 16, 65536, 0.001),
            ("uniform", 1 << 20, 16, 0.1), ("exponential", 1 << 16, 4096, 0.002), ("uniform", 1 << 12, 4096, 0.1)]
    for i, (dist, rng_, nb, p) in enumerate(cfgs):
        s = synth.hist_samples(200_000 + 1000 * i, dist, rng_, seed=i, param=p)
        H = nn.Hist(dev_samples(s, cuda), nb, rng_)
        h = torch.empty(nb, dtype=torch.int32, device=cuda)
        rec = nn.hist_input(H, h, warmup=1, reps=3)
        keep.append(rec)
        cv.add_training_input(nn.addr(rec))
    cv.train(log2c_lo=-1, log2c_hi=3, log2g_lo=-3, log2g_hi=1)
    cost, feat, lab = cv.training_table()
    assert cost.shape == (6, 6) and feat.shape == (6, 3)
    assert np.isinf(cost[2, nn.HIST_SHARED_ES]) and np.isinf(cost[2, nn.HIST_SHARED_DYN])   # 65536 bins
    assert list(lab) == [int(np.argmin(c)) for c in cost]
    v, fsel = cv.select(nn.addr(keep[2]))
    assert v not in (nn.HIST_SHARED_ES, nn.HIST_SHARED_DYN)
    v, c = cv.call(nn.addr(keep[0]))
    assert 0 <= v < 6 and np.isfinite(c)
