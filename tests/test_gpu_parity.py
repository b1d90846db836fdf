"""GPU path (through the C ABI) vs the CPU oracle — the parity gate.

Bars (BASELINE north_star): features and conversions bit-exact; fp32 SpMV
per row |y - y_ref| <= 1e-5 * sum_j |a_ij x_j| + 1e-30; fp64 the same at
1e-12; integer stencils x integer x exact in fp32 for every variant.
"""
import numpy as np
import pytest

import oracle
import synth
from synth import Csr

pytestmark = pytest.mark.gpu

FEAT_KEYS = ("rows", "cols", "nnz", "sum_len", "sum_len2", "max_row", "ndiag", "canonical",
             "mean", "sd", "max_dev", "dia_fill", "ell_fill")


def nitro():
    import paper_conf_ipps_muralidharanshgc14_b200 as n
    return n


def handle(A, cuda, rowptr32=None):
    Ad = synth.to_device(A, cuda, rowptr32=rowptr32)
    return nitro().SpMV.from_csr(Ad), Ad


def small_mats():
    """Several tiles + ragged tails + degenerate cases; (name, host Csr)."""
    yield "2d5_n64_c0", synth.stencil("2d5", 64)
    yield "2d5_n64_rand", synth.stencil("2d5", 64, mode=1, seed=2)
    yield "3d27_n20", synth.stencil("3d27", 20, mode=1, seed=3)
    yield "3d7_n17", synth.stencil("3d7", 17, mode=1, seed=4)
    yield "1d3_n1001", synth.stencil("1d3", 1001, mode=1, seed=5)
    yield "2d9_n33", synth.stencil("2d9", 33, mode=1, seed=6)
    yield "banded_b7_d05", synth.banded(5003, 7, 0.5, seed=7)
    yield "banded_b40_full", synth.banded(2999, 40, 1.0, seed=8)
    yield "uniform_k32", synth.uniform(4099, 32, seed=9)
    yield "uniform_var_k9_rect", synth.uniform(3001, 9, variable=True, seed=10, M=7777)
    yield "uniform_k2", synth.uniform(9000, 2, seed=11)
    yield "rmat12_fp32", synth.rmat(12, 16, seed=12, fp64=False)
    yield "rmat13_fp64", synth.rmat(13, 8, seed=13, fp64=True)
    yield "one_row", Csr(1, 5, np.array([0, 3], np.int64), np.array([0, 2, 4], np.int32),
                         np.array([1.5, -2.0, 0.25], np.float32), False)
    yield "empty_rows", Csr(70, 70, np.array([0] * 35 + [2] * 36, np.int64), np.array([3, 69], np.int32),
                            np.array([1.0, 2.0], np.float32), False)
    yield "nnz0", Csr(40, 33, np.zeros(41, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32), False)
    # mean row length > 64: the nnz-split feature pass K1s
    yield "uniform_k100_rect", synth.uniform(3000, 100, seed=14, M=9000)
    yield "banded_b70_half", synth.banded(4001, 70, 0.5, seed=15)


def long_row_matrix(L=150_000, N=5000, fp64=False, seed=21):
    """Row 17 holds L entries (CSR-vector segments / HYB tail), others 0..5."""
    rng = np.random.default_rng(seed)
    lens = rng.integers(0, 6, N)
    lens[17] = L
    M = max(L + 10, N)
    rp = np.zeros(N + 1, np.int64)
    rp[1:] = np.cumsum(lens)
    cols = []
    for i, l in enumerate(lens):
        cols.append(np.sort(rng.choice(M, l, replace=False)) if l != L else np.arange(L))
    ci = np.concatenate(cols).astype(np.int32)
    v = rng.uniform(-1, 1, rp[-1])
    v[v == 0] = 0.5
    return Csr(N, M, rp, ci, v.astype(np.float64 if fp64 else np.float32), fp64)


def outlier_row_matrix(N=40_000, k=32, L=3000, seed=29):
    """Uniform random rows of k entries plus one row of L: row-length SD stays
    below the mean (no stream mode) while the longest row exceeds 16 steps of
    4V entries, so AUTO keeps K6 for CSR-vector instead of K6v."""
    rng = np.random.default_rng(seed)
    lens = np.full(N, k)
    lens[123] = L
    rp = np.zeros(N + 1, np.int64)
    rp[1:] = np.cumsum(lens)
    ci = np.concatenate([np.sort(rng.choice(N, l, replace=False)) for l in lens]).astype(np.int32)
    v = rng.uniform(-1, 1, rp[-1])
    v[v == 0] = 0.5
    return Csr(N, N, rp, ci, v.astype(np.float32), False)


def check_y(y, y_ref, r, fp64, what=""):
    tol = (1e-12 if fp64 else 1e-5) * r + 1e-30
    err = np.abs(np.asarray(y, np.float64) - y_ref)
    bad = np.nonzero(err > tol)[0]
    assert bad.size == 0, f"{what}: {bad.size} rows out of tolerance, first {bad[:5]}: {err[bad[:5]]} > {tol[bad[:5]]}"


# ------------------------------------------------------------------ features
@pytest.mark.parametrize("name,A", list(small_mats()))
def test_features_bit_exact(cuda, name, A):
    M, _ = handle(A, cuda)
    f = M.features()
    f_ref = oracle.features(A)
    for k in FEAT_KEYS:
        assert f[k] == f_ref[k], (name, k, f[k], f_ref[k])


def test_features_int64_rowptr_and_long_row(cuda):
    A = long_row_matrix()
    M, _ = handle(A, cuda, rowptr32=False)
    f, f_ref = M.features(), oracle.features(A)
    for k in FEAT_KEYS:
        assert f[k] == f_ref[k], k


def mixed_matrix(seed=31, N=3000, M=20000, fp64=False):
    """Every walk of the feature pass in one matrix: rows of similar short length
    (lane per row), groups of very different lengths (whole-warp span walk),
    medium rows, long rows of several kChunk (= 4096) chunks including exact
    multiples, a dense row (runs of equal bitmap words), near-diagonal rows,
    empty rows."""
    rng = np.random.default_rng(seed)
    lens = rng.integers(0, 10, N)
    lens[:320] = 7                                   # 10 groups of equal short rows
    med = rng.choice(np.arange(320, N), 60, replace=False)
    lens[med] = rng.integers(65, 2000, 60)
    longs = {700: 9000, 1201: 4097, 1202: 8192, 2500: 12289, 2999: 4096}
    for r, l in longs.items():
        lens[r] = l
    dense = 5
    lens[dense] = 6000
    lens[400:460] = 0                                # empty run
    cols = []
    for i, l in enumerate(lens):
        if i == dense:
            cols.append(np.arange(100, 100 + l))
        elif 2000 <= i < 2100 and l:
            lo = max(0, i - 4)
            cols.append(np.arange(lo, min(M, lo + l)))
            lens[i] = len(cols[-1])
        else:
            cols.append(np.sort(rng.choice(M, l, replace=False)))
    rp = np.zeros(N + 1, np.int64)
    rp[1:] = np.cumsum(lens)
    ci = np.concatenate(cols).astype(np.int32)
    v = rng.uniform(-1, 1, rp[-1])
    v[v == 0] = 0.5
    return Csr(N, M, rp, ci, v.astype(np.float64 if fp64 else np.float32), fp64)


ROW_KEYS = ("rows", "cols", "nnz", "sum_len", "sum_len2", "max_row", "mean", "sd", "max_dev", "ell_fill")


@pytest.mark.parametrize("name,A", list(small_mats()) + [("mixed", mixed_matrix())])
def test_row_features_level_bit_exact(cuda, name, A):
    """The rowptr-only feature level equals the full pass on every row-length
    feature and reports the column-dependent ones as not evaluated."""
    M, _ = handle(A, cuda, rowptr32=(name != "mixed"))
    f, f_ref = M.row_features(), oracle.features(A)
    for k in ROW_KEYS:
        assert f[k] == f_ref[k], (name, k, f[k], f_ref[k])
    assert f["ndiag"] == -1 and f["dia_fill"] == -1.0 and f["canonical"] == -1


def test_row_features_rejects_broken_rowptr(cuda):
    n = nitro()
    A = Csr(3, 3, np.array([0, 3, 2, 6], np.int64), np.array([0, 1, 2, 0, 1, 2], np.int32),
            np.ones(6, np.float32), False)
    M, _ = handle(A, cuda)
    with pytest.raises(n.NitroError) as e:
        M.row_features()
    assert e.value.code == 2


@pytest.mark.parametrize("rp32", [True, False])
def test_features_mixed_walks(cuda, rp32):
    A = mixed_matrix()
    assert oracle.is_canonical(A)
    M, _ = handle(A, cuda, rowptr32=rp32)
    f, f_ref = M.features(), oracle.features(A)
    for k in FEAT_KEYS:
        assert f[k] == f_ref[k], k


def _shift_rows_case(kind, n, changes):
    """A stencil with edits that break the one-column shift between consecutive
    rows (K1's shifted-row path, rows of >= 8 entries): ("last", r) moves row
    r's last column right, ("mid", r) its middle column, ("first", r) its first
    column left — each where the row stays strictly increasing and in range."""
    A = synth.stencil(kind, n)
    rp = np.asarray(A.rowptr, np.int64)
    ci = A.colidx.copy()
    for how, r in changes:
        a, b = int(rp[r]), int(rp[r + 1])
        if how == "last" and ci[b - 1] + 1 < A.cols:
            ci[b - 1] += 1
        elif how == "first" and ci[a] > 0:
            ci[a] -= 1
        else:  # "mid" (or a blocked edge): the first middle entry with a gap after it
            for e in range(a + 1, b - 1):
                if ci[e] + 1 < ci[e + 1]:
                    ci[e] += 1
                    break
    return Csr(A.rows, A.cols, rp, ci, A.vals, A.fp64)


@pytest.mark.parametrize("kind,n,changes", [
    ("3d27", 16, []),
    ("3d27", 16, [("mid", 1000)]),                                 # one middle entry of an interior row
    ("3d27", 16, [("last", 1024)]),                                # lane 0 of a block
    ("3d27", 16, [("first", 1055)]),                               # lane 31
    ("3d27", 16, [("mid", 1030), ("mid", 1033)]),                 # a few unshifted rows: shifted path
    ("3d27", 16, [("mid", r) for r in range(1030, 1040)]),         # many: the warp walks lane per row
    ("3d27", 16, [("mid", r) for r in range(1030, 1062, 2)] + [("last", 4095)]),
    ("3d27", (40, 12, 6), [("mid", 2000), ("first", 2001)]),       # x-lines longer than a block
    ("2d9", 48, [("mid", 900), ("last", 901)]),
])
def test_features_shifted_rows(cuda, kind, n, changes):
    """K1's shifted-row path (a row equal to its predecessor plus one column is
    not walked): every edit that breaks the shift brings its own diagonals,
    counted bit-exactly against the oracle."""
    if kind not in synth.STENCIL_KINDS:
        pytest.skip(kind)
    B = _shift_rows_case(kind, n, changes)
    assert oracle.is_canonical(B)
    f_ref = oracle.features(B)
    for rp32 in (True, False):
        M, _ = handle(B, cuda, rowptr32=rp32)
        f = M.features()
        for k in FEAT_KEYS:
            assert f[k] == f_ref[k], (k, rp32, f[k], f_ref[k])


@pytest.mark.parametrize("last_ok", [True, False])
def test_features_shifted_rows_column_range(cuda, last_ok):
    """Rows [i, i + 9) of a matrix with M columns: every row is a shift of the
    previous one, so the only check a shifted row adds is its last column < M —
    one past it is rejected (NITRO_E_BAD_MATRIX), exactly at M - 1 is accepted."""
    n = nitro()
    N, L = 256, 9
    M = N + L - 1 if last_ok else N + L - 2
    rp = np.arange(N + 1, dtype=np.int64) * L
    ci = (np.arange(N)[:, None] + np.arange(L)[None, :]).astype(np.int32).ravel()
    B = Csr(N, M, rp, ci, np.ones(N * L, np.float32), False)
    assert oracle.is_canonical(B) == last_ok
    Md, _ = handle(B, cuda)
    if last_ok:
        f, f_ref = Md.features(), oracle.features(B)
        for k in FEAT_KEYS:
            assert f[k] == f_ref[k], k
    else:
        with pytest.raises(n.NitroError) as e:
            Md.features()
        assert e.value.code == 2


@pytest.mark.parametrize("rows", [[1000], [1024], [1055], [1023, 1024], [2000, 2001, 2002], [64 * 64 - 1]])
def test_features_single_row_pattern_change(cuda, rows):
    """The feature pass skips rows whose offset pattern equals the previous
    row's: a single interior row of a 2D 5-pt stencil whose last column moves
    one to the right (lane 0 / lane 31 of a 32-row block, runs of changed rows,
    the last row) brings one new diagonal, which must be counted."""
    n = nitro()
    A = synth.stencil("2d5", 64)
    rp = np.asarray(A.rowptr, np.int64)
    ci = A.colidx.copy()
    for r in rows:
        e = rp[r + 1] - 1
        if r + 1 < A.rows and ci[e] + 1 < A.cols:
            ci[e] += 1
        else:                       # last row: move its first column left instead
            ci[rp[r]] -= 1
    B = Csr(A.rows, A.cols, rp, ci, A.vals, A.fp64)
    assert oracle.is_canonical(B)
    f_ref = oracle.features(B)
    assert f_ref["ndiag"] > 5
    M, _ = handle(B, cuda)
    f = M.features()
    assert f["ndiag"] == f_ref["ndiag"] and f["dia_fill"] == f_ref["dia_fill"]


@pytest.mark.parametrize("where", ["long_chunk_boundary", "long_dup", "medium", "short_var", "short_equal"])
def test_non_canonical_in_every_walk(cuda, where):
    """A broken row is caught whichever walk of the feature pass visits it."""
    n = nitro()
    A = mixed_matrix()
    ci = A.colidx.copy()
    rp = A.rowptr
    row = {"long_chunk_boundary": 700, "long_dup": 2500, "medium": None, "short_var": None, "short_equal": 100}[where]
    if where == "medium":
        row = int(np.nonzero(np.diff(rp) > 64)[0][3])
    if where == "short_var":
        row = int(np.nonzero((np.diff(rp) >= 3) & (np.arange(A.rows) > 500) & (np.diff(rp) < 10))[0][0])
    a = int(rp[row])
    k = {"long_chunk_boundary": 4095, "long_dup": 8192, "short_equal": 1}.get(where, 1)
    if where == "long_dup":
        ci[a + k] = ci[a + k - 1]
    else:
        ci[a + k - 1], ci[a + k] = ci[a + k], ci[a + k - 1]
    B = Csr(A.rows, A.cols, rp, ci, A.vals, A.fp64)
    assert not oracle.is_canonical(B)
    M, _ = handle(B, cuda)
    with pytest.raises(n.NitroError) as e:
        M.features()
    assert e.value.code == 2


@pytest.mark.parametrize("case", ["unsorted", "dup", "oob", "rowptr"])
def test_non_canonical_rejected(cuda, case):
    n = nitro()
    rp = np.array([0, 2, 4, 6], np.int64)
    ci = {"unsorted": [1, 0, 0, 1, 0, 2], "dup": [0, 0, 0, 1, 0, 2], "oob": [0, 1, 0, 3, 0, 2],
          "rowptr": [0, 1, 0, 1, 0, 2]}[case]
    if case == "rowptr":
        rp = np.array([0, 3, 2, 6], np.int64)
    A = Csr(3, 3, rp, np.array(ci, np.int32), np.ones(6, np.float32), False)
    assert not oracle.is_canonical(A)
    M, _ = handle(A, cuda)
    with pytest.raises(n.NitroError) as e:
        M.features()
    assert e.value.code == 2
    with pytest.raises(n.NitroError):
        M.run(n.CSR_VECTOR, __import__("torch").zeros(3, device=cuda))


# ------------------------------------------------------------------ conversions
def _mats_for_conv():
    for name, A in small_mats():
        yield name, A
    yield "long_row", long_row_matrix(L=20_000, N=3000)


@pytest.mark.parametrize("name,A", list(_mats_for_conv()))
def test_conversions_bit_exact(cuda, name, A):
    n = nitro()
    M, _ = handle(A, cuda)
    mask = M.allowed_mask()
    f = oracle.features(A)
    ld = oracle.round_up(A.rows)
    big = 1e18
    M.set_budget(big)
    assert M.allowed_mask() == oracle.allowed_mask(f, ld, 8 if A.fp64 else 4, big)
    mask = M.allowed_mask()
    if mask[n.ELL]:
        K, ld_o, ecol, ev = oracle.csr_to_ell(A)
        info = M.format_info(n.ELL)
        assert (info["width"], info["ld"]) == (K, ld_o)
        assert np.array_equal(M.export(n.PART_ELL_COL), ecol)
        assert np.array_equal(M.export(n.PART_ELL_VAL).astype(np.float64), ev)
    if mask[n.DIA] and A.nnz > 0:
        offs, ld_o, dv = oracle.csr_to_dia(A)
        info = M.format_info(n.DIA)
        assert (info["width"], info["ld"]) == (len(offs), ld_o)
        assert np.array_equal(M.export(n.PART_DIA_OFF), offs)
        assert np.array_equal(M.export(n.PART_DIA_VAL).astype(np.float64), dv)
    K, ld_o, ecol, ev, tr, tc, tv = oracle.csr_to_hyb(A)
    info = M.format_info(n.HYB)
    assert (info["width"], info["ld"], info["tail"]) == (K, ld_o, len(tr))
    assert np.array_equal(M.export(n.PART_HYB_COL), ecol)
    assert np.array_equal(M.export(n.PART_HYB_VAL).astype(np.float64), ev)
    assert np.array_equal(M.export(n.PART_HYB_TROW), tr)
    assert np.array_equal(M.export(n.PART_HYB_TCOL), tc)
    assert np.array_equal(M.export(n.PART_HYB_TVAL).astype(np.float64), tv)


# ------------------------------------------------------------------ SpMV
def _run_all(A, x, cuda, rowptr32=None, budget=1e18):
    import torch
    n = nitro()
    M, _ = handle(A, cuda, rowptr32=rowptr32)
    M.set_budget(budget)
    xd = torch.from_numpy(x).to(cuda)
    out = {}
    for v in range(n.NUM_VARIANTS):
        if not M.allowed(v):
            continue
        y = torch.full((A.rows,), float("nan"), dtype=xd.dtype, device=cuda)  # overwrite semantics
        M.run(v, xd, y)
        y2 = M.run(v, xd)  # repeat: no state carried between multiplies
        torch.cuda.synchronize()
        out[v] = (y.cpu().numpy(), y2.cpu().numpy())
    return out


@pytest.mark.parametrize("name,A", list(small_mats()))
def test_spmv_all_variants_tolerance(cuda, name, A):
    x = synth.vector(A.cols, seed=31, mode=0, fp64=A.fp64)
    y_ref, r = oracle.spmv(A, x)
    res = _run_all(A, x, cuda)
    assert 0 in res and 1 in res and 4 in res
    for v, (y, y2) in res.items():
        check_y(y, y_ref, r, A.fp64, f"{name} v{v}")
        assert np.array_equal(y, y2), (name, v)   # deterministic


@pytest.mark.parametrize("kind,n", [("2d5", 64), ("2d5", 100), ("3d27", 24), ("3d7", 30), ("1d3", 5000), ("2d9", 40)])
def test_spmv_integer_stencil_exact(cuda, kind, n):
    """Integer Poisson stencil x integer x: exact in fp32 for every variant."""
    A = synth.stencil(kind, n)
    x = synth.vector(A.cols, seed=1, mode=1)
    y_ref, _ = oracle.spmv(A, x)
    res = _run_all(A, x, cuda)
    assert len(res) == 5
    for v, (y, _) in res.items():
        assert np.array_equal(y.astype(np.float64), y_ref), v


@pytest.mark.parametrize("fp64", [False, True])
def test_spmv_long_row(cuda, fp64):
    A = long_row_matrix(fp64=fp64)
    x = synth.vector(A.cols, seed=7, fp64=fp64)
    y_ref, r = oracle.spmv(A, x)
    for rp32 in (True, False):
        for v, (y, y2) in _run_all(A, x, cuda, rowptr32=rp32).items():
            check_y(y, y_ref, r, fp64, f"rp32={rp32} v{v}")
            assert np.array_equal(y, y2)


def _csr_impls(A, x, cuda, rowptr32=None, shift=(0, 0, 0)):
    """y of both CSR variants under every kernel implementation.  shift =
    (rowptr, colidx, vals) element offsets of the arrays inside larger device
    buffers, so the staged kernel's 16-byte chunk rounding sees misaligned spans."""
    import torch
    n = nitro()
    Ad = synth.to_device(A, cuda, rowptr32=rowptr32)

    def shifted(t, k):
        if k == 0:
            return t
        buf = torch.zeros(t.numel() + k, dtype=t.dtype, device=cuda)
        buf[k:] = t
        return buf[k:]
    rp, ci, vv = (shifted(t, k) for t, k in zip((Ad.rowptr, Ad.colidx, Ad.vals), shift))
    M = n.SpMV(rp, ci, vv, A.rows, A.cols)
    xd = torch.from_numpy(x).to(cuda)
    out = {}
    for v in (n.CSR_SCALAR, n.CSR_VECTOR):
        for impl in (n.CSR_IMPL_AUTO, n.CSR_IMPL_DIRECT, n.CSR_IMPL_STAGED, n.CSR_IMPL_STREAM, n.CSR_IMPL_VEC4):
            M.set_csr_impl(impl)
            y = torch.full((A.rows,), float("nan"), dtype=xd.dtype, device=cuda)
            M.run(v, xd, y)
            y2 = M.run(v, xd)
            torch.cuda.synchronize()
            out[(v, impl)] = y.cpu().numpy()
            assert np.array_equal(out[(v, impl)], y2.cpu().numpy()), (v, impl)   # deterministic
            if v == n.CSR_VECTOR:   # which row-mode kernel ran (format_info ld: 1 = K6v)
                info = M.format_info(v)
                out[("vec", impl)] = info["width"] > 0 and info["ld"] == 1
    M.close()
    return out


def _impl_mats():
    yield from small_mats()
    yield "long_row_fp32", long_row_matrix()
    yield "long_row_fp64", long_row_matrix(fp64=True, seed=22)
    yield "banded_b33_d01", synth.banded(40_000, 33, 0.1, seed=23)   # CSR-scalar's class in configs[3]
    yield "uniform_var_k3", synth.uniform(50_001, 3, variable=True, seed=24)
    yield "3d27_n40_fp64", synth.stencil("3d27", 40, mode=1, seed=25, fp64=True)
    yield "banded_b40_dense", synth.banded(30_001, 40, 1.0, seed=27)        # consecutive-column runs (K6v x runs)
    yield "banded_b40_dense_fp64", synth.banded(20_003, 40, 1.0, seed=28, fp64=True)
    yield "uniform_k32_outlier_row", outlier_row_matrix()      # AUTO: K6 (longest row beyond the K6v bound)


@pytest.mark.parametrize("name,A", list(_impl_mats()))
def test_csr_impls_bit_identical(cuda, name, A):
    """The TMA row-tile pipeline (auto / forced, incl. tiles computed from
    global memory when their span overflows a stage) and the direct kernels run
    the same per-row arithmetic: y bit-identical, and within the oracle bound.
    The nnz-split stream mode of CSR-vector (K6s; AUTO picks it when the
    row-length SD exceeds the mean) and the vector-load mode (K6v) sum in other
    associations: within the bound, deterministic, and AUTO equals the one it
    picks exactly."""
    n = nitro()
    x = synth.vector(A.cols, seed=41, mode=0, fp64=A.fp64)
    y_ref, r = oracle.spmv(A, x)
    skewed = oracle.features(A)["sd"] > oracle.features(A)["mean"]
    for rp32 in ((True, False) if A.nnz < 2**31 else (False,)):
        out = _csr_impls(A, x, cuda, rowptr32=rp32)
        assert out[("vec", n.CSR_IMPL_VEC4)], name   # arrays from torch: 16-byte aligned
        assert not out[("vec", n.CSR_IMPL_DIRECT)]
        if name == "uniform_k32_outlier_row":
            assert not skewed and not out[("vec", n.CSR_IMPL_AUTO)]   # the K6v row bound sends AUTO to K6
        if name.startswith("banded_b40_dense"):
            assert out[("vec", n.CSR_IMPL_AUTO)]                      # regular rows: AUTO picks K6v
        for (v, impl), y in out.items():
            if v == "vec":
                continue
            check_y(y, y_ref, r, A.fp64, f"{name} v{v} impl{impl} rp32={rp32}")
            auto = impl == n.CSR_IMPL_AUTO
            stream = v == n.CSR_VECTOR and (impl == n.CSR_IMPL_STREAM or (auto and skewed))
            vec = v == n.CSR_VECTOR and not stream and (impl == n.CSR_IMPL_VEC4 or (auto and out[("vec", impl)]))
            want = out[(v, n.CSR_IMPL_STREAM)] if stream else out[(v, n.CSR_IMPL_VEC4)] if vec \
                else out[(v, n.CSR_IMPL_DIRECT)]
            assert np.array_equal(y, want), (name, v, impl, rp32)


@pytest.mark.parametrize("shift", [(1, 1, 1), (3, 2, 1), (2, 3, 3)])
def test_csr_staged_misaligned_spans(cuda, shift):
    A = synth.banded(30_011, 6, 0.7, seed=26)
    x = synth.vector(A.cols, seed=42)
    y_ref, r = oracle.spmv(A, x)
    out = _csr_impls(A, x, cuda, rowptr32=True, shift=shift)
    n = nitro()
    assert not out[("vec", n.CSR_IMPL_VEC4)]   # misaligned col / val: K6v falls back to K6
    for (v, impl), y in out.items():
        if v == "vec":
            continue
        check_y(y, y_ref, r, False, f"shift {shift} v{v} impl{impl}")
        if not (v == n.CSR_VECTOR and impl == n.CSR_IMPL_STREAM):   # misaligned arrays: the scalar-load path of K6s
            assert np.array_equal(y, out[(v, 1)]), (shift, v, impl)


def test_run_host_matches_device(cuda):
    n = nitro()
    A = synth.uniform(10000, 7, variable=True, seed=3)
    x = synth.vector(A.cols, seed=4)
    y_ref, r = oracle.spmv(A, x)
    M, _ = handle(A, cuda)
    for v in range(5):
        if M.allowed(v):
            check_y(M.run_host(v, x), y_ref, r, False, f"v{v}")


@pytest.mark.parametrize("kind", ["3d27_n64", "banded_300k", "uniform_300k_rect"])
def test_run_host_pipelined_bit_identical(cuda, kind):
    """>= 2^17 rows: CSR-scalar / ELL / DIA host-buffer calls run as 4 row chunks
    (x in column pieces, y out per chunk on separate streams); every row must be
    bit-identical to the single-launch device multiply (same kernels, same
    per-row order) and within tolerance of the oracle."""
    import torch
    n = nitro()
    A = {"3d27_n64": lambda: synth.stencil("3d27", 64, mode=1, seed=41),
         "banded_300k": lambda: synth.banded(300_001, 9, 0.5, seed=42),
         "uniform_300k_rect": lambda: synth.uniform(300_007, 5, variable=True, seed=43, M=310_000)}[kind]()
    x = synth.vector(A.cols, seed=44)
    y_ref, r = oracle.spmv(A, x)
    M, _ = handle(A, cuda)
    xd = torch.from_numpy(x).to(cuda)
    for v in (n.CSR_SCALAR, n.ELL, n.DIA):
        if not M.allowed(v):
            continue
        yd = torch.empty(A.rows, dtype=xd.dtype, device=cuda)
        M.run(v, xd, yd)
        torch.cuda.synchronize()
        for rep in range(2):     # the second call reuses streams, events and column bounds
            yh = M.run_host(v, x)
            assert np.array_equal(yh, yd.cpu().numpy()), (kind, v, rep)
        check_y(yh, y_ref, r, False, f"{kind} v{v}")


def test_constraint_blocks_explicit_run(cuda):
    import torch
    n = nitro()
    A = synth.rmat(12, 16, seed=2, fp64=False)
    M, _ = handle(A, cuda)
    assert not M.allowed(n.ELL) and not M.allowed(n.DIA)
    with pytest.raises(n.NitroError) as e:
        M.run(n.DIA, torch.zeros(A.cols, device=cuda))
    assert e.value.code == 4
    M2, _ = handle(synth.stencil("3d27", 10), cuda)
    M2.set_budget(100.0)
    assert not M2.allowed(n.DIA) and not M2.allowed(n.ELL)


def test_timing_and_launch_counts(cuda):
    import torch
    n = nitro()
    A = synth.stencil("3d27", 32, mode=1)
    M, Ad = handle(A, cuda)
    x = synth.vector(A.cols, seed=1, device=cuda)
    y = torch.empty(A.rows, device=cuda)
    for v in range(5):
        med, allt = M.time(v, x, y, warmup=1, reps=5, flush_l2=True)
        assert 0 < med < 0.1 and len(allt) == 5
        assert M.launches(v) == (3 if v == n.HYB and M.format_info(v)["tail"] > 0 else 1)


# ------------------------------------------------------------------ full-size configs (BASELINE configs[1], [2])
def test_c1_3d27_n128_full(cuda):
    """configs[1]: 2,097,152 rows, 55,742,968 nnz, fp32; every variant vs oracle."""
    A = synth.stencil("3d27", 128, mode=1, seed=1)
    x = synth.vector(A.cols, seed=2)
    y_ref, r = oracle.spmv(A, x)
    M, Ad = handle(A, cuda)
    f, f_ref = M.features(), oracle.features(A)
    for k in FEAT_KEYS:
        assert f[k] == f_ref[k], k
    import torch
    xd = torch.from_numpy(x).to(cuda)
    for v in range(5):
        y = M.run(v, xd)
        torch.cuda.synchronize()
        check_y(y.cpu().numpy(), y_ref, r, False, f"v{v}")
        M.release(v)


def test_c2a_uniform_full(cuda):
    """configs[2] uniform: 8,388,608 rows x 32 nnz/row fp32 (ELL-favourable); DIA ruled out."""
    import torch
    n = nitro()
    A = synth.uniform(1 << 23, 32, seed=5)
    x = synth.vector(A.cols, seed=6)
    y_ref, r = oracle.spmv(A, x)
    M, _ = handle(A, cuda)
    assert not M.allowed(n.DIA) and M.allowed(n.ELL)
    xd = torch.from_numpy(x).to(cuda)
    for v in (n.CSR_VECTOR, n.ELL, n.HYB):
        y = M.run(v, xd)
        torch.cuda.synchronize()
        check_y(y.cpu().numpy(), y_ref, r, False, f"v{v}")
        M.release(v)


def test_c2b_rmat_full(cuda):
    """configs[2] power law: R-MAT scale 23, edge factor 16, fp64; ELL/DIA ruled out."""
    import torch
    n = nitro()
    A = synth.rmat(23, 16, seed=7, fp64=True)
    x = synth.vector(A.cols, seed=8, fp64=True)
    y_ref, r = oracle.spmv(A, x)
    M, _ = handle(A, cuda)
    f, f_ref = M.features(), oracle.features(A)
    for k in FEAT_KEYS:
        assert f[k] == f_ref[k], k
    assert not M.allowed(n.DIA) and not M.allowed(n.ELL)
    xd = torch.from_numpy(x).to(cuda)
    for v in (n.CSR_SCALAR, n.CSR_VECTOR, n.HYB):
        y = M.run(v, xd)
        torch.cuda.synchronize()
        check_y(y.cpu().numpy(), y_ref, r, True, f"v{v}")
        if v == n.CSR_VECTOR:   # AUTO: the stream mode (SD > mean) with hot-x staging (power-law columns)
            fi = M.format_info(v)
            assert fi["width"] == 0 and fi["ld"] > 0, fi
        M.release(v)
    # and the same multiply without the staging (NITRO_CSR_IMPL_STREAM keeps it; row mode for reference)
    M.set_csr_impl(n.CSR_IMPL_DIRECT)
    y = M.run(n.CSR_VECTOR, xd)
    torch.cuda.synchronize()
    check_y(y.cpu().numpy(), y_ref, r, True, "csr_vector row mode")


# ------------------------------------------------------------------ select path on the GPU
def test_register_train_select_call(cuda, tmp_path):
    import torch
    n = nitro()
    mats = [synth.stencil("3d27", 24, mode=1), synth.uniform(60000, 30, seed=1), synth.rmat(14, 8, seed=1, fp64=False),
            synth.stencil("1d3", 100000, mode=1), synth.banded(50000, 3, 1.0, seed=2), synth.uniform(80000, 2, seed=3)]
    ctx = n.Context()
    cv = n.CodeVariant(ctx, "spmv")
    cv.register_spmv()
    assert cv.n_variants() == 5 and cv.n_features() == 7
    keep = []
    for A in mats:
        M, Ad = handle(A, cuda)
        x = synth.vector(A.cols, seed=1, device=cuda)
        y = torch.empty(A.rows, device=cuda)
        rec = n.spmv_input(M, x, y, warmup=1, reps=5)
        keep.append((M, Ad, x, y, rec))
        cv.add_training_input(n.addr(rec))
    cv.train(folds=3, log2c_lo=-1, log2c_hi=5, log2g_lo=-3, log2g_hi=1)
    cost, feat, lab = cv.training_table()
    # exhaustive best == argmin of the recorded table (oracle C10), constraints -> inf
    from oracle import select as S
    assert list(lab) == S.exhaustive_best(cost.tolist())
    for (M, *_), row in zip(keep, cost):
        for v in range(5):
            assert np.isfinite(row[v]) == M.allowed(v)
    # features in the table equal the oracle's
    for A, frow in zip(mats, feat):
        fo = oracle.features(A)
        assert list(frow) == [fo[k] for k in S.FEATURE_NAMES]
    p = tmp_path / "m.txt"
    cv.save(p)
    cv2 = n.CodeVariant(ctx, "spmv2")
    cv2.register_spmv()
    cv2.load(p)
    for (M, Ad, x, y, rec) in keep:
        v1, _ = cv.select(n.addr(rec))
        v2, _ = cv2.select(n.addr(rec))
        assert v1 == v2 and M.allowed(v1)
        v3, c3 = cv.call(n.addr(rec))
        assert v3 == v1 and c3 > 0


def test_features_async_then_select(cuda):
    """fix_inputs analogue: the feature pass is enqueued early,
    other GPU work overlaps it, the later features()/select waits for it."""
    import torch
    n = nitro()
    A = synth.stencil("3d27", 40, mode=1, seed=4)
    M, _ = handle(A, cuda)
    M.features_async()
    z = torch.randn(1 << 22, device=cuda).sum()       # unrelated work while K1 runs
    f = M.features()
    f_ref = oracle.features(A)
    for k in FEAT_KEYS:
        assert f[k] == f_ref[k], k
    assert torch.isfinite(z)


_PF_CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import synth, paper_conf_ipps_muralidharanshgc14_b200 as n
dev = torch.device("cuda:0")
out = {}
for name, A in (("3d27", synth.stencil("3d27", 40, mode=1, seed=31)),
                ("band", synth.banded(70_001, 12, 0.6, seed=32)),
                ("3d7_fp64", synth.stencil("3d7", 33, mode=1, seed=33, fp64=True))):
    M = n.SpMV.from_csr(synth.to_device(A, dev))
    M.features()
    x = torch.from_numpy(synth.vector(A.cols, seed=34, fp64=A.fp64)).to(dev)
    for v in (n.ELL, n.DIA, n.HYB):
        if M.allowed(v):
            y = M.run(v, x)
            torch.cuda.synchronize()
            out[f"{name}_{v}"] = y.cpu().numpy()
    M.close()
np.savez(sys.argv[2], **out)
"""


def test_l2_prefetch_is_result_neutral(cuda, tmp_path):
    """The cp.async.bulk L2 prefetches of the DIA / ELL streams are
    pure performance hints: y with them off (NITRO_DIA_PF=0, NITRO_ELL_PF=0) is
    bit-identical to y with the defaults (on)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    script = tmp_path / "pf_child.py"
    script.write_text(_PF_CHILD)
    res = {}
    for tag, env in (("on", {}), ("off", {"NITRO_DIA_PF": "0", "NITRO_ELL_PF": "0"})):
        out = tmp_path / f"{tag}.npz"
        r = subprocess.run([sys.executable, str(script), root, str(out)], env={**os.environ, **env},
                           capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-2000:]
        res[tag] = dict(np.load(out))
    assert res["on"].keys() == res["off"].keys() and len(res["on"]) >= 6
    for k in res["on"]:
        assert np.array_equal(res["on"][k], res["off"][k]), k


# ------------------------------------------------------------------ round-2 robustness cases
def test_dia_more_diagonals_than_shared_offsets(cuda):
    """D > 12288 (the offsets kept in shared memory): a dense 32 x 14000 block
    has 14031 diagonals at fill 1.0, so DIA is allowed and must run correctly
    (offsets past the shared window are read through L1)."""
    n = nitro()
    import torch
    N, M = 32, 14000
    rp = np.arange(N + 1, dtype=np.int64) * M
    ci = np.tile(np.arange(M, dtype=np.int32), N)
    rng = np.random.default_rng(5)
    va = (rng.integers(1, 9, N * M) * rng.choice([-1, 1], N * M)).astype(np.float32)
    A = Csr(N, M, rp, ci, va, False)
    f = oracle.features(A)
    assert f["ndiag"] == N + M - 1 and f["dia_fill"] <= 3.0
    M_, _ = handle(A, cuda)
    assert M_.allowed(n.DIA)
    x = synth.vector(M, seed=1, mode=1)
    y_ref, _ = oracle.spmv(A, x)
    y = M_.run(n.DIA, torch.from_numpy(x).to(cuda))
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().astype(np.float64), y_ref)   # integer data: exact


def test_malformed_rowptr_with_long_rows_is_rejected(cuda):
    """Overlapping rows that each lie inside [0, Z] (rowptr not monotone) and
    are long enough for the long-row task list must give NITRO_E_BAD_MATRIX,
    not a write past the task list."""
    n = nitro()
    Z, N = 20000, 96
    rp = np.zeros(N + 1, np.int64)
    rp[1:32] = Z          # block 0: row 0 has Z entries, the rest are empty
    rp[32] = Z
    rp[33:64] = 0         # block 1: row 32 goes Z -> 0 (negative; flagged)
    rp[64] = 0
    rp[65:N] = Z          # block 2: row 64 again has Z entries
    rp[N] = Z
    ci = np.arange(Z, dtype=np.int32)
    A = Csr(N, Z, rp, ci, np.ones(Z, np.float32), False)
    M, _ = handle(A, cuda)
    with pytest.raises(n.NitroError) as e:
        M.features()
    assert e.value.code == 2
    import torch
    torch.cuda.synchronize()            # no sticky CUDA error left behind
    assert torch.ones(4, device=cuda).sum().item() == 4


def test_binding_rejects_bad_vectors(cuda):
    """The Python binding checks dtype / contiguity / length / device before
    passing a pointer to the C ABI."""
    n = nitro()
    import torch
    A = synth.stencil("2d5", 16)
    M, _ = handle(A, cuda)
    good = torch.zeros(A.cols, dtype=torch.float32, device=cuda)
    for bad in (torch.zeros(A.cols, dtype=torch.float64, device=cuda),
                torch.zeros(2 * A.cols, dtype=torch.float32, device=cuda)[::2],
                torch.zeros(A.cols - 1, dtype=torch.float32, device=cuda),
                torch.zeros(A.cols, dtype=torch.float32)):
        with pytest.raises(ValueError):
            M.run(n.CSR_SCALAR, bad)
        with pytest.raises(ValueError):
            M.run(n.CSR_SCALAR, good, bad[: A.rows] if bad.numel() >= A.rows else bad)
    M.run(n.CSR_SCALAR, good)


def _stream_mats():
    yield "rmat14_fp32", synth.rmat(14, 16, seed=31, fp64=False)
    yield "rmat13_fp64", synth.rmat(13, 8, seed=32, fp64=True)
    yield "long_row", long_row_matrix(L=60_000, N=4000)
    yield "empty_runs", Csr(300, 300, np.array([0] * 100 + [1] * 150 + [40] * 51, np.int64),
                            np.concatenate([[5], np.arange(39)]).astype(np.int32),
                            np.linspace(1, 2, 40).astype(np.float32), False)
    yield "uniform_k1", synth.uniform(5000, 1, seed=33)          # chunks spanning many rows (windows)
    yield "2d5_int", synth.stencil("2d5", 70)


@pytest.mark.parametrize("name,A", list(_stream_mats()))
def test_csr_stream_mode(cuda, name, A):
    """K6s (nnz-split chunks, rows from rowptr by warp binary search, carry
    fixup that stores): within the bound on skewed, long-row, empty-run and
    one-entry-per-row matrices; exact on integer data; empty rows written 0
    (y starts as NaN); deterministic across runs."""
    import torch
    n = nitro()
    exact = name.endswith("_int")
    x = synth.vector(A.cols, seed=7, mode=1 if exact else 0, fp64=A.fp64)
    y_ref, r = oracle.spmv(A, x)
    M, _ = handle(A, cuda)
    M.set_csr_impl(n.CSR_IMPL_STREAM)
    xd = torch.from_numpy(x).to(cuda)
    ys = []
    for _ in range(2):
        y = torch.full((A.rows,), float("nan"), dtype=xd.dtype, device=cuda)
        M.run(n.CSR_VECTOR, xd, y)
        torch.cuda.synchronize()
        ys.append(y.cpu().numpy())
    assert M.format_info(n.CSR_VECTOR)["width"] == 0          # stream mode active
    assert np.all(np.isfinite(ys[0]))                          # every row written (empty rows = 0)
    if exact:
        assert np.array_equal(ys[0].astype(np.float64), y_ref)
    else:
        check_y(ys[0], y_ref, r, A.fp64, name)
    assert np.array_equal(ys[0], ys[1])
