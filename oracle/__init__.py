"""oracle — plain CPU reference of the Nitro SpMV hot path (fp64).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this package.  The product
package (paper_conf_ipps_muralidharanshgc14_b200) never imports it; the two
share no code (only the seeded input generators in synth/, which hold no
arithmetic of the method).

Parts (PAPER.md line cites, readings in SURVEY.md §8(c) / DESIGN.md):
  spmv           C1  P:L38-43 (COO loop, y <- A.x)
  features       C4
  csr_to_ell     C5  P:L200, P:L210          (+ ell_to_csr round trip)
  csr_to_dia     C6  P:L87, P:L126           (+ dia_to_csr round trip)
  csr_to_hyb     C7  not in paper (north star; CUSP family P:L47)
  dia_allowed /
  ell_allowed    C9
  select.*       C10-C13
  hist.*         §8(f) f4 histogram family: counts + features (DESIGN R17)
Parity status of each part is listed in DESIGN.md; the held-out "Nitro %"
value (C13) is parity-unpinned (no reference GPU timings exist).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")


def build(force: bool = False) -> str:
    if not force and os.path.exists(_SO) and os.path.getmtime(_SO) >= os.path.getmtime(_SRC):
        return _SO
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-shared",
                           "-fPIC", "-o", _SO, _SRC, "-lm"], cwd=_HERE)
    return _SO


class Features(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_int64), ("cols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("sum_len", ctypes.c_uint64), ("sum_len2", ctypes.c_uint64),
                ("max_row", ctypes.c_int64), ("ndiag", ctypes.c_int64),
                ("canonical", ctypes.c_int32), ("pad_", ctypes.c_int32),
                ("mean", ctypes.c_double), ("sd", ctypes.c_double), ("max_dev", ctypes.c_double),
                ("dia_fill", ctypes.c_double), ("ell_fill", ctypes.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_ if k != "pad_"}


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        vp, i64 = ctypes.c_void_p, ctypes.c_int64
        L.oracle_spmv.argtypes = [i64, vp, vp, vp, vp, vp, vp]
        L.oracle_spmv.restype = None
        L.oracle_spmv_threads.argtypes = [i64, vp, vp, vp, vp, vp, vp, ctypes.c_int]
        L.oracle_spmv_threads.restype = ctypes.c_int
        L.oracle_features.argtypes = [i64, i64, vp, vp, ctypes.POINTER(Features), vp]
        L.oracle_is_canonical.argtypes = [i64, i64, i64, vp, vp]
        L.oracle_finish_features.argtypes = [i64, i64, i64, ctypes.c_uint64, ctypes.c_uint64, i64, i64,
                                             ctypes.POINTER(Features)]
        L.oracle_finish_features.restype = None
        L.oracle_csr_to_ell.argtypes = [i64, vp, vp, vp, i64, i64, vp, vp]
        L.oracle_ell_to_csr.argtypes = [i64, i64, i64, vp, vp, vp, vp, vp]
        L.oracle_ell_to_csr.restype = i64
        L.oracle_csr_to_dia.argtypes = [i64, i64, vp, vp, vp, i64, vp, i64, vp]
        L.oracle_dia_to_csr.argtypes = [i64, i64, i64, vp, i64, vp, vp, vp, vp]
        L.oracle_dia_to_csr.restype = i64
        L.oracle_hyb_width.argtypes = [i64, vp]
        L.oracle_hyb_width.restype = i64
        L.oracle_hyb_tail_len.argtypes = [i64, vp, i64]
        L.oracle_hyb_tail_len.restype = i64
        L.oracle_csr_to_hyb.argtypes = [i64, vp, vp, vp, i64, i64, vp, vp, vp, vp, vp]
        L.oracle_hyb_to_csr.argtypes = [i64, i64, i64, vp, vp, i64, vp, vp, vp, vp, vp, vp]
        L.oracle_hyb_to_csr.restype = i64
        L.oracle_dia_allowed.argtypes = [ctypes.POINTER(Features), i64, i64, ctypes.c_double]
        L.oracle_ell_allowed.argtypes = [ctypes.POINTER(Features), i64, i64, ctypes.c_double]
        assert L.oracle_features_size() == ctypes.sizeof(Features)
        _lib = L
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data


def _csr(A):
    """(N, M, rowptr int64, colidx int32, vals fp64) contiguous host arrays."""
    rp = np.ascontiguousarray(np.asarray(A.rowptr), dtype=np.int64)
    ci = np.ascontiguousarray(np.asarray(A.colidx), dtype=np.int32)
    v = np.ascontiguousarray(np.asarray(A.vals), dtype=np.float64)   # exact widening of fp32
    return A.rows, A.cols, rp, ci, v


def round_up(n: int, m: int = 32) -> int:
    return ((n + m - 1) // m) * m


def spmv(A, x):
    """C1: y = A.x in fp64, sequential per row; also r_i = sum_k |a_ik x_k|."""
    N, M, rp, ci, v = _csr(A)
    xd = np.ascontiguousarray(np.asarray(x), dtype=np.float64)
    assert xd.shape[0] >= M
    y = np.empty(N, dtype=np.float64)
    r = np.empty(N, dtype=np.float64)
    lib().oracle_spmv(N, _p(rp), _p(ci), _p(v), _p(xd), _p(y), _p(r))
    return y, r


def spmv_threads(A, x, nthreads: int | None = None):
    """C1 with the rows split over host threads (bit-identical to spmv);
    returns (y, r, threads used).  bench.py's all-core CPU baseline only."""
    N, M, rp, ci, v = _csr(A)
    xd = np.ascontiguousarray(np.asarray(x), dtype=np.float64)
    assert xd.shape[0] >= M
    y = np.empty(N, dtype=np.float64)
    r = np.empty(N, dtype=np.float64)
    used = lib().oracle_spmv_threads(N, _p(rp), _p(ci), _p(v), _p(xd), _p(y), _p(r),
                                     int(nthreads or os.cpu_count() or 1))
    return y, r, used


def spmv_prepared(A, x, nthreads: int = 1):
    """C1 loop bound to A and x converted ONCE to the oracle's fp64 / int64
    host layout; returns a no-argument callable that runs oracle_spmv (one
    thread) or oracle_spmv_threads (nthreads > 1) into preallocated y, r.
    bench.py times this callable so the baseline measures the oracle's loop,
    not a per-call dtype conversion of x."""
    N, M, rp, ci, v = _csr(A)
    xd = np.ascontiguousarray(np.asarray(x), dtype=np.float64)
    assert xd.shape[0] >= M
    y = np.empty(N, dtype=np.float64)
    r = np.empty(N, dtype=np.float64)
    L = lib()
    if nthreads <= 1:
        def run():
            L.oracle_spmv(N, _p(rp), _p(ci), _p(v), _p(xd), _p(y), _p(r))
            return 1
    else:
        def run():
            return L.oracle_spmv_threads(N, _p(rp), _p(ci), _p(v), _p(xd), _p(y), _p(r), int(nthreads))
    run.y, run.r = y, r
    return run


def features(A, with_offsets: bool = False):
    """C4 features (dict); optionally also the ascending distinct offsets."""
    N, M, rp, ci, _ = _csr(A)
    f = Features()
    offs = np.empty(max(N + M - 1, 1), dtype=np.int32) if with_offsets else None
    rc = lib().oracle_features(N, M, _p(rp), _p(ci), ctypes.byref(f), _p(offs))
    assert rc == 0
    if with_offsets:
        return f.as_dict(), offs[: f.ndiag].copy()
    return f.as_dict()


def finish_features(N: int, M: int, Z: int, s1: int, s2: int, lmax: int, D: int) -> dict:
    """C4 finishing step alone, from exact integers (e.g. closed forms of a
    matrix too large for the host); 'canonical' is reported as 1."""
    f = Features()
    f.canonical = 1
    lib().oracle_finish_features(N, M, Z, s1, s2, lmax, D, ctypes.byref(f))
    return f.as_dict()


def is_canonical(A) -> bool:
    N, M, rp, ci, _ = _csr(A)
    return bool(lib().oracle_is_canonical(N, M, int(rp[-1]), _p(rp), _p(ci)))


def csr_to_ell(A, K=None, ld=None):
    N, M, rp, ci, v = _csr(A)
    if K is None:
        K = int(np.diff(rp).max()) if N else 0
    ld = round_up(N) if ld is None else ld
    ecol = np.empty(K * ld, dtype=np.int32)
    ev = np.empty(K * ld, dtype=np.float64)
    assert lib().oracle_csr_to_ell(N, _p(rp), _p(ci), _p(v), K, ld, _p(ecol), _p(ev)) == 0
    return K, ld, ecol, ev


def ell_to_csr(N, K, ld, ecol, ev):
    ecol = np.ascontiguousarray(ecol, dtype=np.int32)
    ev = np.ascontiguousarray(ev, dtype=np.float64)
    rp = np.empty(N + 1, dtype=np.int64)
    z = lib().oracle_ell_to_csr(N, K, ld, _p(ecol), _p(ev), _p(rp), None, None)
    ci = np.empty(z, dtype=np.int32)
    v = np.empty(z, dtype=np.float64)
    lib().oracle_ell_to_csr(N, K, ld, _p(ecol), _p(ev), _p(rp), _p(ci), _p(v))
    return rp, ci, v


def csr_to_dia(A, ld=None):
    N, M, rp, ci, v = _csr(A)
    _, offs = features(A, with_offsets=True)
    D = offs.shape[0]
    ld = round_up(N) if ld is None else ld
    dv = np.empty(D * ld, dtype=np.float64)
    assert lib().oracle_csr_to_dia(N, M, _p(rp), _p(ci), _p(v), D, _p(offs), ld, _p(dv)) == 0
    return offs, ld, dv


def dia_to_csr(N, M, offs, ld, dv):
    offs = np.ascontiguousarray(offs, dtype=np.int32)
    dv = np.ascontiguousarray(dv, dtype=np.float64)
    rp = np.empty(N + 1, dtype=np.int64)
    z = lib().oracle_dia_to_csr(N, M, offs.shape[0], _p(offs), ld, _p(dv), _p(rp), None, None)
    ci = np.empty(z, dtype=np.int32)
    v = np.empty(z, dtype=np.float64)
    lib().oracle_dia_to_csr(N, M, offs.shape[0], _p(offs), ld, _p(dv), _p(rp), _p(ci), _p(v))
    return rp, ci, v


def hyb_width(A) -> int:
    N, M, rp, _, _ = _csr(A)
    return int(lib().oracle_hyb_width(N, _p(rp)))


def csr_to_hyb(A, K=None, ld=None):
    N, M, rp, ci, v = _csr(A)
    K = hyb_width(A) if K is None else K
    ld = round_up(N) if ld is None else ld
    Zt = int(lib().oracle_hyb_tail_len(N, _p(rp), K))
    ecol = np.empty(K * ld, dtype=np.int32)
    ev = np.empty(K * ld, dtype=np.float64)
    tr = np.empty(Zt, dtype=np.int32)
    tc = np.empty(Zt, dtype=np.int32)
    tv = np.empty(Zt, dtype=np.float64)
    assert lib().oracle_csr_to_hyb(N, _p(rp), _p(ci), _p(v), K, ld, _p(ecol), _p(ev), _p(tr), _p(tc), _p(tv)) == 0
    return K, ld, ecol, ev, tr, tc, tv


def hyb_to_csr(N, K, ld, ecol, ev, tr, tc, tv):
    args = [np.ascontiguousarray(a, dtype=t) for a, t in
            ((ecol, np.int32), (ev, np.float64), (tr, np.int32), (tc, np.int32), (tv, np.float64))]
    ecol, ev, tr, tc, tv = args
    rp = np.empty(N + 1, dtype=np.int64)
    Zt = tr.shape[0]
    z = lib().oracle_hyb_to_csr(N, K, ld, _p(ecol), _p(ev), Zt, _p(tr), _p(tc), _p(tv), _p(rp), None, None)
    ci = np.empty(z, dtype=np.int32)
    v = np.empty(z, dtype=np.float64)
    lib().oracle_hyb_to_csr(N, K, ld, _p(ecol), _p(ev), Zt, _p(tr), _p(tc), _p(tv), _p(rp), _p(ci), _p(v))
    return rp, ci, v


def _feat_struct(fd: dict) -> Features:
    f = Features()
    for k, _ in Features._fields_:
        if k != "pad_":
            setattr(f, k, fd[k])
    return f


def dia_allowed(fd: dict, ld: int, sv: int, budget_bytes: float) -> bool:
    return bool(lib().oracle_dia_allowed(ctypes.byref(_feat_struct(fd)), ld, sv, budget_bytes))


def ell_allowed(fd: dict, ld: int, sv: int, budget_bytes: float) -> bool:
    return bool(lib().oracle_ell_allowed(ctypes.byref(_feat_struct(fd)), ld, sv, budget_bytes))


def allowed_mask(fd: dict, ld: int, sv: int, budget_bytes: float):
    """[csr_scalar, csr_vector, ell, dia, hyb] allowed flags (C9)."""
    return [True, True, ell_allowed(fd, ld, sv, budget_bytes), dia_allowed(fd, ld, sv, budget_bytes), True]
