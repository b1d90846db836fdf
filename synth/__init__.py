"""synth — seeded synthetic inputs shared by the oracle side and the GPU side.

This module holds NO arithmetic of the method (no SpMV, features or format
conversion).  It decides which (row, col, value) triples a synthetic matrix
holds, and what x holds, from counter-based hashes (gen_core.h), so the host
build (numpy arrays, OpenMP) and the device build (torch CUDA tensors) give
identical inputs.  Matrix classes follow the paper's SpMV workload mix
(§IV: UFL matrices from 9 groups + 13 stencil matrices),
recast as the synthetic recipe of SURVEY.md §8(d) / DESIGN.md "Input recipe".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libsynth.so")
_SRC = [os.path.join(_HERE, "synth.cu"), os.path.join(_HERE, "gen_core.h")]

STENCIL_KINDS = {"1d3": 1, "2d5": 2, "2d9": 3, "3d7": 4, "3d27": 5}


def build(force: bool = False) -> str:
    """Compile libsynth.so in-tree for sm_100a (host part uses OpenMP)."""
    if not force and os.path.exists(_SO) and all(os.path.getmtime(_SO) >= os.path.getmtime(s) for s in _SRC):
        return _SO
    cmd = ["nvcc", "-O3", "-std=c++17", "-shared", "-Xcompiler", "-fPIC,-fopenmp",
           "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
           "-o", _SO, _SRC[0], "-lgomp"]
    subprocess.check_call(cmd, cwd=_HERE)
    return _SO


class SynthParams(ctypes.Structure):
    _fields_ = [("cls", ctypes.c_int32), ("kind", ctypes.c_int32),
                ("nx", ctypes.c_int64), ("ny", ctypes.c_int64), ("nz", ctypes.c_int64),
                ("N", ctypes.c_int64), ("M", ctypes.c_int64),
                ("band", ctypes.c_int32), ("k", ctypes.c_int32),
                ("density", ctypes.c_double), ("variable", ctypes.c_int32),
                ("scale", ctypes.c_int32), ("a", ctypes.c_double), ("b", ctypes.c_double),
                ("c", ctypes.c_double), ("permute", ctypes.c_int32), ("mode", ctypes.c_int32),
                ("seed", ctypes.c_uint64)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        L.synth_lengths.argtypes = [i32, vp, ctypes.POINTER(SynthParams), i64, i64, vp]
        L.synth_fill.argtypes = [i32, vp, ctypes.POINTER(SynthParams), i64, i64, vp, vp, vp, i32]
        L.synth_rmat_keys.argtypes = [i32, vp, ctypes.POINTER(SynthParams), ctypes.c_uint64, ctypes.c_uint64, vp]
        L.synth_values_rc.argtypes = [i32, vp, ctypes.c_uint64, i64, vp, vp, vp, i32]
        L.synth_vector.argtypes = [i32, vp, ctypes.c_uint64, i64, i64, i32, vp, i32]
        for f in ("synth_lengths", "synth_fill", "synth_rmat_keys", "synth_values_rc", "synth_vector", "synth_params_size"):
            getattr(L, f).restype = ctypes.c_int
        assert L.synth_params_size() == ctypes.sizeof(SynthParams), "SynthParams layout mismatch"
        _lib = L
    return _lib


@dataclass
class Csr:
    """A canonical CSR matrix (rowptr int64, colidx int32, vals fp32/fp64).

    Arrays are numpy (host) or torch tensors (device), per ``device``."""
    rows: int
    cols: int
    rowptr: object
    colidx: object
    vals: object
    fp64: bool
    device: str | None = None
    meta: dict = field(default_factory=dict)

    @property
    def nnz(self) -> int:
        return int(self.colidx.shape[0])

    def row(self, i: int):
        """(cols, vals) of row i as numpy arrays (host matrices only)."""
        a, b = int(self.rowptr[i]), int(self.rowptr[i + 1])
        return self.colidx[a:b], self.vals[a:b]


def _ptr(a):
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return a.data_ptr()


def _stream(device):
    if device is None:
        return None
    import torch
    return torch.cuda.current_stream().cuda_stream


def _check(rc, what):
    if rc != 0:
        raise RuntimeError(f"synth: {what} failed with code {rc}")


def _rowwise(p: SynthParams, nrows: int, ncols: int, fp64: bool, device, meta, row0: int = 0) -> Csr:
    L = lib()
    on_dev = 0 if device is None else 1
    s = _stream(device)
    if device is None:
        lens = np.empty(nrows, dtype=np.int32)
        _check(L.synth_lengths(0, None, ctypes.byref(p), row0, nrows, _ptr(lens)), "lengths")
        rowptr = np.zeros(nrows + 1, dtype=np.int64)
        np.cumsum(lens, out=rowptr[1:])
        nnz = int(rowptr[-1])
        col = np.empty(nnz, dtype=np.int32)
        val = np.empty(nnz, dtype=np.float64 if fp64 else np.float32)
    else:
        import torch
        lens = torch.empty(nrows, dtype=torch.int32, device=device)
        _check(L.synth_lengths(on_dev, s, ctypes.byref(p), row0, nrows, _ptr(lens)), "lengths")
        rowptr = torch.zeros(nrows + 1, dtype=torch.int64, device=device)
        torch.cumsum(lens, 0, out=rowptr[1:])
        del lens
        nnz = int(rowptr[-1].item())
        col = torch.empty(nnz, dtype=torch.int32, device=device)
        val = torch.empty(nnz, dtype=torch.float64 if fp64 else torch.float32, device=device)
    _check(L.synth_fill(on_dev, s, ctypes.byref(p), row0, nrows, _ptr(rowptr), _ptr(col), _ptr(val), int(fp64)), "fill")
    return Csr(nrows, ncols, rowptr, col, val, fp64, device, meta)


def stencil(kind: str, n, mode: int = 0, seed: int = 0, fp64: bool = False, device=None,
            row0: int = 0, nrows: int | None = None) -> Csr:
    """Poisson-style stencil on an n^d grid (or explicit (nx, ny, nz)).

    mode 0: centre = npts-1, neighbours = -1 (integers); mode 1: random values.
    row0/nrows select a contiguous row slice (columns stay global)."""
    k = STENCIL_KINDS[kind]
    dim = int(kind[0])
    if isinstance(n, (tuple, list)):
        nx, ny, nz = (list(n) + [1, 1])[:3]
    else:
        nx, ny, nz = (n, n if dim >= 2 else 1, n if dim >= 3 else 1)
    p = SynthParams(cls=1, kind=k, nx=nx, ny=ny, nz=nz, mode=mode, seed=seed)
    N = nx * ny * nz
    if nrows is None:
        nrows = N - row0
    return _rowwise(p, nrows, N, fp64, device,
                    {"class": "stencil", "kind": kind, "grid": (nx, ny, nz), "mode": mode, "seed": seed, "row0": row0},
                    row0=row0)


def banded(N: int, b: int, density: float = 1.0, seed: int = 0, fp64: bool = False, device=None) -> Csr:
    p = SynthParams(cls=2, N=N, M=N, band=b, density=density, seed=seed)
    return _rowwise(p, N, N, fp64, device, {"class": "banded", "b": b, "density": density, "seed": seed})


def uniform(N: int, k: int, variable: bool = False, seed: int = 0, fp64: bool = False, device=None,
            M: int | None = None) -> Csr:
    M = N if M is None else M
    p = SynthParams(cls=3, N=N, M=M, k=k, variable=int(variable), seed=seed)
    return _rowwise(p, N, M, fp64, device, {"class": "uniform", "k": k, "variable": variable, "seed": seed})


def rmat(scale: int, edge_factor: int, a: float = 0.57, b: float = 0.19, c: float = 0.19, seed: int = 0,
         fp64: bool = True, device=None, permute: bool = True) -> Csr:
    """R-MAT (Chakrabarti et al.) graph as a square CSR; duplicate edges merged."""
    L = lib()
    N = 1 << scale
    ne = edge_factor * N
    p = SynthParams(cls=4, scale=scale, a=a, b=b, c=c, permute=int(permute), seed=seed)
    meta = {"class": "rmat", "scale": scale, "edge_factor": edge_factor, "a": a, "b": b, "c": c, "seed": seed}
    mask = N - 1
    if device is None:
        keys = np.empty(ne, dtype=np.uint64)
        _check(L.synth_rmat_keys(0, None, ctypes.byref(p), 0, ne, _ptr(keys)), "rmat")
        keys = np.unique(keys)
        rows = (keys >> np.uint64(scale)).astype(np.int64)
        col = (keys & np.uint64(mask)).astype(np.int32)
        del keys
        rowptr = np.zeros(N + 1, dtype=np.int64)
        np.cumsum(np.bincount(rows, minlength=N), out=rowptr[1:])
        val = np.empty(col.shape[0], dtype=np.float64 if fp64 else np.float32)
        _check(L.synth_values_rc(0, None, seed, col.shape[0], _ptr(rows), _ptr(col), _ptr(val), int(fp64)), "values")
    else:
        import torch
        s = _stream(device)
        keys = torch.empty(ne, dtype=torch.int64, device=device)
        _check(L.synth_rmat_keys(1, s, ctypes.byref(p), 0, ne, _ptr(keys)), "rmat")
        keys = torch.unique(keys, sorted=True)
        rows = keys >> scale
        col = (keys & mask).to(torch.int32)
        del keys
        rowptr = torch.zeros(N + 1, dtype=torch.int64, device=device)
        torch.cumsum(torch.bincount(rows, minlength=N), 0, out=rowptr[1:])
        val = torch.empty(col.shape[0], dtype=torch.float64 if fp64 else torch.float32, device=device)
        _check(L.synth_values_rc(1, s, seed, col.shape[0], _ptr(rows), _ptr(col), _ptr(val), int(fp64)), "values")
        del rows
    return Csr(N, N, rowptr, col, val, fp64, device, meta)


def vector(n: int, seed: int = 1, mode: int = 0, fp64: bool = False, device=None, j0: int = 0):
    """x vector: mode 0 U(-1,1)\\{0}, mode 1 integers U{-8..8}, mode 2 ones."""
    L = lib()
    if device is None:
        out = np.empty(n, dtype=np.float64 if fp64 else np.float32)
        _check(L.synth_vector(0, None, seed, j0, n, mode, _ptr(out), int(fp64)), "vector")
    else:
        import torch
        out = torch.empty(n, dtype=torch.float64 if fp64 else torch.float32, device=device)
        _check(L.synth_vector(1, _stream(device), seed, j0, n, mode, _ptr(out), int(fp64)), "vector")
    return out


def to_device(A: Csr, device="cuda", rowptr32: bool | None = None) -> Csr:
    """Upload a host CSR (the same arrays, bit for bit) to the GPU."""
    import torch
    rp = torch.from_numpy(A.rowptr).to(device)
    if rowptr32 is None:
        rowptr32 = A.nnz < 2**31
    if rowptr32:
        rp = rp.to(torch.int32)
    return Csr(A.rows, A.cols, rp, torch.from_numpy(A.colidx).to(device), torch.from_numpy(A.vals).to(device),
               A.fp64, device, dict(A.meta))


def checksum(A: Csr) -> tuple:
    """Cheap structural/value fingerprint (host arrays)."""
    rp = np.asarray(A.rowptr, dtype=np.int64)
    ci = np.asarray(A.colidx)
    v = np.asarray(A.vals)
    return (A.rows, A.cols, A.nnz, int(rp.sum() % (1 << 61)), int(ci.astype(np.int64).sum()),
            v.view(np.uint32 if v.dtype == np.float32 else np.uint64).astype(np.uint64).sum(dtype=np.uint64).item())


# ---------------------------------------------------------------- histogram samples
HIST_DISTS = ("uniform", "normal", "exponential", "spike", "sorted")


def hist_samples(n: int, dist: str, value_range: int, seed: int = 0, param: float = 0.1) -> np.ndarray:
    """Seeded uint32 histogram inputs over [0, value_range) (host numpy; no
    method arithmetic).  dist: uniform; normal (mean range/2, sd = param *
    range, clipped); exponential (scale = param * range, clipped); spike (a
    fraction param of the samples equal to one value, the rest uniform);
    sorted (uniform, sorted ascending — the paper's "almost sorted" style
    input)."""
    rng = np.random.default_rng(seed)
    hi = value_range - 1
    if dist == "uniform":
        v = rng.integers(0, value_range, n, dtype=np.uint64)
    elif dist == "normal":
        v = np.clip(np.rint(rng.normal(value_range / 2, param * value_range, n)), 0, hi)
    elif dist == "exponential":
        v = np.clip(np.floor(rng.exponential(param * value_range, n)), 0, hi)
    elif dist == "spike":
        v = rng.integers(0, value_range, n, dtype=np.uint64)
        v[rng.random(n) < param] = int(rng.integers(0, value_range))
    elif dist == "sorted":
        v = np.sort(rng.integers(0, value_range, n, dtype=np.uint64))
    else:
        raise ValueError(dist)
    return np.asarray(v, dtype=np.uint64).astype(np.uint32)
