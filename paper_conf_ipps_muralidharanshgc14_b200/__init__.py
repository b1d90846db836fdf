"""paper_conf_ipps_muralidharanshgc14_b200 — B200-native Nitro SpMV code-variant hot path.

Thin Python binding of libnitro.so (include/nitro.h): argument marshalling
only.  Every step of the path — feature pass, conversions, the five SpMV
variants, timing — runs in the library's sm_100a kernels; the SVM training and
selection run in the library's C++ host code.  PyTorch only provides device
memory and streams.  There is no CPU fallback: if libnitro.so is missing the
import fails loudly.
"""
from __future__ import annotations

import ctypes
import math
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# NITRO_LIB: another build of the library (A/B timing of two builds on one box)
LIB_PATH = os.environ.get("NITRO_LIB") or os.path.join(_HERE, "libnitro.so")

CSR_SCALAR, CSR_VECTOR, ELL, DIA, HYB = range(5)
NUM_VARIANTS = 5
CSR_IMPL_AUTO, CSR_IMPL_DIRECT, CSR_IMPL_STAGED, CSR_IMPL_STREAM, CSR_IMPL_VEC4 = range(5)
VARIANT_NAMES = ("csr_scalar", "csr_vector", "ell", "dia", "hyb")
FEATURE_NAMES = ("nnz", "rows", "mean", "sd", "max_dev", "dia_fill", "ell_fill")

# export parts (nitro_spmv_export)
PART_ELL_COL, PART_ELL_VAL, PART_DIA_OFF, PART_DIA_VAL = 0, 1, 2, 3
PART_HYB_COL, PART_HYB_VAL, PART_HYB_TROW, PART_HYB_TCOL, PART_HYB_TVAL = 4, 5, 6, 7, 8
PART_OFFSETS = 9

# histogram family (include/nitro.h §4)
HIST_SORT_ES, HIST_SORT_DYN, HIST_SHARED_ES, HIST_SHARED_DYN, HIST_GLOBAL_ES, HIST_GLOBAL_DYN = range(6)
HIST_NUM_VARIANTS = 6
HIST_VARIANT_NAMES = ("sort_es", "sort_dynamic", "shared_atomic_es", "shared_atomic_dynamic",
                      "global_atomic_es", "global_atomic_dynamic")
HIST_FEATURE_NAMES = ("n", "n_per_bin", "subsample_sd")

STATUS = {0: "OK", 1: "INVALID_ARG", 2: "BAD_MATRIX", 3: "STATE", 4: "CONSTRAINT", 5: "OOM", 6: "CUDA",
          7: "NCCL", 8: "IO", 9: "UNSUPPORTED"}


class NitroError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"nitro {STATUS.get(code, code)}: {msg}")
        self.code = code


if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is not built; run `python __graft_entry__.py` (build()) first")

_L = ctypes.CDLL(LIB_PATH)


class Feat(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_int64), ("cols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("sum_len", ctypes.c_uint64), ("sum_len2", ctypes.c_uint64),
                ("max_row", ctypes.c_int64), ("ndiag", ctypes.c_int64),
                ("canonical", ctypes.c_int32), ("pad_", ctypes.c_int32),
                ("mean", ctypes.c_double), ("sd", ctypes.c_double), ("max_dev", ctypes.c_double),
                ("dia_fill", ctypes.c_double), ("ell_fill", ctypes.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_ if k != "pad_"}


class FormatInfo(ctypes.Structure):
    _fields_ = [("ld", ctypes.c_int64), ("width", ctypes.c_int64), ("tail", ctypes.c_int64),
                ("bytes", ctypes.c_int64), ("compulsory_bytes", ctypes.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class TrainOpts(ctypes.Structure):
    _fields_ = [("folds", ctypes.c_int), ("seed", ctypes.c_uint64), ("tol", ctypes.c_double),
                ("log2c_lo", ctypes.c_int), ("log2c_hi", ctypes.c_int), ("log2c_step", ctypes.c_int),
                ("log2g_lo", ctypes.c_int), ("log2g_hi", ctypes.c_int), ("log2g_step", ctypes.c_int),
                ("verbose", ctypes.c_int), ("timeout_factor", ctypes.c_double)]


class ItuneOpts(ctypes.Structure):
    _fields_ = [("init", ctypes.c_int), ("iters", ctypes.c_int), ("acc", ctypes.c_double),
                ("seed", ctypes.c_uint64), ("prob_folds", ctypes.c_int), ("n_test", ctypes.c_int),
                ("test_feat", ctypes.c_void_p), ("test_cost", ctypes.c_void_p)]


class SpmvInput(ctypes.Structure):
    _fields_ = [("A", ctypes.c_void_p), ("d_x", ctypes.c_void_p), ("d_y", ctypes.c_void_p),
                ("warmup", ctypes.c_int), ("reps", ctypes.c_int), ("flush_l2", ctypes.c_int)]


class HistInput(ctypes.Structure):
    _fields_ = [("H", ctypes.c_void_p), ("d_hist", ctypes.c_void_p),
                ("warmup", ctypes.c_int), ("reps", ctypes.c_int), ("flush_l2", ctypes.c_int)]


VARIANT_FN = ctypes.CFUNCTYPE(ctypes.c_double, ctypes.c_void_p, ctypes.c_void_p)
FEATURE_FN = ctypes.CFUNCTYPE(ctypes.c_double, ctypes.c_void_p, ctypes.c_void_p)
GROUP_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.POINTER(ctypes.c_double), ctypes.c_int,
                            ctypes.c_void_p)
CONSTRAINT_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p)

_vp, _i64, _int, _dbl, _u64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_double, ctypes.c_uint64
_P = ctypes.POINTER
_SIGS = {
    "nitro_last_error": ([], ctypes.c_char_p),
    "nitro_version": ([], ctypes.c_char_p),
    # generic layer
    "nitro_context_create": ([_P(_vp)], _int),
    "nitro_context_destroy": ([_vp], None),
    "nitro_cv_create": ([_vp, ctypes.c_char_p, _P(_vp)], _int),
    "nitro_cv_destroy": ([_vp], None),
    "nitro_cv_add_variant": ([_vp, ctypes.c_char_p, VARIANT_FN, _vp, _P(_int)], _int),
    "nitro_cv_set_default": ([_vp, _int], _int),
    "nitro_cv_add_feature": ([_vp, ctypes.c_char_p, FEATURE_FN, _vp, _P(_int)], _int),
    "nitro_cv_add_feature_group": ([_vp, _P(ctypes.c_char_p), _int, GROUP_FN, _vp], _int),
    "nitro_cv_add_constraint": ([_vp, _int, CONSTRAINT_FN, _vp], _int),
    "nitro_cv_add_training_input": ([_vp, _vp], _int),
    "nitro_train_opts_default": ([_P(TrainOpts)], None),
    "nitro_cv_cost_cutoff": ([], _dbl),
    "nitro_cv_train": ([_vp, _P(TrainOpts)], _int),
    "nitro_cv_train_from_table": ([_vp, _int, _vp, _vp, _P(TrainOpts)], _int),
    "nitro_cv_training_table": ([_vp, _P(_int), _vp, _vp, _vp], _int),
    "nitro_cv_model_info": ([_vp, _P(_dbl), _P(_dbl), _P(_dbl), _P(_int)], _int),
    "nitro_cv_save_model": ([_vp, ctypes.c_char_p], _int),
    "nitro_cv_load_model": ([_vp, ctypes.c_char_p], _int),
    "nitro_cv_set_feature_transform": ([_vp, ctypes.c_uint32, _int], _int),
    "nitro_cv_num_features": ([_vp, _P(_int)], _int),
    "nitro_cv_num_variants": ([_vp, _P(_int)], _int),
    "nitro_cv_select": ([_vp, _vp, _P(_int), _vp], _int),
    "nitro_cv_call": ([_vp, _vp, _P(_int), _P(_dbl)], _int),
    "nitro_cv_predict": ([_vp, _vp, _vp, _P(_int)], _int),
    # svm
    "nitro_svm_fit": ([_int, _int, _vp, _vp, _dbl, _dbl, _dbl, _P(_vp)], _int),
    "nitro_svm_predict": ([_vp, _int, _vp, _vp], _int),
    "nitro_svm_decision": ([_vp, _int, _vp, _vp, _P(_int)], _int),
    "nitro_svm_pair_dual": ([_vp, _int, _vp, _P(_dbl)], _int),
    "nitro_svm_destroy": ([_vp], None),
    "nitro_svm_fold_assign": ([_int, _vp, _int, _u64, _vp], _int),
    "nitro_svm_cv_accuracy": ([_int, _int, _vp, _vp, _dbl, _dbl, _dbl, _int, _u64, _P(_dbl)], _int),
    "nitro_svm_fit_prob": ([_int, _int, _vp, _vp, _dbl, _dbl, _dbl, _int, _u64, _P(_vp)], _int),
    "nitro_svm_probability": ([_vp, _int, _vp, _vp, _P(_int)], _int),
    "nitro_svm_pair_sigmoid": ([_vp, _int, _P(_dbl), _P(_dbl)], _int),
    "nitro_itune_opts_default": ([_P(ItuneOpts)], None),
    "nitro_cv_itune": ([_vp, _P(TrainOpts), _P(ItuneOpts)], _int),
    "nitro_cv_itune_history": ([_vp, _P(_int), _vp, _vp, _vp, _vp], _int),
    # spmv
    "nitro_spmv_create": ([_int, _vp, _i64, _i64, _i64, _vp, _int, _vp, _vp, _int, _P(_vp)], _int),
    "nitro_spmv_set_stream": ([_vp, _vp], _int),
    "nitro_spmv_features": ([_vp, _P(Feat)], _int),
    "nitro_spmv_row_features": ([_vp, _P(Feat)], _int),
    "nitro_spmv_features_async": ([_vp], _int),
    "nitro_spmv_allowed": ([_vp, _int, _P(_int)], _int),
    "nitro_spmv_set_budget": ([_vp, _dbl], _int),
    "nitro_spmv_set_csr_impl": ([_vp, _int], _int),
    "nitro_spmv_prepare": ([_vp, _int], _int),
    "nitro_spmv_format_info": ([_vp, _int, _P(FormatInfo)], _int),
    "nitro_spmv_run": ([_vp, _int, _vp, _vp], _int),
    "nitro_spmv_run_host": ([_vp, _int, _vp, _vp], _int),
    "nitro_spmv_time": ([_vp, _int, _vp, _vp, _int, _int, _int, _P(_dbl), _vp], _int),
    "nitro_spmv_flush_l2": ([_vp], _int),
    "nitro_spmv_launches": ([_vp, _int, _P(_int)], _int),
    "nitro_spmv_export": ([_vp, _int, _vp, ctypes.c_size_t, _P(ctypes.c_size_t)], _int),
    "nitro_spmv_release": ([_vp, _int], _int),
    "nitro_spmv_invalidate": ([_vp], _int),
    "nitro_spmv_destroy": ([_vp], None),
    "nitro_spmv_register": ([_vp], _int),
    # dist
    "nitro_dist_unique_id": ([_vp], _int),
    "nitro_dist_init": ([_vp, _int, _int, _int, _P(_vp)], _int),
    "nitro_dist_destroy": ([_vp], None),
    "nitro_dist_partition": ([_i64, _vp, _int, _vp], _int),
    "nitro_dist_spmv_create": ([_vp, _i64, _vp, _i64, _vp, _int, _vp, _vp, _int, _P(_vp)], _int),
    "nitro_dist_spmv_run": ([_vp, _vp, _int, _vp, _vp], _int),
    "nitro_dist_features": ([_vp, _vp, _P(Feat)], _int),
    "nitro_dist_spmv_run_gathered": ([_vp, _vp, _int, _vp, _vp], _int),
    "nitro_dist_layout": ([_vp, _P(_i64), _P(_i64), _P(_i64)], _int),
    "nitro_dist_init_local": ([_int, _int, _int, _P(_vp)], _int),
    "nitro_dist_loopback_create": ([_int, _int, _P(_vp)], _int),
    "nitro_dist_format_info": ([_vp, _int, _P(FormatInfo)], _int),
    "nitro_dist_loop_create": ([_vp, _vp, _P(_vp)], _int),
    "nitro_dist_loop_destroy": ([_vp], None),
    "nitro_dist_loop_x": ([_vp, _P(_vp)], _int),
    "nitro_dist_loop_start": ([_vp], _int),
    "nitro_dist_loop_step": ([_vp, _int, _vp], _int),
    "nitro_dist_loopback_destroy": ([_vp], None),
    "nitro_dist_init_loopback": ([_vp, _int, _P(_vp)], _int),
    "nitro_dist_spmv_create_ex": ([_vp, _i64, _vp, _i64, _vp, _int, _vp, _vp, _int, _int, _P(_vp)], _int),
    "nitro_dist_exchange_info": ([_vp, _P(_int), _P(_i64), _P(_i64), _P(_i64)], _int),
    "nitro_dist_halo_cols": ([_vp, _vp], _int),
    "nitro_dist_x_local": ([_vp, _P(_vp)], _int),
    # histogram family
    "nitro_hist_create": ([_int, _vp, _i64, _vp, ctypes.c_int32, _u64, _P(_vp)], _int),
    "nitro_hist_destroy": ([_vp], None),
    "nitro_hist_features": ([_vp, _P(_dbl)], _int),
    "nitro_hist_allowed": ([_vp, _int, _P(_int)], _int),
    "nitro_hist_run": ([_vp, _int, _vp], _int),
    "nitro_hist_time": ([_vp, _int, _vp, _int, _int, _int, _P(_dbl)], _int),
    "nitro_hist_register": ([_vp], _int),
}
for _name, (_args, _res) in _SIGS.items():
    _f = getattr(_L, _name)
    _f.argtypes = _args
    _f.restype = _res

EXPORTED = tuple(_SIGS)


def _check(rc):
    if rc != 0:
        raise NitroError(rc, _L.nitro_last_error().decode(errors="replace"))


def version() -> str:
    return _L.nitro_version().decode()


def _ptr(t):
    if t is None:
        return None
    if isinstance(t, np.ndarray):
        return t.ctypes.data
    return t.data_ptr()


def _dev_vec(t, n: int, dtype, device: int, name: str):
    """A device array argument of the C ABI: contiguous, right dtype and
    device, at least n elements (the library reads n elements behind the pointer)."""
    if not t.is_cuda or t.device.index != device:
        raise ValueError(f"{name}: expected a tensor on cuda:{device}, got {t.device}")
    if t.dtype != dtype:
        raise ValueError(f"{name}: expected {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name}: must be contiguous")
    if t.numel() < n:
        raise ValueError(f"{name}: {t.numel()} elements, need {n}")
    return t.data_ptr()


def _np(a, dtype):
    return np.ascontiguousarray(np.asarray(a, dtype=dtype))


# ====================================================================== SpMV layer
class SpMV:
    """A borrowed device CSR matrix (torch CUDA tensors) and its formats.

    rowptr int32/int64 [rows+1], colidx int32 [nnz], vals fp32/fp64 [nnz]."""

    def __init__(self, rowptr, colidx, vals, rows: int, cols: int, stream=None, device: int | None = None):
        import torch
        if not (rowptr.is_cuda and colidx.is_cuda and vals.is_cuda):
            raise ValueError("SpMV needs CUDA tensors")
        if rowptr.dtype not in (torch.int32, torch.int64) or vals.dtype not in (torch.float32, torch.float64):
            raise ValueError("rowptr must be int32/int64 and vals fp32/fp64")
        self._keep = (rowptr, colidx, vals)
        self.rows, self.cols, self.nnz = int(rows), int(cols), int(colidx.numel())
        self.fp64 = vals.dtype == torch.float64
        self.dtype = vals.dtype
        self.device = rowptr.device.index if device is None else device
        _dev_vec(rowptr, self.rows + 1, rowptr.dtype, self.device, "rowptr")
        _dev_vec(colidx, self.nnz, torch.int32, self.device, "colidx")
        _dev_vec(vals, self.nnz, vals.dtype, self.device, "vals")
        if stream is None:
            stream = torch.cuda.current_stream(self.device).cuda_stream
        self.stream = stream
        h = ctypes.c_void_p()
        _check(_L.nitro_spmv_create(self.device, stream, self.rows, self.cols, self.nnz, _ptr(rowptr),
                                    int(rowptr.dtype == torch.int64), _ptr(colidx), _ptr(vals), int(self.fp64),
                                    ctypes.byref(h)))
        self.h = h

    @classmethod
    def from_csr(cls, A, **kw):
        """From a synth.Csr whose arrays live on the GPU."""
        return cls(A.rowptr, A.colidx, A.vals, A.rows, A.cols, **kw)

    def close(self):
        if getattr(self, "h", None):
            _L.nitro_spmv_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def features(self) -> dict:
        f = Feat()
        _check(_L.nitro_spmv_features(self.h, ctypes.byref(f)))
        return f.as_dict()

    def row_features(self) -> dict:
        """Cheap level: rowptr-only pass (ndiag / dia_fill / canonical = -1, not evaluated)."""
        f = Feat()
        _check(_L.nitro_spmv_row_features(self.h, ctypes.byref(f)))
        return f.as_dict()

    def features_async(self):
        _check(_L.nitro_spmv_features_async(self.h))

    def allowed(self, v: int) -> bool:
        ok = ctypes.c_int()
        _check(_L.nitro_spmv_allowed(self.h, v, ctypes.byref(ok)))
        return bool(ok.value)

    def allowed_mask(self):
        return [self.allowed(v) for v in range(NUM_VARIANTS)]

    def set_budget(self, nbytes: float):
        _check(_L.nitro_spmv_set_budget(self.h, float(nbytes)))

    def set_csr_impl(self, impl: int):
        """CSR_IMPL_AUTO / _DIRECT / _STAGED / _STREAM / _VEC4 (nitro_spmv_set_csr_impl)."""
        _check(_L.nitro_spmv_set_csr_impl(self.h, int(impl)))

    def prepare(self, v: int):
        _check(_L.nitro_spmv_prepare(self.h, v))

    def format_info(self, v: int) -> dict:
        fi = FormatInfo()
        _check(_L.nitro_spmv_format_info(self.h, v, ctypes.byref(fi)))
        return fi.as_dict()

    def run(self, v: int, x, y=None):
        import torch
        if y is None:
            y = torch.empty(self.rows, dtype=self.dtype, device=x.device)
        _check(_L.nitro_spmv_run(self.h, v, self._x(x), self._y(y)))
        return y

    def _x(self, x):
        return _dev_vec(x, self.cols, self.dtype, self.device, "x")

    def _y(self, y):
        return _dev_vec(y, self.rows, self.dtype, self.device, "y")

    def run_host(self, v: int, x_host: np.ndarray, y_host: np.ndarray | None = None) -> np.ndarray:
        dt = np.float64 if self.fp64 else np.float32
        if x_host.dtype != dt or not x_host.flags.c_contiguous or x_host.size < self.cols:
            raise ValueError(f"x_host: need a contiguous {np.dtype(dt)} array of >= {self.cols} elements")
        if y_host is None:
            y_host = np.empty(self.rows, dtype=dt)
        if y_host.dtype != dt or not y_host.flags.c_contiguous or y_host.size < self.rows:
            raise ValueError(f"y_host: need a contiguous {np.dtype(dt)} array of >= {self.rows} elements")
        _check(_L.nitro_spmv_run_host(self.h, v, _ptr(x_host), _ptr(y_host)))
        return y_host

    def time(self, v: int, x, y, warmup: int = 3, reps: int = 20, flush_l2: bool = True):
        med = ctypes.c_double()
        allt = np.empty(reps, dtype=np.float64)
        _check(_L.nitro_spmv_time(self.h, v, self._x(x), self._y(y), warmup, reps, int(flush_l2), ctypes.byref(med),
                                  _ptr(allt)))
        return med.value, allt

    def flush_l2(self):
        _check(_L.nitro_spmv_flush_l2(self.h))

    def launches(self, v: int) -> int:
        n = ctypes.c_int()
        _check(_L.nitro_spmv_launches(self.h, v, ctypes.byref(n)))
        return n.value

    def export(self, part: int) -> np.ndarray:
        need = ctypes.c_size_t()
        _check(_L.nitro_spmv_export(self.h, part, None, 0, ctypes.byref(need)))
        is_val = part in (PART_ELL_VAL, PART_DIA_VAL, PART_HYB_VAL, PART_HYB_TVAL)
        dt = (np.float64 if self.fp64 else np.float32) if is_val else np.int32
        out = np.empty(need.value // np.dtype(dt).itemsize, dtype=dt)
        if need.value:
            _check(_L.nitro_spmv_export(self.h, part, _ptr(out), need.value, ctypes.byref(need)))
        return out

    def release(self, v: int = -1):
        _check(_L.nitro_spmv_release(self.h, v))

    def invalidate(self):
        """Matrix contents changed in place: recompute features/formats on next use."""
        _check(_L.nitro_spmv_invalidate(self.h))


# ====================================================================== generic Nitro layer
def train_opts(**kw) -> TrainOpts:
    o = TrainOpts()
    _L.nitro_train_opts_default(ctypes.byref(o))
    for k, v in kw.items():
        setattr(o, k, v)
    return o


class Context:
    def __init__(self):
        h = ctypes.c_void_p()
        _check(_L.nitro_context_create(ctypes.byref(h)))
        self.h = h

    def __del__(self):
        if getattr(self, "h", None):
            _L.nitro_context_destroy(self.h)
            self.h = None


class CodeVariant:
    """nitro_cv: variants, features, constraints, training inputs, model.

    Inputs are opaque pointers (ints); Python callbacks receive the pointer value."""

    def __init__(self, ctx: Context, name: str):
        self.ctx = ctx
        h = ctypes.c_void_p()
        _check(_L.nitro_cv_create(ctx.h, name.encode(), ctypes.byref(h)))
        self.h = h
        self._keep = []

    def __del__(self):
        if getattr(self, "h", None):
            _L.nitro_cv_destroy(self.h)
            self.h = None

    def add_variant(self, name, fn) -> int:
        cb = VARIANT_FN(lambda inp, user: float(fn(inp or 0)))
        self._keep.append(cb)
        i = ctypes.c_int()
        _check(_L.nitro_cv_add_variant(self.h, name.encode(), cb, None, ctypes.byref(i)))
        return i.value

    def set_default(self, vid: int):
        _check(_L.nitro_cv_set_default(self.h, vid))

    def add_feature(self, name, fn) -> int:
        cb = FEATURE_FN(lambda inp, user: float(fn(inp or 0)))
        self._keep.append(cb)
        i = ctypes.c_int()
        _check(_L.nitro_cv_add_feature(self.h, name.encode(), cb, None, ctypes.byref(i)))
        return i.value

    def add_constraint(self, vid: int, fn):
        cb = CONSTRAINT_FN(lambda inp, user: int(bool(fn(inp or 0))))
        self._keep.append(cb)
        _check(_L.nitro_cv_add_constraint(self.h, vid, cb, None))

    def add_training_input(self, inp):
        _check(_L.nitro_cv_add_training_input(self.h, inp))

    def register_spmv(self):
        _check(_L.nitro_spmv_register(self.h))

    def register_hist(self):
        """The six histogram variants, their features and constraints (nitro_hist_register)."""
        _check(_L.nitro_hist_register(self.h))

    def set_feature_transform(self, log_mask: int, clip: bool):
        """log1p of the features in log_mask, clip scaled inputs (nitro_cv_set_feature_transform)."""
        _check(_L.nitro_cv_set_feature_transform(self.h, int(log_mask), int(bool(clip))))

    def train(self, **opts):
        o = train_opts(**opts)
        _check(_L.nitro_cv_train(self.h, ctypes.byref(o)))

    def train_from_table(self, feat, cost, **opts):
        feat = _np(feat, np.float64)
        cost = _np(cost, np.float64)
        o = train_opts(**opts)
        _check(_L.nitro_cv_train_from_table(self.h, feat.shape[0], _ptr(feat), _ptr(cost), ctypes.byref(o)))

    def n_features(self):
        n = ctypes.c_int()
        _check(_L.nitro_cv_num_features(self.h, ctypes.byref(n)))
        return n.value

    def n_variants(self):
        n = ctypes.c_int()
        _check(_L.nitro_cv_num_variants(self.h, ctypes.byref(n)))
        return n.value

    def training_table(self):
        n = ctypes.c_int()
        _check(_L.nitro_cv_training_table(self.h, ctypes.byref(n), None, None, None))
        nv, nf = self.n_variants(), self.n_features()
        cost = np.empty((n.value, nv))
        feat = np.empty((n.value, nf))
        lab = np.empty(n.value, dtype=np.int32)
        _check(_L.nitro_cv_training_table(self.h, ctypes.byref(n), _ptr(cost), _ptr(feat), _ptr(lab)))
        return cost, feat, lab

    def model_info(self) -> dict:
        C, g, a, ns = ctypes.c_double(), ctypes.c_double(), ctypes.c_double(), ctypes.c_int()
        _check(_L.nitro_cv_model_info(self.h, ctypes.byref(C), ctypes.byref(g), ctypes.byref(a), ctypes.byref(ns)))
        return {"C": C.value, "gamma": g.value, "cv_accuracy": a.value, "n_sv": ns.value}

    def save(self, path):
        _check(_L.nitro_cv_save_model(self.h, str(path).encode()))

    def load(self, path):
        _check(_L.nitro_cv_load_model(self.h, str(path).encode()))

    def select(self, inp):
        v = ctypes.c_int()
        f = np.empty(max(self.n_features(), 1))
        _check(_L.nitro_cv_select(self.h, inp, ctypes.byref(v), _ptr(f)))
        return v.value, f

    def call(self, inp):
        v, c = ctypes.c_int(), ctypes.c_double()
        _check(_L.nitro_cv_call(self.h, inp, ctypes.byref(v), ctypes.byref(c)))
        return v.value, c.value

    def itune(self, init=0, iters=0, acc=0.0, seed=0, prob_folds=5, test_feat=None, test_cost=None, **train):
        """Incremental tuning: label a BvSB-chosen subset only.
        Returns the history dict (one entry per refit)."""
        io = ItuneOpts()
        _L.nitro_itune_opts_default(ctypes.byref(io))
        io.init, io.iters, io.acc, io.seed, io.prob_folds = init, iters, acc, seed, prob_folds
        keep = []
        if test_feat is not None:
            tf, tc = _np(test_feat, np.float64), _np(test_cost, np.float64)
            keep = [tf, tc]
            io.n_test, io.test_feat, io.test_cost = tf.shape[0], _ptr(tf), _ptr(tc)
        o = train_opts(**train)
        _check(_L.nitro_cv_itune(self.h, ctypes.byref(o), ctypes.byref(io)))
        del keep
        ns = ctypes.c_int()
        _check(_L.nitro_cv_itune_history(self.h, ctypes.byref(ns), None, None, None, None))
        k = ns.value
        nl, pk = np.empty(k, np.int32), np.empty(k, np.int32)
        ac, pf = np.empty(k), np.empty(k)
        _check(_L.nitro_cv_itune_history(self.h, ctypes.byref(ns), _ptr(nl), _ptr(pk), _ptr(ac), _ptr(pf)))
        return {"n_labelled": nl.tolist(), "picked": pk.tolist(), "test_acc": ac.tolist(), "test_perf": pf.tolist()}

    def predict(self, feat, allowed=None) -> int:
        feat = _np(feat, np.float64)
        al = None if allowed is None else _np([int(bool(a)) for a in allowed], np.int32)
        v = ctypes.c_int()
        _check(_L.nitro_cv_predict(self.h, _ptr(feat), _ptr(al), ctypes.byref(v)))
        return v.value


def spmv_input(A: SpMV, x, y, warmup=3, reps=20, flush_l2=True) -> SpmvInput:
    """Input record for the registered SpMV variants (keep it alive while used)."""
    rec = SpmvInput(A.h.value, A._x(x), A._y(y), warmup, reps, int(flush_l2))
    rec._keep = (A, x, y)
    return rec


class Hist:
    """An even histogram of borrowed device uint32 samples (include/nitro.h §4):
    h[b] = #{i : s_i < range, floor(s_i * nbins / range) = b}."""

    def __init__(self, samples, nbins: int, value_range: int, stream=None):
        import torch
        if samples.dtype not in (torch.int32, torch.uint32):
            raise ValueError("samples: uint32 (or int32 bit pattern) CUDA tensor expected")
        _dev_vec(samples, samples.numel(), samples.dtype, samples.device.index if samples.is_cuda else -1, "samples")
        self._keep = samples
        self.n, self.nbins, self.range = int(samples.numel()), int(nbins), int(value_range)
        self.device = samples.device.index
        if stream is None:
            stream = torch.cuda.current_stream(self.device).cuda_stream
        h = ctypes.c_void_p()
        _check(_L.nitro_hist_create(self.device, stream, self.n, _ptr(samples), self.nbins, self.range,
                                    ctypes.byref(h)))
        self.h = h

    def close(self):
        if getattr(self, "h", None):
            _L.nitro_hist_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def features(self) -> dict:
        out = (ctypes.c_double * 3)()
        _check(_L.nitro_hist_features(self.h, out))
        return dict(zip(HIST_FEATURE_NAMES, list(out)))

    def allowed(self, v: int) -> bool:
        ok = ctypes.c_int()
        _check(_L.nitro_hist_allowed(self.h, v, ctypes.byref(ok)))
        return bool(ok.value)

    def run(self, v: int, hist=None):
        import torch
        if hist is None:
            hist = torch.empty(self.nbins, dtype=torch.int32, device=self._keep.device)
        _check(_L.nitro_hist_run(self.h, v, self._h(hist)))
        return hist

    def time(self, v: int, hist, warmup=3, reps=20, flush_l2=True) -> float:
        t = ctypes.c_double()
        _check(_L.nitro_hist_time(self.h, v, self._h(hist), warmup, reps, int(flush_l2), ctypes.byref(t)))
        return t.value

    def _h(self, hist):
        import torch
        if hist.dtype not in (torch.int32, torch.uint32):
            raise ValueError("hist: int32/uint32 tensor expected")
        return _dev_vec(hist, self.nbins, hist.dtype, self.device, "hist")


def hist_input(H: Hist, hist, warmup=3, reps=20, flush_l2=True) -> HistInput:
    """Input record for the registered histogram variants (keep it alive while used)."""
    rec = HistInput(H.h.value, _ptr(hist), warmup, reps, int(flush_l2))
    rec._keep = (H, hist)
    return rec


def addr(rec) -> int:
    return ctypes.addressof(rec)


# ====================================================================== host SVM primitives
class SVM:
    def __init__(self, X, y, C, gamma, tol=1e-6, probability=False, prob_folds=5, seed=0):
        X = _np(X, np.float64)
        y = _np(y, np.int32)
        h = ctypes.c_void_p()
        if probability:
            _check(_L.nitro_svm_fit_prob(X.shape[0], X.shape[1], _ptr(X), _ptr(y), C, gamma, tol, prob_folds, seed,
                                         ctypes.byref(h)))
        else:
            _check(_L.nitro_svm_fit(X.shape[0], X.shape[1], _ptr(X), _ptr(y), C, gamma, tol, ctypes.byref(h)))
        self.h, self.n, self.d = h, X.shape[0], X.shape[1]

    def probability(self, X):
        X = _np(X, np.float64)
        k = ctypes.c_int()
        _check(_L.nitro_svm_probability(self.h, 0, None, None, ctypes.byref(k)))
        out = np.empty((X.shape[0], k.value))
        _check(_L.nitro_svm_probability(self.h, X.shape[0], _ptr(X), _ptr(out), ctypes.byref(k)))
        return out

    def pair_sigmoid(self, p: int):
        A, B = ctypes.c_double(), ctypes.c_double()
        _check(_L.nitro_svm_pair_sigmoid(self.h, p, ctypes.byref(A), ctypes.byref(B)))
        return A.value, B.value

    def __del__(self):
        if getattr(self, "h", None):
            _L.nitro_svm_destroy(self.h)
            self.h = None

    def predict(self, X):
        X = _np(X, np.float64)
        out = np.empty(X.shape[0], dtype=np.int32)
        _check(_L.nitro_svm_predict(self.h, X.shape[0], _ptr(X), _ptr(out)))
        return out

    def decision(self, X):
        X = _np(X, np.float64)
        npairs = ctypes.c_int()
        _check(_L.nitro_svm_decision(self.h, 0, None, None, ctypes.byref(npairs)))
        out = np.empty((X.shape[0], npairs.value))
        _check(_L.nitro_svm_decision(self.h, X.shape[0], _ptr(X), _ptr(out), ctypes.byref(npairs)))
        return out

    def pair_dual(self, p: int):
        coef = np.empty(self.n)
        rho = ctypes.c_double()
        _check(_L.nitro_svm_pair_dual(self.h, p, _ptr(coef), ctypes.byref(rho)))
        return coef, rho.value


def fold_assign(y, k: int, seed: int = 0) -> np.ndarray:
    y = _np(y, np.int32)
    out = np.empty(y.shape[0], dtype=np.int32)
    _check(_L.nitro_svm_fold_assign(y.shape[0], _ptr(y), k, seed, _ptr(out)))
    return out


def cv_accuracy(X, y, C, gamma, tol=1e-6, folds=5, seed=0) -> float:
    X = _np(X, np.float64)
    y = _np(y, np.int32)
    acc = ctypes.c_double()
    _check(_L.nitro_svm_cv_accuracy(X.shape[0], X.shape[1], _ptr(X), _ptr(y), C, gamma, tol, folds, seed,
                                    ctypes.byref(acc)))
    return acc.value


# ====================================================================== multi-GPU
def _wrap_device(ptr: int, n: int, dtype, device: int):
    """A torch tensor over library-owned device memory (no copy, not owning)."""
    import torch
    itemsize = torch.empty((), dtype=dtype).element_size()

    class _CAI:
        __cuda_array_interface__ = {"shape": (n,), "typestr": "<f8" if itemsize == 8 else "<f4",
                                    "data": (ptr, False), "version": 3, "strides": None}
    with torch.cuda.device(device):
        return torch.as_tensor(_CAI(), device=f"cuda:{device}")


def dist_partition(rowptr_host, nranks: int) -> np.ndarray:
    rp = _np(rowptr_host, np.int64)
    out = np.empty(nranks + 1, dtype=np.int64)
    _check(_L.nitro_dist_partition(rp.shape[0] - 1, _ptr(rp), nranks, _ptr(out)))
    return out


def dist_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(_L.nitro_dist_unique_id(buf))
    return buf.raw


class Loopback:
    """A loopback transport group (nitro_dist_loopback_create): P ranks in one
    process on one GPU, one host thread per rank (``Dist.loopback``)."""

    def __init__(self, nranks: int, device: int = 0):
        h = ctypes.c_void_p()
        _check(_L.nitro_dist_loopback_create(int(nranks), int(device), ctypes.byref(h)))
        self.h, self.nranks, self.device = h, int(nranks), int(device)

    def close(self):
        if getattr(self, "h", None):
            _L.nitro_dist_loopback_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Dist:
    """One rank of the row-partitioned multi-GPU SpMV (NCCL communicator).

    ``Dist.local(rank, nranks, device)`` builds a communicator-less handle whose
    ``run_gathered`` computes that rank's rows from an already gathered x;
    ``Dist.loopback(group, rank)`` a rank of a single-GPU loopback group."""

    def __init__(self, uid: bytes | None, rank: int, nranks: int, device: int, loopback: "Loopback | None" = None):
        h = ctypes.c_void_p()
        self._group = loopback
        if loopback is not None:
            _check(_L.nitro_dist_init_loopback(loopback.h, rank, ctypes.byref(h)))
        elif uid is None:
            _check(_L.nitro_dist_init_local(rank, nranks, device, ctypes.byref(h)))
        else:
            buf = ctypes.create_string_buffer(uid, 128)
            _check(_L.nitro_dist_init(buf, rank, nranks, device, ctypes.byref(h)))
        self.h, self.rank, self.nranks, self.device = h, rank, nranks, device

    @classmethod
    def local(cls, rank: int, nranks: int, device: int = 0):
        return cls(None, rank, nranks, device)

    @classmethod
    def loopback(cls, group: Loopback, rank: int):
        return cls(None, rank, group.nranks, group.device, loopback=group)

    def run_gathered(self, A: "SpMV", v: int, x_gathered, y_local):
        _check(_L.nitro_dist_spmv_run_gathered(self.h, A.h, v, _ptr(x_gathered), _ptr(y_local)))
        return y_local

    @staticmethod
    def exchange_info(A: "SpMV") -> dict:
        m, L, nh, ns = ctypes.c_int(), ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        _check(_L.nitro_dist_exchange_info(A.h, ctypes.byref(m), ctypes.byref(L), ctypes.byref(nh), ctypes.byref(ns)))
        return {"mode": ("allgather", "halo")[m.value], "layout_len": L.value, "halo_len": nh.value,
                "send_len": ns.value}

    @staticmethod
    def halo_cols(A: "SpMV") -> np.ndarray:
        info = Dist.exchange_info(A)
        out = np.empty(info["halo_len"], dtype=np.int32)
        _check(_L.nitro_dist_halo_cols(A.h, _ptr(out) if out.size else None))
        return out

    @staticmethod
    def x_local(A: "SpMV"):
        """torch view of this rank's x block inside the exchange buffer (write x
        there and pass it to run() to skip the per-multiply copy)."""
        import torch
        p = ctypes.c_void_p()
        _check(_L.nitro_dist_x_local(A.h, ctypes.byref(p)))
        return _wrap_device(p.value, A.rows, A.dtype, A.device)

    @staticmethod
    def format_info(A: "SpMV", v: int) -> dict:
        """nitro_dist_format_info: this rank's multiply (all row parts + the exchanged x)."""
        fi = FormatInfo()
        _check(_L.nitro_dist_format_info(A.h, v, ctypes.byref(fi)))
        return fi.as_dict()

    @staticmethod
    def layout(A: "SpMV"):
        B, i0, i1 = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        _check(_L.nitro_dist_layout(A.h, ctypes.byref(B), ctypes.byref(i0), ctypes.byref(i1)))
        return B.value, i0.value, i1.value

    def close(self):
        if getattr(self, "h", None):
            _L.nitro_dist_destroy(self.h)
            self.h = None

    def spmv(self, global_rows, bounds, rowptr, colidx, vals, exchange: int = -1):
        """This rank's row block (global column ids) -> SpMV handle for dist runs.
        exchange: -1 auto, 0 all-gather, 1 halo."""
        import torch
        b = _np(bounds, np.int64)
        h = ctypes.c_void_p()
        _check(_L.nitro_dist_spmv_create_ex(self.h, global_rows, _ptr(b), colidx.numel(), _ptr(rowptr),
                                            int(rowptr.dtype == torch.int64), _ptr(colidx), _ptr(vals),
                                            int(vals.dtype == torch.float64), exchange, ctypes.byref(h)))
        A = SpMV.__new__(SpMV)
        A._keep = (rowptr, colidx, vals)
        A.rows = int(b[self.rank + 1] - b[self.rank])
        A.cols = int(global_rows)
        A.nnz = int(colidx.numel())
        A.fp64 = vals.dtype == torch.float64
        A.dtype = vals.dtype
        A.device = self.device
        A.stream = torch.cuda.current_stream(self.device).cuda_stream
        A.h = h
        _check(_L.nitro_spmv_set_stream(h, A.stream))
        return A

    def run(self, A: SpMV, v: int, x_local, y_local):
        _check(_L.nitro_dist_spmv_run(self.h, A.h, v, _ptr(x_local), _ptr(y_local)))
        return y_local

    def features(self, A: SpMV) -> dict:
        f = Feat()
        _check(_L.nitro_dist_features(self.h, A.h, ctypes.byref(f)))
        return f.as_dict()

    def loop(self, A: SpMV) -> "DistLoop":
        """Solver-loop mode (nitro_dist_loop_*, f3 (ii)): y -> next x fused into the epilogue."""
        return DistLoop(self, A)


class DistLoop:
    """nitro_dist_loop: x_{k+1} = A x_k with the exchange fused into the SpMV epilogue."""

    def __init__(self, D: "Dist", A: SpMV):
        h = ctypes.c_void_p()
        _check(_L.nitro_dist_loop_create(D.h, A.h, ctypes.byref(h)))
        self.h, self.D, self.A = h, D, A

    def x(self):
        """torch view of this rank's block of the current x (write x_0 here, then start())."""
        p = ctypes.c_void_p()
        _check(_L.nitro_dist_loop_x(self.h, ctypes.byref(p)))
        return _wrap_device(p.value, self.A.rows, self.A.dtype, self.A.device)

    def start(self):
        _check(_L.nitro_dist_loop_start(self.h))

    def step(self, v: int, y_local=None):
        _check(_L.nitro_dist_loop_step(self.h, v, None if y_local is None else
                                       _dev_vec(y_local, self.A.rows, self.A.dtype, self.A.device, "y_local")))
        return y_local

    def close(self):
        if getattr(self, "h", None):
            _L.nitro_dist_loop_destroy(self.h)
            self.h = None
