"""Thin ctypes binding of libbro.so (include/bro.h) — argument marshalling only.

Every step of SpMV runs in the library's CUDA kernels; this module converts
numpy / torch arguments to pointers and raises BroError on a non-zero status.
There is no CPU fallback: if libbro.so is missing, importing this module
fails.  PyTorch is used only for device tensors and streams (plumbing).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libbro.so")
if not os.path.exists(_LIB_PATH):
    raise ImportError(f"libbro.so not built ({_LIB_PATH}); run __graft_entry__.build() "
                      "or python -m paper_conf_sc_tangtrwckgtw13_b200._build")
_lib = C.CDLL(_LIB_PATH)

BRO_FP32, BRO_FP64 = 0, 1
BRO_DEVICE_HOST_ONLY = -1
STATUS = {0: "BRO_OK", 1: "BRO_ERR_ARG", 2: "BRO_ERR_INDEX", 3: "BRO_ERR_SHAPE",
          4: "BRO_ERR_OOM", 5: "BRO_ERR_CUDA", 6: "BRO_ERR_UNSUPPORTED"}
PARTS = {
    "ell_words": 0, "ell_bit_alloc": 1, "ell_colptr": 2, "ell_symptr": 3, "ell_vals": 4,
    "coo_words": 5, "coo_base_row": 6, "coo_width": 7, "coo_symptr": 8, "coo_col": 9,
    "coo_vals": 10, "coo_row": 11, "pell_col": 12, "pell_vals": 13, "ell_vcodes": 14, "ell_vdict": 15,
}
FORMATS = {0: "ELL", 1: "COO", 2: "HYB"}


class bro_opts_t(C.Structure):
    _fields_ = [("slice_h", C.c_int32), ("sym_bits", C.c_int32), ("vec_words", C.c_int32),
                ("coo_T", C.c_int32), ("hyb_K", C.c_int64), ("codec", C.c_int32),
                ("min_bits", C.c_int32), ("ell_kernel", C.c_int32), ("pdl", C.c_int32),
                ("x_stage", C.c_int32), ("value_codec", C.c_int32)]


class bro_info_t(C.Structure):
    _fields_ = [("m", C.c_int64), ("n", C.c_int64), ("nnz", C.c_int64),
                ("dtype", C.c_int32), ("codec", C.c_int32), ("format", C.c_int32),
                ("vec_words", C.c_int32), ("slice_h", C.c_int32), ("coo_T", C.c_int32),
                ("ell_kernel", C.c_int32), ("x_stage_bytes", C.c_int32),
                ("K", C.c_int64), ("nnz_ell", C.c_int64),
                ("nnz_coo", C.c_int64), ("n_slices", C.c_int64), ("ell_slots", C.c_int64),
                ("ell_pitch", C.c_int64), ("n_intervals", C.c_int64),
                ("ell_stream_bytes", C.c_int64), ("coo_stream_bytes", C.c_int64),
                ("meta_bytes", C.c_int64), ("index_bytes", C.c_int64), ("value_bytes", C.c_int64),
                ("device_bytes", C.c_int64), ("algorithmic_bytes", C.c_int64),
                ("orig_index_bytes", C.c_int64), ("eta_stream", C.c_double),
                ("eta_total", C.c_double), ("encode_seconds", C.c_double),
                ("value_code_bytes", C.c_int32), ("reserved0", C.c_int32), ("value_dict_size", C.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_P = C.c_void_p
_H = C.c_void_p
_sig = {
    "bro_opts_default": (None, [C.POINTER(bro_opts_t)]),
    "bro_create_ell": (C.c_int, [C.c_int, C.c_int, C.c_int64, C.c_int64, _P, _P, _P,
                                 C.POINTER(bro_opts_t), C.POINTER(_H)]),
    "bro_create_hyb": (C.c_int, [C.c_int, C.c_int, C.c_int64, C.c_int64, _P, _P, _P,
                                 C.POINTER(bro_opts_t), C.POINTER(_H)]),
    "bro_create_coo": (C.c_int, [C.c_int, C.c_int, C.c_int64, C.c_int64, C.c_int64, _P, _P, _P,
                                 C.POINTER(bro_opts_t), C.POINTER(_H)]),
    "bro_spmv": (C.c_int, [_H, _P, _P, _P]),
    "bro_spmv_host": (C.c_int, [_H, _P, _P, _P]),
    "bro_spmv_scatter": (C.c_int, [_H, _P, C.POINTER(C.c_void_p), C.c_int32, _P, _P]),
    "bro_destroy": (C.c_int, [_H]),
    "bro_get_info": (C.c_int, [_H, C.POINTER(bro_info_t)]),
    "bro_export_encoded": (C.c_int, [_H, C.c_int32, _P, C.POINTER(C.c_size_t)]),
    "bro_decode_indices": (C.c_int, [_H, _P, _P, _P]),
    "bro_hyb_K": (C.c_int, [C.c_int64, _P, C.POINTER(C.c_int64)]),
    "bro_reorder_bar": (C.c_int, [C.c_int64, C.c_int64, _P, _P, C.c_int, C.c_int32, C.c_int32, _P]),
    "bro_status_str": (C.c_char_p, [C.c_int]),
    "bro_last_error": (C.c_char_p, []),
    "bro_version": (C.c_int, []),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED_SYMBOLS = tuple(_sig)


class BroError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = _lib.bro_last_error().decode()
        super().__init__(f"{where}: {STATUS.get(status, status)}: {msg}")


def _check(status: int, where: str):
    if status != 0:
        raise BroError(status, where)


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _dtype_code(dtype) -> int:
    dt = np.dtype(dtype)
    if dt == np.float64:
        return BRO_FP64
    if dt == np.float32:
        return BRO_FP32
    raise TypeError(f"unsupported value dtype {dt}")


def bro_opts_default(**overrides) -> bro_opts_t:
    o = bro_opts_t()
    _lib.bro_opts_default(C.byref(o))
    for k, v in overrides.items():
        setattr(o, k, v)
    return o


def _csr_args(row_ptr, col_idx, vals):
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    vals = np.ascontiguousarray(vals)
    return row_ptr, col_idx, vals


def bro_create_ell(device, m, n, row_ptr, col_idx, vals, opts=None) -> int:
    row_ptr, col_idx, vals = _csr_args(row_ptr, col_idx, vals)
    h = _H()
    _check(_lib.bro_create_ell(device, _dtype_code(vals.dtype), m, n, _ptr(row_ptr), _ptr(col_idx),
                               _ptr(vals), C.byref(opts or bro_opts_default()), C.byref(h)),
           "bro_create_ell")
    return h.value


def bro_create_hyb(device, m, n, row_ptr, col_idx, vals, opts=None) -> int:
    row_ptr, col_idx, vals = _csr_args(row_ptr, col_idx, vals)
    h = _H()
    _check(_lib.bro_create_hyb(device, _dtype_code(vals.dtype), m, n, _ptr(row_ptr), _ptr(col_idx),
                               _ptr(vals), C.byref(opts or bro_opts_default()), C.byref(h)),
           "bro_create_hyb")
    return h.value


def bro_create_coo(device, m, n, row_idx, col_idx, vals, opts=None) -> int:
    row_idx = np.ascontiguousarray(row_idx, dtype=np.int32)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    vals = np.ascontiguousarray(vals)
    h = _H()
    _check(_lib.bro_create_coo(device, _dtype_code(vals.dtype), m, n, int(row_idx.size), _ptr(row_idx),
                               _ptr(col_idx), _ptr(vals), C.byref(opts or bro_opts_default()),
                               C.byref(h)), "bro_create_coo")
    return h.value


def bro_spmv(h: int, x_dev_ptr: int, y_dev_ptr: int, stream_ptr: int = 0):
    _check(_lib.bro_spmv(h, x_dev_ptr, y_dev_ptr, stream_ptr or None), "bro_spmv")


BRO_MAX_DST = 8


def bro_spmv_scatter(h: int, x_dev_ptr: int, y_dst_ptrs, y_mc_ptr: int = 0, stream_ptr: int = 0):
    """y stored into every device address of y_dst_ptrs (first = local y), or
    through the multicast address y_mc_ptr (include/bro.h)."""
    n = len(y_dst_ptrs)
    arr = (C.c_void_p * max(n, 1))(*[int(p) for p in y_dst_ptrs])
    _check(_lib.bro_spmv_scatter(h, x_dev_ptr, arr, n, y_mc_ptr or None, stream_ptr or None),
           "bro_spmv_scatter")


def bro_spmv_host(h: int, x: np.ndarray, y: np.ndarray, stream_ptr: int = 0):
    """Raw call: x (n values) and y (m values) must be C-contiguous host arrays
    of the handle's dtype (BroMatrix.spmv_host checks them)."""
    if not (x.flags.c_contiguous and y.flags.c_contiguous):
        raise ValueError("x and y must be C-contiguous")
    _check(_lib.bro_spmv_host(h, _ptr(x), _ptr(y), stream_ptr or None), "bro_spmv_host")


def bro_destroy(h: int):
    _check(_lib.bro_destroy(h), "bro_destroy")


def bro_get_info(h: int) -> dict:
    info = bro_info_t()
    _check(_lib.bro_get_info(h, C.byref(info)), "bro_get_info")
    return info.as_dict()


_PART_DTYPES = {0: np.uint32, 1: np.uint8, 2: np.uint64, 3: np.uint64, 5: np.uint32, 6: np.uint32,
                7: np.uint8, 8: np.uint64, 9: np.int32, 11: np.int32, 12: np.int32, 14: np.uint8}


def bro_export_encoded(h: int, part, value_dtype=None) -> np.ndarray:
    p = PARTS[part] if isinstance(part, str) else int(part)
    n = C.c_size_t(0)
    _check(_lib.bro_export_encoded(h, p, None, C.byref(n)), "bro_export_encoded")
    buf = np.zeros(n.value, dtype=np.uint8)
    _check(_lib.bro_export_encoded(h, p, _ptr(buf), C.byref(n)), "bro_export_encoded")
    dt = _PART_DTYPES.get(p, value_dtype if value_dtype is not None else np.uint8)
    return buf.view(dt)


def bro_decode_indices(h: int, d_ell_cols_ptr: int, d_coo_rows_ptr: int, stream_ptr: int = 0):
    _check(_lib.bro_decode_indices(h, d_ell_cols_ptr or None, d_coo_rows_ptr or None, stream_ptr or None),
           "bro_decode_indices")


def bro_hyb_K(row_ptr) -> int:
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    K = C.c_int64(0)
    _check(_lib.bro_hyb_K(row_ptr.size - 1, _ptr(row_ptr), C.byref(K)), "bro_hyb_K")
    return K.value


def bro_reorder_bar(m, n, row_ptr, col_idx, dtype=np.float64, method=0, window=0) -> np.ndarray:
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    perm = np.zeros(m, dtype=np.int64)
    _check(_lib.bro_reorder_bar(m, n, _ptr(row_ptr), _ptr(col_idx), _dtype_code(dtype), method, window,
                                _ptr(perm)), "bro_reorder_bar")
    return perm


def bro_status_str(s: int) -> str:
    return _lib.bro_status_str(s).decode()


def bro_last_error() -> str:
    return _lib.bro_last_error().decode()


def bro_version() -> int:
    return _lib.bro_version()


# ---------------------------------------------------------------------------
# convenience handle over torch device tensors
# ---------------------------------------------------------------------------

class BroMatrix:
    """Owns one libbro handle.  `fmt` in {"ell", "hyb", "coo"}; codec=1 gives
    BRO-ELL / BRO-HYB / BRO-COO, codec=0 the uncompressed baseline.  Every
    call checks the vectors' dtype, length, contiguity and device before the
    pointers reach the library (the C ABI cannot)."""

    def __init__(self, A, fmt="ell", codec=1, device=0, dtype=None, vec_words=0, hyb_K=-1, min_bits=0,
                 slice_h=0, coo_T=0, ell_kernel=0, pdl=0, x_stage=0, value_codec=0):
        vals = A.vals if dtype is None else A.vals.astype(dtype)
        self.dtype = np.dtype(vals.dtype)
        self.m, self.n, self.fmt, self.device = A.m, A.n, fmt, device
        opts = bro_opts_default(codec=codec, vec_words=vec_words, hyb_K=hyb_K, min_bits=min_bits,
                                slice_h=slice_h, coo_T=coo_T, ell_kernel=ell_kernel, pdl=pdl,
                                x_stage=x_stage, value_codec=value_codec)
        if fmt == "ell":
            self.h = bro_create_ell(device, A.m, A.n, A.row_ptr, A.col, vals, opts)
        elif fmt == "hyb":
            self.h = bro_create_hyb(device, A.m, A.n, A.row_ptr, A.col, vals, opts)
        elif fmt == "coo":
            rows = np.repeat(np.arange(A.m, dtype=np.int32), np.diff(A.row_ptr))
            self.h = bro_create_coo(device, A.m, A.n, rows, A.col, vals, opts)
        else:
            raise ValueError(fmt)
        self.info = bro_get_info(self.h)

    def _tdtype(self):
        import torch
        return torch.float64 if self.dtype == np.float64 else torch.float32

    def _check_vec(self, v, length, name):
        if not (v.is_cuda and v.dtype == self._tdtype() and v.is_contiguous() and v.numel() == length
                and (v.device.index or 0) == self.device):
            raise ValueError(f"{name} must be a contiguous CUDA tensor of the matrix dtype ({self.dtype}), "
                             f"{length} elements, on cuda:{self.device}")

    def spmv(self, x, y=None, stream=None):
        """y = A.x for torch CUDA tensors on the handle's device (async)."""
        import torch
        self._check_vec(x, self.n, "x")
        if y is None:
            y = torch.empty(self.m, dtype=self._tdtype(), device=x.device)
        self._check_vec(y, self.m, "y")
        if stream is None:
            stream = torch.cuda.current_stream(x.device)
        bro_spmv(self.h, x.data_ptr(), y.data_ptr(), stream.cuda_stream)
        return y

    def spmv_scatter(self, x, y_dst_ptrs, y_mc_ptr=0, stream=None):
        """y = A.x stored into every device address of y_dst_ptrs (each m
        values of the matrix dtype; the first is the local y) — the fused
        exchange of dist.py."""
        import torch
        self._check_vec(x, self.n, "x")
        if stream is None:
            stream = torch.cuda.current_stream(x.device)
        bro_spmv_scatter(self.h, x.data_ptr(), y_dst_ptrs, y_mc_ptr, stream.cuda_stream)

    def spmv_host(self, x: np.ndarray, y: np.ndarray = None, stream=None):
        """End to end with host vectors (x: n values, y: m values)."""
        x = np.ascontiguousarray(x, dtype=self.dtype)
        if x.shape != (self.n,):
            raise ValueError(f"x must have {self.n} elements")
        if y is None:
            y = np.empty(self.m, dtype=self.dtype)
        if not (isinstance(y, np.ndarray) and y.dtype == self.dtype and y.shape == (self.m,)
                and y.flags.c_contiguous and y.flags.writeable):
            raise ValueError(f"y must be a writeable C-contiguous {self.dtype} array of {self.m} elements")
        sp = 0
        if stream is not None:
            sp = stream.cuda_stream
        bro_spmv_host(self.h, x, y, sp)
        return y

    def decode_indices(self):
        """GPU decode through the handle's own kernels (decode mode): returns
        (ell_cols, coo_rows) as torch int32 CUDA tensors (include/bro.h)."""
        import torch
        dev = torch.device("cuda", self.device)
        cols = torch.empty(max(self.info["ell_slots"], 1), dtype=torch.int32, device=dev)
        rows = torch.empty(max(self.info["nnz_coo"], 1), dtype=torch.int32, device=dev)
        bro_decode_indices(self.h, cols.data_ptr(), rows.data_ptr(),
                           torch.cuda.current_stream(dev).cuda_stream)
        return cols[:self.info["ell_slots"]], rows[:self.info["nnz_coo"]]

    def export(self, part):
        return bro_export_encoded(self.h, part, self.dtype)

    def close(self):
        if getattr(self, "h", None):
            bro_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
