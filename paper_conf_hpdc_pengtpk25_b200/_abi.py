"""ctypes mirror of include/liteform.h and the loader of liblf.so.

The library must have been built (``python -m paper_conf_hpdc_pengtpk25_b200._build``
or ``__graft_entry__.build()``); importing without it raises -- there is no
fallback implementation.
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("LF_LIB") or os.path.join(_PKG, "liblf.so")  # LF_LIB: experiment builds
HEADER_PATH = os.path.join(os.path.dirname(_PKG), "include", "liteform.h")

LF_MAX_PARTS = 64
_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_I32 = ctypes.c_int32

STATUS = {0: "LF_OK", 1: "LF_ERR_INVALID_ARG", 2: "LF_ERR_UNSORTED_CSR", 3: "LF_ERR_INDEX_OVERFLOW",
          4: "LF_ERR_NO_MEMORY", 5: "LF_ERR_CUDA", 6: "LF_ERR_UNSUPPORTED"}


class LfError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{STATUS.get(status, status)}: {detail}")
        self.status = status
        self.detail = detail


class LfCsr(ctypes.Structure):
    _fields_ = [("n_rows", _I64), ("n_cols", _I64), ("nnz", _I64), ("row_ptr", _P), ("col_ind", _P), ("val", _P)]


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p)


class LfAllocator(ctypes.Structure):
    _fields_ = [("ctx", _P), ("alloc", ALLOC_FN), ("free", FREE_FN)]


class LfCellParams(ctypes.Structure):
    _fields_ = [("use_cell", _I32), ("n_parts", _I32), ("max_width_log2", ctypes.c_int8 * LF_MAX_PARTS),
                ("block_nnz_log2", ctypes.c_int8 * LF_MAX_PARTS)]

    def as_dict(self) -> dict:
        P = self.n_parts
        return {"use_cell": self.use_cell, "n_parts": P, "max_width_log2": list(self.max_width_log2[:P]),
                "block_nnz_log2": list(self.block_nnz_log2[:P])}


class LfConfigureOpts(ctypes.Structure):
    _fields_ = [("max_parts", _I32), ("block_mult_log2", _I32), ("force_parts", _I32),
                ("force_width_log2", _I32), ("force_format", _I32)]


_T32 = _I64 * 32


class LfConfigureStats(ctypes.Structure):
    _fields_ = [("features", ctypes.c_double * 8), ("n_parts", _I32), ("max_log2", _I32 * LF_MAX_PARTS),
                ("chosen_log2", _I32 * LF_MAX_PARTS), ("H", _T32 * LF_MAX_PARTS), ("F", _T32 * LF_MAX_PARTS),
                ("Unat", _T32 * LF_MAX_PARTS), ("Utop", _T32 * LF_MAX_PARTS), ("cost", _T32 * LF_MAX_PARTS),
                ("group_union_ratio", ctypes.c_double), ("spmm_grouped", _I32), ("spmm_tc", _I32),
                ("window_span_mean", ctypes.c_double), ("window_over_frac", ctypes.c_double)]


class LfBucket(ctypes.Structure):
    _fields_ = [("part", _I32), ("width_log2", _I32), ("rows_per_block", _I32), ("pad_", _I32),
                ("n_rows", _I64), ("n_rows_pad", _I64), ("row_off", _I64), ("slot_off", _I64)]


class LfCellArrays(ctypes.Structure):
    _fields_ = [("n_rows", _I64), ("n_cols", _I64), ("nnz", _I64), ("n_cell_rows", _I64), ("n_slots", _I64),
                ("n_buckets", _I32), ("pad_", _I32), ("row_ind", _P), ("col_ind", _P), ("val", _P),
                ("buckets", ctypes.POINTER(LfBucket)), ("params", LfCellParams)]


LF_MAX_DST = 8


class LfSpmmOpts(ctypes.Structure):
    _fields_ = [("n_dst", _I32), ("pad_", _I32), ("dst", ctypes.POINTER(ctypes.c_void_p)), ("row_base", _I64)]


# every symbol include/liteform.h declares, with its ctypes signature
SIGNATURES = {
    "lf_cell_configure": (_I32, [ctypes.POINTER(LfCsr), _I32, ctypes.POINTER(LfConfigureOpts),
                                 ctypes.POINTER(LfCellParams), ctypes.POINTER(LfConfigureStats), _P]),
    "lf_cell_build": (_I32, [ctypes.POINTER(LfCsr), ctypes.POINTER(LfCellParams), ctypes.POINTER(LfConfigureStats),
                             ctypes.POINTER(LfAllocator), _P, ctypes.POINTER(ctypes.c_void_p)]),
    "lf_spmm": (_I32, [_P, _P, _I64, _I32, _P, _I64, _P]),
    "lf_predict": (_I32, [ctypes.POINTER(ctypes.c_double), _I32, ctypes.POINTER(_I32), ctypes.POINTER(_I32)]),
    "lf_spmm_kernel_name": (ctypes.c_char_p, [_P, _I32]),
    "lf_spmm_ex": (_I32, [_P, _P, _I64, _I32, _P, _I64, ctypes.POINTER(LfSpmmOpts), _P]),
    "lf_csr_spmm": (_I32, [ctypes.POINTER(LfCsr), _P, _I64, _I32, _P, _I64, _P]),
    "lf_cell_view": (_I32, [_P, ctypes.POINTER(LfCellArrays)]),
    "lf_cell_destroy": (_I32, [_P]),
    "lf_status_string": (ctypes.c_char_p, [_I32]),
    "lf_last_error_detail": (ctypes.c_char_p, []),
    "lf_abi_version": (_I32, []),
}


def load(path: str = LIB_PATH) -> ctypes.CDLL:
    if not os.path.exists(path):
        raise ImportError(f"{path} is missing: build it with `python -m paper_conf_hpdc_pengtpk25_b200._build` "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(path)
    for name, (res, args) in SIGNATURES.items():
        if os.environ.get("LF_LIB") and not hasattr(L, name):
            continue  # an experiment / comparison build of another revision (LF_LIB) may predate a call
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    if L.lf_abi_version() != 1:
        raise ImportError("liblf.so ABI version mismatch")
    return L


lib = load()


def check(status: int) -> None:
    if status != 0:
        raise LfError(status, (lib.lf_last_error_detail() or b"").decode())


# ---- PyTorch caching allocator bridge ------------------------------------
_alloc_obj = None


def torch_allocator() -> LfAllocator:
    """lf_allocator backed by torch.cuda's caching allocator (stream-aware)."""
    global _alloc_obj
    if _alloc_obj is None:
        import torch

        @ALLOC_FN
        def _alloc(ctx, nbytes, stream):
            try:
                return int(torch.cuda.caching_allocator_alloc(int(nbytes), torch.cuda.current_device(),
                                                              int(stream or 0)))
            except Exception:
                return None

        @FREE_FN
        def _free(ctx, ptr, nbytes, stream):
            torch.cuda.caching_allocator_delete(int(ptr))

        _alloc_obj = (LfAllocator(None, _alloc, _free), _alloc, _free)
    return _alloc_obj[0]
