"""LiteForm hot path on B200: CSR -> CELL conversion and the CELL SpMM.

Thin Python binding over ``liblf.so`` (C ABI in ``include/liteform.h``):
argument marshalling only -- every step of the path runs in the library's
sm_100a kernels.  PyTorch provides device memory (through its caching
allocator), streams and process groups.  There is no CPU fallback: importing
this package without the built library raises.

    import paper_conf_hpdc_pengtpk25_b200 as lf
    A = lf.Csr(row_ptr, col_ind, val, n_cols)          # CUDA tensors
    params, stats = lf.configure(A, J)                  # eq. 7 + Algorithm 3
    M = lf.CellMatrix.build(A, params)                  # GPU CSR -> CELL
    C = M.spmm(B)                                       # C = A . B
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import torch

from . import _abi
from ._abi import (LF_MAX_PARTS, LfCsr, LfCellParams, LfConfigureOpts, LfConfigureStats, LfCellArrays,
                   LfError, lib)

__all__ = ["Csr", "CellMatrix", "configure", "predict", "csr_spmm", "library_path", "LfError", "LF_MAX_PARTS"]


def library_path() -> str:
    return _abi.LIB_PATH


def _stream(stream=None) -> int:
    if stream is None:
        stream = torch.cuda.current_stream()
    return int(stream.cuda_stream) if hasattr(stream, "cuda_stream") else int(stream)


@dataclass
class Csr:
    """CSR operand on the GPU: int64 row_ptr[I+1], int32 col_ind, float32 val.
    ``row_ptr`` may be a slice of a larger CSR (row shard): positions stay
    absolute indexes into col_ind / val."""
    row_ptr: torch.Tensor
    col_ind: torch.Tensor
    val: torch.Tensor
    n_cols: int
    nnz: int | None = None

    def __post_init__(self):
        for name, t, dt in (("row_ptr", self.row_ptr, torch.int64), ("col_ind", self.col_ind, torch.int32),
                            ("val", self.val, torch.float32)):
            if not t.is_cuda or t.dtype != dt or not t.is_contiguous():
                raise TypeError(f"{name} must be a contiguous CUDA {dt} tensor")
        if self.nnz is None:
            self.nnz = int(self.row_ptr[-1].item() - self.row_ptr[0].item()) if self.row_ptr.numel() else 0

    @property
    def n_rows(self) -> int:
        return self.row_ptr.numel() - 1

    def c(self) -> LfCsr:
        return LfCsr(self.n_rows, self.n_cols, self.nnz, self.row_ptr.data_ptr(), self.col_ind.data_ptr(),
                     self.val.data_ptr())

    @staticmethod
    def from_host(h, device="cuda", non_blocking=False) -> "Csr":
        """From a host CSR with numpy arrays (gen.CSR)."""
        def to(a, dt):
            return torch.from_numpy(a).to(device=device, dtype=dt, non_blocking=non_blocking)
        return Csr(to(h.row_ptr, torch.int64), to(h.col_ind, torch.int32), to(h.val, torch.float32), h.n_cols,
                   int(h.row_ptr[-1] - h.row_ptr[0]))


def configure(A: Csr, J: int, *, max_parts: int = 0, block_mult_log2: int = 0, force_parts: int = 0,
              force_width_log2: int = -1, force_format: int = 0, stream=None):
    """Automatic CELL composition (section 5): returns
    (LfCellParams, LfConfigureStats).  force_parts / force_format = 0 leave
    P / the format to the predictor (lf_predict)."""
    opts = LfConfigureOpts(max_parts, block_mult_log2, force_parts, force_width_log2, force_format)
    params = LfCellParams()
    stats = LfConfigureStats()
    csr = A.c()
    _abi.check(lib.lf_cell_configure(ctypes.byref(csr), int(J), ctypes.byref(opts), ctypes.byref(params),
                                     ctypes.byref(stats), _stream(stream)))
    return params, stats


def predict(features, max_parts: int = 0) -> tuple[int, int]:
    """lf_predict (sections 5.1-5.2): (use_cell, P) from the 8 Table 2/3
    features (n_rows, n_cols, nnz, mean, min, max, std of row lengths, J).
    Host only; no GPU needed."""
    f = (ctypes.c_double * 8)(*[float(x) for x in features])
    u, p = ctypes.c_int32(), ctypes.c_int32()
    _abi.check(lib.lf_predict(f, int(max_parts), ctypes.byref(u), ctypes.byref(p)))
    return int(u.value), int(p.value)


def make_params(n_parts: int, e, k=None, use_cell: int = 1) -> LfCellParams:
    """Explicit CELL parameters: P partitions, max width 2^e[p], block 2^k[p]."""
    if isinstance(e, int):
        e = [e] * n_parts
    if k is None:
        k = list(e)
    elif isinstance(k, int):
        k = [k] * n_parts
    p = LfCellParams()
    p.use_cell = use_cell
    p.n_parts = n_parts
    for i in range(n_parts):
        p.max_width_log2[i] = int(e[i])
        p.block_nnz_log2[i] = int(k[i])
    return p


class CellMatrix:
    """A built CELL handle (lf_cell*).  Device arrays are owned by the handle
    and allocated through PyTorch's caching allocator."""

    def __init__(self, handle, A: Csr, params: LfCellParams):
        self._h = handle
        self._A = A  # keeps the CSR alive (use_cell = 0 reads it at spmm time)
        self.params = params
        self.n_rows = A.n_rows
        self.n_cols = A.n_cols

    @staticmethod
    def build(A: Csr, params: LfCellParams, stats: LfConfigureStats | None = None, stream=None) -> "CellMatrix":
        """GPU CSR -> CELL.  Passing the stats lf.configure returned for this A
        lets the build run without a host synchronisation."""
        h = ctypes.c_void_p()
        csr = A.c()
        _abi.check(lib.lf_cell_build(ctypes.byref(csr), ctypes.byref(params),
                                     ctypes.byref(stats) if stats is not None else None,
                                     ctypes.byref(_abi.torch_allocator()), _stream(stream), ctypes.byref(h)))
        return CellMatrix(h, A, params)

    def spmm(self, B: torch.Tensor, out: torch.Tensor | None = None, stream=None, dst=None,
             row_base: int = 0) -> torch.Tensor | None:
        """C = A . B (overwrites out).  B: [K, J] fp32 CUDA, row-major (row stride = ldb).

        dst: fused row exchange (lf_spmm_ex) -- a list of full-C destinations
        (tensors [I_total, J] with unit column stride and a common row stride,
        or raw device addresses); row i of this matrix is written to row
        row_base + i of every destination straight from the kernel, and out is
        not used.  Returns out (None with dst)."""
        if B.dtype != torch.float32 or not B.is_cuda or B.dim() != 2 or B.stride(1) != 1:
            raise TypeError("B must be a 2-D CUDA float32 tensor with unit column stride")
        if B.shape[0] != self.n_cols:
            raise ValueError(f"B has {B.shape[0]} rows, A has {self.n_cols} columns")
        J = B.shape[1]
        if dst is not None:
            ptrs, ldc = [], None
            for t in dst:
                if isinstance(t, torch.Tensor):
                    if t.dtype != torch.float32 or t.dim() != 2 or t.stride(1) != 1 or t.shape[1] != J:
                        raise ValueError("each destination must be [I_total, J] float32 with unit column stride")
                    if t.shape[0] < row_base + self.n_rows:
                        raise ValueError("destination has fewer rows than row_base + n_rows")
                    if ldc is not None and t.stride(0) != ldc:
                        raise ValueError("destinations must share one row stride")
                    ldc = t.stride(0)
                    ptrs.append(t.data_ptr())
                else:
                    ptrs.append(int(t))
            ldc = max(ldc or J, J)
            arr = (ctypes.c_void_p * len(ptrs))(*ptrs)
            opts = _abi.LfSpmmOpts(len(ptrs), 0, ctypes.cast(arr, ctypes.POINTER(ctypes.c_void_p)), int(row_base))
            self._J = J
            _abi.check(lib.lf_spmm_ex(self._h, B.data_ptr(), max(B.stride(0), J), J, None, ldc, ctypes.byref(opts),
                                      _stream(stream)))
            return None
        if out is None:
            out = torch.empty((self.n_rows, J), dtype=torch.float32, device=B.device)
        if out.shape != (self.n_rows, J) or out.stride(1) != 1 or out.dtype != torch.float32:
            raise ValueError("out must be [I, J] float32 with unit column stride")
        self._J = J
        _abi.check(lib.lf_spmm(self._h, B.data_ptr(), max(B.stride(0), J), J, out.data_ptr(),
                               max(out.stride(0), J), _stream(stream)))
        return out

    def path(self, J: int | None = None) -> str:
        """Kernel family lf_spmm runs for this handle (aligned B / C, ldb = ldc = J)."""
        J = int(J if J is not None else getattr(self, "_J", 0) or 0)
        return (lib.lf_spmm_kernel_name(self._h, J) or b"").decode()

    def view(self) -> dict:
        """The CELL arrays (zero-copy CUDA tensors valid while self lives) and the
        bucket table (list of dicts)."""
        v = LfCellArrays()
        _abi.check(lib.lf_cell_view(self._h, ctypes.byref(v)))
        dev = torch.cuda.current_device()

        def wrap(ptr, n, typestr, dtype):
            if n == 0 or not ptr:
                return torch.empty(0, dtype=dtype, device="cuda")
            obj = type("CAI", (), {"__cuda_array_interface__": {
                "shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 2}})()
            return torch.as_tensor(obj, device=f"cuda:{dev}")

        buckets = [{f: getattr(v.buckets[i], f) for f, _ in _abi.LfBucket._fields_ if f != "pad_"}
                   for i in range(v.n_buckets)]
        return {"row_ind": wrap(v.row_ind, v.n_cell_rows, "<i4", torch.int32),
                "col_ind": wrap(v.col_ind, v.n_slots, "<i4", torch.int32),
                "val": wrap(v.val, v.n_slots, "<f4", torch.float32),
                "buckets": buckets, "n_cell_rows": v.n_cell_rows, "n_slots": v.n_slots}

    def close(self):
        if self._h:
            lib.lf_cell_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def csr_spmm(A: Csr, B: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """Algorithm 1 on the GPU directly from CSR (the fixed-format path)."""
    J = B.shape[1]
    if out is None:
        out = torch.empty((A.n_rows, J), dtype=torch.float32, device=B.device)
    csr = A.c()
    _abi.check(lib.lf_csr_spmm(ctypes.byref(csr), B.data_ptr(), max(B.stride(0), J), J, out.data_ptr(),
                               max(out.stride(0), J), _stream(stream)))
    return out
