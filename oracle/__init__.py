"""CPU oracle for LiteForm's hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` leg may import this package.  The
product path (``paper_conf_hpdc_pengtpk25_b200``) never imports it and shares
no code with it.

The arithmetic lives in plain C (``lf_oracle.c``, fp64, each function citing
the PAPER.md passage it follows); this module only marshals numpy arrays.
Readings of the paper that the oracle adopts are SURVEY.md 8(c) C1-C17,
restated in DESIGN.md.  Parity status: every function is pinned by
``tests/test_oracle_*.py`` except the format/partition *predictor*, which the
oracle does not implement ("parity unpinned").
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lf_oracle.c")
_LIB = os.path.join(_HERE, "liblforacle.so")


def build(force: bool = False) -> str:
    """gcc -O2 -fopenmp, no -ffast-math (SURVEY 8(d) timing protocol)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11", "-Wall",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class Bucket(ctypes.Structure):
    _fields_ = [("part", ctypes.c_int32), ("width_log2", ctypes.c_int32), ("rows_per_block", ctypes.c_int32),
                ("pad_", ctypes.c_int32), ("n_rows", ctypes.c_int64), ("n_rows_pad", ctypes.c_int64),
                ("row_off", ctypes.c_int64), ("slot_off", ctypes.c_int64)]


BUCKET_DTYPE = np.dtype([("part", np.int32), ("width_log2", np.int32), ("rows_per_block", np.int32),
                         ("pad_", np.int32), ("n_rows", np.int64), ("n_rows_pad", np.int64),
                         ("row_off", np.int64), ("slot_off", np.int64)])

_lib = None
_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_I32 = ctypes.c_int32


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.lfo_spmm_csr.argtypes = [_I64, _P, _I64, _P, _P, _P, _P, _I64, _P, _P]
        _lib.lfo_csr_to_cell.argtypes = [_I64, _I64, _P, _P, _P, _I32, _P, _P, _P, _P, _P, _P, _P, _P, _P]
        _lib.lfo_csr_to_cell.restype = ctypes.c_int
        _lib.lfo_cell_to_csr.argtypes = [_I64, _I32, _P, _P, _P, _P, _P, _P, _P]
        _lib.lfo_cell_to_csr.restype = _I64
        _lib.lfo_cell_spmm.argtypes = [_I64, _I64, _I32, _P, _P, _P, _P, _P, _I64, _P]
        _lib.lfo_partition_cost.argtypes = [_I64, _I64, _P, _P, _I32, _I32, _I32, _I64]
        _lib.lfo_partition_cost.restype = _I64
        _lib.lfo_partition_max_log2.argtypes = [_I64, _I64, _P, _P, _I32, _I32]
        _lib.lfo_partition_max_log2.restype = _I32
        _lib.lfo_build_buckets.argtypes = [_I64, _I64, _P, _P, _I32, _I32, _I64]
        _lib.lfo_build_buckets.restype = _I32
        _lib.lfo_build_buckets_literal.argtypes = [_I64, _I64, _P, _P, _I32, _I32, _I64]
        _lib.lfo_build_buckets_literal.restype = _I64
        _lib.lfo_partition_stats.argtypes = [_I64, _I64, _P, _P, _I32, _I32, _P, _P, _P, _P]
        _lib.lfo_features.argtypes = [_I64, _I64, _P, _P]
        _lib.lfo_set_threads.argtypes = [_I32]
        _lib.lfo_set_threads.restype = _I32
    return _lib


def _c(a, dtype):
    a = np.ascontiguousarray(a, dtype=dtype)
    return a, a.ctypes.data


def spmm_csr(A, B: np.ndarray, rows: np.ndarray | None = None, with_abs: bool = True):
    """Algorithm 1 in fp64.  Returns (C, Cabs) as float64 [n_out, J]; rows
    selects a sample of output rows (full-size parity checks)."""
    rp, prp = _c(A.row_ptr, np.int64)
    ci, pci = _c(A.col_ind, np.int32)
    va, pva = _c(A.val, np.float32)
    B = np.ascontiguousarray(B, dtype=np.float32)
    J = B.shape[1]
    if rows is None:
        n_out, prow = A.n_rows, None
    else:
        rows, prow = _c(rows, np.int64)
        n_out = len(rows)
    C = np.empty((n_out, J), np.float64)
    Cabs = np.empty((n_out, J), np.float64) if with_abs else None
    _L().lfo_spmm_csr(n_out, prow, J, prp, pci, pva, B.ctypes.data if B.size else None, J, C.ctypes.data,
                      Cabs.ctypes.data if with_abs else None)
    return C, Cabs


@dataclass
class Cell:
    """Oracle CELL arrays (readings C1-C7)."""
    row_ind: np.ndarray      # int32 [R_tot]
    col_ind: np.ndarray      # int32 [S_tot]
    val: np.ndarray          # float32 [S_tot]
    buckets: np.ndarray      # BUCKET_DTYPE [n_buckets]
    n_rows: int              # I of the source matrix


def _params(P, e, k):
    e = np.ascontiguousarray(np.broadcast_to(np.asarray(e, np.int8), (P,)))
    k = np.ascontiguousarray(np.broadcast_to(np.asarray(k, np.int8), (P,)))
    return e, k


def csr_to_cell(A, P: int, e, k=None) -> Cell:
    """CSR -> CELL with P partitions, max width 2^e[p], block 2^k[p] slots
    (k defaults to e: multiplier 1, reading C2)."""
    e, k = _params(P, e, e if k is None else k)
    rp, prp = _c(A.row_ptr, np.int64)
    ci, pci = _c(A.col_ind, np.int32)
    va, pva = _c(A.val, np.float32)
    R, S, nb = _I64(), _I64(), _I32()
    L = _L()
    rc = L.lfo_csr_to_cell(A.n_rows, A.n_cols, prp, pci, pva, P, e.ctypes.data, k.ctypes.data, ctypes.byref(R),
                           ctypes.byref(S), ctypes.byref(nb), None, None, None, None)
    if rc != 0:
        raise ValueError("bad CELL parameters")
    row_ind = np.empty(R.value, np.int32)
    col_ind = np.empty(S.value, np.int32)
    val = np.empty(S.value, np.float32)
    buckets = np.zeros(nb.value, BUCKET_DTYPE)
    rc = L.lfo_csr_to_cell(A.n_rows, A.n_cols, prp, pci, pva, P, e.ctypes.data, k.ctypes.data, ctypes.byref(R),
                           ctypes.byref(S), ctypes.byref(nb), row_ind.ctypes.data, col_ind.ctypes.data,
                           val.ctypes.data, buckets.ctypes.data)
    assert rc == 0
    return Cell(row_ind, col_ind, val, buckets, A.n_rows)


def cell_to_csr(cell: Cell):
    """Inverse conversion; returns (row_ptr, col_ind, val)."""
    I = cell.n_rows
    rp = np.empty(I + 1, np.int64)
    ci = np.empty(max(len(cell.col_ind), 1), np.int32)
    va = np.empty(max(len(cell.col_ind), 1), np.float32)
    b = np.ascontiguousarray(cell.buckets)
    nnz = _L().lfo_cell_to_csr(I, len(b), b.ctypes.data, cell.row_ind.ctypes.data, cell.col_ind.ctypes.data,
                               cell.val.ctypes.data, rp.ctypes.data, ci.ctypes.data, va.ctypes.data)
    if nnz < 0:
        raise ValueError("real slot inside a padding row")
    return rp, ci[:nnz], va[:nnz]


def cell_spmm(cell: Cell, B: np.ndarray) -> np.ndarray:
    """Algorithm 2 over every block of every bucket, fp64."""
    B = np.ascontiguousarray(B, dtype=np.float32)
    J = B.shape[1]
    C = np.empty((cell.n_rows, J), np.float64)
    b = np.ascontiguousarray(cell.buckets)
    _L().lfo_cell_spmm(cell.n_rows, J, len(b), b.ctypes.data, cell.row_ind.ctypes.data, cell.col_ind.ctypes.data,
                       cell.val.ctypes.data, B.ctypes.data if B.size else None, J, C.ctypes.data)
    return C


def partition_cost(A, P: int, p: int, e: int, J: int) -> int:
    """Eq. 7 summed over partition p's buckets for max width 2^e (materialised)."""
    rp, prp = _c(A.row_ptr, np.int64)
    ci, pci = _c(A.col_ind, np.int32)
    return int(_L().lfo_partition_cost(A.n_rows, A.n_cols, prp, pci, P, p, e, J))


def partition_max_log2(A, P: int, p: int) -> int:
    rp, prp = _c(A.row_ptr, np.int64)
    ci, pci = _c(A.col_ind, np.int32)
    return int(_L().lfo_partition_max_log2(A.n_rows, A.n_cols, prp, pci, P, p))


def build_buckets(A, P: int, p: int, J: int) -> int:
    """Algorithm 3 (exponent space): log2 of the partition's max width, -1 if empty."""
    rp, prp = _c(A.row_ptr, np.int64)
    ci, pci = _c(A.col_ind, np.int32)
    return int(_L().lfo_build_buckets(A.n_rows, A.n_cols, prp, pci, P, p, J))


def build_buckets_literal(A, P: int, p: int, J: int) -> int:
    """Algorithm 3 read literally in width space; returns the WIDTH."""
    rp, prp = _c(A.row_ptr, np.int64)
    ci, pci = _c(A.col_ind, np.int32)
    return int(_L().lfo_build_buckets_literal(A.n_rows, A.n_cols, prp, pci, P, p, J))


def configure(A, P: int, J: int, block_mult_log2: int = 0):
    """Per-partition (e_p, k_p) via Algorithm 3; empty partitions get e=k=0."""
    e = []
    for p in range(P):
        ep = build_buckets(A, P, p, J)
        e.append(max(ep, 0))
    e = np.array(e, np.int8)
    return e, (e + block_mult_log2).astype(np.int8)


def partition_stats(A, P: int, p: int):
    """(H, F, Unat, Utop) int64[32] from their set definitions."""
    rp, prp = _c(A.row_ptr, np.int64)
    ci, pci = _c(A.col_ind, np.int32)
    out = [np.zeros(32, np.int64) for _ in range(4)]
    _L().lfo_partition_stats(A.n_rows, A.n_cols, prp, pci, P, p, *[o.ctypes.data for o in out])
    return tuple(out)


def features(A) -> np.ndarray:
    """Table 2 features: n_rows, n_cols, nnz, mean, min, max, std of row nnz."""
    rp, prp = _c(A.row_ptr, np.int64)
    out = np.zeros(7, np.float64)
    _L().lfo_features(A.n_rows, A.n_cols, prp, out.ctypes.data)
    return out


def set_threads(n: int = 0) -> int:
    """OpenMP threads of the oracle's parallel loops (n <= 0: unchanged);
    returns the count now in effect."""
    return int(_L().lfo_set_threads(int(n)))
