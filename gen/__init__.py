"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds none of the method's arithmetic (no bucketing, cost model or
SpMM): only matrix *shapes* and value distributions, per DESIGN.md "Input
recipe" and SURVEY.md section 8(d).  Generation runs in C (``lf_gen.c``,
OpenMP, counter-based RNG so the output does not depend on the thread count).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lf_gen.c")
_LIB = os.path.join(_HERE, "liblfgen.so")

# value kinds (lf_gen.c lfgen_fill_values)
GRID = 0      # 2^-23 grid in [-1, 1)
INT = 1       # integers in [lo, hi]
POS = 2       # 2^-24 grid in [0, 1)
ONE = 3       # constant 1.0

STREAM_VAL = 0x56414C00
STREAM_B = 0x42000000


def build(force: bool = False) -> str:
    """Compile lf_gen.c into liblfgen.so (gcc -O2 -fopenmp)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11", "-Wall",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class _Csr(ctypes.Structure):
    _fields_ = [("n_rows", ctypes.c_int64), ("n_cols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.POINTER(ctypes.c_int64)), ("col_ind", ctypes.POINTER(ctypes.c_int32))]


_lib = None


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.lfgen_u64.restype = ctypes.c_uint64
        _lib.lfgen_u64.argtypes = [ctypes.c_uint64] * 3
        _lib.lfgen_free.argtypes = [ctypes.POINTER(_Csr)]
        _lib.lfgen_rmat.argtypes = [ctypes.c_int32, ctypes.c_int64, ctypes.c_double, ctypes.c_double,
                                    ctypes.c_double, ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
                                    ctypes.POINTER(_Csr)]
        _lib.lfgen_uniform.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_double, ctypes.c_uint64,
                                       ctypes.POINTER(_Csr)]
        _lib.lfgen_stencil27.argtypes = [ctypes.c_int64, ctypes.POINTER(_Csr)]
        _lib.lfgen_banded.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.POINTER(_Csr)]
        _lib.lfgen_powerlaw.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_double, ctypes.c_uint64,
                                        ctypes.POINTER(_Csr)]
        _lib.lfgen_blockdiag.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.POINTER(_Csr)]
        _lib.lfgen_arrowhead.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.POINTER(_Csr)]
        _lib.lfgen_fill_values.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64, ctypes.c_uint64,
                                           ctypes.c_int32, ctypes.c_int32, ctypes.c_int32]
    return _lib


@dataclass
class CSR:
    """Host CSR: int64 row_ptr[n_rows+1], int32 col_ind[nnz], float32 val[nnz]."""
    n_rows: int
    n_cols: int
    row_ptr: np.ndarray
    col_ind: np.ndarray
    val: np.ndarray
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1] - self.row_ptr[0])

    def row_lengths(self) -> np.ndarray:
        return np.diff(self.row_ptr)


def u64(seed: int, stream: int, idx: int) -> int:
    return int(_L().lfgen_u64(seed, stream, idx))


def fill(n: int, seed: int, stream: int, kind: int = GRID, lo: int = 0, hi: int = 0) -> np.ndarray:
    out = np.empty(int(n), dtype=np.float32)
    rc = _L().lfgen_fill_values(out.ctypes.data, int(n), seed, stream, kind, lo, hi)
    if rc != 0:
        raise ValueError(f"lfgen_fill_values rc={rc}")
    return out


def dense(rows: int, cols: int, seed: int, kind: int = GRID, lo: int = -15, hi: int = 15,
          stream: int = STREAM_B) -> np.ndarray:
    """Dense row-major [rows, cols] float32 (the B operand)."""
    return fill(rows * cols, seed, stream, kind, lo, hi).reshape(rows, cols)


def _take(c: _Csr, rc: int, seed: int, kind: int, lo: int, hi: int, name: str) -> CSR:
    if rc != 0:
        raise ValueError(f"generator {name} failed rc={rc}")
    try:
        n, nnz = c.n_rows, c.nnz
        rp = np.ctypeslib.as_array(c.row_ptr, shape=(n + 1,)).copy()
        ci = np.ctypeslib.as_array(c.col_ind, shape=(max(nnz, 1),))[:nnz].copy() if nnz else \
            np.zeros(0, np.int32)
    finally:
        _L().lfgen_free(ctypes.byref(c))
    val = fill(nnz, seed, STREAM_VAL, kind, lo, hi)
    return CSR(int(n), int(c.n_cols), rp, ci, val, name)


def rmat(scale: int, edge_factor: int = 16, a: float = 0.57, b: float = 0.19, c: float = 0.19,
         seed: int = 0, permute: bool = False, dedup: bool = True, kind: int = GRID, lo: int = -3,
         hi: int = 3) -> CSR:
    """R-MAT / Graph500 power law, rows = source vertex."""
    m = _Csr()
    rc = _L().lfgen_rmat(scale, edge_factor, a, b, c, seed, int(permute), int(dedup), ctypes.byref(m))
    return _take(m, rc, seed, kind, lo, hi, f"rmat{scale}")


def uniform(n_rows: int, n_cols: int, p: float, seed: int = 0, kind: int = GRID, lo: int = -3,
            hi: int = 3) -> CSR:
    """Erdos-Renyi with per-entry probability p (config 1: 1024^2, p = 1/64)."""
    m = _Csr()
    rc = _L().lfgen_uniform(n_rows, n_cols, p, seed, ctypes.byref(m))
    return _take(m, rc, seed, kind, lo, hi, f"uniform{n_rows}")


def stencil27(n: int, seed: int = 0, kind: int = GRID, lo: int = -3, hi: int = 3) -> CSR:
    """27-point stencil on an n^3 grid (config 3 uses n = 126: 2,000,376 rows)."""
    m = _Csr()
    rc = _L().lfgen_stencil27(n, ctypes.byref(m))
    return _take(m, rc, seed, kind, lo, hi, f"stencil27_{n}")


def banded(n_rows: int, hw: int, n_cols: int | None = None, seed: int = 0, kind: int = GRID,
           lo: int = -3, hi: int = 3) -> CSR:
    m = _Csr()
    rc = _L().lfgen_banded(n_rows, n_rows if n_cols is None else n_cols, hw, ctypes.byref(m))
    return _take(m, rc, seed, kind, lo, hi, f"banded{n_rows}_{hw}")


def powerlaw(n: int, total_nnz: int, sigma: float = 1.2, seed: int = 0, kind: int = GRID, lo: int = -3,
             hi: int = 3) -> CSR:
    """Lognormal-degree Chung-Lu graph; config 4 (reddit-shaped): n=232,965,
    total_nnz=114,615,892, sigma=1.2 (Table 4)."""
    m = _Csr()
    rc = _L().lfgen_powerlaw(n, total_nnz, sigma, seed, ctypes.byref(m))
    return _take(m, rc, seed, kind, lo, hi, f"powerlaw{n}")


def blockdiag(n: int, b: int, seed: int = 0, kind: int = GRID, lo: int = -3, hi: int = 3) -> CSR:
    """Dense b x b diagonal blocks."""
    m = _Csr()
    rc = _L().lfgen_blockdiag(n, b, ctypes.byref(m))
    return _take(m, rc, seed, kind, lo, hi, f"blockdiag{n}_{b}")


def arrowhead(n: int, w: int, seed: int = 0, kind: int = GRID, lo: int = -3, hi: int = 3) -> CSR:
    """w dense rows + w dense columns + the diagonal."""
    m = _Csr()
    rc = _L().lfgen_arrowhead(n, w, ctypes.byref(m))
    return _take(m, rc, seed, kind, lo, hi, f"arrowhead{n}_{w}")


def mixed_suite(sizes=(1 << 16, 1 << 18, 1 << 20), seeds=(0,)):
    """BASELINE.json configs[4]: the mixed-skew suite --
    yields (name, thunk) so callers generate one matrix at a time."""
    for n in sizes:
        sc = n.bit_length() - 1
        for sd in seeds:
            yield f"er_{n}_{sd}", (lambda n=n, sd=sd: uniform(n, n, 16.0 / n, sd))
            for a in (0.45, 0.57, 0.70):
                b = (1.0 - a) / 3.0 if a != 0.57 else 0.19
                yield f"rmat{a}_{n}_{sd}", (lambda sc=sc, a=a, b=b, sd=sd: rmat(sc, 16, a, b, b, seed=sd))
            for sg in (0.5, 1.0, 1.5, 2.0):
                yield f"lognormal{sg}_{n}_{sd}", (lambda n=n, sg=sg, sd=sd: powerlaw(n, 16 * n, sg, sd))
            for hw in (4, 16, 64):
                yield f"band{hw}_{n}_{sd}", (lambda n=n, hw=hw, sd=sd: banded(n, hw, seed=sd))
            # GNN-degree lognormal graphs (Reddit-shaped, mean degree 128 / 512 over
            # n/4 rows): the regime where B outgrows L2 and rows are long enough
            # for column partitions (P > 1) to pay off
            for deg in (128, 512):
                yield f"gnn{deg}_{n}_{sd}", (lambda n=n, deg=deg, sd=sd: powerlaw(n // 4, deg * (n // 4), 1.2, sd))
            g = round(n ** (1.0 / 3.0))
            yield f"stencil27_{g}", (lambda g=g: stencil27(g))
            for bb in (8, 32):
                yield f"blockdiag{bb}_{n}", (lambda n=n, bb=bb: blockdiag(n, bb))
            yield f"arrowhead_{n}", (lambda n=n: arrowhead(n, 4))


def random_small(n_rows: int, n_cols: int, max_len: int, seed: int, dup: bool = True,
                 zeros: bool = True, empty_frac: float = 0.2, kind: int = INT, lo: int = -3,
                 hi: int = 3) -> CSR:
    """Tiny irregular CSR for edge-case tests: empty rows, duplicate column
    indices, explicit zero values, lengths 0..max_len (numpy, seeded)."""
    rng = np.random.default_rng(seed)
    lens = rng.integers(0, max_len + 1, size=n_rows)
    lens[rng.random(n_rows) < empty_frac] = 0
    if n_cols == 0:
        lens[:] = 0
    rows = []
    for i in range(n_rows):
        if dup:
            cols = np.sort(rng.integers(0, max(n_cols, 1), size=lens[i]))
        else:
            k = min(lens[i], n_cols)
            cols = np.sort(rng.choice(n_cols, size=k, replace=False)) if k else np.zeros(0, np.int64)
        rows.append(cols.astype(np.int32))
    rp = np.zeros(n_rows + 1, np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    ci = np.concatenate(rows).astype(np.int32) if rows else np.zeros(0, np.int32)
    val = fill(len(ci), seed, STREAM_VAL, kind, lo, hi)
    if zeros and len(val):
        val[rng.random(len(val)) < 0.1] = 0.0
    return CSR(n_rows, n_cols, rp, ci, val, f"small{seed}")


# BASELINE.json configs; J per config
CONFIGS = {
    "c1_uniform1024": dict(J=32),
    "c2_rmat20": dict(J=128),
    "c2p_rmat20_perm": dict(J=128),
    "c3_stencil126": dict(J=64),
    # configs[2] read literally ("banded FEM-like 2M rows, ~50M nnz"): a band
    # of half-width 12 around the diagonal, 25 nonzeros per interior row
    "c3b_banded2M": dict(J=64),
    "c4_reddit": dict(J=256),
}


def config(name: str, seed: int = 0, kind: int = GRID, lo: int = -3, hi: int = 3) -> tuple[CSR, int]:
    """The matrices of BASELINE.json configs[0..3] and their J."""
    if name == "c1_uniform1024":
        m = uniform(1024, 1024, 1.0 / 64.0, seed, kind, lo, hi)
    elif name == "c2_rmat20":
        m = rmat(20, 16, seed=seed, kind=kind, lo=lo, hi=hi)
    elif name == "c2p_rmat20_perm":
        # the same R-MAT with rows and columns permuted ("also
        # report a permuted variant"): hub rows / columns scattered over the index range
        m = rmat(20, 16, seed=seed, permute=True, kind=kind, lo=lo, hi=hi)
    elif name == "c3_stencil126":
        m = stencil27(126, seed, kind, lo, hi)
    elif name == "c3b_banded2M":
        m = banded(2_000_000, 12, seed=seed, kind=kind, lo=lo, hi=hi)
    elif name == "c4_reddit":
        m = powerlaw(232965, 114615892, 1.2, seed, kind, lo, hi)
    else:
        raise KeyError(name)
    m.name = name
    return m, CONFIGS[name]["J"]
