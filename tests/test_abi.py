"""The C-ABI library loads and exports every symbol include/liteform.h
declares; the ctypes mirror matches the header's struct layout (no GPU)."""
import ctypes
import os
import re
import subprocess

import pytest

from conftest import ROOT

HEADER = os.path.join(ROOT, "include", "liteform.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lf_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for n in ("lf_cell_configure", "lf_cell_build", "lf_spmm", "lf_cell_view", "lf_cell_destroy",
              "lf_csr_spmm", "lf_status_string", "lf_last_error_detail", "lf_abi_version"):
        assert n in names


def test_library_exports_every_declared_symbol():
    from paper_conf_hpdc_pengtpk25_b200 import _abi
    L = ctypes.CDLL(_abi.LIB_PATH)
    for n in declared_functions():
        assert hasattr(L, n), n
    assert set(declared_functions()) == set(_abi.SIGNATURES)
    assert L.lf_abi_version() == 1
    out = subprocess.run(["nm", "-D", "--defined-only", _abi.LIB_PATH], capture_output=True, text=True).stdout
    exported = {ln.split()[-1] for ln in out.splitlines() if " T " in ln}
    assert {n for n in exported if n.startswith("lf_")} == set(declared_functions())


def test_status_strings_without_gpu():
    from paper_conf_hpdc_pengtpk25_b200 import _abi
    assert _abi.lib.lf_status_string(0) == b"LF_OK"
    assert _abi.lib.lf_status_string(5) == b"LF_ERR_CUDA"


def test_null_arguments_rejected_on_host():
    """Host-side argument checks run before any CUDA call (works without a GPU)."""
    from paper_conf_hpdc_pengtpk25_b200 import _abi
    L = _abi.lib
    assert L.lf_cell_build(None, None, None, None, None, None) == 1
    p = _abi.LfCellParams()
    p.n_parts = 0
    A = _abi.LfCsr(4, 4, 0, 8, 0, 0)
    h = ctypes.c_void_p()
    assert L.lf_cell_build(ctypes.byref(A), ctypes.byref(p), None, None, None, ctypes.byref(h)) == 1
    assert b"n_parts" in L.lf_last_error_detail()
    p.n_parts, p.use_cell = 1, 1
    p.max_width_log2[0], p.block_nnz_log2[0] = 3, 2
    assert L.lf_cell_build(ctypes.byref(A), ctypes.byref(p), None, None, None, ctypes.byref(h)) == 1
    A2 = _abi.LfCsr(1 << 28, 4, 0, 8, 0, 0)
    p.block_nnz_log2[0] = 3
    assert L.lf_cell_build(ctypes.byref(A2), ctypes.byref(p), None, None, None, ctypes.byref(h)) == 3
    assert L.lf_spmm(None, None, 0, 4, None, 4, None) == 1
    assert L.lf_cell_configure(ctypes.byref(A), 0, None, ctypes.byref(p), None, None) == 1


LAYOUT_C = r"""
#include <stdio.h>
#include <stddef.h>
#include "liteform.h"
#define O(T, f) printf(#T "." #f " %zu\n", offsetof(T, f))
#define S(T) printf(#T " %zu\n", sizeof(T))
int main(void) {
  S(lf_csr); O(lf_csr, row_ptr); O(lf_csr, val);
  S(lf_allocator); O(lf_allocator, free);
  S(lf_cell_params); O(lf_cell_params, block_nnz_log2);
  S(lf_configure_opts);
  S(lf_configure_stats); O(lf_configure_stats, max_log2); O(lf_configure_stats, H); O(lf_configure_stats, cost);
  S(lf_bucket); O(lf_bucket, slot_off);
  S(lf_cell_arrays); O(lf_cell_arrays, row_ind); O(lf_cell_arrays, buckets); O(lf_cell_arrays, params);
  return 0;
}
"""


def test_ctypes_layout_matches_header(tmp_path):
    from paper_conf_hpdc_pengtpk25_b200 import _abi
    src = tmp_path / "layout.c"
    src.write_text(LAYOUT_C)
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    got = dict(ln.rsplit(" ", 1) for ln in subprocess.check_output([str(exe)], text=True).splitlines())
    m = {"lf_csr": _abi.LfCsr, "lf_allocator": _abi.LfAllocator, "lf_cell_params": _abi.LfCellParams,
         "lf_configure_opts": _abi.LfConfigureOpts, "lf_configure_stats": _abi.LfConfigureStats,
         "lf_bucket": _abi.LfBucket, "lf_cell_arrays": _abi.LfCellArrays}
    for key, v in got.items():
        if "." in key:
            t, f = key.split(".")
            assert getattr(m[t], f).offset == int(v), key
        else:
            assert ctypes.sizeof(m[key]) == int(v), key


def test_product_does_not_import_oracle():
    """The product path never reaches oracle/ (no CPU fallback)."""
    pkg = os.path.join(ROOT, "paper_conf_hpdc_pengtpk25_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in re.sub(r"#.*|//.*", "", txt).replace("no oracle", ""), f
