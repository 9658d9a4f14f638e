"""Build liblf.so in-tree with nvcc for sm_100a (no JIT, no torch extension)."""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OBJ = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "liblf.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
         "--expt-relaxed-constexpr", "-I", os.path.join(ROOT, "include"), "-I", CSRC]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "kernels", "*.cu")))


def _headers():
    return (glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h"))
            + glob.glob(os.path.join(ROOT, "include", "*.h")))


def _newest(paths):
    return max((os.path.getmtime(p) for p in paths), default=0.0)


def src_hash(defs=()) -> str:
    """sha1 of every source and header, the flags and the -D macros: liblf.so
    is reused only when it was built from exactly these (a stamp file next to
    it), never on timestamps alone (a pushed or copied binary keeps its mtime)."""
    import hashlib
    h = hashlib.sha1(" ".join([NVCC, *ARCH, *FLAGS, *defs]).encode())
    for f in sorted(sources() + _headers() + [__file__]):
        with open(f, "rb") as fh:
            h.update(os.path.relpath(f, ROOT).encode() + b"\0" + fh.read())
    return h.hexdigest()


def build(force: bool = False, verbose: bool = False, defs=(), out: str | None = None) -> str:
    """defs: extra -D macros (experiment variants go to `out` / build_<tag>/)."""
    global OBJ
    lib = out or LIB
    obj_dir = OBJ if not defs else OBJ + "_" + "_".join(d.replace("=", "") for d in defs)
    srcs = sources()
    stamp = lib + ".srchash"
    want = src_hash(defs)
    if not force and os.path.exists(lib) and os.path.exists(stamp):
        with open(stamp) as f:
            if f.read().strip() == want:
                return lib
    os.makedirs(obj_dir, exist_ok=True)
    hdr_t = _newest(_headers() + [__file__])

    def compile_one(src):
        obj = os.path.join(obj_dir, os.path.basename(src).replace(".cu", ".o"))
        if force or not os.path.exists(obj) or os.path.getmtime(obj) < max(os.path.getmtime(src), hdr_t):
            cmd = [NVCC, *ARCH, *FLAGS, *[f"-D{d}" for d in defs], "-Xptxas", "-v" if verbose else "-O3", "-c", src, "-o", obj]
            r = subprocess.run(cmd, capture_output=True, text=True)
            if r.returncode != 0:
                raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
            if verbose:
                print(r.stderr)
        return obj

    with cf.ThreadPoolExecutor(max_workers=min(8, len(srcs))) as ex:
        objs = list(ex.map(compile_one, srcs))
    tmp = lib + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-cudart", "static"])
    os.replace(tmp, lib)
    with open(stamp, "w") as f:
        f.write(want + "\n")
    return lib


if __name__ == "__main__":
    import sys
    defs = [a[2:] for a in sys.argv[1:] if a.startswith("-D")]
    outs = [a[6:] for a in sys.argv[1:] if a.startswith("--out=")]
    print(build(force="-f" in sys.argv, verbose="-v" in sys.argv, defs=defs, out=outs[0] if outs else None))
