"""Phase timing on one config (CUDA events): configure, build, spmm.
python scripts/spmm_time.py [config] [key=val ...]   (parts=, width=, iters=)"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2_rmat20"
opt = dict(a.split("=") for a in sys.argv[2:])
iters = int(opt.pop("iters", 20))
J_over = opt.pop("J", None)
kw = {}
if "parts" in opt:
    kw["force_parts"] = int(opt["parts"])
if "width" in opt:
    kw["force_width_log2"] = int(opt["width"])
if "fmt" in opt:
    kw["force_format"] = int(opt["fmt"])
if "mult" in opt:
    kw["block_mult_log2"] = int(opt["mult"])
A_h, J = gen.config(cfg)
if J_over:
    J = int(J_over)
A = lf.Csr.from_host(A_h)
B = torch.from_numpy(gen.dense(A_h.n_cols, J, 0)).cuda()
C = torch.empty((A_h.n_rows, J), device="cuda")
U = int(np.count_nonzero(np.bincount(A_h.col_ind, minlength=A_h.n_cols)))
bytes_alg = 8 * A_h.nnz + 4 * U * J + 4 * A_h.n_rows * J
ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
t = {"configure": [], "build": [], "spmm": []}
for it in range(iters + 3):
    e0, e1, e2, e3 = ev(), ev(), ev(), ev()
    e0.record()
    params, stats = lf.configure(A, J, **kw)
    e1.record()
    M = lf.CellMatrix.build(A, params, stats)
    e2.record()
    M.spmm(B, out=C)
    e3.record()
    torch.cuda.synchronize()
    if it >= 3:
        t["configure"].append(e0.elapsed_time(e1))
        t["build"].append(e1.elapsed_time(e2))
        t["spmm"].append(e2.elapsed_time(e3))
    if it < iters + 2:
        M.close()
# spmm alone, back to back
s0, s1 = ev(), ev()
s0.record()
for _ in range(iters):
    M.spmm(B, out=C)
s1.record()
torch.cuda.synchronize()
sp = s0.elapsed_time(s1) / iters
out = {k: round(float(np.median(v)), 4) for k, v in t.items()}
out.update(cfg=cfg, J=J, lib=os.path.basename(lf.library_path()), params=params.as_dict(), spmm_loop_ms=round(sp, 4),
           gflops=round(2 * A_h.nnz * J / sp / 1e6, 1), alg_gbs=round(bytes_alg / sp / 1e6, 1),
           frac=round(bytes_alg / sp / 1e6 / 6552, 3), slots=int(M.view()["n_slots"]))
print(json.dumps(out), flush=True)
