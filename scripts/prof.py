"""Short driver for ncu: configure + build + spmm on a BASELINE config, a few
iterations (python scripts/prof.py [config] [iters] [extra: parts=P width=E])."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2_rmat20"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 3
kw = {}
for a in sys.argv[3:]:
    k, v = a.split("=")
    kw[{"parts": "force_parts", "width": "force_width_log2"}[k]] = int(v)
A_h, J = gen.config(cfg)
A = lf.Csr.from_host(A_h)
B = torch.from_numpy(gen.dense(A_h.n_cols, J, 0)).cuda()
C = torch.empty((A_h.n_rows, J), device="cuda")
for _ in range(iters):
    params, stats = lf.configure(A, J, **kw)
    M = lf.CellMatrix.build(A, params, stats)
    M.spmm(B, out=C)
    M.close()
torch.cuda.synchronize()
print("done", params.as_dict())
