"""configure + build once, then N lf_spmm launches (ncu target).
python scripts/spmm_once.py CONFIG J [N]   -- prints the kernel path"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402

cfg, J = sys.argv[1], int(sys.argv[2])
n = int(sys.argv[3]) if len(sys.argv) > 3 else 2
A_h, _ = gen.config(cfg)
A = lf.Csr.from_host(A_h)
B = torch.from_numpy(gen.dense(A_h.n_cols, J, 0)).cuda()
C = torch.empty((A_h.n_rows, J), device="cuda")
params, stats = lf.configure(A, J)
M = lf.CellMatrix.build(A, params, stats)
torch.cuda.synchronize()
for _ in range(n):
    M.spmm(B, out=C)
torch.cuda.synchronize()
print("path", M.path(J), params.as_dict(), flush=True)
