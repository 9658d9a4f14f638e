"""NEXT-2 / Fig. 11 analogue: sweep the max bucket width 2^e of a
config, report eq. 7's cost (GPU statistics) beside the measured SpMM time,
and the Spearman rank correlation.  python scripts/costmodel_sweep.py c4_reddit"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c4_reddit"
A_h, J = gen.config(cfg)
A = lf.Csr.from_host(A_h)
B = torch.from_numpy(gen.dense(A_h.n_cols, J, 0)).cuda()
C = torch.empty((A_h.n_rows, J), device="cuda")
p0, st0 = lf.configure(A, J)
top = st0.max_log2[0]
rows = []
for e in range(0, top + 1):
    params, st = lf.configure(A, J, force_width_log2=e)
    M = lf.CellMatrix.build(A, params, st)
    for _ in range(3):
        M.spmm(B, out=C)
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 10
    ev0.record()
    for _ in range(n):
        M.spmm(B, out=C)
    ev1.record()
    torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1) / n
    rows.append({"e": e, "cost": int(st.cost[0][e]), "spmm_ms": ms, "slots": int(M.view()["n_slots"]),
                 "gflops": 2 * A_h.nnz * J / ms / 1e6})
    M.close()
costs = np.array([r["cost"] for r in rows], float)
times = np.array([r["spmm_ms"] for r in rows])
rk = lambda x: np.argsort(np.argsort(x))  # noqa: E731
rho = float(np.corrcoef(rk(costs), rk(times))[0, 1])
print(json.dumps({"cfg": cfg, "J": J, "alg3_e": int(p0.max_width_log2[0]), "argmin_cost_e": int(np.argmin(costs)),
                  "argmin_time_e": int(np.argmin(times)), "spearman": rho, "rows": rows}))
