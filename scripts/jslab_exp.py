"""Experiment: C = A.B at J = 128 as S column slabs of J/S (strided lf_spmm
views of B and C), so each pass's B working set is 1/S of the rows' bytes.
python scripts/jslab_exp.py CFG"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2_rmat20"
A_h, J = gen.config(cfg)
J = int(os.environ.get("J", J))
A = lf.Csr.from_host(A_h)
B = torch.from_numpy(gen.dense(A_h.n_cols, J, 0)).cuda()
C = torch.empty((A_h.n_rows, J), device="cuda")
params, stats = lf.configure(A, J)
M = lf.CellMatrix.build(A, params, stats)
ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
ref = M.spmm(B, out=torch.empty_like(C)).clone()
for rep in range(2):
    for S in (1, 2, 4, 8):
        w = J // S
        def run():
            for s in range(S):
                M.spmm(B[:, s * w:(s + 1) * w], out=C[:, s * w:(s + 1) * w])
        for _ in range(3):
            run()
        s0, s1 = ev(), ev()
        s0.record()
        for _ in range(10):
            run()
        s1.record()
        torch.cuda.synchronize()
        ok = bool(torch.equal(C, ref)) if S == 1 else float((C - ref).abs().max())
        print(json.dumps({"cfg": cfg, "J": J, "slabs": S, "ms": round(s0.elapsed_time(s1) / 10, 4), "check": ok}), flush=True)
