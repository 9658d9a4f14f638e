"""Small inputs through every kernel of liblf.so, for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck): configure (speculative and
features-first paths), build (stats-sized and GPU-counted), the per-slot,
grouped, mma.sync, tcgen05 (windowed) and CSR SpMM kernels, P > 1, folded rows, J tails.
Checks results against the oracle so a run that "passes" computed the right
thing.   python scripts/sanitize_cases.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402


def check(M, A_h, J, env=None):
    B_h = gen.dense(A_h.n_cols, J, 1, gen.INT, -15, 15)
    C = M.spmm(torch.from_numpy(B_h).cuda()).cpu().numpy().astype(np.float64)
    assert np.array_equal(C, oracle.spmm_csr(A_h, B_h)[0]), (A_h.name, J, env)


cases = [(gen.config("c1_uniform1024", kind=gen.INT)[0], (32, 7)),
         (gen.rmat(10, 16, seed=1, kind=gen.INT), (64, 128)),
         (gen.banded(2048, 12, seed=2, kind=gen.INT), (64, 128)),
         (gen.arrowhead(2048, 4, seed=3, kind=gen.INT), (32,))]
os.environ["LF_TC"] = "1"  # build the per-group windows of the tcgen05 path in every handle
for A_h, Js in cases:
    A = lf.Csr.from_host(A_h)
    for J in Js:
        for P in (1, 3):
            params, stats = lf.configure(A, J, force_parts=P, force_format=1)
            for M in (lf.CellMatrix.build(A, params, stats), lf.CellMatrix.build(A, params)):
                os.environ["LF_TC"] = "0"
                check(M, A_h, J)
                for env in ("LF_GROUPED", "LF_MMA", "LF_TC"):
                    os.environ[env] = "1"
                    check(M, A_h, J, env)
                    os.environ[env] = "0"
                os.environ["LF_TC"] = "1"
                M.close()
        params, stats = lf.configure(A, J)  # predictor path
        M = lf.CellMatrix.build(A, params, stats)
        check(M, A_h, J)
        C = lf.csr_spmm(A, torch.from_numpy(gen.dense(A_h.n_cols, J, 1, gen.INT, -15, 15)).cuda())
torch.cuda.synchronize()
print("sanitize cases ok")
