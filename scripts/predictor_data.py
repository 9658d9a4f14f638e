"""NEXT-1 training data (run on the B200): for every matrix of the mixed-skew
suite (BASELINE.json configs[4]) and J in {32..512}, the Table 2 / Table 3
features and the measured times of the plain CSR
kernel (Alg. 1) and of CELL SpMM with P in {1, 2, 4, 8} (Alg. 3 widths).
Labels follow section 5.1-5.2:
  use_cell = CELL (best P) >= 1.1x faster than the fixed CSR kernel
  parts    = the P with the lowest CELL time.
python scripts/predictor_data.py OUT.jsonl [sizes...]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402

out = sys.argv[1]
sizes = tuple(int(x) for x in sys.argv[2:]) or (1 << 16, 1 << 18, 1 << 20)
ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731


def timed(fn, n=8):
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    a, b = ev(), ev()
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n


g = torch.Generator(device="cuda")
g.manual_seed(0)
with open(out, "w") as f:
    for name, thunk in gen.mixed_suite(sizes, seeds=(0, 1)):
        t0 = time.time()
        A_h = thunk()
        A = lf.Csr.from_host(A_h)
        for J in (32, 64, 128, 256, 512):
            # timing only: B's values do not change the work, so draw it on the device
            B = torch.rand((A_h.n_cols, J), device="cuda", generator=g) * 2 - 1
            C = torch.empty((A_h.n_rows, J), device="cuda")
            _, st = lf.configure(A, J, force_parts=1)
            rec = {"name": name, "J": J, "features": list(st.features), "n_rows": A_h.n_rows, "nnz": A_h.nnz,
                   "t_csr": timed(lambda: lf.csr_spmm(A, B, out=C)), "t_cell": {}}
            for P in (1, 2, 4, 8):
                params, stp = lf.configure(A, J, force_parts=P, force_format=1)
                M = lf.CellMatrix.build(A, params, stp)
                rec["t_cell"][P] = timed(lambda: M.spmm(B, out=C))
                rec.setdefault("widths", {})[P] = list(params.max_width_log2[:P])
                M.close()
            best = min(rec["t_cell"], key=rec["t_cell"].get)
            rec["parts"] = int(best)
            rec["use_cell"] = int(rec["t_csr"] >= 1.1 * rec["t_cell"][best])
            f.write(json.dumps(rec) + "\n")
            f.flush()
            del B, C
        print(name, A_h.n_rows, A_h.nnz, round(time.time() - t0, 1), file=sys.stderr, flush=True)
