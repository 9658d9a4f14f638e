"""Host-side latency of each API call in the bench step (c2): wall time of the
Python call (no extra syncs), and GPU phase time by events.  Diagnostic."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2_rmat20"
A_h, J = gen.config(cfg)
A = lf.Csr.from_host(A_h)
B = torch.from_numpy(gen.dense(A_h.n_cols, J, 0)).cuda()
C = torch.empty((A_h.n_rows, J), device="cuda")
rec = []
for it in range(30):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    params, stats = lf.configure(A, J)
    t1 = time.perf_counter()
    M = lf.CellMatrix.build(A, params, stats)
    t2 = time.perf_counter()
    M.spmm(B, out=C)
    t3 = time.perf_counter()
    M.close()
    t4 = time.perf_counter()
    torch.cuda.synchronize()
    t5 = time.perf_counter()
    if it >= 5:
        rec.append((t1 - t0, t2 - t1, t3 - t2, t4 - t3, t5 - t0))
import numpy as np  # noqa: E402
r = np.median(np.array(rec), axis=0) * 1e6
print(f"host us: configure {r[0]:.1f} build {r[1]:.1f} spmm {r[2]:.1f} close {r[3]:.1f} | step wall {r[4]:.1f}")
# allocator callback cost
al = lf._abi.torch_allocator()
t0 = time.perf_counter()
for _ in range(200):
    p = al.alloc(None, 1 << 20, 0)
    al.free(None, p, 1 << 20, 0)
print(f"allocator alloc+free via ctypes: {(time.perf_counter() - t0) / 200 * 1e6:.1f} us")
