"""c1 (uniform 1024^2, J = 32, launch-latency bound): lf_spmm
timed back to back and as 200 calls captured in one CUDA graph (per-call
latency).  python scripts/c1_graph.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_hpdc_pengtpk25_b200 as lf  # noqa: E402

import ctypes  # noqa: E402
import glob  # noqa: E402
cudart = ctypes.CDLL(sorted(glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                                                   "libcudart.so*")))[0])

A_h, J = gen.config("c1_uniform1024")
A = lf.Csr.from_host(A_h)
B_h = gen.dense(A_h.n_cols, J, 0)
B = torch.from_numpy(B_h).cuda()
C = torch.empty((A_h.n_rows, J), device="cuda")
out = {"cfg": "c1_uniform1024", "J": J, "nnz": A_h.nnz}
for fmt in (1, 2):  # CELL, fixed CSR (the predictor's choice for c1)
    print("fmt", fmt, flush=True)
    s = torch.cuda.Stream()
    # the handle is built on the stream the graph is captured on: its launches
    # then take the single-stream path (kernel launches only, capture-safe)
    params, stats = lf.configure(A, J, force_format=fmt, stream=s)
    M = lf.CellMatrix.build(A, params, stats, stream=s)
    print("last error after build:", cudart.cudaGetLastError(), flush=True)
    with torch.cuda.stream(s):
        for _ in range(5):
            M.spmm(B, out=C, stream=s)
    s.synchronize()
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    e0, e1 = ev(), ev()
    e0.record(s)
    for _ in range(200):
        M.spmm(B, out=C, stream=s)
    e1.record(s)
    s.synchronize()
    loop_us = e0.elapsed_time(e1) / 200 * 1e3
    print("loop_us", loop_us, "last error:", cudart.cudaGetLastError(), flush=True)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(200):
            M.spmm(B, out=C, stream=torch.cuda.current_stream())
    print("after capture, last error:", cudart.cudaGetLastError(), flush=True)
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    e0.record()
    for _ in range(10):
        g.replay()
    e1.record()
    torch.cuda.synchronize()
    graph_us = e0.elapsed_time(e1) / 2000 * 1e3
    Cref, Cabs = oracle.spmm_csr(A_h, B_h)
    ok = bool(np.all(np.abs(C.cpu().numpy().astype(np.float64) - Cref) <= 1e-5 * Cabs))
    out["cell" if fmt == 1 else "csr"] = {"path": M.path(), "loop_us": round(loop_us, 2), "graph_us": round(graph_us, 2),
                                          "gflops_graph": round(2 * A_h.nnz * J / (graph_us * 1e-6) / 1e9, 1),
                                          "parity": ok}
    M.close()
print(json.dumps(out), flush=True)
