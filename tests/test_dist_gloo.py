"""Row-sharded multi-process logic (paper_conf_hpdc_pengtpk25_b200.dist) on CPU
with the gloo backend, world size 2 (no GPU): shard boundaries and the C
all-gather.  Each rank computes its row block with the oracle (test-only);
the gathered C must equal the unsharded oracle result exactly."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, mode, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_hpdc_pengtpk25_b200 import dist as lfd
        A = gen.rmat(10, 8, seed=3, kind=gen.INT, lo=-3, hi=3)
        J = 24
        B = gen.dense(A.n_cols, J, 3, gen.INT, -15, 15)
        bounds = lfd.shard_bounds(A.row_ptr, world, J, mode)
        lo, hi = int(bounds[rank]), int(bounds[rank + 1])
        C_loc, _ = oracle.spmm_csr(A, B, rows=np.arange(lo, hi, dtype=np.int64), with_abs=False)
        C = lfd.gather_rows(torch.from_numpy(C_loc.astype(np.float64)), bounds)
        full, _ = oracle.spmm_csr(A, B, with_abs=False)
        ok = bool(np.array_equal(C.numpy(), full))
        # large-J mode: column slabs of B, each rank's slab of C, gathered
        for Jc in (J, 26):  # equal slabs (one permuting copy) and unequal ones (12 + 14: padded)
            Bc = gen.dense(A.n_cols, Jc, 3, gen.INT, -15, 15)
            fullc, _ = oracle.spmm_csr(A, Bc, with_abs=False)
            cb = lfd.col_bounds(Jc, world)
            j0, j1 = int(cb[rank]), int(cb[rank + 1])
            C_slab, _ = oracle.spmm_csr(A, np.ascontiguousarray(Bc[:, j0:j1]), with_abs=False)
            Cc = lfd.gather_cols(torch.from_numpy(C_slab.astype(np.float64)), cb)
            ok = ok and bool(np.array_equal(Cc.numpy(), fullc))
        q.put((rank, ok, bounds.tolist()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["nnz", "bytes"])
def test_rowsharded_gather_world2(mode):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, mode, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=180) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert all(ok for _, ok, _ in res)
    assert res[0][2] == res[1][2]


def test_col_bounds_properties():
    from paper_conf_hpdc_pengtpk25_b200 import dist as lfd
    for J in (1, 4, 30, 128, 256, 512, 1000):
        for world in (1, 2, 3, 4, 8):
            b = lfd.col_bounds(J, world)
            assert b[0] == 0 and b[-1] == J and len(b) == world + 1 and np.all(np.diff(b) >= 0)
            assert all(x % 4 == 0 for x in b[1:-1])
            w = np.diff(b)
            assert w.max() - w[w > 0].min() <= 4 if (w > 0).any() else True


def test_shard_bounds_properties():
    from paper_conf_hpdc_pengtpk25_b200 import dist as lfd
    A = gen.rmat(12, 16, seed=1)
    for world in (1, 2, 3, 4, 8):
        for mode in ("nnz", "bytes"):
            b = lfd.shard_bounds(A.row_ptr, world, 128, mode)
            assert b[0] == 0 and b[-1] == A.n_rows and np.all(np.diff(b) >= 0) and len(b) == world + 1
            w = lfd.row_weights(A.row_ptr, 128, mode)
            shares = [w[b[r]:b[r + 1]].sum() for r in range(world)]
            # contiguous split: each shard within one row's weight of the ideal share
            assert max(shares) <= w.sum() / world + w.max() + 1
    # empty matrix and more ranks than rows
    rp = np.zeros(4, np.int64)
    b = lfd.shard_bounds(rp, 8, 4, "nnz")
    assert b[0] == 0 and b[-1] == 3 and np.all(np.diff(b) >= 0)
