"""Multi-GPU entry points over NCCL on the GPU: row sharding
with B replicated and the large-J column split, against the oracle.

* world size 1 (one GPU, in-process NCCL group): spmm_rowsharded and
  spmm_colsplit run their whole code path (shard bounds, per-rank configure
  and build from a row_ptr view, local SpMM in place, the NCCL exchange /
  all-gather) and must equal the fp64 oracle exactly on integer inputs;
* world size 2 over NCCL (skipped with fewer than 2 GPUs): each rank's
  gathered C equals the oracle.
"""
import os
import socket

import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.fixture(scope="module")
def nccl1():
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(_port())
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    assert dist.get_world_size() == 1
    yield dist
    dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["nnz", "bytes"])
@pytest.mark.parametrize("J", [64, 128])
def test_rowsharded_world1(nccl1, mode, J):
    import paper_conf_hpdc_pengtpk25_b200 as lf
    from paper_conf_hpdc_pengtpk25_b200 import dist as lfd
    A_h = gen.rmat(13, 16, seed=7, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, J, 7, gen.INT, -15, 15)
    A = lf.Csr.from_host(A_h)
    C, bounds = lfd.spmm_rowsharded(A, torch.from_numpy(B_h).cuda(), J, mode=mode)
    assert list(bounds) == [0, A_h.n_rows]
    assert np.array_equal(C.cpu().numpy().astype(np.float64), oracle.spmm_csr(A_h, B_h)[0])


@pytest.mark.parametrize("J", [256, 260])
def test_colsplit_world1(nccl1, J):
    import paper_conf_hpdc_pengtpk25_b200 as lf
    from paper_conf_hpdc_pengtpk25_b200 import dist as lfd
    A_h = gen.powerlaw(4000, 300000, 1.2, seed=2, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, J, 2, gen.INT, -15, 15)
    A = lf.Csr.from_host(A_h)
    C, cb = lfd.spmm_colsplit(A, torch.from_numpy(B_h).cuda())
    assert list(cb) == [0, J]
    assert np.array_equal(C.cpu().numpy().astype(np.float64), oracle.spmm_csr(A_h, B_h)[0])


def _worker2(rank, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=2, device_id=torch.device("cuda", rank))
    try:
        import paper_conf_hpdc_pengtpk25_b200 as lf
        from paper_conf_hpdc_pengtpk25_b200 import dist as lfd
        A_h = gen.rmat(12, 16, seed=9, kind=gen.INT, lo=-3, hi=3)
        B_h = gen.dense(A_h.n_cols, 128, 9, gen.INT, -15, 15)
        A = lf.Csr.from_host(A_h)
        B = torch.from_numpy(B_h).cuda()
        ref = oracle.spmm_csr(A_h, B_h)[0]
        C, _ = lfd.spmm_rowsharded(A, B, 128)
        ok = bool(np.array_equal(C.cpu().numpy().astype(np.float64), ref))
        C2, _ = lfd.spmm_colsplit(A, B)
        ok = ok and bool(np.array_equal(C2.cpu().numpy().astype(np.float64), ref))
        q.put((rank, ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2, reason="needs 2 GPUs")
def test_two_ranks_nccl():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker2, args=(r, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=600) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    assert all(ok for _, ok in res), res
