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
        C3, _ = lfd.spmm_rowsharded_fused(A, B, 128)  # kernels write into both ranks' C over NVLink
        torch.cuda.synchronize()
        ok = ok and bool(np.array_equal(C3.cpu().numpy().astype(np.float64), ref))
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


FUSED_CASES = [("rmat", 1, "0"), ("rmat", 3, "0"), ("band", 1, "1"), ("band", 1, "0"), ("stencil", 1, "0"),
               ("band_p2", 2, "1")]


@pytest.mark.parametrize("kind,P,tc", FUSED_CASES)
@pytest.mark.parametrize("J", [64, 128])
def test_fused_exchange_local_destinations(kind, P, tc, J, monkeypatch):
    """lf_spmm_ex's fused row exchange on one GPU: a row shard of A writes its C
    rows straight into TWO full-C destinations (standing in for two ranks'
    buffers) at row_base; both hold Alg. 1's rows exactly (integer inputs),
    rows outside the shard stay untouched.  Per-slot (R-MAT), tcgen05 windowed
    and grouped (band, stencil) kernels, P > 1 (red.add rows pre-zeroed in
    every destination)."""
    import paper_conf_hpdc_pengtpk25_b200 as lf
    monkeypatch.setenv("LF_TC", tc)
    monkeypatch.setenv("LF_GROUPED", "1" if kind == "stencil" or (kind == "band" and tc == "0") else "0")
    A_h = {"rmat": lambda: gen.rmat(13, 16, seed=3, kind=gen.INT, lo=-3, hi=3),
           "band": lambda: gen.banded(9000, 12, seed=3, kind=gen.INT, lo=-3, hi=3),
           "band_p2": lambda: gen.banded(9000, 12, seed=4, kind=gen.INT, lo=-3, hi=3),
           "stencil": lambda: gen.stencil27(20, seed=3, kind=gen.INT, lo=-3, hi=3)}[kind]()
    B_h = gen.dense(A_h.n_cols, J, 3, gen.INT, -15, 15)
    I = A_h.n_rows
    lo, hi = I // 3, (2 * I) // 3
    A = lf.Csr.from_host(A_h)
    shard = lf.Csr(A.row_ptr[lo:hi + 1], A.col_ind, A.val, A.n_cols)
    params = lf.make_params(P, [5] * P)
    M = lf.CellMatrix.build(shard, params)
    dsts = [torch.full((I, J), float("nan"), device="cuda") for _ in range(2)]
    assert M.spmm(torch.from_numpy(B_h).cuda(), dst=dsts, row_base=lo) is None
    torch.cuda.synchronize()
    ref = oracle.spmm_csr(A_h, B_h, rows=np.arange(lo, hi, dtype=np.int64))[0]
    for D in dsts:
        Dh = D.cpu().numpy().astype(np.float64)
        assert np.array_equal(Dh[lo:hi], ref)
        assert np.isnan(Dh[:lo]).all() and np.isnan(Dh[hi:]).all()


def test_fused_exchange_errors():
    import paper_conf_hpdc_pengtpk25_b200 as lf
    A_h = gen.rmat(10, 8, seed=1)
    A = lf.Csr.from_host(A_h)
    M = lf.CellMatrix.build(A, lf.make_params(1, 5))
    B = torch.ones(A_h.n_cols, 32, device="cuda")
    with pytest.raises(lf.LfError):
        M.spmm(B, dst=[0], row_base=0)  # NULL destination
    with pytest.raises(lf.LfError):
        M.spmm(B, dst=[torch.zeros(A_h.n_rows, 32, device="cuda")] * 9)  # more than LF_MAX_DST
    params, _ = lf.configure(A, 32, force_format=2)
    Mc = lf.CellMatrix.build(A, params)
    with pytest.raises(lf.LfError):
        Mc.spmm(B, dst=[torch.zeros(A_h.n_rows, 32, device="cuda")])  # CSR format: unsupported


def test_fused_rowsharded_world1(nccl1):
    """dist.spmm_rowsharded_fused at world size 1: symmetric-memory C, the
    kernels write through the destination list, equal to Alg. 1."""
    import paper_conf_hpdc_pengtpk25_b200 as lf
    from paper_conf_hpdc_pengtpk25_b200 import dist as lfd
    A_h = gen.rmat(13, 16, seed=8, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, 128, 8, gen.INT, -15, 15)
    C, bounds = lfd.spmm_rowsharded_fused(lf.Csr.from_host(A_h), torch.from_numpy(B_h).cuda(), 128)
    torch.cuda.synchronize()
    assert list(bounds) == [0, A_h.n_rows]
    assert np.array_equal(C.cpu().numpy().astype(np.float64), oracle.spmm_csr(A_h, B_h)[0])
