"""GPU parity of the grouped (column-merged) SpMM path against the oracle.

The grouped paths (cell_spmm.cu) apply when every
bucket has W <= 32, B / C are 16-byte aligned and J <= 256: kGroupRows
consecutive CELL rows share one gather per distinct column.  It must give the
same C as Algorithm 1: exactly on integer inputs (any atomic / summation
order), within max|C - C_ref| <= 1e-5 (|A|.|B|) on float inputs.  LF_GROUPED=1
forces it (LF_GROUPED=0 forbids it) for the lf_spmm calls of a test.
"""
import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = 1e-5


@pytest.fixture(scope="module")
def lf():
    import paper_conf_hpdc_pengtpk25_b200 as m
    return m


@pytest.fixture(params=["LF_GROUPED", "LF_MMA"])
def grouped(request, monkeypatch):
    """Both grouped paths: the CUDA-core one (LF_GROUPED) and the tensor-core
    one (LF_MMA: 16-row groups, 3xTF32 mma.sync; J in {64, 128}, otherwise
    the launch falls back to the per-slot path)."""
    monkeypatch.setenv("LF_GROUPED", "0")
    monkeypatch.setenv("LF_MMA", "0")
    monkeypatch.setenv(request.param, "1")
    return request.param


def run(lf, A_h, B_h, P, e, k=None):
    A = lf.Csr.from_host(A_h)
    M = lf.CellMatrix.build(A, lf.make_params(P, e, k))
    C = M.spmm(torch.from_numpy(B_h).cuda()).cpu().numpy().astype(np.float64)
    return C, M


CASES = []
for s in range(12):
    rng = np.random.default_rng(100 + s)
    P = int(rng.integers(1, 4))
    e = rng.integers(0, 6, size=P).tolist()          # every W <= 32
    k = [x + int(rng.integers(0, 3)) for x in e]     # blocks of 1..4 rows of the max bucket
    CASES.append((s, int(rng.integers(1, 400)), int(rng.integers(1, 300)), P, e, k))


@pytest.mark.parametrize("seed,I,K,P,e,k", CASES)
@pytest.mark.parametrize("J", [4, 32, 64, 96, 128, 256])  # 256: falls back to the per-slot path
def test_grouped_integer_exact(lf, grouped, seed, I, K, P, e, k, J):
    """Duplicates, explicit zeros, empty rows, folded rows (l > W), P > 1."""
    A_h = gen.random_small(I, K, 90, seed, dup=True, zeros=True, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(K, J, seed, gen.INT, -15, 15)
    C, _ = run(lf, A_h, B_h, P, e, k)
    Cref, _ = oracle.spmm_csr(A_h, B_h)
    assert np.array_equal(C, Cref)


@pytest.mark.parametrize("J", [32, 64, 128, 256])
def test_grouped_stencil_float(lf, grouped, J):
    """27-point stencil (the banded workload the grouped path is for)."""
    A_h = gen.stencil27(14, seed=3)
    B_h = gen.dense(A_h.n_cols, J, 3)
    C, _ = run(lf, A_h, B_h, 1, 5)
    Cref, Cabs = oracle.spmm_csr(A_h, B_h)
    assert np.all(np.abs(C - Cref) <= TOL * Cabs)


@pytest.mark.parametrize("hw,e", [(2, 2), (8, 4), (15, 5), (40, 5)])
def test_grouped_banded_float(lf, grouped, hw, e):
    """Banded rows of 2hw+1 entries: hw=40 folds every row into 3 CELL rows."""
    A_h = gen.banded(3000, hw, seed=4)
    B_h = gen.dense(A_h.n_cols, 64, 4)
    C, _ = run(lf, A_h, B_h, 2, [e, e])
    Cref, Cabs = oracle.spmm_csr(A_h, B_h)
    assert np.all(np.abs(C - Cref) <= TOL * Cabs)


@pytest.mark.parametrize("env", ["LF_GROUPED", "LF_MMA"])
@pytest.mark.parametrize("J", [64, 128])
def test_grouped_equals_per_slot_path(lf, monkeypatch, env, J):
    """Same handle, per-slot vs grouped path: equal on integer inputs (R-MAT:
    most 16-row groups exceed the tensor-core path's 64 distinct columns and
    take its per-row fallback); repeated launches (queue counters reset by
    the last warp) stay equal."""
    A_h = gen.rmat(12, 16, seed=5, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, J, 5, gen.INT, -15, 15)
    A = lf.Csr.from_host(A_h)
    M = lf.CellMatrix.build(A, lf.make_params(1, 5))
    Bd = torch.from_numpy(B_h).cuda()
    monkeypatch.setenv("LF_GROUPED", "0")
    monkeypatch.setenv("LF_MMA", "0")
    C0 = M.spmm(Bd).cpu().numpy()
    monkeypatch.setenv(env, "1")
    for _ in range(3):
        assert np.array_equal(M.spmm(Bd).cpu().numpy(), C0)


def test_grouped_full_stencil_sampled(lf, grouped):
    """Config 3 (27-point stencil, 126^3, J = 64) at full size, CELL forced,
    sampled rows against the oracle."""
    A_h, J = gen.config("c3_stencil126")
    A = lf.Csr.from_host(A_h)
    params, stats = lf.configure(A, J, force_format=1, force_parts=1)
    M = lf.CellMatrix.build(A, params, stats)
    B_h = gen.dense(A_h.n_cols, J, 0)
    C = M.spmm(torch.from_numpy(B_h).cuda()).cpu().numpy().astype(np.float64)
    rng = np.random.default_rng(0)
    rows = np.unique(np.concatenate([rng.integers(0, A_h.n_rows, 3000), [0, A_h.n_rows - 1]])).astype(np.int64)
    Cref, Cabs = oracle.spmm_csr(A_h, B_h, rows)
    assert np.all(np.abs(C[rows] - Cref) <= TOL * Cabs)


@pytest.mark.parametrize("name,want", [("banded", 1), ("blockdiag32", 1), ("stencil", 1), ("rmat", 0),
                                       ("blockdiag8", 0)])
def test_grouped_heuristic(lf, monkeypatch, name, want):
    """lf_cell_configure's sampled group-union ratio picks the grouped path
    where it measured faster (banded, 32-wide dense blocks, 27-point stencil),
    not on R-MAT or rows of 8; lf_spmm on the automatically chosen path
    matches the oracle."""
    monkeypatch.delenv("LF_GROUPED", raising=False)
    A_h = {"banded": lambda: gen.banded(20000, 12, seed=6), "blockdiag32": lambda: gen.blockdiag(16384, 32, seed=6),
           "stencil": lambda: gen.stencil27(24, seed=6), "rmat": lambda: gen.rmat(14, 16, seed=6),
           "blockdiag8": lambda: gen.blockdiag(16384, 8, seed=6)}[name]()
    A = lf.Csr.from_host(A_h)
    params, stats = lf.configure(A, 64, force_format=1, force_parts=1)
    assert stats.spmm_grouped == want, stats.group_union_ratio
    M = lf.CellMatrix.build(A, params, stats)
    B_h = gen.dense(A_h.n_cols, 64, 6)
    C = M.spmm(torch.from_numpy(B_h).cuda()).cpu().numpy().astype(np.float64)
    Cref, Cabs = oracle.spmm_csr(A_h, B_h)
    assert np.all(np.abs(C - Cref) <= TOL * Cabs)


@pytest.mark.parametrize("J,ldb,ldc", [(64, 68, 72), (128, 132, 256), (32, 36, 32), (60, 64, 64)])
def test_grouped_strided(lf, grouped, J, ldb, ldc):
    """Row strides ldb / ldc > J (16-byte multiples: the grouped paths run;
    J = 60 is not a multiple of 64, so the tensor-core path falls back)."""
    A_h = gen.banded(3000, 12, seed=7, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, J, 7, gen.INT, -15, 15)
    A = lf.Csr.from_host(A_h)
    M = lf.CellMatrix.build(A, lf.make_params(1, 5))
    big = torch.full((A_h.n_cols, ldb), float("nan"), device="cuda")
    big[:, :J] = torch.from_numpy(B_h).cuda()
    out = torch.full((A_h.n_rows, ldc), float("nan"), device="cuda")[:, :J]
    C = M.spmm(big[:, :J], out=out).cpu().numpy().astype(np.float64)
    Cref, _ = oracle.spmm_csr(A_h, B_h)
    assert np.array_equal(C, Cref)


def test_grouped_edge_cases(lf, grouped):
    """No entries (C exactly +0.0), fewer rows than a group, one column,
    NaN in B rows that no nonzero references (must not leak through the
    zero-valued entries of a group)."""
    A_h = gen.CSR(7, 5, np.zeros(8, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32))
    M = lf.CellMatrix.build(lf.Csr.from_host(A_h), lf.make_params(1, 2))
    C = M.spmm(torch.full((5, 64), 3.0, device="cuda"), out=torch.full((7, 64), float("nan"), device="cuda"))
    assert torch.equal(C, torch.zeros(7, 64, device="cuda"))
    for I, K in ((1, 1), (3, 1), (3, 40), (5, 2)):
        A_h = gen.random_small(I, K, 30, I + K, dup=True, zeros=True, kind=gen.INT)
        B_h = gen.dense(K, 64, 3, gen.INT, -15, 15)
        C, _ = run(lf, A_h, B_h, 1, 5)
        Cref, _ = oracle.spmm_csr(A_h, B_h)
        assert np.array_equal(C, Cref)
    # rows 0..3 use columns {0, 1} / {2} only: B rows 3.. hold NaN and are never read
    A_h = gen.CSR(4, 6, np.array([0, 2, 3, 4, 5], np.int64), np.array([0, 1, 2, 0, 1], np.int32),
                  np.array([1, 2, 3, 4, 5], np.float32))
    B_h = np.full((6, 64), np.nan, np.float32)
    B_h[:3] = gen.dense(3, 64, 4, gen.INT, -15, 15)
    C, _ = run(lf, A_h, B_h, 1, 5)
    Cref, _ = oracle.spmm_csr(A_h, np.nan_to_num(B_h))
    assert np.array_equal(C, Cref)
