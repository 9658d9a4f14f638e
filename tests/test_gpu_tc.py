"""GPU parity of the tcgen05 windowed path (cell_spmm_tc.cu) against the oracle.

Groups of 128 CELL rows of a W <= 32 bucket are contracted on the tensor cores
over their B-row window (kind::tf32, 3xTF32 split, A operand in TMEM).  It
must give Alg. 1's C: EXACTLY on integer inputs (small integers are tf32-exact,
so the lo parts vanish and every partial sum is an exact fp32 integer), within
max|C - C_ref| <= 1e-5 (|A|.|B|) on float inputs.  LF_TC=1 forces the path
(the per-group windows are built at lf_cell_build when LF_TC=1 or when the
sizes are GPU-counted), LF_TC=0 forbids it.
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


@pytest.fixture
def tc(monkeypatch):
    monkeypatch.setenv("LF_TC", "1")
    monkeypatch.setenv("LF_GROUPED", "0")


def run(lf, A_h, B_h, P, e, k=None, ldb=None, ldc=None):
    A = lf.Csr.from_host(A_h)
    M = lf.CellMatrix.build(A, lf.make_params(P, e, k))
    J = B_h.shape[1]
    Bd = torch.from_numpy(B_h).cuda()
    if ldb is not None:
        big = torch.full((B_h.shape[0], ldb), float("nan"), device="cuda")
        big[:, :J] = Bd
        Bd = big[:, :J]
    out = None if ldc is None else torch.full((A_h.n_rows, ldc), float("nan"), device="cuda")[:, :J]
    C = M.spmm(Bd, out=out).cpu().numpy().astype(np.float64)
    return C, M


@pytest.mark.parametrize("J", [32, 64, 96, 100, 128])
@pytest.mark.parametrize("n,hw", [(1000, 12), (4096, 3), (777, 31), (300, 60), (5000, 100)])
def test_tc_banded_integer_exact(lf, tc, n, hw, J):
    """Bands of several half-widths (windows up to the 256-row cap), ragged
    last group, edge rows in smaller buckets, folded rows (hw > 15 at W = 32:
    a group holds several sub-rows per source row, combined with red.add)."""
    A_h = gen.banded(n, hw, seed=n + hw, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, J, 3, gen.INT, -15, 15)
    C, M = run(lf, A_h, B_h, 1, 5)
    assert M.path(J) == "cell_spmm_tc_kernel"
    assert np.array_equal(C, oracle.spmm_csr(A_h, B_h)[0])


CASES = []
for s in range(10):
    rng = np.random.default_rng(900 + s)
    P = int(rng.integers(1, 4))
    e = rng.integers(0, 6, size=P).tolist()
    k = [x + int(rng.integers(0, 3)) for x in e]
    CASES.append((s, int(rng.integers(1, 700)), int(rng.integers(1, 400)), P, e, k))


@pytest.mark.parametrize("seed,I,K,P,e,k", CASES)
@pytest.mark.parametrize("J", [32, 128])
def test_tc_random_integer_exact(lf, tc, seed, I, K, P, e, k, J):
    """Duplicates (summed), explicit zeros, empty rows, folded rows, P > 1
    (several CELL rows per C row: red.add), windows both inside and beyond the
    cap (uniform columns over K up to 400)."""
    A_h = gen.random_small(I, K, 90, seed, dup=True, zeros=True, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(K, J, seed, gen.INT, -15, 15)
    C, _ = run(lf, A_h, B_h, P, e, k)
    assert np.array_equal(C, oracle.spmm_csr(A_h, B_h)[0])


@pytest.mark.parametrize("J", [32, 128])
def test_tc_wide_window_fallback(lf, tc, J):
    """Uniform columns over 3000: every group's window exceeds the 256-row cap,
    so all groups take the in-kernel CUDA-core fallback; a band glued below
    mixes tensor-core and fallback groups in one launch."""
    U_h = gen.uniform(3000, 3000, 1 / 200, seed=11, kind=gen.INT, lo=-3, hi=3)
    Bd_h = gen.banded(3000, 12, seed=11, kind=gen.INT, lo=-3, hi=3)
    rp = np.concatenate([U_h.row_ptr, Bd_h.row_ptr[1:] + U_h.row_ptr[-1]]).astype(np.int64)
    A_h = gen.CSR(6000, 3000, rp, np.concatenate([U_h.col_ind, Bd_h.col_ind]), np.concatenate([U_h.val, Bd_h.val]))
    B_h = gen.dense(3000, J, 11, gen.INT, -15, 15)
    C, M = run(lf, A_h, B_h, 1, 5)
    assert M.path(J) == "cell_spmm_tc_kernel"
    assert np.array_equal(C, oracle.spmm_csr(A_h, B_h)[0])


@pytest.mark.parametrize("J", [64, 128])
@pytest.mark.parametrize("kind", ["band", "blockdiag32", "blockdiag8", "pos"])
def test_tc_float_tolerance(lf, tc, kind, J):
    if kind == "band":
        A_h, B_h = gen.banded(20000, 12, seed=1), gen.dense(20000, J, 1)
    elif kind == "blockdiag32":
        A_h, B_h = gen.blockdiag(16384, 32, seed=2), gen.dense(16384, J, 2)
    elif kind == "blockdiag8":
        A_h, B_h = gen.blockdiag(16384, 8, seed=3), gen.dense(16384, J, 3)
    else:  # GNN-style all-positive: the adversarial case for a relative bound
        A_h, B_h = gen.banded(9000, 12, seed=4, kind=gen.ONE), gen.dense(9000, J, 4, gen.POS)
    C, M = run(lf, A_h, B_h, 1, 5)
    assert M.path(J) == "cell_spmm_tc_kernel"
    Cref, Cabs = oracle.spmm_csr(A_h, B_h)
    err = np.abs(C - Cref)
    assert np.all(err <= TOL * Cabs), float((err / np.maximum(Cabs, 1e-300)).max())


@pytest.mark.parametrize("J,ldb,ldc", [(64, 68, 72), (128, 132, 256), (32, 36, 32), (60, 64, 64)])
def test_tc_strided(lf, tc, J, ldb, ldc):
    A_h = gen.banded(3000, 12, seed=7, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, J, 7, gen.INT, -15, 15)
    C, _ = run(lf, A_h, B_h, 1, 5, ldb=ldb, ldc=ldc)
    assert np.array_equal(C, oracle.spmm_csr(A_h, B_h)[0])


def test_tc_unreferenced_rows_never_read(lf, tc):
    """B rows inside a group's window that no nonzero references hold NaN / Inf:
    they must not reach C (the loaders read only referenced window rows and
    put exact zeros elsewhere; 0 x NaN would be NaN)."""
    n = 600
    rows = [[i - (i % 4), i - (i % 4) + 3] for i in range(n)]  # columns 4q and 4q+3 only
    rp = np.concatenate([[0], np.cumsum([len(r) for r in rows])]).astype(np.int64)
    ci = np.concatenate([np.array(r, np.int32) for r in rows])
    A_h = gen.CSR(n, n, rp, ci, gen.fill(len(ci), 5, 1, gen.INT, -3, 3))
    B_h = gen.dense(n, 64, 5, gen.INT, -15, 15)
    B_bad = B_h.copy()
    B_bad[1::4] = np.nan
    B_bad[2::4] = np.inf
    C, M = run(lf, A_h, B_bad, 1, 5)
    assert M.path(64) == "cell_spmm_tc_kernel"
    assert np.array_equal(C, oracle.spmm_csr(A_h, B_h)[0])


def test_tc_equals_other_paths_repeated(lf, monkeypatch):
    """Same handle: per-slot, grouped and tcgen05 paths give the same C on
    integer inputs; repeated TC launches (persistent CTAs, TMEM allocated and
    freed per launch, mbarrier phases) stay equal."""
    monkeypatch.setenv("LF_TC", "1")
    A_h = gen.banded(50000, 12, seed=9, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, 128, 9, gen.INT, -15, 15)
    A = lf.Csr.from_host(A_h)
    M = lf.CellMatrix.build(A, lf.make_params(1, 5))
    Bd = torch.from_numpy(B_h).cuda()
    ref = oracle.spmm_csr(A_h, B_h)[0]
    outs = [M.spmm(Bd).cpu().numpy() for _ in range(5)]
    monkeypatch.setenv("LF_TC", "0")
    monkeypatch.setenv("LF_GROUPED", "1")
    outs.append(M.spmm(Bd).cpu().numpy())
    monkeypatch.setenv("LF_GROUPED", "0")
    outs.append(M.spmm(Bd).cpu().numpy())
    for C in outs:
        assert np.array_equal(C.astype(np.float64), ref)


@pytest.mark.parametrize("name,want", [("banded", 1), ("blockdiag32", 1), ("stencil", 0), ("rmat", 0),
                                       ("uniform", 0)])
def test_tc_heuristic(lf, monkeypatch, name, want):
    """lf_cell_configure's sampled 128-row windows choose the tcgen05 path for
    banded / block-diagonal matrices, not for the stencil (window ~ 2 planes),
    R-MAT or uniform columns; the chosen path matches the oracle."""
    monkeypatch.delenv("LF_TC", raising=False)
    monkeypatch.delenv("LF_GROUPED", raising=False)
    A_h = {"banded": lambda: gen.banded(20000, 12, seed=6), "blockdiag32": lambda: gen.blockdiag(16384, 32, seed=6),
           "stencil": lambda: gen.stencil27(24, seed=6), "rmat": lambda: gen.rmat(14, 16, seed=6),
           "uniform": lambda: gen.uniform(8192, 8192, 1 / 512, seed=6)}[name]()
    A = lf.Csr.from_host(A_h)
    params, stats = lf.configure(A, 128, force_format=1, force_parts=1)
    assert stats.spmm_tc == want, (stats.window_span_mean, stats.window_over_frac)
    M = lf.CellMatrix.build(A, params, stats)
    assert (M.path(128) == "cell_spmm_tc_kernel") == bool(want)
    B_h = gen.dense(A_h.n_cols, 128, 6)
    C = M.spmm(torch.from_numpy(B_h).cuda()).cpu().numpy().astype(np.float64)
    Cref, Cabs = oracle.spmm_csr(A_h, B_h)
    assert np.all(np.abs(C - Cref) <= TOL * Cabs)


@pytest.mark.parametrize("J", [64, 128])
def test_tc_full_c3b(lf, monkeypatch, J):
    """Config c3b (band half-width 12, 2M rows) at full size through configure
    (which picks the tcgen05 path), the bench's launch configuration: CELL
    bit-exact, sampled C rows within tolerance, integer-valued run exact on
    sampled rows."""
    monkeypatch.delenv("LF_TC", raising=False)
    monkeypatch.delenv("LF_GROUPED", raising=False)
    A_h, _ = gen.config("c3b_banded2M")
    A = lf.Csr.from_host(A_h)
    params, stats = lf.configure(A, J)
    assert params.use_cell == 1 and stats.spmm_tc == 1
    M = lf.CellMatrix.build(A, params, stats)
    assert M.path(J) == "cell_spmm_tc_kernel"
    B_h = gen.dense(A_h.n_cols, J, 0)
    C = M.spmm(torch.from_numpy(B_h).cuda()).cpu().numpy().astype(np.float64)
    rng = np.random.default_rng(0)
    rows = np.unique(np.concatenate([rng.integers(0, A_h.n_rows, 4000), np.arange(0, 300),
                                     np.arange(A_h.n_rows - 300, A_h.n_rows)])).astype(np.int64)
    Cref, Cabs = oracle.spmm_csr(A_h, B_h, rows)
    assert np.all(np.abs(C[rows] - Cref) <= TOL * Cabs)
    Ai_h, _ = gen.config("c3b_banded2M", kind=gen.INT, lo=-3, hi=3)
    Bi_h = gen.dense(A_h.n_cols, J, 1, gen.INT, -15, 15)
    Mi = lf.CellMatrix.build(lf.Csr.from_host(Ai_h), params, stats)
    Ci = Mi.spmm(torch.from_numpy(Bi_h).cuda()).cpu().numpy().astype(np.float64)
    assert np.array_equal(Ci[rows], oracle.spmm_csr(Ai_h, Bi_h, rows)[0])


def test_tc_edge_cases(lf, tc):
    """No entries (C exactly +0.0), fewer rows than a group, a single column,
    empty rows between real ones, J just above the 32 minimum; and J = 256 /
    J = 16, which the windowed path does not take (per-slot / grouped path
    instead, same result)."""
    A_h = gen.CSR(7, 5, np.zeros(8, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32))
    M = lf.CellMatrix.build(lf.Csr.from_host(A_h), lf.make_params(1, 2))
    C = M.spmm(torch.full((5, 64), 3.0, device="cuda"), out=torch.full((7, 64), float("nan"), device="cuda"))
    assert torch.equal(C, torch.zeros(7, 64, device="cuda"))
    for I, K, J in ((1, 1, 32), (3, 1, 36), (130, 40, 64), (129, 300, 128), (5, 2, 16), (200, 200, 256)):
        A_h = gen.random_small(I, K, 30, I + K, dup=True, zeros=True, kind=gen.INT)
        B_h = gen.dense(K, J, 3, gen.INT, -15, 15)
        C, M = run(lf, A_h, B_h, 1, 5)
        assert np.array_equal(C, oracle.spmm_csr(A_h, B_h)[0]), (I, K, J)
        want_tc = 32 <= J <= 128
        assert (M.path(J) == "cell_spmm_tc_kernel") == want_tc, (J, M.path(J))
    # rows with no entries interleaved with banded rows
    A_b = gen.banded(1000, 12, seed=12, kind=gen.INT, lo=-3, hi=3)
    keep = np.arange(1000) % 3 != 1
    l = np.diff(A_b.row_ptr) * keep
    rp = np.concatenate([[0], np.cumsum(l)]).astype(np.int64)
    idx = np.concatenate([np.arange(A_b.row_ptr[i], A_b.row_ptr[i + 1]) for i in range(1000) if keep[i]])
    A_h = gen.CSR(1000, 1000, rp, A_b.col_ind[idx], A_b.val[idx])
    B_h = gen.dense(1000, 128, 4, gen.INT, -15, 15)
    C, M = run(lf, A_h, B_h, 1, 5)
    assert M.path(128) == "cell_spmm_tc_kernel"
    assert np.array_equal(C, oracle.spmm_csr(A_h, B_h)[0])
