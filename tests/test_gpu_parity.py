"""GPU parity: the CUDA path (through the C ABI) against the oracle.

* builder (a1, a4, a5): every CELL array and the bucket table BIT-EXACT;
* configure statistics (a2) and eq. 7 / Algorithm 3 (a3): exact integers;
* SpMM (a6, a7): integer-valued inputs (|A| <= 3, |B| <= 15, every partial
  sum < 2^24) must match EXACTLY whatever the atomic order; float inputs
  within max|C - C_ref| <= 1e-5 * (|A|.|B|) elementwise (BASELINE.json);
* full-size BASELINE configs in the bench's launch configuration on sampled
  rows, plus edge cases (empty, ragged, J not a multiple of 4, ldb/ldc > J,
  K < P, empty partitions).
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


def build(lf, A_h, P, e, k=None):
    A = lf.Csr.from_host(A_h)
    M = lf.CellMatrix.build(A, lf.make_params(P, e, k))
    return A, M


def assert_cell_equal(M, cell):
    v = M.view()
    torch.cuda.synchronize()
    assert np.array_equal(v["row_ind"].cpu().numpy(), cell.row_ind)
    assert np.array_equal(v["col_ind"].cpu().numpy(), cell.col_ind)
    assert np.array_equal(v["val"].cpu().numpy().view(np.int32), cell.val.view(np.int32))
    got = [(b["part"], b["width_log2"], b["rows_per_block"], b["n_rows"], b["n_rows_pad"], b["row_off"],
            b["slot_off"]) for b in v["buckets"]]
    exp = [tuple(int(b[f]) for f in ("part", "width_log2", "rows_per_block", "n_rows", "n_rows_pad", "row_off",
                                     "slot_off")) for b in cell.buckets]
    assert got == exp


def spmm_check(M, A_h, B_h, exact=False, rows=None, ldb=None, ldc=None):
    J = B_h.shape[1]
    Bd = torch.from_numpy(B_h).cuda()
    if ldb is not None:
        big = torch.full((B_h.shape[0], ldb), float("nan"), device="cuda")
        big[:, :J] = Bd
        Bd = big[:, :J]
    out = None
    if ldc is not None:
        out = torch.full((A_h.n_rows, ldc), float("nan"), device="cuda")[:, :J]
    C = M.spmm(Bd, out=out).cpu().numpy().astype(np.float64)
    Cref, Cabs = oracle.spmm_csr(A_h, B_h, rows)
    if rows is not None:
        C = C[rows]
    if exact:
        assert np.array_equal(C, Cref)
    else:
        err = np.abs(C - Cref)
        assert np.all(err <= TOL * Cabs), float((err / np.maximum(Cabs, 1e-300)).max())
    return C


SMALL = []
for s in range(20):
    rng = np.random.default_rng(s)
    P = int(rng.integers(1, 6))
    e = rng.integers(0, 7, size=P).tolist()
    k = [x + int(rng.integers(0, 3)) for x in e]
    SMALL.append((s, int(rng.integers(0, 300)), int(rng.integers(1, 200)), P, e, k))


@pytest.mark.parametrize("seed,I,K,P,e,k", SMALL)
def test_builder_bit_exact_small(lf, seed, I, K, P, e, k):
    A_h = gen.random_small(I, K, 90, seed, dup=True, zeros=True)
    _, M = build(lf, A_h, P, e, k)
    assert_cell_equal(M, oracle.csr_to_cell(A_h, P, e, k))


@pytest.mark.parametrize("seed,I,K,P,e,k", SMALL[:10])
@pytest.mark.parametrize("J", [1, 3, 4, 32, 64, 96, 128, 256, 512, 520])
def test_spmm_integer_exact(lf, seed, I, K, P, e, k, J):
    A_h = gen.random_small(I, K, 90, seed, dup=True, zeros=True, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(K, J, seed, gen.INT, -15, 15)
    _, M = build(lf, A_h, P, e, k)
    spmm_check(M, A_h, B_h, exact=True)


@pytest.mark.parametrize("J,ldb,ldc", [(4, 8, 12), (32, 36, 40), (7, 9, 11), (128, 132, 256)])
def test_spmm_strided(lf, J, ldb, ldc):
    A_h = gen.rmat(11, 16, seed=1, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, J, 1, gen.INT, -15, 15)
    _, M = build(lf, A_h, 2, [3, 4])
    spmm_check(M, A_h, B_h, exact=True, ldb=ldb, ldc=ldc)


@pytest.mark.parametrize("P", [1, 3])
@pytest.mark.parametrize("J", [32, 128, 256])
def test_spmm_tolerance_float(lf, P, J):
    A_h = gen.rmat(13, 16, seed=2)
    B_h = gen.dense(A_h.n_cols, J, 2)
    params, _ = lf.configure(lf.Csr.from_host(A_h), J, force_parts=P)
    A = lf.Csr.from_host(A_h)
    M = lf.CellMatrix.build(A, params)
    spmm_check(M, A_h, B_h)


@pytest.mark.parametrize("P", [1, 3])
def test_build_with_stats_equals_counted(lf, P):
    """lf_cell_build with the configure statistics (no host sync) produces the
    same arrays as the GPU-counted path, and both equal the oracle."""
    A_h = gen.rmat(12, 16, seed=11)
    A = lf.Csr.from_host(A_h)
    params, stats = lf.configure(A, 64, force_parts=P)
    M1 = lf.CellMatrix.build(A, params, stats)
    M2 = lf.CellMatrix.build(A, params)
    P_ = params.n_parts
    cell = oracle.csr_to_cell(A_h, P_, list(params.max_width_log2[:P_]), list(params.block_nnz_log2[:P_]))
    assert_cell_equal(M1, cell)
    assert_cell_equal(M2, cell)
    with pytest.raises(lf.LfError):
        _, st1 = lf.configure(A, 64, force_parts=P + 1)
        lf.CellMatrix.build(A, params, st1)


def test_spmm_positive_gnn_style(lf):
    """All-positive values (val = 1, B in [0,1)): the adversarial case for the
    relative tolerance; long rows fold."""
    A_h = gen.powerlaw(3000, 400000, 1.5, seed=3, kind=gen.ONE)
    B_h = gen.dense(A_h.n_cols, 64, 3, gen.POS)
    A = lf.Csr.from_host(A_h)
    params, _ = lf.configure(A, 64)
    M = lf.CellMatrix.build(A, params)
    spmm_check(M, A_h, B_h)


def test_configure_stats_and_alg3_match_oracle(lf):
    for A_h, Ps in ((gen.rmat(12, 16, seed=5), (1, 2, 5)), (gen.random_small(200, 150, 120, 9), (1, 4)),
                    (gen.stencil27(9), (1, 3))):
        A = lf.Csr.from_host(A_h)
        for P in Ps:
            for J in (32, 128):
                params, st = lf.configure(A, J, force_parts=P)
                assert params.n_parts == P
                for p in range(P):
                    H, F, Un, Ut = oracle.partition_stats(A_h, P, p)
                    assert list(st.H[p]) == H.tolist()
                    assert list(st.F[p]) == F.tolist()
                    assert list(st.Unat[p]) == Un.tolist()
                    assert list(st.Utop[p]) == Ut.tolist()
                    top = oracle.partition_max_log2(A_h, P, p)
                    assert st.max_log2[p] == top
                    for e in range(top + 1):
                        assert st.cost[p][e] == oracle.partition_cost(A_h, P, p, e, J)
                    assert st.chosen_log2[p] == oracle.build_buckets(A_h, P, p, J)
                    assert params.max_width_log2[p] == max(oracle.build_buckets(A_h, P, p, J), 0)
        f = oracle.features(A_h)
        assert list(st.features[:3]) == f[:3].tolist() and list(st.features[4:6]) == f[4:6].tolist()
        assert st.features[3] == pytest.approx(f[3], rel=1e-14)
        assert st.features[6] == pytest.approx(f[6], rel=1e-9)


def _hot_column_csr(n_rows: int, n_cols: int, seed: int) -> "gen.CSR":
    """Every row holds column 7 plus 0..5 random columns: >= 2^20 nonzeros in
    rows of several natural buckets, a third of them in one column."""
    rng = np.random.default_rng(seed)
    lens = rng.integers(0, 6, size=n_rows)
    rp = np.zeros(n_rows + 1, np.int64)
    rp[1:] = np.cumsum(lens + 1)
    ci = np.empty(int(rp[-1]), np.int32)
    extra = rng.integers(8, n_cols, size=int(lens.sum())).astype(np.int32)
    ci[rp[:-1]] = 7
    pos = np.repeat(rp[:-1] + 1, lens) + (np.arange(int(lens.sum())) - np.repeat(np.cumsum(lens) - lens, lens))
    ci[pos] = extra
    for i in np.flatnonzero(lens > 1):  # rows sorted by column (CSR contract)
        ci[rp[i]:rp[i + 1]] = np.sort(ci[rp[i]:rp[i + 1]])
    return gen.CSR(n_rows, n_cols, rp, ci, gen.fill(len(ci), seed, gen.STREAM_VAL, gen.INT, -3, 3), "hotcol")


@pytest.mark.parametrize("case", ["rmat16", "hotcol"])
def test_configure_large_inputs_match_oracle(lf, case):
    """Column marking (stats_mark_kernel) on >= 2^20 nonzeros in tiles of
    several natural buckets: a power-law matrix, and one with a third of its
    nonzeros in a single column (every tile marks that column).  Unat / Utop
    / H / F and Algorithm 3 == the oracle at P = 1 and 3."""
    A_h = gen.rmat(16, 20, seed=3) if case == "rmat16" else _hot_column_csr(1 << 20, 40000, 4)
    assert A_h.nnz >= 1 << 20
    A = lf.Csr.from_host(A_h)
    for P in (1, 3):
        params, st = lf.configure(A, 64, force_parts=P, force_format=1)
        for p in range(P):
            H, F, Un, Ut = oracle.partition_stats(A_h, P, p)
            assert list(st.H[p]) == H.tolist() and list(st.F[p]) == F.tolist()
            assert list(st.Unat[p]) == Un.tolist() and list(st.Utop[p]) == Ut.tolist()
            assert st.chosen_log2[p] == oracle.build_buckets(A_h, P, p, 64)


def test_configure_very_long_rows(lf):
    """Natural buckets up to t = 22 (rows of 1 .. 2^21 + 3 nonzeros, one of them
    2^21 + 3 long, plus empty rows): H / F / Unat / Utop per bucket (the P = 1
    statistics pass keeps H[t], F[t] of bucket t in lane t) == the oracle."""
    rng = np.random.default_rng(11)
    lens = np.concatenate([[0, 1, 2, 3, 5, 33, 1000, (1 << 21) + 3, 0, 70000], rng.integers(0, 40, 3000)])
    n_cols = 1 << 22
    rows = [np.sort(rng.choice(n_cols, size=int(l), replace=False)).astype(np.int32) if l else np.zeros(0, np.int32)
            for l in lens]
    rp = np.zeros(len(lens) + 1, np.int64)
    rp[1:] = np.cumsum(lens)
    ci = np.concatenate(rows)
    A_h = gen.CSR(len(lens), n_cols, rp, ci, gen.fill(len(ci), 11, gen.STREAM_VAL, gen.INT, -3, 3), "longrows")
    A = lf.Csr.from_host(A_h)
    params, st = lf.configure(A, 32, force_parts=1, force_format=1)
    H, F, Un, Ut = oracle.partition_stats(A_h, 1, 0)
    assert list(st.H[0]) == H.tolist() and list(st.F[0]) == F.tolist()
    assert list(st.Unat[0]) == Un.tolist() and list(st.Utop[0]) == Ut.tolist()
    assert st.max_log2[0] == 22 and st.chosen_log2[0] == oracle.build_buckets(A_h, 1, 0, 32)


def test_golden_configure_on_gpu(lf):
    """The hand-worked eq. 7 examples, through the GPU statistics."""
    from conftest import read_golden
    for name in ("cost_5x8.txt", "cost_separating_2x16.txt"):
        g = read_golden(name)
        rows = g["rows"]
        rp = np.concatenate([[0], np.cumsum([len(r) for r in rows])]).astype(np.int64)
        ci = np.concatenate([np.array(r, np.int32) for r in rows])
        A_h = gen.CSR(len(rows), g["K"][0], rp, ci, np.ones(len(ci), np.float32))
        params, st = lf.configure(lf.Csr.from_host(A_h), g["J"][0], force_parts=1)
        assert list(st.cost[0][:len(g["cost"])]) == g["cost"]
        assert params.max_width_log2[0] == g["alg3_e"][0]


def test_edge_cases(lf):
    # no rows
    A_h = gen.CSR(0, 5, np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32))
    _, M = build(lf, A_h, 1, 2)
    assert M.spmm(torch.ones(5, 4, device="cuda")).shape == (0, 4)
    # no entries: C must be exactly +0.0
    A_h = gen.CSR(7, 5, np.zeros(8, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32))
    _, M = build(lf, A_h, 2, 2)
    C = M.spmm(torch.full((5, 8), 3.0, device="cuda"), out=torch.full((7, 8), float("nan"), device="cuda"))
    assert torch.equal(C, torch.zeros(7, 8, device="cuda"))
    # K < P (empty partitions), J = 0
    A_h = gen.random_small(20, 3, 5, 2, kind=gen.INT)
    _, M = build(lf, A_h, 5, [1, 2, 0, 3, 1])
    assert_cell_equal(M, oracle.csr_to_cell(A_h, 5, [1, 2, 0, 3, 1]))
    B_h = gen.dense(3, 5, 2, gen.INT)
    spmm_check(M, A_h, B_h, exact=True)
    assert M.spmm(torch.zeros(3, 0, device="cuda")).shape == (20, 0)


def test_csr_path_and_errors(lf):
    A_h = gen.rmat(11, 16, seed=8, kind=gen.INT)
    B_h = gen.dense(A_h.n_cols, 64, 8, gen.INT)
    A = lf.Csr.from_host(A_h)
    C = lf.csr_spmm(A, torch.from_numpy(B_h).cuda()).cpu().numpy()
    assert np.array_equal(C.astype(np.float64), oracle.spmm_csr(A_h, B_h)[0])
    params, _ = lf.configure(A, 64, force_format=2)
    assert params.use_cell == 0
    M = lf.CellMatrix.build(A, params)
    spmm_check(M, A_h, B_h, exact=True)
    with pytest.raises(lf.LfError):
        lf.CellMatrix.build(A, lf.make_params(1, 4, 3))


def test_row_shard_view(lf):
    """row_ptr slice with a non-zero base (row sharding) builds the same CELL as
    the standalone slice."""
    A_h = gen.rmat(11, 16, seed=6)
    lo, hi = 300, 1500
    A = lf.Csr.from_host(A_h)
    shard = lf.Csr(A.row_ptr[lo:hi + 1], A.col_ind, A.val, A.n_cols)
    sub = gen.CSR(hi - lo, A_h.n_cols, A_h.row_ptr[lo:hi + 1] - A_h.row_ptr[lo],
                  A_h.col_ind[A_h.row_ptr[lo]:A_h.row_ptr[hi]], A_h.val[A_h.row_ptr[lo]:A_h.row_ptr[hi]])
    M = lf.CellMatrix.build(shard, lf.make_params(2, [4, 3]))
    assert_cell_equal(M, oracle.csr_to_cell(sub, 2, [4, 3]))
    B_h = gen.dense(A_h.n_cols, 32, 6)
    spmm_check(M, sub, B_h)


# ---- full-size BASELINE configs, the bench's launch configuration ----------
FULL = ["c1_uniform1024", "c2_rmat20", "c2p_rmat20_perm", "c3_stencil126", "c3b_banded2M"]


@pytest.mark.parametrize("name", FULL)
def test_full_config_parity(lf, name):
    A_h, J = gen.config(name)
    A = lf.Csr.from_host(A_h)
    params, stats = lf.configure(A, J)
    # the predictor's decision is the one lf_predict makes on the same features,
    # except that the grouped CELL path overrides a CSR verdict (lf_api.cu)
    pu, pp = lf.predict(list(stats.features))
    assert params.n_parts == pp
    assert params.use_cell == (1 if stats.spmm_grouped else pu)
    if params.use_cell == 0:  # fixed CSR format chosen: check CELL at the predicted P too
        params, stats = lf.configure(A, J, force_parts=params.n_parts, force_format=1)
    M = lf.CellMatrix.build(A, params, stats)  # the bench's path: sizes from the stats, no sync
    P = params.n_parts
    cell = oracle.csr_to_cell(A_h, P, list(params.max_width_log2[:P]), list(params.block_nnz_log2[:P]))
    assert_cell_equal(M, cell)
    B_h = gen.dense(A_h.n_cols, J, 0)
    rng = np.random.default_rng(0)
    l = A_h.row_lengths()
    rows = np.unique(np.concatenate([rng.integers(0, A_h.n_rows, 3000), np.argsort(l)[-50:],
                                     np.flatnonzero(l == 0)[:50], [0, A_h.n_rows - 1]])).astype(np.int64)
    spmm_check(M, A_h, B_h, rows=rows)


def test_full_reddit_parity(lf):
    """c4 (Reddit-shaped, 114.6M nnz) on its production path: the predictor's P
    (8 on B200), widths from the GPU statistics.  The widths must equal the
    oracle's Algorithm 3 per partition, the WHOLE CELL (every array, every
    bucket) must equal the oracle's bit for bit, and sampled C rows (incl. the
    20 longest) must be within tolerance."""
    A_h, J = gen.config("c4_reddit")
    A = lf.Csr.from_host(A_h)
    params, stats = lf.configure(A, J)
    P = params.n_parts
    assert params.use_cell == 1
    e_or, _ = oracle.configure(A_h, P, J)
    assert list(params.max_width_log2[:P]) == e_or.tolist()
    M = lf.CellMatrix.build(A, params, stats)  # bench path: sizes from the stats, no sync
    cell = oracle.csr_to_cell(A_h, P, list(params.max_width_log2[:P]), list(params.block_nnz_log2[:P]))
    assert_cell_equal(M, cell)
    del cell
    B_h = gen.dense(A_h.n_cols, J, 0)
    rng = np.random.default_rng(1)
    l = A_h.row_lengths()
    rows = np.unique(np.concatenate([rng.integers(0, A_h.n_rows, 500), np.argsort(l)[-20:]])).astype(np.int64)
    spmm_check(M, A_h, B_h, rows=rows)


def test_reddit_shard_p8(lf):
    """A 1/8 row shard of c4 (the multi-GPU unit of work, nnz-balanced bounds)
    configured and built from a row_ptr VIEW with a non-zero base at P = 8:
    configure == the oracle's Algorithm 3 on the standalone sub-CSR, CELL bit-exact,
    C exact on integer inputs."""
    from paper_conf_hpdc_pengtpk25_b200 import dist as lfd
    A_h, J = gen.config("c4_reddit", kind=gen.INT, lo=-3, hi=3)
    bounds = lfd.shard_bounds(A_h.row_ptr, 8, J, "nnz")
    lo, hi = int(bounds[3]), int(bounds[4])
    p0, p1 = int(A_h.row_ptr[lo]), int(A_h.row_ptr[hi])
    sub = gen.CSR(hi - lo, A_h.n_cols, A_h.row_ptr[lo:hi + 1] - p0, A_h.col_ind[p0:p1], A_h.val[p0:p1])
    A = lf.Csr.from_host(A_h)
    shard = lf.Csr(A.row_ptr[lo:hi + 1], A.col_ind, A.val, A.n_cols, p1 - p0)
    params, stats = lf.configure(shard, J, force_parts=8, force_format=1)
    e_or, _ = oracle.configure(sub, 8, J)
    assert list(params.max_width_log2[:8]) == e_or.tolist()
    for p in range(8):
        top = oracle.partition_max_log2(sub, 8, p)
        assert stats.max_log2[p] == top
        for e in range(max(0, e_or[p] - 1), min(top, e_or[p] + 1) + 1):
            assert stats.cost[p][e] == oracle.partition_cost(sub, 8, p, e, J)
    M = lf.CellMatrix.build(shard, params, stats)
    assert_cell_equal(M, oracle.csr_to_cell(sub, 8, list(params.max_width_log2[:8]),
                                            list(params.block_nnz_log2[:8])))
    B_h = gen.dense(A_h.n_cols, J, 5, gen.INT, -15, 15)
    rng = np.random.default_rng(2)
    rows = np.unique(np.concatenate([rng.integers(0, sub.n_rows, 400),
                                     np.argsort(sub.row_lengths())[-10:]])).astype(np.int64)
    spmm_check(M, sub, B_h, exact=True, rows=rows)


@pytest.mark.parametrize("name", ["c2_rmat20", "c2p_rmat20_perm", "c3_stencil126", "c3b_banded2M"])
def test_full_configure_matches_oracle(lf, name):
    """Full-size configure (nnz > 2^25 takes the features-first path on c3 /
    c3b) against the oracle at the P the predictor chose: every eq. 7 cost of
    every partition, the statistics tables (P = 1) and Algorithm 3's e_p."""
    A_h, J = gen.config(name)
    A = lf.Csr.from_host(A_h)
    for Jx in (J, 128):
        params, st = lf.configure(A, Jx, force_format=1)
        P = params.n_parts
        e_or, k_or = oracle.configure(A_h, P, Jx)
        assert list(params.max_width_log2[:P]) == e_or.tolist()
        assert list(params.block_nnz_log2[:P]) == k_or.tolist()
        for p in range(P):
            top = oracle.partition_max_log2(A_h, P, p)
            assert st.max_log2[p] == top
            assert [st.cost[p][e] for e in range(top + 1)] == \
                [oracle.partition_cost(A_h, P, p, e, Jx) for e in range(top + 1)]
            if P == 1 and Jx == J:
                H, F, Un, Ut = oracle.partition_stats(A_h, P, p)
                assert list(st.H[p]) == H.tolist() and list(st.F[p]) == F.tolist()
                assert list(st.Unat[p]) == Un.tolist() and list(st.Utop[p]) == Ut.tolist()


@pytest.mark.parametrize("P", [6, 7, 8])
@pytest.mark.parametrize("seed", range(4))
def test_builder_bit_exact_many_parts(lf, P, seed):
    """P >= 6 (c4's production P is 8): random widths and block multipliers on
    random CSR with duplicates / explicit zeros, and configure-chosen widths on
    an R-MAT, both bit-exact; integer SpMM exact."""
    rng = np.random.default_rng(500 + 10 * P + seed)
    A_h = gen.random_small(int(rng.integers(50, 400)), int(rng.integers(P, 300)), 120, seed, dup=True, zeros=True,
                           kind=gen.INT, lo=-3, hi=3)
    e = rng.integers(0, 7, size=P).tolist()
    k = [x + int(rng.integers(0, 3)) for x in e]
    _, M = build(lf, A_h, P, e, k)
    assert_cell_equal(M, oracle.csr_to_cell(A_h, P, e, k))
    spmm_check(M, A_h, gen.dense(A_h.n_cols, 64, seed, gen.INT, -15, 15), exact=True)
    R_h = gen.rmat(12, 16, seed=seed, kind=gen.INT, lo=-3, hi=3)
    R = lf.Csr.from_host(R_h)
    params, stats = lf.configure(R, 128, force_parts=P, force_format=1)
    M2 = lf.CellMatrix.build(R, params, stats)
    assert_cell_equal(M2, oracle.csr_to_cell(R_h, P, list(params.max_width_log2[:P]),
                                             list(params.block_nnz_log2[:P])))
    spmm_check(M2, R_h, gen.dense(R_h.n_cols, 128, seed, gen.INT, -15, 15), exact=True)


@pytest.mark.parametrize("width", [None, 12])
def test_long_rows_split_into_pieces(lf, width):
    """Rows wider than 2^kPieceLog2 = 1024 slots (the dense rows of an
    arrowhead matrix, Algorithm 3 picks W = 2^14 here; or a forced 2^12 on
    R-MAT) are processed as several wide tasks that red.add into the row:
    the CELL arrays are unchanged and C stays within tolerance."""
    if width is None:
        A_h = gen.arrowhead(1 << 14, 4, seed=1)
        kw = dict(force_parts=1, force_format=1)
    else:
        A_h = gen.rmat(14, 16, seed=4)
        kw = dict(force_parts=1, force_format=1, force_width_log2=width)
    A = lf.Csr.from_host(A_h)
    for J in (64, 128, 512, 640):
        params, stats = lf.configure(A, J, **kw)
        assert params.max_width_log2[0] > 10
        M = lf.CellMatrix.build(A, params, stats)
        cell = oracle.csr_to_cell(A_h, 1, [params.max_width_log2[0]], [params.block_nnz_log2[0]])
        assert_cell_equal(M, cell)
        spmm_check(M, A_h, gen.dense(A_h.n_cols, J, 7))


def test_repeated_launches_reuse_counter_slots(lf):
    """More launches than the handle's counter ring (64 slots, each reset by
    its kernel's last warp), on two streams: every result stays correct."""
    A_h = gen.rmat(12, 16, seed=3, kind=gen.INT)
    B_h = gen.dense(A_h.n_cols, 64, 3, gen.INT)
    A = lf.Csr.from_host(A_h)
    M = lf.CellMatrix.build(A, lf.make_params(1, 4))
    B = torch.from_numpy(B_h).cuda()
    ref = oracle.spmm_csr(A_h, B_h)[0]
    s2 = torch.cuda.Stream()
    torch.cuda.synchronize()
    outs = []
    for it in range(150):
        st = s2 if it % 3 == 0 else torch.cuda.current_stream()
        with torch.cuda.stream(st):
            outs.append(M.spmm(B, stream=st))
    torch.cuda.synchronize()
    for C in outs[::7] + outs[-3:]:
        assert np.array_equal(C.cpu().numpy().astype(np.float64), ref)


def test_host_pipeline_overlapped(lf):
    """HostPipeline: host CSR + B in, host C out, double-buffered over three
    streams; several different problems in flight give their own results."""
    from paper_conf_hpdc_pengtpk25_b200.pipeline import HostPipeline
    J = 64
    probs = []
    for seed in range(4):
        A_h = gen.rmat(11, 8 + 4 * seed, seed=seed, kind=gen.INT)
        B_h = gen.dense(A_h.n_cols, J, seed, gen.INT)
        probs.append((A_h, B_h))
    I, K = probs[0][0].n_rows, probs[0][0].n_cols
    pipe = HostPipeline(I, K, max(a.nnz for a, _ in probs), J)
    outs = []
    for it in range(8):
        A_h, B_h = probs[it % 4]
        h = [torch.from_numpy(x).pin_memory() for x in (A_h.row_ptr, A_h.col_ind, A_h.val, B_h)]
        hC = torch.empty((I, J), dtype=torch.float32).pin_memory()
        pipe.submit(*h, hC)
        outs.append((it % 4, hC))
    pipe.synchronize()
    for i, hC in outs:
        A_h, B_h = probs[i]
        assert np.array_equal(hC.numpy().astype(np.float64), oracle.spmm_csr(A_h, B_h)[0])


@pytest.mark.parametrize("n_lanes", [2, 3])
def test_steps_in_flight_on_lanes(lf, n_lanes):
    """bench.py's pipelined steps: configure -> build -> SpMM of the SAME A issued
    on alternating streams, each lane with its own C, the previous step's SpMM
    still running when the next step's configure and build synchronise the
    host; every step's result is exact."""
    A_h = gen.rmat(13, 16, seed=11, kind=gen.INT)
    J = 64
    B_h = gen.dense(A_h.n_cols, J, 11, gen.INT)
    A = lf.Csr.from_host(A_h)
    B = torch.from_numpy(B_h).cuda()
    ref = oracle.spmm_csr(A_h, B_h)[0]
    lanes = [torch.cuda.current_stream()] + [torch.cuda.Stream() for _ in range(n_lanes - 1)]
    torch.cuda.synchronize()
    got = []
    for it in range(4 * n_lanes):
        st = lanes[it % n_lanes]
        with torch.cuda.stream(st):
            C = torch.full((A_h.n_rows, J), float("nan"), device="cuda")
            params, stats = lf.configure(A, J, stream=st)
            M = lf.CellMatrix.build(A, params, stats, stream=st)
            M.spmm(B, out=C, stream=st)
            M.close()
        got.append(C)
    torch.cuda.synchronize()
    for C in got:
        assert np.array_equal(C.cpu().numpy().astype(np.float64), ref)


def test_build_rejects_foreign_stats(lf):
    """lf_cell_build sizes its arrays from the stats, so it must refuse stats of
    another matrix (same P), stats of a CSR-format configure (tables zeroed)
    and stats whose tables were tampered with -- an error, never an
    out-of-bounds write."""
    A_h = gen.rmat(11, 16, seed=1)
    B_h = gen.rmat(11, 8, seed=2)
    A, Bm = lf.Csr.from_host(A_h), lf.Csr.from_host(B_h)
    pa, sa = lf.configure(A, 64, force_parts=2, force_format=1)
    _, sb = lf.configure(Bm, 64, force_parts=2, force_format=1)
    with pytest.raises(lf.LfError):
        lf.CellMatrix.build(A, pa, sb)  # another matrix
    _, scsr = lf.configure(A, 64, force_parts=2, force_format=2)
    with pytest.raises(lf.LfError):
        lf.CellMatrix.build(A, pa, scsr)  # CSR format: no tables
    sa.F[0][0] -= 1
    with pytest.raises(lf.LfError):
        lf.CellMatrix.build(A, pa, sa)  # tables do not cover A
    sa.F[0][0] += 1
    M = lf.CellMatrix.build(A, pa, sa)
    assert_cell_equal(M, oracle.csr_to_cell(A_h, 2, list(pa.max_width_log2[:2]), list(pa.block_nnz_log2[:2])))


def test_destroy_after_spmm_on_other_stream(lf):
    """lf_spmm on a second stream, then close() right away: the free is ordered
    (through the recorded event) after that launch, so memory the build stream
    reuses and overwrites immediately cannot corrupt the running SpMM."""
    A_h = gen.rmat(16, 16, seed=5, kind=gen.INT, lo=-3, hi=3)
    B_h = gen.dense(A_h.n_cols, 128, 5, gen.INT, -15, 15)
    A = lf.Csr.from_host(A_h)
    B = torch.from_numpy(B_h).cuda()
    ref = oracle.spmm_csr(A_h, B_h)[0]
    s2 = torch.cuda.Stream()
    for it in range(3):
        params, stats = lf.configure(A, 128)
        M = lf.CellMatrix.build(A, params, stats)  # build stream = current stream
        torch.cuda.current_stream().synchronize()
        s2.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s2):
            C = M.spmm(B, stream=s2)
        M.close()
        junk = torch.full((64 << 20,), -7.0, device="cuda")  # reuses the freed pool on the build stream
        del junk
        s2.synchronize()
        assert np.array_equal(C.cpu().numpy().astype(np.float64), ref)


def test_kernel_name(lf):
    A_h = gen.banded(4096, 12, seed=0)
    A = lf.Csr.from_host(A_h)
    p, s = lf.configure(A, 64, force_format=1)
    M = lf.CellMatrix.build(A, p, s)
    assert M.path(64) in ("cell_spmm_grouped_kernel", "cell_spmm_tc_kernel")
    R_h = gen.rmat(12, 16, seed=0)
    R = lf.Csr.from_host(R_h)
    p, s = lf.configure(R, 128, force_format=1)
    assert lf.CellMatrix.build(R, p, s).path(128) == "cell_spmm_kernel"
    p, s = lf.configure(R, 128, force_format=2)
    assert lf.CellMatrix.build(R, p, s).path(128) == "csr_spmm_kernel"


def test_spmm_in_cuda_graph(lf):
    """lf_spmm on the handle's build stream launches kernels only, so it can be
    captured in a CUDA graph: 8 captured launches (more than one counter
    slot each replay), replayed 3 times, give Alg. 1's C each time; the
    fixed-CSR kernel too."""
    A_h = gen.rmat(12, 16, seed=21, kind=gen.INT)
    A = lf.Csr.from_host(A_h)
    J = 64
    B_h = gen.dense(A_h.n_cols, J, 21, gen.INT, -15, 15)
    B = torch.from_numpy(B_h).cuda()
    Cref = oracle.spmm_csr(A_h, B_h)[0]
    for fmt in (1, 2):
        s = torch.cuda.Stream()
        params, stats = lf.configure(A, J, force_format=fmt, stream=s)
        M = lf.CellMatrix.build(A, params, stats, stream=s)
        C = torch.empty((A_h.n_rows, J), device="cuda")
        with torch.cuda.stream(s):
            M.spmm(B, out=C, stream=s)  # warm (not captured)
        s.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(8):
                M.spmm(B, out=C, stream=torch.cuda.current_stream())
        for _ in range(3):
            C.fill_(float("nan"))
            g.replay()
            torch.cuda.synchronize()
            assert np.array_equal(C.cpu().numpy().astype(np.float64), Cref), M.path()
        M.close()
