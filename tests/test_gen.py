"""Generators (gen/): determinism, structure and the closed forms of the shapes."""
import numpy as np

import gen
from conftest import read_golden


def _check_csr(m, dedup=True):
    assert m.row_ptr[0] == 0 and len(m.row_ptr) == m.n_rows + 1
    assert np.all(np.diff(m.row_ptr) >= 0)
    assert len(m.col_ind) == m.nnz == len(m.val)
    if m.nnz:
        assert m.col_ind.min() >= 0 and m.col_ind.max() < m.n_cols
    rows = np.repeat(np.arange(m.n_rows), np.diff(m.row_ptr))
    d = np.diff(m.col_ind.astype(np.int64))
    same = rows[1:] == rows[:-1]
    assert np.all(d[same] > 0) if dedup else np.all(d[same] >= 0)


def test_counter_rng_is_pure():
    assert gen.u64(1, 2, 3) == gen.u64(1, 2, 3)
    assert gen.u64(1, 2, 3) != gen.u64(1, 2, 4)
    a = gen.fill(1000, 7, 9)
    b = gen.fill(1000, 7, 9)
    assert np.array_equal(a.view(np.int32), b.view(np.int32))


def test_value_kinds():
    g = gen.fill(100000, 0, 1, gen.GRID)
    assert g.min() >= -1.0 and g.max() < 1.0
    assert np.all((g.astype(np.float64) + 1.0) * 2**23 == np.round((g.astype(np.float64) + 1.0) * 2**23))
    assert np.all((g == 0) | (np.abs(g) >= 2.0**-23))  # no denormals
    i = gen.fill(100000, 0, 1, gen.INT, -3, 3)
    assert set(np.unique(i)) == set(range(-3, 4))
    p = gen.fill(1000, 0, 1, gen.POS)
    assert p.min() >= 0 and p.max() < 1
    assert np.all(gen.fill(10, 0, 1, gen.ONE) == 1)


def test_uniform_config1_shape():
    m, J = gen.config("c1_uniform1024")
    _check_csr(m)
    assert J == 32 and m.n_rows == m.n_cols == 1024
    assert 15000 < m.nnz < 17800   # E = 16384, sd ~ 127
    m2, _ = gen.config("c1_uniform1024")
    assert np.array_equal(m.col_ind, m2.col_ind)


def test_rmat_small():
    m = gen.rmat(12, 16, seed=3)
    _check_csr(m)
    assert m.n_rows == 4096
    assert 0.6 * 16 * 4096 < m.nnz <= 16 * 4096
    # power law: row 0 (all-zero bits, probability (a+b)^12) is among the longest
    l = m.row_lengths()
    assert l[0] >= np.percentile(l, 99)
    mp = gen.rmat(12, 16, seed=3, permute=True)
    _check_csr(mp)
    assert mp.nnz == m.nnz
    assert sorted(mp.row_lengths()) == sorted(l)


def test_stencil_census_golden():
    g = read_golden("stencil27_census.txt")
    n = g["n"][0]
    m = gen.stencil27(n)
    _check_csr(m)
    l, c = np.unique(m.row_lengths(), return_counts=True)
    assert dict(zip(l.tolist(), c.tolist())) == {8: g["8"][0], 12: g["12"][0], 18: g["18"][0], 27: g["27"][0]}
    assert m.nnz == g["nnz"][0] == (3 * n - 2) ** 3


def test_banded():
    m = gen.banded(100, 4)
    _check_csr(m)
    assert m.nnz == 100 * 9 - 2 * (4 + 3 + 2 + 1)


def test_powerlaw_exact_total():
    m = gen.powerlaw(5000, 200000, 1.2, seed=1)
    _check_csr(m)
    assert m.nnz == 200000
    l = m.row_lengths()
    assert l.min() >= 1
    assert l.max() > 8 * np.median(l)  # heavy skew


def test_random_small_edge_cases():
    m = gen.random_small(50, 20, 40, seed=5)
    _check_csr(m, dedup=False)
    assert (m.row_lengths() == 0).any()
    assert (m.val == 0).any()


def test_banded_config_closed_form():
    """c3b_banded2M (BASELINE configs[2] read literally): half-width 12 band on
    2,000,000 rows -> 25 n - 2 (1 + ... + 12) nonzeros, columns i-12..i+12."""
    A, J = gen.config("c3b_banded2M")
    n = 2_000_000
    assert (A.n_rows, A.n_cols, J) == (n, n, 64)
    assert A.nnz == 25 * n - 2 * 78
    rp, ci = np.asarray(A.row_ptr), np.asarray(A.col_ind)
    for i in (0, 5, 12, 999_999, n - 13, n - 1):
        assert np.array_equal(ci[rp[i]:rp[i + 1]], np.arange(max(i - 12, 0), min(i + 12, n - 1) + 1))
