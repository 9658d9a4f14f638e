"""Pins for the oracle's Algorithm 1 (lfo_spmm_csr) and Algorithm 2
(lfo_cell_spmm) against closed forms (no GPU).

* dense GEMM on tiny integer-valued inputs: every product and partial sum is
  an integer < 2^53, so fp64 is exact and equality is ==;
* A = I  ->  C == B;  A = D.P (power-of-two diagonal times permutation) -> exact;
* Alg. 2 over the oracle's CELL arrays == Alg. 1 exactly on integer inputs
  (any P, folding), and bit-for-bit on float inputs when P = 1 with no folding
  (same additions in the same order, P:L589-620 vs P:L132-147).
"""
import numpy as np
import pytest

import gen
import oracle


def dense_of(A, absval=False):
    D = np.zeros((A.n_rows, A.n_cols), np.float64)
    rows = np.repeat(np.arange(A.n_rows), np.diff(A.row_ptr))
    v = A.val.astype(np.float64)
    np.add.at(D, (rows, A.col_ind.astype(np.int64)), np.abs(v) if absval else v)
    return D


@pytest.mark.parametrize("seed", range(12))
def test_alg1_equals_dense_gemm(seed):
    rng = np.random.default_rng(seed)
    I, K, J = rng.integers(1, 40), rng.integers(1, 40), rng.integers(1, 20)
    A = gen.random_small(I, K, 3 * K, seed, dup=True, zeros=True)
    B = gen.dense(K, J, seed, gen.INT, -15, 15)
    C, Cabs = oracle.spmm_csr(A, B)
    assert np.array_equal(C, dense_of(A) @ B.astype(np.float64))
    assert np.array_equal(Cabs, dense_of(A, True) @ np.abs(B.astype(np.float64)))


def test_alg1_identity():
    n, J = 300, 17
    A = gen.CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32), np.ones(n, np.float32))
    B = gen.dense(n, J, 4)
    C, _ = oracle.spmm_csr(A, B)
    assert np.array_equal(C, B.astype(np.float64))


def test_alg1_scaled_permutation():
    n, J = 257, 9
    rng = np.random.default_rng(0)
    perm = rng.permutation(n).astype(np.int32)
    d = (2.0 ** rng.integers(-4, 5, size=n)) * rng.choice([-1, 1], size=n)
    A = gen.CSR(n, n, np.arange(n + 1, dtype=np.int64), perm, d.astype(np.float32))
    B = gen.dense(n, J, 1)
    C, _ = oracle.spmm_csr(A, B)
    assert np.array_equal(C, d[:, None] * B[perm].astype(np.float64))


def test_alg1_row_sample_matches_full():
    A = gen.rmat(10, 8, seed=2)
    B = gen.dense(A.n_cols, 33, 2)
    C, Ca = oracle.spmm_csr(A, B)
    rows = np.array([0, 5, 1023, 17, 17], np.int64)
    Cs, Cas = oracle.spmm_csr(A, B, rows)
    assert np.array_equal(Cs, C[rows]) and np.array_equal(Cas, Ca[rows])


def test_alg1_empty_and_zero_width():
    A = gen.CSR(5, 3, np.zeros(6, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32))
    C, _ = oracle.spmm_csr(A, gen.dense(3, 4, 0))
    assert np.array_equal(C, np.zeros((5, 4)))
    C, _ = oracle.spmm_csr(A, np.zeros((3, 0), np.float32))
    assert C.shape == (5, 0)


@pytest.mark.parametrize("seed", range(16))
def test_alg2_equals_alg1_integer_exact(seed):
    rng = np.random.default_rng(100 + seed)
    I, K, J = rng.integers(1, 60), rng.integers(1, 60), rng.integers(1, 12)
    A = gen.random_small(I, K, 70, seed)
    P = int(rng.integers(1, 6))
    e = rng.integers(0, 6, size=P)
    k = e + rng.integers(0, 3, size=P)
    cell = oracle.csr_to_cell(A, P, e, k)
    B = gen.dense(K, J, seed, gen.INT, -15, 15)
    C1, _ = oracle.spmm_csr(A, B)
    C2 = oracle.cell_spmm(cell, B)
    assert np.array_equal(C1, C2)


def test_alg2_bitwise_p1_no_folding():
    A = gen.rmat(11, 8, seed=7)  # float values on the 2^-23 grid
    e = oracle.partition_max_log2(A, 1, 0)
    cell = oracle.csr_to_cell(A, 1, [e], [e])
    B = gen.dense(A.n_cols, 16, 7)
    C1, _ = oracle.spmm_csr(A, B)
    C2 = oracle.cell_spmm(cell, B)
    assert np.array_equal(C1.view(np.int64), C2.view(np.int64))


def test_cell_spmm_thread_count_independent():
    """lfo_cell_spmm splits the output columns over threads: the fp64 result
    is bit-identical with 1 thread and with all threads (float inputs, folded
    rows, P > 1 so several CELL rows add into one C row)."""
    A = gen.rmat(10, 16, seed=4)
    B = gen.dense(A.n_cols, 37, 4)
    cell = oracle.csr_to_cell(A, 3, [2, 3, 1])
    n_all = oracle.set_threads(0)
    try:
        oracle.set_threads(1)
        C1 = oracle.cell_spmm(cell, B)
        oracle.set_threads(max(4, n_all))
        C4 = oracle.cell_spmm(cell, B)
    finally:
        oracle.set_threads(n_all)
    assert np.array_equal(C1.view(np.int64), C4.view(np.int64))
    Cref, Cabs = oracle.spmm_csr(A, B)
    assert np.all(np.abs(C1 - Cref) <= 1e-12 * Cabs)
