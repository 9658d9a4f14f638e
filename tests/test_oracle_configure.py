"""Pins for the oracle's cost model (eq. 7) and Algorithm 3
(P:L913-947), no GPU.

* the two hand-worked examples in tests/golden/ (costs, exponent-space and
  literal readings of Alg. 3);
* the natural-bucket statistics (lfo_partition_stats, set definitions over the
  UNfolded buckets) reproduce the materialised eq. 7 cost (lfo_partition_cost,
  folded buckets) -- two independent formulations must agree exactly;
* Alg. 3 equals the brute-force argmin whenever the cost's "go right"
  predicate is monotone (unimodal sequence);
* Table 2 features equal numpy statistics.
"""
import numpy as np
import pytest

import gen
import oracle
from conftest import read_golden


def golden_matrix(g):
    rows = g["rows"]
    rp = np.concatenate([[0], np.cumsum([len(r) for r in rows])]).astype(np.int64)
    ci = np.concatenate([np.array(r, np.int32) for r in rows])
    return gen.CSR(len(rows), g["K"][0], rp, ci, np.ones(len(ci), np.float32))


@pytest.mark.parametrize("name", ["cost_5x8.txt", "cost_separating_2x16.txt"])
def test_golden_cost_and_alg3(name):
    g = read_golden(name)
    A = golden_matrix(g)
    J = g["J"][0]
    costs = [oracle.partition_cost(A, 1, 0, e, J) for e in range(len(g["cost"]))]
    assert costs == g["cost"]
    assert oracle.build_buckets(A, 1, 0, J) == g["alg3_e"][0]
    assert oracle.build_buckets_literal(A, 1, 0, J) == g["literal_width"][0]


def cost_from_stats(stats, e, J):
    H, F, Un, Ut = stats
    c = 0
    for b in range(e):
        if H[b]:
            c += 2 * H[b] * (1 << b) + Un[b] * J + H[b] * J
    if F[e]:
        c += 2 * F[e] * (1 << e) + Ut[e] * J + F[e] * J
    return int(c)


@pytest.mark.parametrize("seed", range(10))
def test_stats_identity(seed):
    rng = np.random.default_rng(seed)
    A = gen.random_small(int(rng.integers(1, 50)), int(rng.integers(1, 50)), 80, seed)
    P = int(rng.integers(1, 5))
    J = int(rng.integers(1, 300))
    for p in range(P):
        st = oracle.partition_stats(A, P, p)
        top = oracle.partition_max_log2(A, P, p)
        for e in range(0, max(top, 0) + 1):
            assert cost_from_stats(st, e, J) == oracle.partition_cost(A, P, p, e, J)


def test_stats_identity_rmat():
    A = gen.rmat(11, 16, seed=4)
    for P in (1, 3):
        for p in range(P):
            st = oracle.partition_stats(A, P, p)
            for e in range(oracle.partition_max_log2(A, P, p) + 1):
                assert cost_from_stats(st, e, 128) == oracle.partition_cost(A, P, p, e, 128)


def test_alg3_equals_argmin_when_unimodal():
    n_unimodal = 0
    for seed in range(40):
        rng = np.random.default_rng(500 + seed)
        A = gen.random_small(int(rng.integers(2, 60)), int(rng.integers(2, 60)), 120, seed, empty_frac=0.1)
        P = int(rng.integers(1, 3))
        J = int(rng.choice([1, 4, 32, 128]))
        for p in range(P):
            top = oracle.partition_max_log2(A, P, p)
            if top < 0:
                assert oracle.build_buckets(A, P, p, J) == -1
                continue
            c = [oracle.partition_cost(A, P, p, e, J) for e in range(top + 1)]
            go_right = [c[m] > c[m + 1] for m in range(top)]
            if go_right == sorted(go_right, reverse=True):  # True..True False..False
                n_unimodal += 1
                assert oracle.build_buckets(A, P, p, J) == int(np.argmin(c))
    assert n_unimodal >= 20


def test_alg3_rmat_lands_on_argmin():
    A = gen.rmat(12, 16, seed=0)
    for J in (32, 128):
        c = [oracle.partition_cost(A, 1, 0, e, J) for e in range(oracle.partition_max_log2(A, 1, 0) + 1)]
        assert oracle.build_buckets(A, 1, 0, J) == int(np.argmin(c))


def test_features():
    A = gen.rmat(10, 8, seed=3)
    f = oracle.features(A)
    l = A.row_lengths().astype(np.float64)
    assert f[:3].tolist() == [A.n_rows, A.n_cols, A.nnz]
    assert f[3] == pytest.approx(l.mean(), rel=1e-15)
    assert f[4:6].tolist() == [l.min(), l.max()]
    assert f[6] == pytest.approx(l.std(), rel=1e-12)
