"""Pins for the oracle's CSR->CELL converter (lfo_csr_to_cell) and its
inverse (lfo_cell_to_csr), no GPU.

* lossless round trip CELL->CSR == CSR, bit for bit (explicit zeros,
  duplicate columns, empty rows, K < P, P not dividing K);
* invariants recomputed here from numpy segment lengths: bucket ranges
  2^(t-1) < l <= 2^t (Fig. 3 labels), folded rows only in the max
  bucket with ceil(l/W) sub-rows, R_t * 2^t = 2^k
  (P:L532-537, L817-820), padding encoding (-1, +0.0) (Fig. 4, C5),
  ascending source rows inside a bucket (C6), partition-major order (C7);
* closed forms: a regular matrix (every row length L) and the 27-point
  stencil census.
"""
import numpy as np
import pytest

import gen
import oracle
from conftest import read_golden


def seg_lengths(A, P):
    """[I, P] segment lengths with S = ceil(K/P) (reading C3)."""
    S = -(-A.n_cols // P) if A.n_cols else 0
    out = np.zeros((A.n_rows, P), np.int64)
    for i in range(A.n_rows):
        cols = A.col_ind[A.row_ptr[i]:A.row_ptr[i + 1]]
        for p in range(P):
            lo, hi = p * S, min(p * S + S, A.n_cols)
            out[i, p] = np.searchsorted(cols, hi, "left") - np.searchsorted(cols, lo, "left")
    return out


def nat_bucket(l):
    return int(np.ceil(np.log2(l))) if l > 1 else 0


def check_invariants(A, P, e, k, cell):
    L = seg_lengths(A, P)
    b = cell.buckets
    # order (C7) and offsets
    keys = list(zip(b["part"], b["width_log2"]))
    assert keys == sorted(keys) and len(set(keys)) == len(keys)
    r_off = s_off = 0
    for bk in b:
        p, t = int(bk["part"]), int(bk["width_log2"])
        W, R = 1 << t, int(bk["rows_per_block"])
        assert R * W == 1 << int(k[p]) and t <= e[p]
        assert bk["row_off"] == r_off and bk["slot_off"] == s_off
        assert bk["n_rows_pad"] % R == 0 and bk["n_rows"] <= bk["n_rows_pad"] < bk["n_rows"] + R
        assert bk["n_rows"] > 0
        rows = cell.row_ind[r_off:r_off + bk["n_rows_pad"]]
        real, pad = rows[:bk["n_rows"]], rows[bk["n_rows"]:]
        assert np.all(pad == -1)
        assert np.all(np.diff(real) >= 0)  # C6
        slots_c = cell.col_ind[s_off:s_off + bk["n_rows_pad"] * W].reshape(-1, W)
        slots_v = cell.val[s_off:s_off + bk["n_rows_pad"] * W].reshape(-1, W)
        assert np.all(slots_c[bk["n_rows"]:] == -1)
        assert np.all(slots_v[bk["n_rows"]:].view(np.int32) == 0)
        # which rows belong here, and how many sub-rows each
        exp_rows = []
        for i in range(A.n_rows):
            l = L[i, p]
            if l == 0:
                continue
            ti = min(nat_bucket(l), int(e[p]))
            if ti == t:
                if t < e[p]:
                    assert (1 << t) // 2 < l <= (1 << t)
                exp_rows += [i] * (-(-l // W))
                # slot contents of this row's last sub-row: real then (-1, +0.0)
        assert real.tolist() == exp_rows
        for q, i in enumerate(real):
            c = slots_c[q]
            nreal = int((c >= 0).sum())
            assert np.all(c[:nreal] >= 0) and np.all(c[nreal:] == -1)
            assert np.all(slots_v[q, nreal:].view(np.int32) == 0)
        r_off += int(bk["n_rows_pad"])
        s_off += int(bk["n_rows_pad"]) * W
    assert r_off == len(cell.row_ind) and s_off == len(cell.col_ind)


CASES = []
for s in range(24):
    rng = np.random.default_rng(s)
    CASES.append((s, int(rng.integers(0, 40)), int(rng.integers(0, 30)), int(rng.integers(1, 7))))


@pytest.mark.parametrize("seed,I,K,P", CASES)
def test_round_trip_and_invariants(seed, I, K, P):
    rng = np.random.default_rng(1000 + seed)
    A = gen.random_small(I, K, 45, seed, dup=True, zeros=True)
    e = rng.integers(0, 6, size=P)
    k = e + rng.integers(0, 3, size=P)
    cell = oracle.csr_to_cell(A, P, e, k)
    rp, ci, va = oracle.cell_to_csr(cell)
    assert np.array_equal(rp, A.row_ptr)
    assert np.array_equal(ci, A.col_ind)
    assert np.array_equal(va.view(np.int32), A.val.view(np.int32))
    check_invariants(A, P, e, k, cell)


def test_round_trip_generated():
    A = gen.rmat(12, 16, seed=1)
    for P, e in [(1, [5]), (3, [4, 6, 2]), (8, [3] * 8)]:
        cell = oracle.csr_to_cell(A, P, e)
        rp, ci, va = oracle.cell_to_csr(cell)
        assert np.array_equal(rp, A.row_ptr) and np.array_equal(ci, A.col_ind)
        assert np.array_equal(va.view(np.int32), A.val.view(np.int32))


def test_fig3_bucket_ranges():
    g = read_golden("fig3_bucket_ranges.txt")
    for line_key in ("1", "2", "3"):
        t, lo, hi = int(line_key), *g[line_key]
        # one row per length lo+1..hi; all must land in bucket t (width 2^t)
        lens = list(range(lo + 1, hi + 1))
        rows = [list(range(l)) for l in lens]
        rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
        A = gen.CSR(len(rows), 16, rp, np.concatenate(rows).astype(np.int32),
                    np.ones(int(rp[-1]), np.float32))
        cell = oracle.csr_to_cell(A, 1, [4])
        assert len(cell.buckets) == 1 and cell.buckets[0]["width_log2"] == t


@pytest.mark.parametrize("L,I,mult", [(1, 10, 0), (3, 17, 0), (5, 33, 2), (16, 9, 1), (27, 50, 1)])
def test_closed_form_regular(L, I, mult):
    """Every row holds exactly L entries -> one bucket of width 2^ceil_log2 L,
    ceil(I/R) blocks of R = 2^k / 2^e rows."""
    K = 64
    cols = np.sort((np.arange(I)[:, None] + np.arange(L)[None, :] * 2) % K, axis=1).astype(np.int32)
    A = gen.CSR(I, K, np.arange(I + 1, dtype=np.int64) * L, cols.ravel(), gen.fill(I * L, 0, 1))
    e = nat_bucket(L)
    cell = oracle.csr_to_cell(A, 1, [e], [e + mult])
    assert len(cell.buckets) == 1
    R = 1 << mult
    n_pad = -(-I // R) * R
    b = cell.buckets[0]
    assert (b["width_log2"], b["n_rows"], b["n_rows_pad"]) == (e, I, n_pad)
    assert len(cell.col_ind) == n_pad * (1 << e)


def test_closed_form_stencil_buckets():
    n = 7
    A = gen.stencil27(n)
    cell = oracle.csr_to_cell(A, 1, [5])
    got = {int(b["width_log2"]): int(b["n_rows"]) for b in cell.buckets}
    assert got == {3: 8, 4: 12 * (n - 2), 5: 6 * (n - 2) ** 2 + (n - 2) ** 3}
    # folding at W = 8: 12 -> 2 sub-rows, 18 -> 3, 27 -> 4
    cell = oracle.csr_to_cell(A, 1, [3])
    assert len(cell.buckets) == 1
    assert int(cell.buckets[0]["n_rows"]) == 8 + 2 * 12 * (n - 2) + 3 * 6 * (n - 2) ** 2 + 4 * (n - 2) ** 3


def test_bad_params():
    A = gen.random_small(5, 5, 3, 0)
    with pytest.raises(ValueError):
        oracle.csr_to_cell(A, 1, [3], [2])  # k < e


def concat_real_slots(cell):
    """Walk the CELL arrays in storage order (buckets partition-major, ascending
    width, R7) and append every real slot of CELL row r (col >= 0) to its source
    row rowInd[r], in slot order: (cols, val bits) per source row."""
    rows = [[] for _ in range(cell.n_rows)]
    for b in cell.buckets:
        W = 1 << int(b["width_log2"])
        for q in range(int(b["n_rows_pad"])):
            r = int(b["row_off"]) + q
            i = int(cell.row_ind[r])
            s0 = int(b["slot_off"]) + q * W
            cs = cell.col_ind[s0:s0 + W]
            vs = cell.val[s0:s0 + W].view(np.int32)
            if i < 0:
                assert np.all(cs == -1) and np.all(vs == 0)  # padding row (R5)
                continue
            real = cs >= 0
            n = int(real.sum())
            assert np.all(real[:n]) and not np.any(real[n:])  # real slots form a prefix
            rows[i].extend(zip(cs[:n].tolist(), vs[:n].tolist()))
    return rows


@pytest.mark.parametrize("seed", range(12))
def test_slot_order_pin(seed):
    """Reading R6 pinned WITHOUT the round trip's sort: the real slots of a
    source row's CELL sub-rows, concatenated in storage order, ARE its CSR
    entries in CSR order (values bit-identical), for every P, width and fold.
    A swapped pair of sub-rows, a reversed slot order or a bucket out of
    partition order (R7) fails this even when the round trip's stable sort
    would hide it.  (Fig. 4.)"""
    rng = np.random.default_rng(7000 + seed)
    I, K = int(rng.integers(1, 60)), int(rng.integers(1, 90))
    P = int(rng.integers(1, 9))
    A = gen.random_small(I, K, 80, seed, dup=True, zeros=True)
    e = rng.integers(0, 5, size=P)
    k = e + rng.integers(0, 3, size=P)
    cell = oracle.csr_to_cell(A, P, e, k)
    got = concat_real_slots(cell)
    for i in range(I):
        a, b = int(A.row_ptr[i]), int(A.row_ptr[i + 1])
        exp = list(zip(A.col_ind[a:b].tolist(), A.val[a:b].view(np.int32).tolist()))
        assert got[i] == exp, i


def test_slot_order_pin_catches_a_swap():
    """The pin above is not vacuous: swapping two sub-rows of a folded row in
    an otherwise valid CELL breaks it, while the sorted round trip still passes
    when the swapped sub-rows hold distinct columns."""
    A = gen.CSR(1, 16, np.array([0, 6], np.int64), np.arange(0, 12, 2, dtype=np.int32),
                np.arange(1, 7, dtype=np.float32))
    cell = oracle.csr_to_cell(A, 1, [1])  # W = 2: 3 sub-rows of 2
    cell.col_ind[[0, 1, 2, 3]] = cell.col_ind[[2, 3, 0, 1]]
    cell.val[[0, 1, 2, 3]] = cell.val[[2, 3, 0, 1]]
    rp, ci, va = oracle.cell_to_csr(cell)
    assert np.array_equal(ci, A.col_ind)  # the round trip is blind to the swap
    assert concat_real_slots(cell)[0] != list(zip(A.col_ind.tolist(), A.val.view(np.int32).tolist()))
