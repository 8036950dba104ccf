"""Pins for the HH-CPU four-block oracle (PAPER Alg. 3, Section V-A
L285-L291): C = A_H B_H + A_H B_L + A_L B_H + A_L B_L with "high" = more than t non-zeros (L274), the
sqrt(n)-row sampler (reading R20: the principal sub-matrix on a uniform random index set) and the
extrapolation t_A = t_s^2 (L291)."""
import numpy as np
import pytest

import oracle
import sginputs as gen


def _dense(R, n, p):
    d = np.zeros((n, p))
    for s, i in enumerate(R.rows):
        d[i, R.col[R.row_ptr[s]:R.row_ptr[s + 1]]] += R.val[R.row_ptr[s]:R.row_ptr[s + 1]]
    return d


def _pattern(R, n, p):
    d = np.zeros((n, p), dtype=bool)
    for s, i in enumerate(R.rows):
        d[i, R.col[R.row_ptr[s]:R.row_ptr[s + 1]]] = True
    return d


def test_hand_example_blocks():
    """4x4 hand case, t = 1: rows 0, 2 of A have 2 entries (high), rows 1, 3 one (low); the same rows of
    B (A = B). A = [[1,2,0,0],[0,0,3,0],[4,0,0,5],[0,6,0,0]] (row/col ids), so
      A_H B_H: row 0: k in {0} (B_0 high) -> 1*[1,2,0,0] = [1,2,0,0];  row 2: k in {0} -> 4*[1,2,0,0] = [4,8,0,0]
      A_H B_L: row 0: k = 1 (B_1 low) -> 2*[0,0,3,0] = [0,0,6,0];  row 2: k = 3 -> 5*[0,6,0,0] = [0,30,0,0]
      A_L B_H: row 1: k = 2 (B_2 high) -> 3*[4,0,0,5] = [12,0,0,15]; row 3: k = 1 is low -> nothing
      A_L B_L: row 3: k = 1 -> 6*[0,0,3,0] = [0,0,18,0];  row 1: k = 2 is high -> nothing."""
    rp = np.array([0, 2, 3, 5, 6], dtype=np.int64)
    col = np.array([0, 1, 2, 0, 3, 1], dtype=np.int32)
    val = np.array([1, 2, 3, 4, 5, 6], dtype=np.float64)
    A = gen.CSR(4, 4, rp, col, val, "hand")
    want = {
        (1, 1): {0: [1, 2, 0, 0], 2: [4, 8, 0, 0]},
        (1, 0): {0: [0, 0, 6, 0], 2: [0, 30, 0, 0]},
        (0, 1): {1: [12, 0, 0, 15]},
        (0, 0): {3: [0, 0, 18, 0]},
    }
    for (xa, yb), rows in want.items():
        R = oracle.hh_block(A, A, 1, xa, yb)
        d = _dense(R, 4, 4)
        ref = np.zeros((4, 4))
        for i, r in rows.items():
            ref[i] = r
        assert np.array_equal(d, ref), (xa, yb)
    # Phase IV: the sum of the four blocks is A*A (dense brute force)
    C = oracle.hh_combine([oracle.hh_block(A, A, 1, x, y) for x in (0, 1) for y in (0, 1)])
    Ad = A.to_dense()
    assert np.array_equal(_dense(C, 4, 4), Ad @ Ad)


@pytest.mark.parametrize("name,t", [("rmat9", 8), ("rmat9", 20), ("C1", 7), ("rmat10", 0), ("rmat10", 64)])
def test_four_blocks_sum_to_the_product(name, t):
    """Phase IV equals O1 exactly in integer-value mode: structure (union of the block patterns) and
    values; every product (i, k, j) falls in exactly one block (work adds up to w_i)."""
    A = gen.config(name, mode="int")
    full = oracle.spgemm(A, A)
    blocks = [oracle.hh_block(A, A, t, x, y) for x in (0, 1) for y in (0, 1)]
    C = oracle.hh_combine(blocks)
    assert np.array_equal(C.row_ptr, full.row_ptr) and np.array_equal(C.col, full.col)
    assert np.array_equal(C.val, full.val)
    ones = gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, np.ones_like(A.val), "ones")
    w = oracle.row_work(A, A)
    tot = np.zeros(A.nrows)
    for x in (0, 1):
        for y in (0, 1):
            R = oracle.hh_block(ones, ones, t, x, y)
            for s in range(A.nrows):
                tot[s] += R.val[R.row_ptr[s]:R.row_ptr[s + 1]].sum()
    assert np.array_equal(tot, w.astype(np.float64))


def test_degenerate_thresholds():
    """t >= max nnz: every row low, A_L B_L is the whole product; t = -1: every row high (even empty
    ones: 0 > -1), A_H B_H is the whole product; the other blocks are empty."""
    A = gen.config("rmat9", mode="int")
    full = oracle.spgemm(A, A)
    big = int(np.diff(A.row_ptr).max())
    for t, keep in ((big, (0, 0)), (-1, (1, 1))):
        for x in (0, 1):
            for y in (0, 1):
                R = oracle.hh_block(A, A, t, x, y)
                if (x, y) == keep:
                    assert np.array_equal(R.col, full.col) and np.array_equal(R.val, full.val)
                else:
                    assert R.nnz == 0


def test_sqrt_n_sampler_is_the_principal_submatrix():
    A = gen.config("rmat10")
    n = A.nrows
    rows, rp, col, pos = oracle.hh_sample(A, seed=3)
    s = len(rows)
    assert np.all(np.diff(rows) > 0) and np.all(col < s) and rp[-1] == len(col)
    Ad = A.to_dense()
    sub = np.zeros((s, s))
    for r in range(s):
        sub[r, col[rp[r]:rp[r + 1]]] = A.val[pos[rp[r]:rp[r + 1]]]
        assert np.all(np.diff(col[rp[r]:rp[r + 1]]) > 0), "relabelled columns stay sorted"
    assert np.array_equal(sub, Ad[np.ix_(rows, rows)])
    # ~sqrt(n) rows: Binomial(n, 1/sqrt(n)) within 4 sigma
    f = 1.0 / np.sqrt(n)
    assert abs(s - n * f) < 4 * np.sqrt(n * f * (1 - f))
    # f = 1 keeps everything: A' = A
    rows, rp, col, pos = oracle.hh_sample(A, seed=3, f=1.0)
    assert np.array_equal(rp, A.row_ptr) and np.array_equal(col, A.col) and np.array_equal(pos, np.arange(A.nnz))


def test_extrapolation_is_t_squared():
    for t in (0, 1, 7, 31, 1000):
        assert oracle.hh_extrapolate(t) == t * t
