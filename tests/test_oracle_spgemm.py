"""Pins for oracle O1 (Gustavson SpGEMM, PAPER L74 / Alg. 2 l.5-6 L222-L223) and O2 (row work,
PAPER L206). Each test checks the oracle against something other than itself: dense brute force,
closed forms (identity, permutation, diagonal, tridiagonal), invariants, and scipy.sparse.
"""
import numpy as np
import pytest

import oracle
import sginputs as gen


def _dense_of(R, nrows, ncols):
    d = np.zeros((nrows, ncols))
    for s in range(len(R.rows)):
        lo, hi = R.row_ptr[s], R.row_ptr[s + 1]
        d[R.rows[s], R.col[lo:hi]] = R.val[lo:hi]
    return d


def _pattern_of(R, nrows, ncols):
    d = np.zeros((nrows, ncols), dtype=bool)
    for s in range(len(R.rows)):
        lo, hi = R.row_ptr[s], R.row_ptr[s + 1]
        d[R.rows[s], R.col[lo:hi]] = True
    return d


def _assert_canonical(R):
    for s in range(len(R.rows)):
        c = R.col[R.row_ptr[s]:R.row_ptr[s + 1]]
        assert np.all(np.diff(c) > 0), "columns must be strictly ascending"


@pytest.mark.parametrize("n,m,p,dens,seed", [
    (1, 1, 1, 1.0, 1), (7, 5, 9, 0.3, 2), (16, 16, 16, 0.2, 3), (33, 17, 40, 0.15, 4),
    (64, 64, 64, 0.08, 5), (64, 30, 64, 0.25, 6), (20, 64, 8, 0.1, 7)])
@pytest.mark.parametrize("mode", ["real", "int"])
def test_dense_brute_force(n, m, p, dens, seed, mode):
    A = gen.random_pattern(n, m, dens, seed, mode)
    B = gen.random_pattern(m, p, dens, seed + 100, mode)
    R = oracle.spgemm(A, B, with_absmag=True)
    _assert_canonical(R)
    Ad, Bd = A.to_dense(), B.to_dense()
    # structure: boolean matmul of the patterns (structural semantics, reading R9)
    pat = (Ad != 0).astype(np.int64) @ (Bd != 0).astype(np.int64) > 0
    assert np.array_equal(_pattern_of(R, n, p), pat)
    ref = Ad @ Bd
    got = _dense_of(R, n, p)
    if mode == "int":
        assert np.array_equal(got, ref)
    else:
        mag = np.abs(Ad) @ np.abs(Bd)
        assert np.all(np.abs(got - ref) <= 1e-14 * mag + 0.0)


def test_identity_bit_exact():
    A = gen.config("C1")
    I = gen.identity(A.nrows)
    for R in (oracle.spgemm(A, I), oracle.spgemm(I, A)):
        assert np.array_equal(R.row_ptr, A.row_ptr)
        assert np.array_equal(R.col, A.col)
        assert np.array_equal(R.val, A.val)


def test_permutation_rows_and_columns():
    A = gen.config("C1")
    n = A.nrows
    P = gen.permutation(n, seed=9)
    pi = P.col  # P[i, pi[i]] = 1
    # (P A) row i = A row pi[i]
    R = oracle.spgemm(P, A)
    for i in range(0, n, 37):
        lo, hi = A.row_ptr[pi[i]], A.row_ptr[pi[i] + 1]
        assert np.array_equal(R.col[R.row_ptr[i]:R.row_ptr[i + 1]], A.col[lo:hi])
        assert np.array_equal(R.val[R.row_ptr[i]:R.row_ptr[i + 1]], A.val[lo:hi])
    # (A P)[i, pi[k]] = A[i, k]: columns relabelled then re-sorted
    R = oracle.spgemm(A, P)
    for i in range(0, n, 41):
        lo, hi = A.row_ptr[i], A.row_ptr[i + 1]
        order = np.argsort(pi[A.col[lo:hi]])
        assert np.array_equal(R.col[R.row_ptr[i]:R.row_ptr[i + 1]], pi[A.col[lo:hi]][order])
        assert np.array_equal(R.val[R.row_ptr[i]:R.row_ptr[i + 1]], A.val[lo:hi][order])


def test_diagonal_scaling_bit_exact():
    A = gen.config("C1")
    d = np.linspace(0.25, 4.0, A.nrows)
    D = gen.diagonal(A.nrows, d)
    R = oracle.spgemm(D, A)
    assert np.array_equal(R.col, A.col)
    rows = np.repeat(np.arange(A.nrows), np.diff(A.row_ptr))
    assert np.array_equal(R.val, d[rows] * A.val)  # one product per entry -> exact


@pytest.mark.parametrize("n,al,be,ga", [(8, 2, 3, 5), (12, -1, 4, 7), (5, 3, -2, 1)])
def test_tridiagonal_square_closed_form(n, al, be, ga):
    """T = tridiag(al (sub), be (diag), ga (super)). Expanding (T^2)_{ij} = sum_k T_ik T_kj:
    (T^2)_{i,i-2} = al^2, (T^2)_{i,i-1} = 2 al be, (T^2)_{i,i+1} = 2 be ga, (T^2)_{i,i+2} = ga^2,
    (T^2)_{i,i} = be^2 + al ga [i >= 1] + ga al [i <= n-2]."""
    T = gen.tridiag(n, al, be, ga)
    R = oracle.spgemm(T, T)
    for i in range(n):
        exp = {i: be * be + (al * ga if i >= 1 else 0) + (ga * al if i <= n - 2 else 0)}
        if i - 2 >= 0: exp[i - 2] = al * al
        if i - 1 >= 0: exp[i - 1] = 2 * al * be
        if i + 1 <= n - 1: exp[i + 1] = 2 * be * ga
        if i + 2 <= n - 1: exp[i + 2] = ga * ga
        lo, hi = R.row_ptr[i], R.row_ptr[i + 1]
        got = dict(zip(R.col[lo:hi].tolist(), R.val[lo:hi].tolist()))
        assert got == {k: float(v) for k, v in exp.items()}, (i, got, exp)
    # row work w = (5, 8, 9, ..., 9, 8, 5) and row nnz (3, 4, 5, ..., 5, 4, 3) for n >= 4
    if n >= 4:
        w = oracle.row_work(T, T)
        assert w[0] == 5 and w[1] == 8 and w[-2] == 8 and w[-1] == 5
        assert np.all(w[2:-2] == 9)
        u = np.diff(R.row_ptr)
        assert list(u[:2]) == [3, 4] and list(u[-2:]) == [4, 3] and np.all(u[2:-2] == 5)


def test_tridiagonal_survey_values():
    """The hand-checked values quoted in SURVEY §8(c) O1 pin (v): alpha=2, beta=3, gamma=5, n=8
    give interior diagonal 29, end diagonal 19, super 30, sub 12, super-2 25, sub-2 4."""
    T = gen.tridiag(8, 2, 3, 5)
    d = _dense_of(oracle.spgemm(T, T), 8, 8)
    assert d[3, 3] == 29 and d[0, 0] == 19 and d[3, 4] == 30 and d[3, 2] == 12
    assert d[3, 5] == 25 and d[3, 1] == 4


@pytest.mark.parametrize("name", ["C1", "rmat10"])
def test_all_ones_row_sums_equal_work(name):
    """With all-ones values c_ij counts the products landing on (i, j): sum_j c_ij = w_i
    and sum_ij c_ij = W, exactly."""
    A = gen.config(name, mode="ones")
    R = oracle.spgemm(A, A)
    w = oracle.row_work(A, A)
    rs = np.add.reduceat(R.val, R.row_ptr[:-1].clip(max=max(R.nnz - 1, 0))) if R.nnz else np.zeros(A.nrows)
    rs[np.diff(R.row_ptr) == 0] = 0
    assert np.array_equal(rs.astype(np.int64), w)
    assert int(R.val.sum()) == int(w.sum())


@pytest.mark.parametrize("name", ["C1", "rmat11"])
def test_scipy_cross_check(name):
    A = gen.config(name)
    R = oracle.spgemm(A, A, with_absmag=True)
    S = (A.to_scipy() @ A.to_scipy()).tocsr()
    S.sort_indices()
    assert np.array_equal(R.row_ptr, S.indptr.astype(np.int64))
    assert np.array_equal(R.col, S.indices.astype(np.int32))
    assert np.all(np.abs(R.val - S.data) <= 1e-13 * R.absmag)


def test_scipy_cross_check_er_rows_subset():
    A = gen.config("C2")
    rows = np.arange(0, A.nrows, 997, dtype=np.int64)
    R = oracle.spgemm(A, A, rows=rows)
    S = (A.to_scipy()[rows] @ A.to_scipy()).tocsr()
    S.sort_indices()
    assert np.array_equal(R.row_ptr, S.indptr.astype(np.int64))
    assert np.array_equal(R.col, S.indices.astype(np.int32))
    assert np.allclose(R.val, S.data, rtol=1e-13, atol=0)


def test_row_nnz_bounded_by_work_and_width():
    A = gen.config("rmat11")
    w = oracle.row_work(A, A)
    u = oracle.counts(A, A)
    assert np.all(u <= np.minimum(w, A.ncols))
    assert np.all((u == 0) == (w == 0))


def test_fp32_inputs_promote_to_fp64():
    A = gen.config("C1", dtype="f32")
    R = oracle.spgemm(A, A)
    Ad = A.to_dense()  # float32 values widened exactly
    ref = Ad @ Ad
    got = _dense_of(R, A.nrows, A.ncols)
    assert np.allclose(got, ref, rtol=1e-14, atol=0)


def test_empty_and_degenerate():
    Z = gen.empty_rows(5, 7)
    B = gen.random_pattern(7, 4, 0.5, 3)
    R = oracle.spgemm(Z, B)
    assert R.nnz == 0 and np.all(R.row_ptr == 0)
    A = gen.random_pattern(6, 7, 0.3, 4)
    R = oracle.spgemm(A, gen.empty_rows(7, 3))
    assert R.nnz == 0
    assert len(oracle.spgemm(A, B, rows=np.zeros(0, dtype=np.int64)).rows) == 0


# ---- O2 -------------------------------------------------------------------------------------

@pytest.mark.parametrize("name", ["C1", "rmat12"])
def test_work_outer_product_identity(name):
    """sum_i w_i = sum_k colnnz_A(k) * rownnz_B(k) (outer-product form of L_AB = A x V_B)."""
    A = gen.config(name)
    w = oracle.row_work(A, A)
    colnnz = np.bincount(A.col, minlength=A.ncols).astype(np.int64)
    rownnz = np.diff(A.row_ptr)
    assert int(w.sum()) == int((colnnz * rownnz).sum())


def test_work_is_spmv_with_row_counts():
    """L_AB = A x V_B as an SpMV on the pattern, in fp64 (exact below 2^53)."""
    A = gen.config("rmat12")
    w = oracle.row_work(A, A)
    VB = np.diff(A.row_ptr).astype(np.float64)
    pat = A.to_scipy().copy()
    pat.data[:] = 1.0
    assert np.array_equal((pat @ VB).astype(np.int64), w)


def _struct_dense(A):
    d = np.zeros((A.nrows, A.ncols), dtype=np.int64)
    for i in range(A.nrows):
        d[i, A.col[A.row_ptr[i]:A.row_ptr[i + 1]]] = 1
    return d


@pytest.mark.parametrize("mode", ["signed", "zeros"])
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_structural_zeros_and_exact_cancellation(mode, seed):
    """Reading R9 (structural semantics): C has an entry wherever a product exists, kept when its
    value is 0 — by exact cancellation (signed integers) or from explicitly stored zeros. Structure
    = boolean product of the STORED patterns; values = the dense integer product, bit-exact."""
    A = gen.random_pattern(48, 40, 0.15, seed, mode)
    B = gen.random_pattern(40, 56, 0.15, seed + 50, mode)
    R = oracle.spgemm(A, B)
    _assert_canonical(R)
    pat = _struct_dense(A) @ _struct_dense(B) > 0
    assert np.array_equal(_pattern_of(R, 48, 56), pat)
    assert np.array_equal(_dense_of(R, 48, 56), A.to_dense() @ B.to_dense())
    zeros = int((R.val == 0).sum())
    assert zeros > 0, "the fixture must produce structural zeros"
    assert R.nnz == int(pat.sum())


@pytest.mark.parametrize("name", ["C1", "rmat11"])
def test_moments_digest_vs_scipy_structure(name):
    """oracle.moments (per-row u, sum c, c^2, c^3 mod 2^64; the structure digest the C3 parity test
    uses) equals the same sums over scipy.sparse's A@A pattern (an independent SpGEMM)."""
    A = gen.config(name)
    S = A.to_scipy()
    P = (S @ S).tocsr()
    P.sort_indices()
    m = oracle.moments(A, A)
    for i in range(A.nrows):
        c = P.indices[P.indptr[i]:P.indptr[i + 1]].astype(np.uint64)
        assert int(m[i, 0]) == len(c)
        assert m[i, 1] == c.sum(dtype=np.uint64)
        assert m[i, 2] == (c * c).sum(dtype=np.uint64)
        assert m[i, 3] == (c * c * c).sum(dtype=np.uint64)
