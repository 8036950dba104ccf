"""GPU parity of the HH-CPU four-block variant (PAPER Alg. 3,
Section V-A) against the oracle (oracle.hh_block / hh_combine / hh_sample / hh_extrapolate)."""
import numpy as np
import pytest
import torch

import oracle
import sginputs as gen
from _util import compare_rows

pytestmark = pytest.mark.gpu

sg = pytest.importorskip("paper_conf_icpp_hardhikbrks17_b200")


def _host(C):
    return C.row_ptr.cpu().numpy(), C.col.cpu().numpy(), C.val.cpu().numpy()


@pytest.mark.parametrize("name,t", [("rmat12", 16), ("rmat12", 64), ("C1", 8), ("rmat14", 100)])
def test_filter_matches_oracle_classes(name, t):
    A = gen.config(name)
    dA = sg.DeviceCSR.from_host(A)
    d = np.diff(A.row_ptr)
    for high in (True, False):
        F = sg.sg_hh_filter(dA, t, high)
        rp, col, val = _host(F)
        keep = (d > t) == high
        assert np.array_equal(np.diff(rp), np.where(keep, d, 0))
        idx = np.concatenate([np.arange(A.row_ptr[i], A.row_ptr[i + 1]) for i in np.nonzero(keep)[0]] or [np.zeros(0, int)])
        assert np.array_equal(col, A.col[idx]) and np.array_equal(val, A.val[idx])


@pytest.mark.parametrize("name,t", [("rmat12", 16), ("rmat13", 40), ("C1", 8)])
def test_four_blocks_equal_oracle_blocks(name, t):
    """Each block A_X B_Y on the hot path equals oracle.hh_block (integer values: bit-exact)."""
    A = gen.config(name, mode="int")
    dA = sg.DeviceCSR.from_host(A)
    F = {1: sg.sg_hh_filter(dA, t, True), 0: sg.sg_hh_filter(dA, t, False)}
    for x in (0, 1):
        for y in (0, 1):
            if F[x].nnz == 0 or F[y].nnz == 0:
                assert oracle.hh_block(A, A, t, x, y).nnz == 0
                continue
            C, _ = sg.spgemm(F[x], F[y], 0.05, 3)
            R = oracle.hh_block(A, A, t, x, y)
            rp, col, val = _host(C)
            assert np.array_equal(rp, R.row_ptr)
            assert np.array_equal(col, R.col) and np.array_equal(val, R.val)


@pytest.mark.parametrize("mode,dtype", [("int", "f64"), ("real", "f64"), ("real", "f32"), ("signed", "f64")])
def test_spgemm_hh_equals_the_product(mode, dtype):
    """Phase IV (P + Q as [P Q] * [I; I]) over the four blocks gives C = A*A: structure bit-exact,
    values bit-exact for integer values and within the north-star tolerance otherwise."""
    A = gen.config("rmat13", mode=mode, dtype=dtype)
    dA = sg.DeviceCSR.from_host(A)
    C, info = sg.spgemm_hh(dA, dA, 24)
    R = oracle.spgemm(A, A, with_absmag=True)
    rp, col, val = _host(C)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, dtype, exact_values=mode in ("int", "signed"))
    assert sum(info["blocks"].values()) >= R.nnz  # the blocks overlap in structure; their union is C


def test_add_keeps_structural_zeros():
    """P + (-P): every entry of P stays, with value 0 (reading R9)."""
    A = gen.config("C1", mode="int")
    dA = sg.DeviceCSR.from_host(A)
    N = sg.DeviceCSR(dA.nrows, dA.ncols, dA.row_ptr, dA.col, -dA.val)
    S = sg.sg_hh_add(dA, N)
    rp, col, val = _host(S)
    assert np.array_equal(rp, A.row_ptr) and np.array_equal(col, A.col) and not val.any()


@pytest.mark.parametrize("name,seed,f", [("rmat12", 3, None), ("rmat14", 5, None), ("C1", 1, 0.2), ("rmat10", 2, 1.0)])
def test_sample_equals_oracle(name, seed, f):
    A = gen.config(name)
    dA = sg.DeviceCSR.from_host(A)
    rows, As, pos = sg.sg_hh_sample(dA, seed, f)
    orows, orp, ocol, opos = oracle.hh_sample(A, seed, f)
    assert np.array_equal(rows.cpu().numpy(), orows)
    assert np.array_equal(As.row_ptr.cpu().numpy(), orp)
    assert np.array_equal(As.col.cpu().numpy(), ocol) and np.array_equal(pos.cpu().numpy(), opos)
    assert np.array_equal(As.val.cpu().numpy(), A.val[opos])


def test_hh_threshold_runs_sample_identify_extrapolate():
    A = gen.config("rmat14")
    dA = sg.DeviceCSR.from_host(A)
    tA, info = sg.hh_threshold(dA, seed=1, reps=1)
    assert tA == oracle.hh_extrapolate(info["t_s"])
    assert info["sample_rows"] > 0 and len(info["curve"]) >= 2
    ts = min(info["curve"], key=lambda k: info["curve"][k])
    assert int(ts) == info["t_s"]
