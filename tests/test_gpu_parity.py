"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the same seeded inputs.

Structure (C.row_ptr, C.col) and every integer quantity (w, classes, sample set, thresholds, cuts)
must be bit-exact; values within rtol * sum_k |a_ik b_kj| (1e-12 fp64, 1e-5 fp32; north_star), and
bit-exact in integer-value mode (R11).
"""
import numpy as np
import pytest
import torch

import oracle
import sginputs as gen
from _util import compare_rows

pytestmark = pytest.mark.gpu

sg = pytest.importorskip("paper_conf_icpp_hardhikbrks17_b200")


def _dev(H):
    return sg.DeviceCSR.from_host(H)


@pytest.fixture
def dense_log2():
    """Forces the dense-window bound (sg_set_option(SG_OPT_DENSE_LOG2, m)); restored afterwards."""
    old = sg.get_option(sg.SG_OPT_DENSE_LOG2)
    yield lambda m: sg.set_option(sg.SG_OPT_DENSE_LOG2, m)
    sg.set_option(sg.SG_OPT_DENSE_LOG2, old)


def _model_from(cm_sg):
    o = oracle.CostModel()
    for k, v in cm_sg.as_dict().items():
        setattr(o, k, v)
    return o


def _full_product(A, B, thr):
    dA, dB = _dev(A), (_dev(B) if B is not A else None)
    dB = dB or dA
    plan = sg.sg_symbolic(dA, dB, thr)
    col, val = sg.sg_numeric(plan, dA, dB)
    torch.cuda.synchronize()
    info = plan.info()
    cls = plan.classes().cpu().numpy()
    out = plan.row_ptr.cpu().numpy(), col.cpu().numpy(), val.cpu().numpy()
    plan.destroy()
    return out, info, cls


# ---- a1 row work ----------------------------------------------------------------------------

@pytest.mark.parametrize("name", ["C1", "C2", "rmat12", "rmat16"])
def test_row_work_bit_exact(name):
    A = gen.config(name)
    w, W = sg.sg_row_work(_dev(A), _dev(A), with_total=True)
    wo = oracle.row_work(A, A)
    assert np.array_equal(w.cpu().numpy(), wo)
    assert W == int(wo.sum())


def test_row_work_subrange_and_empty():
    A = gen.config("rmat12")
    dA = _dev(A)
    w = sg.sg_row_work(dA, dA, 100, 2000).cpu().numpy()
    assert np.array_equal(w, oracle.row_work(A, A)[100:2000])
    assert sg.sg_row_work(dA, dA, 5, 5).numel() == 0


# ---- a3 sampler ---------------------------------------------------------------------------------

@pytest.mark.parametrize("n,f,seed", [(1000, 0.05, 1), (262_144, 0.01, 7), (1 << 20, 0.1, 3), (777, 1.0, 2)])
def test_sample_rows_bit_exact(n, f, seed):
    S = sg.sg_sample_rows(n, f, seed).cpu().numpy()
    assert np.array_equal(S, oracle.sample_rows(n, seed, f))


@pytest.mark.parametrize("name,f,seed", [("C1", 0.2, 1), ("C2", 0.01, 3), ("rmat12", 0.05, 5),
                                         ("rmat14", 0.02, 11), ("rmat14", 1.0, 0)])
def test_sampled_threshold_bit_exact(name, f, seed):
    A = gen.config(name)
    dA = _dev(A)
    cm = sg.sg_default_cost_model()
    thr, rep = sg.sg_sample_threshold(dA, dA, f, seed, cm)
    o = oracle.sampled_threshold(A, A, f, seed, _model_from(cm))
    assert thr == o.thr
    assert rep["sample_rows"] == len(o.rows)
    assert rep["sample_nonempty"] == o.nonempty
    assert rep["J_min"] == o.Jmin
    assert rep["W_est_L"] == o.W_est_L and rep["W_est_H"] == o.W_est_H


@pytest.mark.parametrize("seed", range(4))
def test_sampled_threshold_random_models(seed):
    rng = np.random.default_rng(seed)
    A = gen.config("rmat12")
    dA = _dev(A)
    cm = sg.CostModel(kappa_L=int(rng.integers(0, 5000)), lambda_L=int(rng.integers(1, 200)),
                      sigma_L=int(rng.integers(0, 5)), rho_L=int(rng.integers(0, 300)),
                      kappa_H=int(rng.integers(0, 10**6)), lambda_H=int(rng.integers(1, 200)),
                      tau_H=int(rng.integers(0, 1000)), mu_H=int(rng.integers(0, 300)),
                      tiles_fixed=int(rng.integers(1, 5)), capu=int(rng.choice([0, 1024, 4096])),
                      cap_L=int(rng.integers(16, 4097)))
    thr, rep = sg.sg_sample_threshold(dA, dA, 0.1, seed, cm)
    o = oracle.sampled_threshold(A, A, 0.1, seed, _model_from(cm))
    assert thr == o.thr and rep["J_min"] == o.Jmin
    ts, Js = sg.sg_exhaustive_threshold(dA, dA, cm)
    to, Jo = oracle.exhaustive_threshold(A, A, _model_from(cm))
    assert (ts, Js) == (to, Jo)


def test_cost_curve_matches_plain_J():
    A = gen.config("rmat11")
    dA = _dev(A)
    cm = sg.sg_default_cost_model()
    ts = [0, 1, 7, 64, 500, 4096, 10**6]
    J = sg.sg_cost_curve(dA, dA, ts, cm)
    w = oracle.row_work(A, A)
    u = oracle.counts(A, A)
    a = np.diff(A.row_ptr)
    assert J == [oracle.J(_model_from(cm), w, a, u, t) for t in ts]


@pytest.mark.parametrize("name,kind", [("C1", "first"), ("rmat12", "first"), ("rmat12", "random"),
                                       ("rmat14_unperm", "first"), ("rmat14_unperm", "sqrt")])
def test_threshold_on_explicit_rows_bit_exact(name, kind):
    """Identify on a caller-chosen sample (predetermined first rows, random rows with repeats, sqrt(n)
    rows): the GPU thr and J_min equal the oracle's argmin over exactly those rows."""
    A = gen.rmat(14, permute=False) if name == "rmat14_unperm" else gen.config(name)
    dA = _dev(A)
    cm = sg.sg_default_cost_model()
    n = A.nrows
    rng = np.random.default_rng(3)
    rows = {"first": np.arange(max(n // 50, 1)), "random": rng.integers(0, n, size=n // 20),
            "sqrt": np.sort(rng.choice(n, size=int(np.sqrt(n)), replace=False))}[kind].astype(np.int64)
    thr, rep = sg.sg_threshold_on_rows(dA, dA, rows, cm)
    w = oracle.row_work(A, A)[rows]
    a = np.diff(A.row_ptr)[rows]
    u = oracle.counts(A, A, rows)
    t_o, J_o = oracle.threshold(_model_from(cm), w, a, u)
    assert (thr, rep["J_min"]) == (t_o, J_o)
    assert rep["sample_rows"] == len(rows) and rep["sample_nonempty"] == int((w > 0).sum())


def test_threshold_on_rows_rejects_bad_rows():
    A = gen.config("C1")
    dA = _dev(A)
    with pytest.raises(sg.SgError) as e:
        sg.sg_threshold_on_rows(dA, dA, np.array([0, 5, A.nrows], dtype=np.int64))
    assert "INVALID_ARG" in str(e.value)


def test_empty_sample_is_an_error():
    Z = gen.empty_rows(50, 50)
    dZ = _dev(Z)
    with pytest.raises(sg.SgError) as e:
        sg.sg_sample_threshold(dZ, dZ, 0.5, 1)
    assert "EMPTY_SAMPLE" in str(e.value)


# ---- a4 partition -------------------------------------------------------------------------------

@pytest.mark.parametrize("name", ["C2", "rmat14"])
@pytest.mark.parametrize("G", [1, 2, 3, 8])
def test_partition_bit_exact(name, G):
    A = gen.config(name)
    cuts, W = sg.sg_partition(_dev(A), _dev(A), G)
    w = oracle.row_work(A, A)
    assert cuts == list(oracle.partition(w, G))
    assert W == int(w.sum())


def test_partition_plateaus_and_ties():
    # rows with zero work create plateaus in the prefix; ties go to the smaller boundary
    A = gen.banded(64, [0], [1.0])
    rp = A.row_ptr.copy()
    keep = np.ones(64, bool)
    keep[10:30] = False  # empty rows 10..29
    cols, vals, nrp = [], [], [0]
    for i in range(64):
        if keep[i]:
            cols.append(i); vals.append(1.0)
        nrp.append(len(cols))
    A = gen.CSR(64, 64, np.array(nrp, np.int64), np.array(cols, np.int32), np.array(vals), "plateau")
    for G in (2, 3, 5, 7):
        cuts, _ = sg.sg_partition(_dev(A), _dev(A), G)
        assert cuts == list(oracle.partition(oracle.row_work(A, A), G))


@pytest.mark.parametrize("name", ["C1", "rmat12", "rmat12u", "rmat14u"])
@pytest.mark.parametrize("G", [1, 2, 3, 8])
def test_partition_cost_bit_exact(name, G):
    """NEXT #2 (R19): the sample's per-class compression and the cost-weighted cuts,
    bit-exact against the oracle (permuted and un-permuted R-MAT: hubs at low row ids)."""
    A = gen.rmat(int(name[4:-1]), 16, seed=1, permute=False) if name.endswith("u") else gen.config(name)
    dA = _dev(A)
    cm = sg.sg_default_cost_model()
    thr, rep = sg.sg_sample_threshold(dA, dA, 0.05, 3, cm)
    o = oracle.sampled_threshold(A, A, 0.05, 3, _model_from(cm))
    assert thr == o.thr
    comp = oracle.sample_comp(o)
    assert [rep["U_est_L"], rep["W_est_L"], rep["U_est_H"], rep["W_est_H"]] == comp.tolist()
    cuts, tot = sg.sg_partition_cost(dA, dA, G, thr, comp.tolist(), cm)
    ocuts, otot = oracle.partition_cost(_model_from(cm), thr, comp, oracle.row_work(A, A), np.diff(A.row_ptr), G)
    assert cuts == ocuts.tolist() and tot == otot


@pytest.mark.parametrize("name", ["rmat12", "rmat14u"])
def test_partition_cost_default_partition_model(name):
    """cm = NULL selects sg_default_partition_model; same cuts as the oracle with it."""
    A = gen.rmat(int(name[4:-1]), 16, seed=1, permute=False) if name.endswith("u") else gen.config(name)
    dA = _dev(A)
    thr, rep = sg.sg_sample_threshold(dA, dA, 0.05, 3)
    comp = [rep["U_est_L"], rep["W_est_L"], rep["U_est_H"], rep["W_est_H"]]
    pm = sg.sg_default_partition_model()
    assert pm.rho_L > 0 and pm.lambda_H > 0
    for G in (2, 8):
        cuts, tot = sg.sg_partition_cost(dA, dA, G, thr, comp)
        ocuts, otot = oracle.partition_cost(_model_from(pm), thr, comp, oracle.row_work(A, A), np.diff(A.row_ptr), G)
        assert cuts == ocuts.tolist() and tot == otot


def test_partition_cost_edge_cases():
    A = gen.config("rmat10")
    dA = _dev(A)
    cm = sg.sg_default_cost_model()
    w, a = oracle.row_work(A, A), np.diff(A.row_ptr)
    for thr, comp in [(0, [0, 0, 0, 0]), (4096, [5, 7, 0, 0]), (100, [1, 1, 1, 1]), (1, [0, 3, 9, 10])]:
        cuts, tot = sg.sg_partition_cost(dA, dA, 5, thr, comp, cm)
        ocuts, otot = oracle.partition_cost(_model_from(cm), thr, comp, w, a, 5)
        assert cuts == ocuts.tolist() and tot == otot
    with pytest.raises(RuntimeError):
        sg.sg_partition_cost(dA, dA, 0, 10, [1, 1, 1, 1], cm)
    with pytest.raises(RuntimeError):
        sg.sg_partition_cost(dA, dA, 2, 10, [-1, 1, 1, 1], cm)


# ---- a5-a8 symbolic + numeric ---------------------------------------------------------------------

def _csr_from_sets(nrows, ncols, rows, seed):
    rng = np.random.default_rng(seed)
    rp, cols = [0], []
    for r in rows:
        c = np.unique(np.asarray(r, dtype=np.int64))
        cols.append(c)
        rp.append(rp[-1] + len(c))
    col = np.concatenate(cols).astype(np.int32) if cols else np.zeros(0, np.int32)
    val = 0.5 + rng.random(col.shape[0])
    return gen.CSR(nrows, ncols, np.array(rp, np.int64), col, val, "sets")


@pytest.mark.parametrize("f32", [False, True])
def test_rank_kernel_big_tile_ranges(f32):
    """A heavy (rank-kernel) row whose columns crowd one 8192-column tile far beyond half the range
    capacity: such a tile must form a range of its own (sg_heavy.cu range plan)."""
    rng = np.random.default_rng(5)
    p, m = 1 << 20, 200
    brows = []
    for k in range(m):
        brows.append(np.concatenate([rng.integers(5 * 8192, 6 * 8192, 100), rng.integers(0, 8192, 10),
                                     rng.integers(9 * 8192, 10 * 8192, 10), rng.integers(0, p, 5)]))
    B = _csr_from_sets(m, p, brows, 1)
    A = _csr_from_sets(5, m, [np.arange(m), np.arange(0, m, 2), [], rng.integers(0, m, 10), np.arange(150)], 2)
    if f32:
        A, B = A.astype("f32"), B.astype("f32")
    (rp, col, val), info, cls = _full_product(A, B, 0)
    assert info["n_heavy"] == 4 and info["n_dense"] == 0
    R = oracle.spgemm(A, B, with_absmag=True)
    assert np.array_equal(rp, R.row_ptr)
    assert int(np.diff(rp)[0]) > 10000
    compare_rows(rp, col, val, R, "f32" if f32 else "f64")


@pytest.mark.parametrize("name", ["C1", "rmat10", "rmat12"])
@pytest.mark.parametrize("thr", [0, 1, 64, 300, 4096])
def test_full_product_bit_exact_structure(name, thr):
    A = gen.config(name)
    (rp, col, val), info, cls = _full_product(A, A, thr)
    R = oracle.spgemm(A, A, with_absmag=True)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, "f64")
    w = oracle.row_work(A, A)
    exp_cls = np.where(w == 0, 0, np.where(w > thr, 2, 1))
    assert np.array_equal(cls, exp_cls)
    assert info["n_heavy"] == int((exp_cls == 2).sum()) and info["flops"] == int(w.sum())


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_integer_values_bit_exact(dtype):
    A = gen.config("rmat12", mode="int", dtype=dtype)
    for thr in (0, 128, 4096):
        (rp, col, val), _, _ = _full_product(A, A, thr)
        R = oracle.spgemm(A, A, with_absmag=True)
        compare_rows(rp, col, val, R, dtype, exact_values=True)


def test_fp32_tolerance():
    A = gen.config("rmat12", dtype="f32")
    (rp, col, val), _, _ = _full_product(A, A, 256)
    assert val.dtype == np.float32
    R = oracle.spgemm(A, A, with_absmag=True)
    compare_rows(rp, col, val, R, "f32")


def test_er_2pow18_full():
    """Config 2 (ER 2^18, 16/row), every row, at the sampled threshold."""
    A = gen.config("C2")
    dA = _dev(A)
    thr, _ = sg.sg_sample_threshold(dA, dA, 0.01, 1)
    (rp, col, val), _, _ = _full_product(A, A, thr)
    R = oracle.spgemm(A, A, with_absmag=True)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, "f64")


@pytest.mark.parametrize("thr", [0, 2048])
def test_rmat16_heavy_ranges(thr):
    """Several heavy rows span many column tiles / hashed ranges (p = 65536 -> 8 tiles)."""
    A = gen.config("rmat16")
    (rp, col, val), info, _ = _full_product(A, A, thr)
    R = oracle.spgemm(A, A, with_absmag=True)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, "f64")
    assert info["n_ranges"] > 0


def test_rmat18_sampled_rows():
    """R-MAT 18 (config 5): structure bit-exact on every row (row_ptr), values on a seeded row
    sample plus the 64 heaviest rows."""
    A = gen.config("R18")
    dA = _dev(A)
    thr, _ = sg.sg_sample_threshold(dA, dA, 0.01, 1)
    (rp, col, val), _, _ = _full_product(A, A, thr)
    u = oracle.counts(A, A)
    assert np.array_equal(np.diff(rp), u)
    w = oracle.row_work(A, A)
    rows = np.union1d(oracle.sample_rows(A.nrows, 99, 0.002), np.argsort(w)[-64:]).astype(np.int64)
    R = oracle.spgemm(A, A, rows=rows, with_absmag=True)
    compare_rows(rp, col, val, R, "f64")


def test_special_matrices():
    n = 3000
    A = gen.config("C1")
    I = gen.identity(A.nrows)
    for X, Y in ((A, I), (I, A)):
        (rp, col, val), _, _ = _full_product(X, Y, 64)
        assert np.array_equal(rp, A.row_ptr) and np.array_equal(col, A.col) and np.array_equal(val, A.val)
    P = gen.permutation(n, 4)
    T = gen.tridiag(n, 2.0, 3.0, 5.0)
    for X, Y in ((P, T), (T, P), (T, T)):
        for thr in (0, 8):
            (rp, col, val), _, _ = _full_product(X, Y, thr)
            R = oracle.spgemm(X, Y, with_absmag=True)
            assert np.array_equal(rp, R.row_ptr)
            compare_rows(rp, col, val, R, "f64", exact_values=True)


def test_rectangular_and_ragged():
    A = gen.random_pattern(37, 5000, 0.01, 3)
    B = gen.random_pattern(5000, 70000, 0.002, 4)
    for thr in (0, 16, 4096):
        (rp, col, val), _, _ = _full_product(A, B, thr)
        R = oracle.spgemm(A, B, with_absmag=True)
        assert np.array_equal(rp, R.row_ptr)
        compare_rows(rp, col, val, R, "f64")


def test_empty_inputs():
    Z = gen.empty_rows(100, 100)
    (rp, col, val), info, cls = _full_product(Z, Z, 10)
    assert np.all(rp == 0) and col.size == 0 and info["n_empty"] == 100
    A = gen.random_pattern(1, 1, 1.0, 1)
    (rp, col, val), _, _ = _full_product(A, A, 0)
    assert list(rp) == [0, 1] and list(col) == [0]


def test_row_subrange_concatenation_equals_whole():
    A = gen.config("rmat12")
    dA = _dev(A)
    cuts, _ = sg.sg_partition(dA, dA, 3)
    whole = oracle.spgemm(A, A)
    cols, nnzs = [], []
    for g in range(3):
        plan = sg.sg_symbolic(dA, dA, 512, cuts[g], cuts[g + 1])
        c, v = sg.sg_numeric(plan, dA, dA)
        cols.append(c.cpu().numpy())
        nnzs.append(plan.nnz)
        plan.destroy()
    assert np.array_equal(np.concatenate(cols), whole.col)


def test_errors():
    A = gen.config("C1")
    dA = _dev(A)
    with pytest.raises(sg.SgError, match="INVALID_ARG"):
        sg.sg_symbolic(dA, dA, sg.SG_CAP_L_MAX + 1)
    with pytest.raises(sg.SgError, match="INVALID_ARG"):
        sg.sg_sample_threshold(dA, dA, 0.0, 1)
    B = _dev(gen.random_pattern(7, 9, 0.3, 1))
    with pytest.raises(sg.SgError, match="SHAPE"):
        sg.sg_symbolic(dA, B, 10)
    A32 = _dev(A.astype("f32"))
    with pytest.raises(sg.SgError, match="DTYPE"):
        sg.sg_symbolic(dA, A32, 10)


def test_gather_single_rank_nccl():
    """sg_gather through a real NCCL communicator (world size 1 on the one-GPU box): the global
    row_ptr and the gathered col/val equal the local result."""
    import os
    import socket
    import torch.distributed as dist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    try:
        dist.barrier()
        comm = dist.group.WORLD._get_backend(dev)._comm_ptr()
        A = gen.config("rmat12")
        dA = _dev(A)
        plan = sg.sg_symbolic(dA, dA, 256)
        col, val = sg.sg_numeric(plan, dA, dA)
        rp, gcol, gval, tot = sg.sg_gather(plan, comm, A.nrows, col, val, gather_values=True, nnz_global=plan.nnz)
        torch.cuda.synchronize()
        assert tot == plan.nnz
        assert torch.equal(rp, plan.row_ptr)
        assert torch.equal(gcol, col) and torch.equal(gval, val)
        plan.destroy()
    finally:
        dist.destroy_process_group()


def test_rmat22_multi_window_row_subset():
    """p = 2^22 columns: four 2^20-column symbolic windows, T = 512 column tiles (config 4's
    matrix). Rows [0, n/256) at the sampled threshold: structure bit-exact on every row of the
    subset (row_ptr vs oracle counts), values on a seeded sample plus the heaviest rows."""
    A = gen.config("C4")
    dA = _dev(A)
    thr, _ = sg.sg_sample_threshold(dA, dA, 0.002, 1)
    re = A.nrows // 256
    plan = sg.sg_symbolic(dA, dA, thr, 0, re)
    col, val = sg.sg_numeric(plan, dA, dA)
    torch.cuda.synchronize()
    rp = plan.row_ptr.cpu().numpy()
    rows = np.arange(re, dtype=np.int64)
    assert np.array_equal(np.diff(rp), oracle.counts(A, A, rows))
    w = oracle.row_work(A, A)[:re]
    pick = np.union1d(oracle.sample_rows(re, 5, 0.01), np.argsort(w)[-16:]).astype(np.int64)
    R = oracle.spgemm(A, A, rows=pick, with_absmag=True)
    compare_rows(rp, col.cpu().numpy(), val.cpu().numpy(), R, "f64")
    plan.destroy()


@pytest.mark.parametrize("dw", ["0", "62"])
@pytest.mark.parametrize("name,thr", [("rmat12", 0), ("rmat16", 2048), ("C1", 16)])
def test_dense_window_path_forced(dense_log2, name, thr, dw):
    """Every heavy row on the dense-window kernel (SG_OPT_DENSE_LOG2 = 0) or none (62): same C either way."""
    dense_log2(int(dw))
    A = gen.config(name)
    (rp, col, val), info, _ = _full_product(A, A, thr)
    R = oracle.spgemm(A, A, with_absmag=True)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, "f64")
    assert info["n_dense"] == (info["n_heavy"] if dw == "0" else 0)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_dense_window_integer_values_exact(dense_log2, dtype):
    """Dense-window accumulation in integer-value mode: values bit-exact (R11); includes
    rows with more than 1024 k entries (multi-chunk) at R-MAT 16."""
    dense_log2(0)
    A = gen.config("rmat16", mode="int", dtype=dtype)
    (rp, col, val), info, _ = _full_product(A, A, 1024)
    assert int(np.diff(A.row_ptr).max()) > 1024
    R = oracle.spgemm(A, A, with_absmag=True)
    compare_rows(rp, col, val, R, dtype, exact_values=True)
    assert info["n_dense"] == info["n_heavy"] > 0


@pytest.fixture
def hash_light():
    old = sg.get_option(sg.SG_OPT_VARIANT)
    sg.set_option(sg.SG_OPT_VARIANT, old | 16)
    yield
    sg.set_option(sg.SG_OPT_VARIANT, old)


@pytest.mark.parametrize("scale,thr", [(14, 4096), (16, 1024)])
def test_light_skewed_rows_sorted_path(scale, thr, hash_light):
    """Un-permuted R-MAT (hubs at low ids): light rows whose columns crowd the order-preserving
    hash's homes take the uniform-hash + bitonic-sort path; C is unchanged (structure bit-exact).
    (SG_OPT_VARIANT bit 4: every light bin on the hash path, so the skew detection runs for all.)"""
    A = gen.rmat(scale, permute=False)
    (rp, col, val), info, _ = _full_product(A, A, thr)
    R = oracle.spgemm(A, A, with_absmag=True)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, "f64")
    assert info["n_light_sorted"] > 0


def test_light_sorted_path_integer_values_exact(hash_light):
    A = gen.rmat(14, permute=False, mode="int")
    (rp, col, val), info, _ = _full_product(A, A, 4096)
    R = oracle.spgemm(A, A, with_absmag=True)
    compare_rows(rp, col, val, R, "f64", exact_values=True)
    assert info["n_light_sorted"] > 0


@pytest.mark.parametrize("name", ["C2", "rmat16"])
def test_uniform_rows_keep_the_order_preserving_path(name, hash_light):
    """Permuted / uniform inputs: (almost) no light row is flagged as column-skewed."""
    A = gen.config(name)
    _, info, _ = _full_product(A, A, 4096)
    assert info["n_light_sorted"] <= max(1, info["n_light"] // 100)


@pytest.mark.parametrize("blocks", [1, 3, 8])
def test_spgemm_to_host_blocks(blocks):
    """Row-blocked C streamed to the host while later blocks compute equals the oracle."""
    A = gen.config("rmat12")
    dA = _dev(A)
    R = oracle.spgemm(A, A, with_absmag=True)
    parts = []

    def sink(g, r0, r1, drp, dcol, dval):  # runs with the copy stream current
        parts.append((g, r0, r1, drp[:-1].to("cpu", non_blocking=True), dcol.to("cpu", non_blocking=True),
                      dval.to("cpu", non_blocking=True)))

    info = sg.spgemm_to_host(dA, dA, sink, blocks=blocks, sample_frac=0.05, seed=3)
    torch.cuda.synchronize()
    off = info["offsets"]
    assert info["nnz"] == R.nnz and len(parts) == blocks
    rp = np.zeros(A.nrows + 1, dtype=np.int64)
    col = np.zeros(R.nnz, dtype=np.int32)
    val = np.zeros(R.nnz, dtype=np.float64)
    for g, r0, r1, prp, pc, pv in parts:
        rp[r0:r1] = prp.numpy() + off[g]
        col[off[g]:off[g + 1]] = pc.numpy()
        val[off[g]:off[g + 1]] = pv.numpy()
    rp[A.nrows] = off[-1]
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, "f64")


def test_spgemm_to_host_more_blocks_than_rows_and_empty():
    """Degenerate row blocking: more blocks than rows (empty blocks), and an empty matrix."""
    A = gen.config("C1")
    small = gen.CSR(3, A.ncols, A.row_ptr[:4].copy(), A.col[:A.row_ptr[3]].copy(), A.val[:A.row_ptr[3]].copy(), "3rows")
    dS, dA = _dev(small), _dev(A)
    got = []
    info = sg.spgemm_to_host(dS, dA, lambda g, r0, r1, rp, c, v: got.append((r0, r1, int(c.numel()))), blocks=8,
                             thr=16)
    torch.cuda.synchronize()
    R = oracle.spgemm(small, A)
    assert info["nnz"] == R.nnz and sum(x[2] for x in got) == R.nnz and len(got) == 8
    E = gen.CSR(0, A.ncols, np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0), "empty")
    dE = _dev(E)
    info = sg.spgemm_to_host(dE, dA, lambda *a: None, blocks=4, thr=16)
    assert info["nnz"] == 0
    cuts, tot = sg.sg_partition_cost(dE, dA, 3, 16, [0, 0, 0, 0])
    assert cuts == [0, 0, 0, 0] and tot == 0

