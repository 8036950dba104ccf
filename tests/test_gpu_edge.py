"""GPU parity on the method's edge cases: exact cancellation and explicitly stored zeros (structural
semantics, reading R9) with every kernel path forced, in fp64, fp32 and integer values.

Values here are small signed integers ({-2,-1,1,2} or {-1,0,1,2}, sginputs modes "signed" / "zeros"),
so every sum is an exact integer below 2^24: values must be BIT-EXACT in fp64 and fp32 alike, and an
entry whose sum is 0 must still be present (C's structure = the boolean product of the stored
patterns, PAPER L74 / Alg. 2 l.5-6, L222-L223). The heavy kernels decide occupancy by "the
accumulator was exactly 0.0 when this product arrived" (sg_dense2.cu, sg_heavy.cu), which is exactly
what these inputs stress.
"""
import numpy as np
import pytest
import torch

import oracle
import sginputs as gen
from _util import compare_rows

pytestmark = pytest.mark.gpu

sg = pytest.importorskip("paper_conf_icpp_hardhikbrks17_b200")

# path -> (thr, dense_log2, variant): light = every row with w <= cap_L on the light kernels (the sorted
# warp path for w <= 512, the order-preserving hash above; light_hash: the hash for every bin); rank =
# every non-empty row heavy on the rank kernels (rows of <= 64 k entries on the warp-tile kernel, forced by
# variant bit 5 at these sizes, the rest on the CTA kernel; rank_cta: the CTA kernel for all); dense = every non-empty row heavy on the
# dense-window kernel
PATHS = {"light": (4096, 62, 0), "light_hash": (4096, 62, 16), "rank": (0, 62, 32), "rank_cta": (0, 62, 8),
         "dense": (0, 0, 0), "mixed": (256, 10, 32)}


@pytest.fixture
def options():
    old = (sg.get_option(sg.SG_OPT_DENSE_LOG2), sg.get_option(sg.SG_OPT_VARIANT), sg.get_option(sg.SG_OPT_TP_MAX_BYTES))
    yield
    sg.set_option(sg.SG_OPT_DENSE_LOG2, old[0])
    sg.set_option(sg.SG_OPT_VARIANT, old[1])
    sg.set_option(sg.SG_OPT_TP_MAX_BYTES, old[2])


def _run(A, thr):
    dA = sg.DeviceCSR.from_host(A)
    plan = sg.sg_symbolic(dA, dA, thr)
    col, val = sg.sg_numeric(plan, dA, dA)
    torch.cuda.synchronize()
    info = plan.info()
    out = plan.row_ptr.cpu().numpy(), col.cpu().numpy(), val.cpu().numpy()
    plan.destroy()
    return out, info


@pytest.mark.parametrize("path", list(PATHS))
@pytest.mark.parametrize("mode", ["signed", "zeros"])
@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_cancellation_and_stored_zeros_every_path(options, path, mode, dtype):
    thr, dl, var = PATHS[path]
    sg.set_option(sg.SG_OPT_DENSE_LOG2, dl)
    sg.set_option(sg.SG_OPT_VARIANT, var)
    A = gen.config("rmat13", mode=mode, dtype=dtype)
    (rp, col, val), info = _run(A, thr)
    R = oracle.spgemm(A, A)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, dtype, exact_values=True)
    assert int((R.val == 0).sum()) > 0, "fixture must contain structural zeros"
    if path == "dense":
        assert info["n_dense"] == info["n_heavy"] > 0
    if path == "rank":
        assert info["n_dense"] == 0 and info["n_heavy"] > 0


@pytest.mark.parametrize("variant", [0, 1])
def test_cancellation_dense_kernel_variants(options, variant):
    """Both dense-window kernels (SG_OPT_VARIANT 0: sg_dense2.cu, 1: sg_dense.cu) on multi-chunk rows
    (more than 1024 k entries at R-MAT 16) with signed values: bit-exact."""
    sg.set_option(sg.SG_OPT_VARIANT, variant)
    sg.set_option(sg.SG_OPT_DENSE_LOG2, 0)
    A = gen.config("rmat16", mode="signed")
    assert int(np.diff(A.row_ptr).max()) > 1024
    (rp, col, val), info = _run(A, 1024)
    R = oracle.spgemm(A, A)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, "f64", exact_values=True)
    assert info["n_dense"] > 0


@pytest.mark.parametrize("mode", ["signed", "zeros"])
def test_sorted_light_path_with_cancellation(options, mode):
    """Un-permuted R-MAT (column-skewed light rows take the uniform-hash + bitonic-sort path; variant bit 4
    keeps every light bin on the hash path, whose skew detection routes them there)."""
    sg.set_option(sg.SG_OPT_VARIANT, 16)
    A = gen.rmat(14, permute=False, mode=mode)
    (rp, col, val), info = _run(A, 4096)
    R = oracle.spgemm(A, A)
    compare_rows(rp, col, val, R, "f64", exact_values=True)
    assert info["n_light_sorted"] > 0


def test_all_zero_values_keep_full_structure(options):
    """Every stored value 0: C's values are all 0 and its structure is the full boolean product."""
    A = gen.config("rmat12")
    Z = gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, np.zeros_like(A.val), "zeros")
    for thr, dl, var in PATHS.values():
        sg.set_option(sg.SG_OPT_DENSE_LOG2, dl)
        sg.set_option(sg.SG_OPT_VARIANT, var)
        (rp, col, val), _ = _run(Z, thr)
        R = oracle.spgemm(A, A)
        assert np.array_equal(rp, R.row_ptr) and np.array_equal(col, R.col)
        assert not val.any()


def test_negative_zero_products_are_structural(options):
    """-0.0 inputs: products are +-0.0, every entry exists and compares equal to 0."""
    A = gen.config("C1")
    N = gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, np.full_like(A.val, -0.0), "negzero")
    for thr, dl, var in PATHS.values():
        sg.set_option(sg.SG_OPT_DENSE_LOG2, dl)
        sg.set_option(sg.SG_OPT_VARIANT, var)
        (rp, col, val), _ = _run(N, thr)
        R = oracle.spgemm(A, A)
        assert np.array_equal(rp, R.row_ptr) and np.array_equal(col, R.col)
        assert np.all(val == 0)


@pytest.mark.parametrize("name", ["C1", "rmat14"])
def test_kernel_variants_same_c(options, name):
    """Every SG_OPT_VARIANT computes the same C (integer values: bit-exact), equal to the oracle: the
    warp-tile vs CTA rank kernels (bits 3 and 5) and the sorted warp light path vs the order-preserving hash
    (bit 4), at a threshold that puts rows on both light and heavy paths."""
    A = gen.config(name, mode="int")
    R = oracle.spgemm(A, A)
    dA = sg.DeviceCSR.from_host(A)
    thr = sg.sg_sample_threshold(dA, dA, 0.05, 1)[0]
    outs = []
    for var in (0, 8, 16, 24, 32, 48):
        sg.set_option(sg.SG_OPT_VARIANT, var)
        (rp, col, val), info = _run(A, thr)
        assert np.array_equal(rp, R.row_ptr)
        compare_rows(rp, col, val, R, "f64", exact_values=True)
        outs.append((col, val))
    for col, val in outs[1:]:
        assert np.array_equal(col, outs[0][0]) and np.array_equal(val, outs[0][1])


@pytest.mark.parametrize("path", ["rank", "rank_cta", "dense", "mixed"])
def test_heavy_paths_without_tile_pointers(options, path):
    """SG_OPT_TP_MAX_BYTES = 0: no B tile-pointer table (the table grows with rows x columns); every
    heavy kernel finds its B-row segments by binary search and C is unchanged (integer values: bit-exact)."""
    thr, dl, var = PATHS[path]
    sg.set_option(sg.SG_OPT_DENSE_LOG2, dl)
    sg.set_option(sg.SG_OPT_VARIANT, var)
    sg.set_option(sg.SG_OPT_TP_MAX_BYTES, 0)
    A = gen.config("rmat13", mode="int")
    (rp, col, val), info = _run(A, thr)
    R = oracle.spgemm(A, A)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, "f64", exact_values=True)


def test_gather_rows_equals_host_gather_and_checks_ids():
    """sg_gather_rows (the Sample step's A_S = A[S, :]): bit-exact against a host gather, any order and
    repeated ids; an id out of range is INVALID_ARG."""
    A = gen.config("rmat12")
    dA = sg.DeviceCSR.from_host(A)
    rng = np.random.default_rng(5)
    rows = np.concatenate([rng.choice(A.nrows, 300, replace=False), [0, 0, A.nrows - 1]])
    S = sg.sg_gather_rows(dA, torch.as_tensor(rows, device="cuda"))
    lens = np.diff(A.row_ptr)[rows]
    rp = np.concatenate([[0], np.cumsum(lens)])
    idx = np.concatenate([np.arange(A.row_ptr[r], A.row_ptr[r + 1]) for r in rows])
    assert np.array_equal(S.row_ptr.cpu().numpy(), rp)
    assert np.array_equal(S.col.cpu().numpy(), A.col[idx])
    assert np.array_equal(S.val.cpu().numpy(), A.val[idx])
    with pytest.raises(sg.SgError, match="INVALID_ARG"):
        sg.sg_gather_rows(dA, torch.as_tensor([0, A.nrows], device="cuda"))


def test_measured_threshold_is_the_fastest_evaluated_candidate():
    """measured_threshold (the paper's Identify by running the algorithm on the sample): the threshold it
    returns is a grid point, the fastest of the candidates it timed, and the hot path at that threshold
    computes the oracle's C. (Timing itself is not pinned: parity unpinned by nature.)"""
    A = gen.config("rmat14")
    dA = sg.DeviceCSR.from_host(A)
    thr, rep = sg.measured_threshold(dA, dA, sample_frac=0.05, seed=2)
    T = rep["T_ms"]
    assert thr in T and len(T) >= 5 and rep["sample_rows"] > 0
    assert T[thr] == min(T.values())
    (rp, col, val), _ = _run(A, thr)
    R = oracle.spgemm(A, A, with_absmag=True)
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col, val, R, "f64")


def test_tile_kernel_rank_windows_of_a_dense_tile(options):
    """A tile with more outputs than the warp-tile kernel's accumulator (512 entries) is accumulated in
    rank windows: rows of <= 64 k entries whose B rows fill most of tile 0 (8192 columns) — integer values,
    bit-exact against the oracle, with the warp-tile kernel forced (variant bit 5) and no dense-window rows."""
    rng = np.random.default_rng(11)
    n, p = 256, 20000
    rows, cols = [], []
    for i in range(n):  # B = A: row i holds 40-64 columns, most of them in [0, 8192)
        k = int(rng.integers(40, 65))
        c = np.unique(np.concatenate([rng.choice(8192, k - 4, replace=False), rng.choice(np.arange(8192, p), 4)]))
        rows.append(np.full(c.size, i)); cols.append(c)
    r = np.concatenate(rows); c = np.concatenate(cols)
    rp = np.zeros(n + 1, dtype=np.int64); np.add.at(rp, r + 1, 1); rp = np.cumsum(rp)
    val = rng.integers(1, 5, size=c.size).astype(np.float64)
    # B: p x p, rows [0, n) as generated, the rest empty; A: the same pattern with columns folded into
    # [0, n) (every k of A hits a non-empty B row), so each row of C fills most of tile 0
    Brp = np.concatenate([rp, np.full(p - n, rp[-1], dtype=np.int64)])
    B = gen.CSR(p, p, Brp, c.astype(np.int32), val, "dense-tile-B")
    Ac = (c % n).astype(np.int64)
    order = np.lexsort((Ac, r))
    r2, c2, v2 = r[order], Ac[order], val[order]
    keep = np.ones(r2.size, bool); keep[1:] = (r2[1:] != r2[:-1]) | (c2[1:] != c2[:-1])
    r2, c2, v2 = r2[keep], c2[keep], v2[keep]
    rp2 = np.zeros(n + 1, dtype=np.int64); np.add.at(rp2, r2 + 1, 1); rp2 = np.cumsum(rp2)
    A = gen.CSR(n, p, rp2, c2.astype(np.int32), v2, "dense-tile-A")
    sg.set_option(sg.SG_OPT_DENSE_LOG2, 62)
    sg.set_option(sg.SG_OPT_VARIANT, 32)
    dA, dB = sg.DeviceCSR.from_host(A), sg.DeviceCSR.from_host(B)
    plan = sg.sg_symbolic(dA, dB, 0)
    col, cval = sg.sg_numeric(plan, dA, dB)
    torch.cuda.synchronize()
    R = oracle.spgemm(A, B)
    crp = plan.row_ptr.cpu().numpy()
    assert np.array_equal(crp, R.row_ptr)
    assert int(np.diff(R.row_ptr).max()) > 512  # some tile holds more outputs than one accumulator window
    compare_rows(crp, col.cpu().numpy(), cval.cpu().numpy(), R, "f64", exact_values=True)
    plan.destroy()


def _random_csr(rng, nrows, ncols, deg, name):
    rows, cols = [], []
    for i in range(nrows):
        c = np.unique(rng.integers(0, ncols, size=int(rng.integers(1, 2 * deg))))
        rows.append(np.full(c.size, i)); cols.append(c)
    r = np.concatenate(rows); c = np.concatenate(cols)
    rp = np.zeros(nrows + 1, dtype=np.int64); np.add.at(rp, r + 1, 1)
    return gen.CSR(nrows, ncols, np.cumsum(rp), c.astype(np.int32), rng.integers(1, 5, size=c.size).astype(np.float64), name)


def test_light_sorted_and_hash_bins_in_one_plan():
    """The sorted light path needs c < 2^(32 - log2 U): with B.ncols = 2^24 bin 8 (U = 256) is sorted and
    bin 9 (U = 512) falls back to the hash path in the same plan; C bit-exact against the oracle."""
    rng = np.random.default_rng(4)
    A = _random_csr(rng, 2048, 2048, 20, "A")
    B = _random_csr(rng, 2048, 1 << 24, 20, "B")
    dA, dB = sg.DeviceCSR.from_host(A), sg.DeviceCSR.from_host(B)
    plan = sg.sg_symbolic(dA, dB, 4096)
    col, val = sg.sg_numeric(plan, dA, dB)
    torch.cuda.synchronize()
    R = oracle.spgemm(A, B)
    w = oracle.row_work(A, B)
    assert ((w > 256) & (w <= 512)).any() and ((w > 128) & (w <= 256)).any()  # both bins populated
    crp = plan.row_ptr.cpu().numpy()
    assert np.array_equal(crp, R.row_ptr)
    compare_rows(crp, col.cpu().numpy(), val.cpu().numpy(), R, "f64", exact_values=True)
    plan.destroy()
