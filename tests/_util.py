"""Shared test helpers (comparison of a device C against the oracle)."""
import numpy as np

RTOL = {"f64": 1e-12, "f32": 1e-5}   # north_star tolerances, relative to sum_k |a_ik b_kj| (R16)


def compare_rows(rp, col, val, R, dtype, rows_local=None, exact_values=False):
    """rp/col/val: full device result on host (numpy); R: oracle RowsResult for the rows
    `R.rows` (global ids == local ids unless rows_local is given)."""
    rows = R.rows if rows_local is None else rows_local
    for s, i in enumerate(rows):
        lo, hi = int(rp[i]), int(rp[i + 1])
        olo, ohi = int(R.row_ptr[s]), int(R.row_ptr[s + 1])
        assert hi - lo == ohi - olo, f"row {i}: nnz {hi - lo} != oracle {ohi - olo}"
    # gather the device rows in oracle order
    idx = np.concatenate([np.arange(int(rp[i]), int(rp[i + 1])) for i in rows]) if len(rows) else np.zeros(0, np.int64)
    gc, gv = col[idx], val[idx].astype(np.float64)
    assert np.array_equal(gc, R.col), "column structure differs"
    if exact_values:
        assert np.array_equal(gv, R.val), "values differ (integer mode must be bit-exact)"
    else:
        err = np.abs(gv - R.val)
        tol = RTOL[dtype] * R.absmag
        bad = err > tol
        assert not bad.any(), f"{bad.sum()} values out of tolerance; worst rel {np.max(err / np.maximum(R.absmag, 1e-300))}"
