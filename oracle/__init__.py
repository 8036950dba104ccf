"""oracle — TEST INFRASTRUCTURE ONLY (not part of the product path).

Plain CPU implementation of the hot path of Mallipeddi et al., ICPP 2017
(/root/reference/PAPER.md, cited "PAPER Lnnn"), used to prove the CUDA path right. Only
``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import it. The product package never imports it and shares no code
with it; the only shared module is ``sginputs`` (seeded input generators, no method arithmetic).

Functions and the passage each follows (details in oracle.cpp's header):

* ``row_work``            O2  w_i = sum_{k in A_i} nnz(B_k)
* ``spgemm`` / ``counts`` O1  Gustavson, sorted-map accumulator
* ``moments``             O1  per-row structure digest (u, sum c^1..3) PAPER L74, L222-L223
* ``sample_rows``         sampler, Bernoulli(f) by SplitMix64       PAPER L92 (uniform sampling)
* ``J`` / ``threshold``   O4  Identify: best candidate on the sample PAPER L87-L89, L232-L236
* ``sampled_threshold``   Sample -> Identify -> Extrapolate(identity)
* ``partition``           O3  closest-prefix cuts
* ``heavy_share``         O6  split percentage r(t)
* ``gap_report``          O6  sampled-vs-exhaustive gaps

Every function is pinned by ``tests/test_oracle_*.py`` against closed forms, brute force,
scipy, invariants and the hand-computed worked example in ``tests/golden/``; see DESIGN.md §5.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.cpp")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fopenmp", "-fPIC", "-shared", "-o", _SO, src])
    return _SO


class CostModel(ctypes.Structure):
    """Per-row path costs in integer picoseconds:
    c_L = kappa_L + lambda_L*w + sigma_L*u*ceil(log2 max(u,2)) + rho_L*u
    c_H = kappa_H + lambda_H*w + tau_H*a*R(u) + mu_H*u,  R(u) = tiles_fixed if capu == 0 else max(1, tiles_fixed, ceil(u/capu))
    """
    _fields_ = [(n, ctypes.c_int64) for n in (
        "kappa_L", "lambda_L", "sigma_L", "rho_L",
        "kappa_H", "lambda_H", "tau_H", "mu_H",
        "tiles_fixed", "capu", "cap_L")]

    def as_dict(self):
        return {n: int(getattr(self, n)) for n, _ in self._fields_}


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        i64, u64 = ctypes.c_int64, ctypes.c_uint64
        lib.oracle_threads.restype = ctypes.c_int
        lib.oracle_hash.restype = u64
        lib.oracle_hash.argtypes = [u64, u64, u64]
        lib.oracle_tag_sample.restype = u64
        lib.oracle_row_work.argtypes = [i64, P, P, P, P]
        lib.oracle_spgemm_count.argtypes = [P, P, P, P, i64, P, P]
        lib.oracle_spgemm_moments.argtypes = [P, P, P, P, i64, P, P]
        lib.oracle_hh_block_count.argtypes = [P, P, P, P, i64, ctypes.c_int, ctypes.c_int, i64, P, P]
        lib.oracle_hh_block_fill.argtypes = [P, P, P, ctypes.c_int, P, P, P, ctypes.c_int, i64, ctypes.c_int,
                                             ctypes.c_int, i64, P, P, P, P]
        lib.oracle_hh_sample.restype = i64
        lib.oracle_hh_sample.argtypes = [i64, P, P, u64, ctypes.c_double, P, P, P, P]
        lib.oracle_hh_extrapolate.restype = i64
        lib.oracle_hh_extrapolate.argtypes = [i64]
        lib.oracle_spgemm_fill.argtypes = [P, P, P, ctypes.c_int, P, P, P, ctypes.c_int, i64, P, P, P, P, P]
        lib.oracle_sample_rows.restype = i64
        lib.oracle_sample_rows.argtypes = [i64, i64, u64, ctypes.c_double, P]
        CMP = ctypes.POINTER(CostModel)
        lib.oracle_cost_L.restype = i64
        lib.oracle_cost_L.argtypes = [CMP, i64, i64, i64]
        lib.oracle_cost_H.restype = i64
        lib.oracle_cost_H.argtypes = [CMP, i64, i64, i64]
        lib.oracle_J.argtypes = [CMP, i64, P, P, P, i64, ctypes.POINTER(i64), ctypes.POINTER(u64)]
        lib.oracle_threshold.restype = i64
        lib.oracle_threshold.argtypes = [CMP, i64, P, P, P, ctypes.POINTER(i64), ctypes.POINTER(u64)]
        lib.oracle_partition.argtypes = [i64, P, ctypes.c_int, P]
        lib.oracle_row_cost.restype = i64
        lib.oracle_row_cost.argtypes = [CMP, i64, P, i64, i64]
        lib.oracle_partition_cost.argtypes = [CMP, i64, P, i64, P, P, ctypes.c_int, P, ctypes.POINTER(i64)]
        lib.oracle_heavy_share.restype = ctypes.c_double
        lib.oracle_heavy_share.argtypes = [i64, P, i64]
        _lib = lib
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def threads() -> int:
    return int(_L().oracle_threads())


def hash3(seed: int, tag: int, j: int) -> int:
    return int(_L().oracle_hash(seed, tag, j))




def tag_sample() -> int:
    return int(_L().oracle_tag_sample())


# ---- O2 -------------------------------------------------------------------------------------

def row_work(A, B) -> np.ndarray:
    w = np.empty(A.nrows, dtype=np.int64)
    _L().oracle_row_work(A.nrows, _p(A.row_ptr), _p(A.col), _p(B.row_ptr), _p(w))
    return w


# ---- O1 -------------------------------------------------------------------------------------

def counts(A, B, rows=None) -> np.ndarray:
    rows = np.arange(A.nrows, dtype=np.int64) if rows is None else np.ascontiguousarray(rows, dtype=np.int64)
    u = np.empty(rows.shape[0], dtype=np.int64)
    if rows.shape[0]:
        _L().oracle_spgemm_count(_p(A.row_ptr), _p(A.col), _p(B.row_ptr), _p(B.col), rows.shape[0], _p(rows), _p(u))
    return u


@dataclass
class RowsResult:
    """C restricted to a row list: row s occupies [row_ptr[s], row_ptr[s+1]) of col/val."""
    rows: np.ndarray
    row_ptr: np.ndarray
    col: np.ndarray
    val: np.ndarray
    absmag: np.ndarray | None = None
    ncols: int = 0

    @property
    def nnz(self):
        return int(self.row_ptr[-1])


def moments(A, B, rows=None) -> np.ndarray:
    """Per listed row (u_i, sum c, sum c^2, sum c^3) over the columns of C_i, sums mod 2^64 (uint64[n, 4])."""
    rows = np.arange(A.nrows, dtype=np.int64) if rows is None else np.ascontiguousarray(rows, dtype=np.int64)
    out = np.zeros((rows.shape[0], 4), dtype=np.uint64)
    if rows.shape[0]:
        _L().oracle_spgemm_moments(_p(A.row_ptr), _p(A.col), _p(B.row_ptr), _p(B.col), rows.shape[0], _p(rows), _p(out))
    return out


def spgemm(A, B, rows=None, with_absmag: bool = False) -> RowsResult:
    """C = A*B (fp64 values) for the listed rows (all rows by default)."""
    assert A.ncols == B.nrows
    rows = np.arange(A.nrows, dtype=np.int64) if rows is None else np.ascontiguousarray(rows, dtype=np.int64)
    u = counts(A, B, rows)
    rp = np.zeros(rows.shape[0] + 1, dtype=np.int64)
    np.cumsum(u, out=rp[1:])
    nnz = int(rp[-1])
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=np.float64)
    mag = np.empty(nnz, dtype=np.float64) if with_absmag else None
    if rows.shape[0]:
        _L().oracle_spgemm_fill(_p(A.row_ptr), _p(A.col), _p(A.val), int(A.val.dtype == np.float32),
                                _p(B.row_ptr), _p(B.col), _p(B.val), int(B.val.dtype == np.float32),
                                rows.shape[0], _p(rows), _p(rp), _p(col), _p(val),
                                _p(mag) if mag is not None else None)
    return RowsResult(rows, rp, col, val, mag, B.ncols)


# ---- sampler --------------------------------------------------------------------------------

def sample_rows(n: int, seed: int, f: float, row_begin: int = 0, row_end: int | None = None) -> np.ndarray:
    row_end = n if row_end is None else row_end
    out = np.empty(max(row_end - row_begin, 0), dtype=np.int64)
    c = _L().oracle_sample_rows(row_begin, row_end, seed, f, _p(out))
    return out[:c].copy()


# ---- O4 -------------------------------------------------------------------------------------

def cost_L(cm: CostModel, w: int, a: int, u: int) -> int:
    return int(_L().oracle_cost_L(ctypes.byref(cm), w, a, u))


def cost_H(cm: CostModel, w: int, a: int, u: int) -> int:
    return int(_L().oracle_cost_H(ctypes.byref(cm), w, a, u))


def _i128(hi, lo) -> int:
    return (int(hi) << 64) + int(lo)


def J(cm: CostModel, w, a, u, t: int) -> int:
    w, a, u = (np.ascontiguousarray(x, dtype=np.int64) for x in (w, a, u))
    hi, lo = ctypes.c_int64(), ctypes.c_uint64()
    _L().oracle_J(ctypes.byref(cm), w.shape[0], _p(w), _p(a), _p(u), t, ctypes.byref(hi), ctypes.byref(lo))
    return _i128(hi.value, lo.value)


def threshold(cm: CostModel, w, a, u) -> tuple[int, int]:
    """(thr, Jmin) over the given rows' (w, a, u)."""
    w, a, u = (np.ascontiguousarray(x, dtype=np.int64) for x in (w, a, u))
    hi, lo = ctypes.c_int64(), ctypes.c_uint64()
    t = _L().oracle_threshold(ctypes.byref(cm), w.shape[0], _p(w), _p(a), _p(u), ctypes.byref(hi), ctypes.byref(lo))
    return int(t), _i128(hi.value, lo.value)


@dataclass
class SampleResult:
    thr: int
    rows: np.ndarray
    w: np.ndarray
    a: np.ndarray
    u: np.ndarray
    Jmin: int
    nonempty: int = 0
    W_est_L: int = 0
    W_est_H: int = 0


def sampled_threshold(A, B, f: float, seed: int, cm: CostModel, w_all=None) -> SampleResult:
    """Sample (Bernoulli(f) rows, B intact) -> Identify (argmin J on the sample) ->
    Extrapolate (identity, r = r')."""
    w_all = row_work(A, B) if w_all is None else w_all
    S = sample_rows(A.nrows, seed, f)
    w = w_all[S]
    a = np.diff(A.row_ptr)[S]
    u = counts(A, B, S)
    thr, Jmin = threshold(cm, w, a, u)
    nz = int((w > 0).sum())
    return SampleResult(thr, S, w, a, u, Jmin, nz, int(w[(w > 0) & (w <= thr)].sum()), int(w[w > thr].sum()))


def exhaustive_threshold(A, B, cm: CostModel, w_all=None, u_all=None) -> tuple[int, int]:
    """thr* over every row: needs u for every row, i.e. the full symbolic."""
    w_all = row_work(A, B) if w_all is None else w_all
    u_all = counts(A, B) if u_all is None else u_all
    return threshold(cm, w_all, np.diff(A.row_ptr), u_all)


# ---- HH four-block variant (NEXT #4; Alg. 3) ----------------------------------

def hh_block(A, B, t: int, xa: int, yb: int, rows=None) -> RowsResult:
    """Block A_X B_Y of the HH-CPU decomposition (X = xa, Y = yb; 1 = high: more than t non-zeros)."""
    rows = np.arange(A.nrows, dtype=np.int64) if rows is None else np.ascontiguousarray(rows, dtype=np.int64)
    L = _L()
    u = np.zeros(rows.shape[0], dtype=np.int64)
    if rows.shape[0]:
        L.oracle_hh_block_count(_p(A.row_ptr), _p(A.col), _p(B.row_ptr), _p(B.col), t, xa, yb, rows.shape[0], _p(rows), _p(u))
    rp = np.zeros(rows.shape[0] + 1, dtype=np.int64)
    np.cumsum(u, out=rp[1:])
    col = np.empty(int(rp[-1]), dtype=np.int32)
    val = np.empty(int(rp[-1]), dtype=np.float64)
    if rows.shape[0]:
        L.oracle_hh_block_fill(_p(A.row_ptr), _p(A.col), _p(A.val), int(A.val.dtype == np.float32), _p(B.row_ptr),
                               _p(B.col), _p(B.val), int(B.val.dtype == np.float32), t, xa, yb, rows.shape[0],
                               _p(rows), _p(rp), _p(col), _p(val))
    return RowsResult(rows, rp, col, val, None, B.ncols)


def hh_combine(blocks) -> RowsResult:
    """Phase IV: the four blocks added row by row (same row list in every block)."""
    rows = blocks[0].rows
    out_rp = [0]
    cols, vals = [], []
    for s in range(len(rows)):
        acc = {}
        for R in blocks:
            for c, v in zip(R.col[R.row_ptr[s]:R.row_ptr[s + 1]], R.val[R.row_ptr[s]:R.row_ptr[s + 1]]):
                acc[int(c)] = acc.get(int(c), 0.0) + float(v)
        ks = sorted(acc)
        cols.extend(ks)
        vals.extend(acc[k] for k in ks)
        out_rp.append(len(cols))
    return RowsResult(rows, np.array(out_rp, dtype=np.int64), np.array(cols, dtype=np.int32),
                      np.array(vals, dtype=np.float64), None, blocks[0].ncols)


def hh_sample(A, seed: int, f: float | None = None):
    """Phase I Sample (L285-L287): returns (kept row ids, A' as (row_ptr, col, source positions)); f
    defaults to 1/sqrt(n)."""
    n = A.nrows
    f = 1.0 / max(1.0, np.sqrt(n)) if f is None else f
    rows = np.empty(max(n, 1), dtype=np.int64)
    rp = np.empty(max(n, 1) + 1, dtype=np.int64)
    col = np.empty(max(A.nnz, 1), dtype=np.int32)
    pos = np.empty(max(A.nnz, 1), dtype=np.int64)
    s = int(_L().oracle_hh_sample(n, _p(A.row_ptr), _p(A.col), seed, f, _p(rows), _p(rp), _p(col), _p(pos)))
    m = int(rp[s])
    return rows[:s].copy(), rp[:s + 1].copy(), col[:m].copy(), pos[:m].copy()


def hh_extrapolate(t_s: int) -> int:
    return int(_L().oracle_hh_extrapolate(int(t_s)))


# ---- O3 -------------------------------------------------------------------------------------

def partition(w, G: int) -> np.ndarray:
    w = np.ascontiguousarray(w, dtype=np.int64)
    cuts = np.empty(G + 1, dtype=np.int64)
    _L().oracle_partition(w.shape[0], _p(w), G, _p(cuts))
    return cuts


def sample_comp(res: "SampleResult") -> np.ndarray:
    """(U_L, W_L, U_H, W_H): sums of u and w over the sampled rows of each class at res.thr."""
    w, u = res.w, res.u
    L = (w > 0) & (w <= res.thr)
    H = w > res.thr
    return np.array([int(u[L].sum()), int(w[L].sum()), int(u[H].sum()), int(w[H].sum())], dtype=np.int64)


def row_cost(cm: CostModel, thr: int, comp, w: int, a: int) -> int:
    comp = np.ascontiguousarray(comp, dtype=np.int64)
    return int(_L().oracle_row_cost(ctypes.byref(cm), thr, _p(comp), w, a))


def partition_cost(cm: CostModel, thr: int, comp, w, a, G: int) -> tuple[np.ndarray, int]:
    """Cost-weighted cuts (NEXT #2, R19) and the total modeled cost."""
    w, a = (np.ascontiguousarray(x, dtype=np.int64) for x in (w, a))
    comp = np.ascontiguousarray(comp, dtype=np.int64)
    cuts = np.empty(G + 1, dtype=np.int64)
    tot = ctypes.c_int64()
    _L().oracle_partition_cost(ctypes.byref(cm), thr, _p(comp), w.shape[0], _p(w), _p(a), G, _p(cuts), ctypes.byref(tot))
    return cuts, int(tot.value)


# ---- O6 -------------------------------------------------------------------------------------

def heavy_share(w, t: int) -> float:
    w = np.ascontiguousarray(w, dtype=np.int64)
    return float(_L().oracle_heavy_share(w.shape[0], _p(w), t))


def gap_report(w_all, a_all, u_all, cm: CostModel, thr_s: int, thr_star: int | None = None) -> dict:
    """Sampled-vs-exhaustive gaps (reading R2): primary dr = |r(thr_s) - r(thr*)| in
    percentage points of work share; also delta_rel = |thr_s - thr*| / max(thr*, 1) and
    dJ = J(thr_s)/J(thr*) - 1 on the full matrix."""
    if thr_star is None:
        thr_star, _ = threshold(cm, w_all, a_all, u_all)
    Js = J(cm, w_all, a_all, u_all, thr_s)
    Jb = J(cm, w_all, a_all, u_all, thr_star)
    rs, rb = heavy_share(w_all, thr_s), heavy_share(w_all, thr_star)
    return {
        "thr_s": int(thr_s), "thr_star": int(thr_star),
        "r_s": rs, "r_star": rb, "dr_pp": abs(rs - rb),
        "delta_rel": abs(thr_s - thr_star) / max(thr_star, 1),
        "dJ": (Js / Jb - 1.0) if Jb else 0.0,
    }
