"""Seeded synthetic inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This package holds none of the method's arithmetic (no row work, no products, no thresholds):
it only builds canonical CSR matrices — sorted, unique column indices per row — whose
structure and values are pure functions of (parameters, seed). See DESIGN.md §3 for the
recipe and SURVEY.md §8(c) Q4/Q10–Q13 for the readings it implements.

The heavy lifting (hashing tens of millions of edges, sort + dedupe) lives in ``gen.c``,
compiled in-tree to ``libsginputs.so`` by ``build()`` (or lazily on first use).
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libsginputs.so")
_lib = None

VAL_REAL, VAL_INT, VAL_ONES, VAL_SIGNED, VAL_ZEROS = 0, 1, 2, 3, 4
# real U[0.5,1.5); int {1,2,3,4}; ones; signed {-2,-1,1,2} (exact cancellation); zeros {-1,0,1,2} (stored zeros)
_MODES = {"real": VAL_REAL, "int": VAL_INT, "ones": VAL_ONES, "signed": VAL_SIGNED, "zeros": VAL_ZEROS}


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-fPIC", "-shared", "-o", _SO, src])
    return _SO


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        i64, u64, i32 = ctypes.c_int64, ctypes.c_uint64, ctypes.c_int
        lib.sginputs_hash.restype = u64
        lib.sginputs_hash.argtypes = [u64, u64, u64]
        lib.sginputs_er_edges.argtypes = [i64, i64, i64, u64, P, P]
        lib.sginputs_rmat_edges.argtypes = [i32, i64, u64, u64, u64, u64, i32, P, P]
        lib.sginputs_rmat_perm.argtypes = [i64, u64, P]
        lib.sginputs_csr_from_edges.restype = i64
        lib.sginputs_csr_from_edges.argtypes = [i64, i64, P, P, P, P]
        lib.sginputs_values.argtypes = [i64, i64, P, P, u64, i32, i32, P]
        _lib = lib
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


@dataclass
class CSR:
    """Canonical CSR on the host: row_ptr int64[n+1], col int32[nnz] sorted/unique per row,
    val float64 or float32[nnz]."""
    nrows: int
    ncols: int
    row_ptr: np.ndarray
    col: np.ndarray
    val: np.ndarray
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    @property
    def dtype(self) -> str:
        return "f32" if self.val.dtype == np.float32 else "f64"

    def astype(self, dtype: str) -> "CSR":
        npd = np.float32 if dtype == "f32" else np.float64
        return CSR(self.nrows, self.ncols, self.row_ptr, self.col, self.val.astype(npd), self.name)

    def to_dense(self) -> np.ndarray:
        d = np.zeros((self.nrows, self.ncols), dtype=np.float64)
        rows = np.repeat(np.arange(self.nrows), np.diff(self.row_ptr))
        d[rows, self.col] = self.val
        return d

    def to_scipy(self):
        import scipy.sparse as sp
        return sp.csr_matrix((self.val.astype(np.float64), self.col, self.row_ptr),
                             shape=(self.nrows, self.ncols))


def hash3(seed: int, tag: int, j: int) -> int:
    return int(_L().sginputs_hash(seed, tag, j))


def _csr_from_edges(n, p, ei, ej, seed, mode, dtype, name):
    lib = _L()
    m = ei.shape[0]
    rp = np.empty(n + 1, dtype=np.int64)
    col = np.empty(max(m, 1), dtype=np.int32)
    nnz = lib.sginputs_csr_from_edges(n, m, _p(ei), _p(ej), _p(rp), _p(col))
    col = col[:nnz].copy()
    return _with_values(CSR(n, p, rp, col, np.empty(0), name), seed, mode, dtype)


def _with_values(A: CSR, seed: int, mode: str, dtype: str) -> CSR:
    is32 = dtype == "f32"
    val = np.empty(A.nnz, dtype=np.float32 if is32 else np.float64)
    if A.nnz:
        _L().sginputs_values(A.nrows, A.ncols, _p(A.row_ptr), _p(A.col), seed, _MODES[mode], int(is32), _p(val))
    A.val = val
    return A


def er(n: int, d: float, seed: int = 1, p: int | None = None, mode: str = "real", dtype: str = "f64") -> CSR:
    """ER G(n, m) with m = round(d*n) uniform (i, j) pairs, deduped."""
    p = n if p is None else p
    m = int(round(d * n))
    ei = np.empty(m, dtype=np.int32)
    ej = np.empty(m, dtype=np.int32)
    _L().sginputs_er_edges(n, p, m, seed, _p(ei), _p(ej))
    return _csr_from_edges(n, p, ei, ej, seed, mode, dtype, f"er_n{n}_d{d}_s{seed}")


def _fx64(x: float) -> int:
    """2^64 fixed point of a probability (host-side, once)."""
    return min(int(math.ldexp(x, 64)), (1 << 64) - 1)


def rmat(scale: int, ef: int = 16, a: float = 0.57, b: float = 0.19, c: float = 0.19, seed: int = 1,
         permute: bool = True, mode: str = "real", dtype: str = "f64") -> CSR:
    """R-MAT(scale, ef; a, b, c), d = 1-a-b-c, permuted labels, directed, self-loops kept."""
    n = 1 << scale
    m = ef * n
    ei = np.empty(m, dtype=np.int32)
    ej = np.empty(m, dtype=np.int32)
    _L().sginputs_rmat_edges(scale, m, _fx64(a), _fx64(a + b), _fx64(a + b + c), seed, int(permute), _p(ei), _p(ej))
    return _csr_from_edges(n, n, ei, ej, seed, mode, dtype, f"rmat{scale}_ef{ef}_s{seed}{'' if permute else '_unperm'}")


def rmat_perm(scale: int, seed: int) -> np.ndarray:
    n = 1 << scale
    perm = np.empty(n, dtype=np.int32)
    _L().sginputs_rmat_perm(n, seed, _p(perm))
    return perm


# ---- special matrices (closed-form pins) -------------------------------------------------

def identity(n: int, dtype: str = "f64") -> CSR:
    return CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32),
               np.ones(n, dtype=np.float32 if dtype == "f32" else np.float64), f"I{n}")


def permutation(n: int, seed: int = 1, dtype: str = "f64") -> CSR:
    """P with P[i, pi(i)] = 1, pi the seeded label permutation (rank of hash)."""
    keys = np.array([hash3(seed, 0x5045524d55544531, v) for v in range(n)], dtype=np.uint64)
    pi = np.empty(n, dtype=np.int32)
    pi[np.argsort(keys, kind="stable")] = np.arange(n, dtype=np.int32)
    return CSR(n, n, np.arange(n + 1, dtype=np.int64), pi,
               np.ones(n, dtype=np.float32 if dtype == "f32" else np.float64), f"P{n}_s{seed}")


def diagonal(n: int, diag: np.ndarray, dtype: str = "f64") -> CSR:
    return CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32),
               np.asarray(diag, dtype=np.float32 if dtype == "f32" else np.float64), f"D{n}")


def banded(n: int, offsets: list[int], coeffs: list[float], dtype: str = "f64") -> CSR:
    """Toeplitz band: A[i, i+o] = coeff for each (o, coeff), columns in range."""
    order = np.argsort(offsets)
    offs = [offsets[k] for k in order]
    cf = [coeffs[k] for k in order]
    rp = [0]
    cols, vals = [], []
    for i in range(n):
        for o, c in zip(offs, cf):
            j = i + o
            if 0 <= j < n:
                cols.append(j)
                vals.append(c)
        rp.append(len(cols))
    return CSR(n, n, np.array(rp, dtype=np.int64), np.array(cols, dtype=np.int32),
               np.array(vals, dtype=np.float32 if dtype == "f32" else np.float64), f"band{n}")


def tridiag(n: int, alpha: float, beta: float, gamma: float, dtype: str = "f64") -> CSR:
    """T = tridiag(alpha (sub), beta (diag), gamma (super))."""
    return banded(n, [-1, 0, 1], [alpha, beta, gamma], dtype)


def empty_rows(n: int, p: int, dtype: str = "f64") -> CSR:
    return CSR(n, p, np.zeros(n + 1, dtype=np.int64), np.zeros(0, dtype=np.int32),
               np.zeros(0, dtype=np.float32 if dtype == "f32" else np.float64), f"Z{n}x{p}")


def random_pattern(n: int, p: int, density: float, seed: int, mode: str = "real", dtype: str = "f64") -> CSR:
    """Small ER-like pattern with an expected density (for brute-force pins)."""
    m = int(round(density * n * p))
    ei = np.empty(m, dtype=np.int32)
    ej = np.empty(m, dtype=np.int32)
    if m:
        _L().sginputs_er_edges(n, p, m, seed, _p(ei), _p(ej))
    return _csr_from_edges(n, p, ei, ej, seed, mode, dtype, f"rand{n}x{p}_s{seed}")


# ---- BASELINE.json configs ---------------------------------------------------------------

CONFIGS = {
    # name: (builder, description) — BASELINE.json "configs" in order
    "C1": "uniform-random sparse 1000x1000, ~8 nnz/row, fp64, C=A*A",
    "C2": "Erdos-Renyi 2^18 rows, 16 nnz/row, C=A*A, fp64",
    "C3": "R-MAT scale 20, edge factor 16 (a=0.57,b=c=0.19), C=A*A",
    "C4": "R-MAT scale 22, 8xB200 sharded",
    "R18": "R-MAT scale 18 (threshold sweep, config 5)",
    "R18u": "R-MAT scale 18, un-permuted labels (config 5 ablation)",
}


def config(name: str, seed: int = 1, mode: str = "real", dtype: str = "f64") -> CSR:
    if name == "C1":
        return er(1000, 8, seed, mode=mode, dtype=dtype)
    if name == "C2":
        return er(1 << 18, 16, seed, mode=mode, dtype=dtype)
    if name == "C3":
        return rmat(20, 16, seed=seed, mode=mode, dtype=dtype)
    if name == "C4":
        return rmat(22, 16, seed=seed, mode=mode, dtype=dtype)
    if name == "R18":
        return rmat(18, 16, seed=seed, mode=mode, dtype=dtype)
    if name == "R18u":  # config 5's un-permuted variant (hubs at low ids; the Fig. 7 randomness ablation)
        return rmat(18, 16, seed=seed, permute=False, mode=mode, dtype=dtype)
    if name.startswith("rmat"):
        return rmat(int(name[4:]), 16, seed=seed, mode=mode, dtype=dtype)
    raise KeyError(name)
