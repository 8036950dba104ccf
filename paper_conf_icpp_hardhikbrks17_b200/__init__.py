"""paper_conf_icpp_hardhikbrks17_b200 — B200-native sampled-threshold Gustavson SpGEMM.

A thin ctypes binding over the C ABI of ``libsg.so`` (declared in ``include/sg.h``). Every step of
the path runs in the library's sm_100a kernels; this module only marshals arguments. PyTorch is
used for device memory, streams and ``torch.distributed`` process groups. There is no CPU
fallback: importing works anywhere the library builds, but every call needs a CUDA device and the
compiled ``libsg.so``; without them it raises.

Entry points keep the C names (``sg_sample_threshold``, ``sg_partition``, ``sg_symbolic``,
``sg_numeric``, ``sg_gather``, ...) plus ``spgemm()``, the one-call user API:
Sample -> Identify -> Extrapolate picks the routing threshold, then the
two-phase Gustavson product (Alg. 2 l.5-6 L222-L223) runs on the device.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import torch

from . import _build

__all__ = [
    "DeviceCSR", "CostModel", "SampleReport", "PlanInfo", "SgError", "Plan", "lib", "load",
    "sg_row_work", "sg_sample_rows", "sg_sample_threshold", "sg_threshold_on_rows", "sg_exhaustive_threshold",
    "sg_cost_curve",
    "sg_partition", "sg_symbolic", "sg_numeric", "sg_gather", "sg_default_cost_model", "spgemm",
    "sg_gather_rows", "measured_threshold",
    "SG_CAP_L_MAX",
]

SG_CAP_L_MAX = 4096
_STATUS = ["SG_OK", "SG_ERR_INVALID_ARG", "SG_ERR_SHAPE", "SG_ERR_DTYPE", "SG_ERR_NOT_CANONICAL",
           "SG_ERR_EMPTY_SAMPLE", "SG_ERR_OOM", "SG_ERR_CUDA", "SG_ERR_NCCL", "SG_ERR_OVERFLOW"]

# every symbol include/sg.h declares (checked by tests/test_abi.py)
EXPORTS = ["sg_status_string", "sg_version", "sg_default_cost_model", "sg_row_work", "sg_partition_cost", "sg_default_partition_model", "sg_sample_threshold",
           "sg_exhaustive_threshold", "sg_cost_curve", "sg_partition", "sg_symbolic", "sg_numeric", "sg_gather",
           "sg_plan_get_info", "sg_plan_get_classes", "sg_plan_get_work", "sg_plan_destroy", "sg_sample_rows",
           "sg_profile_enable", "sg_launch_count", "sg_profile_count", "sg_profile_read", "sg_profile_reset",
           "sg_gather_layout", "sg_threshold_on_rows", "sg_set_option", "sg_get_option",
           "sg_sym_c_create", "sg_sym_c_buffers", "sg_sym_c_layout", "sg_sym_c_assemble", "sg_sym_c_destroy",
           "sg_copy_device", "sg_default_cost_model_for", "sg_hh_filter", "sg_hh_hstack", "sg_hh_identity2", "sg_hh_sample",
           "sg_gather_rows"]

SG_OPT_VALIDATE, SG_OPT_DENSE_LOG2, SG_OPT_VARIANT, SG_OPT_L2_PERSIST, SG_OPT_TP_MAX_BYTES = 0, 1, 2, 3, 4


class SgError(RuntimeError):
    def __init__(self, code: int, where: str):
        self.code = code
        name = _STATUS[code] if 0 <= code < len(_STATUS) else f"status {code}"
        super().__init__(f"{where}: {name}")


class CsrView(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("ncols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p), ("val", ctypes.c_void_p),
                ("dtype", ctypes.c_int)]


class CostModel(ctypes.Structure):
    """sg_cost_model (integer picoseconds)."""
    _fields_ = [(n, ctypes.c_int64) for n in (
        "kappa_L", "lambda_L", "sigma_L", "rho_L", "kappa_H", "lambda_H", "tau_H", "mu_H",
        "tiles_fixed", "capu", "cap_L")]

    def as_dict(self):
        return {n: int(getattr(self, n)) for n, _ in self._fields_}


class SampleReport(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in (
        "sample_rows", "sample_nonempty", "thr", "W_est_L", "W_est_H", "J_min", "U_est_L", "U_est_H")]

    def comp(self):
        """The sample's per-class compression (U_L, W_L, U_H, W_H) for sg_partition_cost."""
        return [int(self.U_est_L), int(self.W_est_L), int(self.U_est_H), int(self.W_est_H)]

    def as_dict(self):
        return {n: int(getattr(self, n)) for n, _ in self._fields_}


class PlanInfo(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in (
        "row_begin", "row_end", "thr", "n_empty", "n_light", "n_heavy", "nnz_c", "flops", "n_ranges")] + [
        ("light_bins", ctypes.c_int64 * 13), ("n_dense", ctypes.c_int64), ("dense_log2", ctypes.c_int64),
        ("n_light_sorted", ctypes.c_int64)]

    def as_dict(self):
        d = {n: int(getattr(self, n)) for n, _ in self._fields_ if n != "light_bins"}
        d["light_bins"] = [int(x) for x in self.light_bins]
        return d


_lib = None


def load(build_if_missing: bool = True):
    """Loads libsg.so (building it with nvcc if missing). Raises if it cannot."""
    global _lib
    if _lib is not None:
        return _lib
    so = os.environ.get("SG_LIB_PATH", _build.SO)  # A/B experiments may point at another build
    if not os.path.exists(so):
        if not build_if_missing:
            raise ImportError(f"{so} is missing; run __graft_entry__.build()")
        _build.build()
    L = ctypes.CDLL(so)
    P, i64, u64, st = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64, ctypes.c_int
    V = ctypes.POINTER(CsrView)
    CM = ctypes.POINTER(CostModel)
    pi64 = ctypes.POINTER(ctypes.c_int64)
    sigs = {
        "sg_status_string": (ctypes.c_char_p, [st]),
        "sg_version": (ctypes.c_char_p, []),
        "sg_default_cost_model": (None, [CM]),
        "sg_default_partition_model": (None, [CM]),
        "sg_row_work": (st, [V, V, i64, i64, P, pi64, P]),
        "sg_sample_rows": (st, [i64, i64, ctypes.c_double, u64, P, i64, pi64, P]),
        "sg_sample_threshold": (st, [V, V, ctypes.c_double, u64, CM, pi64, ctypes.POINTER(SampleReport), P]),
        "sg_threshold_on_rows": (st, [V, V, P, i64, CM, pi64, ctypes.POINTER(SampleReport), P]),
        "sg_exhaustive_threshold": (st, [V, V, CM, pi64, pi64, P]),
        "sg_cost_curve": (st, [V, V, CM, i64, P, P, P]),
        "sg_partition": (st, [V, V, ctypes.c_int, P, pi64, P]),
        "sg_partition_cost": (st, [V, V, ctypes.c_int, i64, CM, P, P, pi64, P]),
        "sg_symbolic": (st, [V, V, i64, i64, i64, P, pi64, ctypes.POINTER(ctypes.c_void_p), P]),
        "sg_numeric": (st, [P, V, V, P, P, P]),
        "sg_gather": (st, [P, P, ctypes.c_int, P, P, P, P, i64, P, P, i64, pi64, P]),
        "sg_set_option": (st, [ctypes.c_int, i64]),
        "sg_sym_c_create": (st, [P, i64, i64, ctypes.c_int, ctypes.POINTER(P)]),
        "sg_sym_c_buffers": (st, [P, ctypes.POINTER(P), ctypes.POINTER(P), ctypes.POINTER(P)]),
        "sg_sym_c_layout": (st, [P, P, pi64, pi64, P]),
        "sg_sym_c_assemble": (st, [P, P, P, P]),
        "sg_sym_c_destroy": (None, [P]),
        "sg_copy_device": (st, [P, P, i64, P]),
        "sg_default_cost_model_for": (None, [i64, ctypes.POINTER(CostModel)]),
        "sg_hh_filter": (st, [P, i64, ctypes.c_int, P, P, P, pi64, P]),
        "sg_hh_hstack": (st, [P, P, P, P, P, P]),
        "sg_hh_identity2": (st, [i64, ctypes.c_int, P, P, P, P]),
        "sg_hh_sample": (st, [P, ctypes.c_uint64, ctypes.c_double, P, P, P, P, P, pi64, pi64, P]),
        "sg_gather_rows": (st, [V, P, i64, P, P, P, i64, pi64, P]),
        "sg_get_option": (i64, [ctypes.c_int]),
        "sg_plan_get_info": (st, [P, ctypes.POINTER(PlanInfo)]),
        "sg_plan_get_classes": (st, [P, P, P]),
        "sg_plan_get_work": (st, [P, P, P]),
        "sg_plan_destroy": (None, [P]),
        "sg_profile_enable": (None, [ctypes.c_int]),
        "sg_launch_count": (i64, []),
        "sg_profile_count": (i64, []),
        "sg_profile_read": (i64, [P, P, i64]),
        "sg_profile_reset": (None, []),
        "sg_gather_layout": (st, [P, ctypes.c_int, P, P, pi64, pi64]),
    }
    for name, (res, args) in sigs.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def lib():
    return load()


def _check(code: int, where: str):
    if code != 0:
        raise SgError(code, where)


def _stream():
    return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)


def _ptr(t: torch.Tensor | None):
    return ctypes.c_void_p(t.data_ptr() if t is not None and t.numel() > 0 else 0)


def _require_cuda():
    if not torch.cuda.is_available():
        raise RuntimeError("paper_conf_icpp_hardhikbrks17_b200 needs a CUDA device (no CPU fallback)")


@dataclass
class DeviceCSR:
    """CSR resident in device memory (torch tensors): row_ptr int64, col int32, val f64|f32."""
    nrows: int
    ncols: int
    row_ptr: torch.Tensor
    col: torch.Tensor
    val: torch.Tensor

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    @property
    def dtype_code(self) -> int:
        return 1 if self.val.dtype == torch.float32 else 0

    def view(self) -> CsrView:
        return CsrView(self.nrows, self.ncols, self.nnz, _ptr(self.row_ptr), _ptr(self.col), _ptr(self.val),
                       self.dtype_code)

    @staticmethod
    def from_host(H, device="cuda", pin: bool = False, non_blocking: bool = False) -> "DeviceCSR":
        """From any object with nrows, ncols, row_ptr, col, val (numpy arrays)."""
        def t(x):
            x = torch.from_numpy(x)
            if pin:
                x = x.pin_memory()
            return x.to(device, non_blocking=non_blocking)
        return DeviceCSR(int(H.nrows), int(H.ncols), t(H.row_ptr), t(H.col), t(H.val))

    def to_host(self):
        return (self.row_ptr.cpu().numpy(), self.col.cpu().numpy(), self.val.cpu().numpy())


def sg_default_cost_model(p: int | None = None) -> CostModel:
    """The calibrated default model; with p (= B.ncols) the exact model calls with cm=None use."""
    cm = CostModel()
    if p is None:
        lib().sg_default_cost_model(ctypes.byref(cm))
    else:
        lib().sg_default_cost_model_for(int(p), ctypes.byref(cm))
    return cm


def sg_default_partition_model() -> CostModel:
    """The cost model sg_partition_cost uses when none is given (fitted to measured shard times)."""
    cm = CostModel()
    lib().sg_default_partition_model(ctypes.byref(cm))
    return cm


def _cmref(cm):
    return ctypes.byref(cm) if cm is not None else None


def sg_row_work(A: DeviceCSR, B: DeviceCSR, row_begin: int = 0, row_end: int | None = None,
                with_total: bool = False):
    _require_cuda()
    row_end = A.nrows if row_end is None else row_end
    w = torch.empty(max(row_end - row_begin, 0), dtype=torch.int64, device=A.row_ptr.device)
    tot = ctypes.c_int64(0)
    _check(lib().sg_row_work(ctypes.byref(A.view()), ctypes.byref(B.view()), row_begin, row_end, _ptr(w),
                             ctypes.byref(tot) if with_total else None, _stream()), "sg_row_work")
    return (w, int(tot.value)) if with_total else w


def sg_sample_rows(n: int, sample_frac: float, seed: int, row_begin: int = 0, row_end: int | None = None,
                   device="cuda") -> torch.Tensor:
    _require_cuda()
    row_end = n if row_end is None else row_end
    out = torch.empty(max(row_end - row_begin, 1), dtype=torch.int64, device=device)
    c = ctypes.c_int64(0)
    _check(lib().sg_sample_rows(row_begin, row_end, sample_frac, seed, _ptr(out), out.numel(), ctypes.byref(c),
                                _stream()), "sg_sample_rows")
    return out[: c.value]


def sg_gather_rows(A: DeviceCSR, rows: torch.Tensor) -> DeviceCSR:
    """A_S = the rows `rows` of A (all of A's columns), built on the device (sg_gather_rows)."""
    _require_cuda()
    rows = rows.to(device=A.row_ptr.device, dtype=torch.int64).contiguous()
    nr = rows.numel()
    rp = torch.empty(nr + 1, dtype=torch.int64, device=A.row_ptr.device)
    nz = ctypes.c_int64(0)
    cap = 0
    while True:
        col = torch.empty(max(cap, 1), dtype=torch.int32, device=A.row_ptr.device)
        val = torch.empty(max(cap, 1), dtype=A.val.dtype, device=A.row_ptr.device)
        code = lib().sg_gather_rows(ctypes.byref(A.view()), _ptr(rows), nr, _ptr(rp), _ptr(col), _ptr(val), cap,
                                    ctypes.byref(nz), _stream())
        if code == _STATUS.index("SG_ERR_SHAPE") and nz.value > cap:
            cap = int(nz.value)  # second call with the size the first one returned
            continue
        _check(code, "sg_gather_rows")
        break
    m = int(nz.value)
    return DeviceCSR(nr, A.ncols, rp, col[:m], val[:m])


def _threshold_grid(cap: int = SG_CAP_L_MAX) -> list[int]:
    ts, k = {0, cap}, 0
    while round(16 * 2 ** (k / 4)) <= cap:
        ts.add(int(round(16 * 2 ** (k / 4))))
        k += 1
    return sorted(ts)


def measured_threshold(A: DeviceCSR, B: DeviceCSR, sample_frac: float = 0.01, seed: int = 1, reps: int = 1,
                       grid: list[int] | None = None):
    """The paper's measured Identify ("identify the best threshold for the sample by running
    the algorithm"; L141): Sample the rows S (sg_sample_rows, R3/R4), build A_S = A[S, :] with B
    whole (sg_gather_rows), time sg_symbolic + sg_numeric of A_S B on the device at the candidate thresholds
    of a geometric grid — every 8th point first, then the 17 points around the fastest — and Extrapolate the
    fastest t unchanged (L236). The default Identify of sg_sample_threshold evaluates the calibrated cost
    model instead (deterministic, the parity-tested one). Returns (thr, {"T_ms": {t: ms}, "sample_rows": |S|})."""
    _require_cuda()
    S = sg_sample_rows(A.nrows, sample_frac, seed, device=A.row_ptr.device)
    if S.numel() == 0:
        raise SgError(_STATUS.index("SG_ERR_EMPTY_SAMPLE"), "measured_threshold")
    AS = sg_gather_rows(A, S)
    G = grid or _threshold_grid()
    timed: dict[int, float] = {}

    def T(t: int) -> float:
        if t not in timed:
            best = None
            for _ in range(max(1, reps)):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(torch.cuda.current_stream())
                plan = sg_symbolic(AS, B, t)
                col, val = sg_numeric(plan, AS, B)
                e1.record(torch.cuda.current_stream())
                torch.cuda.synchronize()
                plan.destroy()
                del col, val
                ms = e0.elapsed_time(e1)
                best = ms if best is None else min(best, ms)
            timed[t] = best
        return timed[t]

    thr = _coarse_fine(G, T)
    return thr, {"T_ms": dict(sorted(timed.items())), "sample_rows": int(S.numel())}


def _coarse_fine(G: list[int], T) -> int:
    """The measured Identify's search over the sorted grid G: every 8th point (and the last), then the 17
    points around the fastest of those; returns the fastest point evaluated (host logic, CPU-tested)."""
    coarse = G[::8] + ([G[-1]] if (len(G) - 1) % 8 else [])
    k = G.index(min(coarse, key=T))
    return min(G[max(0, k - 8): k + 9], key=T)


def sg_sample_threshold(A: DeviceCSR, B: DeviceCSR, sample_frac: float, seed: int, cm: CostModel | None = None):
    """Sample -> Identify -> Extrapolate. Returns (thr, SampleReport dict)."""
    _require_cuda()
    thr = ctypes.c_int64(0)
    rep = SampleReport()
    _check(lib().sg_sample_threshold(ctypes.byref(A.view()), ctypes.byref(B.view()), sample_frac, seed, _cmref(cm),
                                     ctypes.byref(thr), ctypes.byref(rep), _stream()), "sg_sample_threshold")
    return int(thr.value), rep.as_dict()


def sg_threshold_on_rows(A: DeviceCSR, B: DeviceCSR, rows, cm: CostModel | None = None):
    """Identify on an explicit row sample (device or host int64 row ids). Returns (thr, SampleReport dict)."""
    _require_cuda()
    r = torch.as_tensor(rows, dtype=torch.int64, device=A.row_ptr.device).contiguous()
    thr = ctypes.c_int64(0)
    rep = SampleReport()
    _check(lib().sg_threshold_on_rows(ctypes.byref(A.view()), ctypes.byref(B.view()), ctypes.c_void_p(r.data_ptr()),
                                      r.numel(), _cmref(cm), ctypes.byref(thr), ctypes.byref(rep), _stream()),
           "sg_threshold_on_rows")
    return int(thr.value), rep.as_dict()


def sg_exhaustive_threshold(A: DeviceCSR, B: DeviceCSR, cm: CostModel | None = None):
    _require_cuda()
    thr, J = ctypes.c_int64(0), ctypes.c_int64(0)
    _check(lib().sg_exhaustive_threshold(ctypes.byref(A.view()), ctypes.byref(B.view()), _cmref(cm),
                                         ctypes.byref(thr), ctypes.byref(J), _stream()), "sg_exhaustive_threshold")
    return int(thr.value), int(J.value)


def sg_cost_curve(A: DeviceCSR, B: DeviceCSR, ts, cm: CostModel | None = None) -> list[int]:
    import numpy as np
    _require_cuda()
    t = np.ascontiguousarray(ts, dtype=np.int64)
    J = np.zeros(t.shape[0], dtype=np.int64)
    _check(lib().sg_cost_curve(ctypes.byref(A.view()), ctypes.byref(B.view()), _cmref(cm), t.shape[0],
                               t.ctypes.data_as(ctypes.c_void_p), J.ctypes.data_as(ctypes.c_void_p), _stream()),
           "sg_cost_curve")
    return [int(x) for x in J]


def sg_partition(A: DeviceCSR, B: DeviceCSR, nparts: int):
    """Returns (cuts list of nparts+1, W)."""
    import numpy as np
    _require_cuda()
    cuts = np.zeros(nparts + 1, dtype=np.int64)
    W = ctypes.c_int64(0)
    _check(lib().sg_partition(ctypes.byref(A.view()), ctypes.byref(B.view()), nparts,
                              cuts.ctypes.data_as(ctypes.c_void_p), ctypes.byref(W), _stream()), "sg_partition")
    return [int(x) for x in cuts], int(W.value)


def sg_partition_cost(A: DeviceCSR, B: DeviceCSR, nparts: int, thr: int, comp, cm=None):
    """Cost-weighted cuts (NEXT #2, R19): returns (cuts list of nparts+1, total modeled cost
    in ps). comp = (U_L, W_L, U_H, W_H), e.g. SampleReport.comp() of the sg_sample_threshold call."""
    import numpy as np
    _require_cuda()
    cuts = np.zeros(nparts + 1, dtype=np.int64)
    cc = np.ascontiguousarray(comp, dtype=np.int64)
    tot = ctypes.c_int64(0)
    _check(lib().sg_partition_cost(ctypes.byref(A.view()), ctypes.byref(B.view()), nparts, int(thr), _cmref(cm),
                                   cc.ctypes.data_as(ctypes.c_void_p), cuts.ctypes.data_as(ctypes.c_void_p),
                                   ctypes.byref(tot), _stream()), "sg_partition_cost")
    return [int(x) for x in cuts], int(tot.value)


class Plan:
    """Owns an sg_plan* and the C.row_ptr it was built with."""

    def __init__(self, handle: ctypes.c_void_p, row_ptr: torch.Tensor, nnz: int, dtype: torch.dtype,
                 row_begin: int, row_end: int):
        self.handle = handle
        self.row_ptr = row_ptr
        self.nnz = nnz
        self.dtype = dtype
        self.row_begin, self.row_end = row_begin, row_end

    def info(self) -> dict:
        pi = PlanInfo()
        _check(lib().sg_plan_get_info(self.handle, ctypes.byref(pi)), "sg_plan_get_info")
        return pi.as_dict()

    def classes(self) -> torch.Tensor:
        out = torch.empty(self.row_end - self.row_begin, dtype=torch.int8, device=self.row_ptr.device)
        _check(lib().sg_plan_get_classes(self.handle, _ptr(out), _stream()), "sg_plan_get_classes")
        return out

    def work(self) -> torch.Tensor:
        out = torch.empty(self.row_end - self.row_begin, dtype=torch.int64, device=self.row_ptr.device)
        _check(lib().sg_plan_get_work(self.handle, _ptr(out), _stream()), "sg_plan_get_work")
        return out

    def destroy(self):
        if self.handle:
            lib().sg_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


def sg_symbolic(A: DeviceCSR, B: DeviceCSR, thr: int, row_begin: int = 0, row_end: int | None = None) -> Plan:
    _require_cuda()
    row_end = A.nrows if row_end is None else row_end
    rp = torch.empty(row_end - row_begin + 1, dtype=torch.int64, device=A.row_ptr.device)
    nnz = ctypes.c_int64(0)
    h = ctypes.c_void_p(0)
    _check(lib().sg_symbolic(ctypes.byref(A.view()), ctypes.byref(B.view()), thr, row_begin, row_end, _ptr(rp),
                             ctypes.byref(nnz), ctypes.byref(h), _stream()), "sg_symbolic")
    return Plan(h, rp, int(nnz.value), A.val.dtype, row_begin, row_end)


def sg_numeric(plan: Plan, A: DeviceCSR, B: DeviceCSR, out=None):
    """Returns (C_col int32[nnz], C_val[nnz]); `out` may pass preallocated (col, val)."""
    _require_cuda()
    if out is None:
        col = torch.empty(plan.nnz, dtype=torch.int32, device=A.row_ptr.device)
        val = torch.empty(plan.nnz, dtype=plan.dtype, device=A.row_ptr.device)
    else:
        col, val = out
    _check(lib().sg_numeric(plan.handle, ctypes.byref(A.view()), ctypes.byref(B.view()), _ptr(col), _ptr(val),
                            _stream()), "sg_numeric")
    return col, val


def sg_gather(plan: Plan, comm_ptr: int, n_global: int, local_col=None, local_val=None, gather_values: bool = False,
              nnz_global: int | None = None):
    """Assembles the row-distributed C over NCCL (comm_ptr: ncclComm_t as int, e.g.
    ProcessGroupNCCL._comm_ptr()). n_global = rows of the global C (A.nrows); with gather_values,
    nnz_global = total nnz of C (e.g. the sum of every rank's plan.nnz). The library checks both
    against the gathered layout on every rank (SgError(SHAPE) everywhere if too small).
    Returns (row_ptr_global, col_global|None, val_global|None, nnz_total)."""
    _require_cuda()
    dev = plan.row_ptr.device
    rp = torch.empty(n_global + 1, dtype=torch.int64, device=dev)
    col = val = None
    cap = 0
    if gather_values:
        if nnz_global is None:
            raise ValueError("gather_values needs nnz_global (the total nnz of C over all ranks)")
        col = torch.empty(nnz_global, dtype=torch.int32, device=dev)
        val = torch.empty(nnz_global, dtype=plan.dtype, device=dev)
        cap = nnz_global
    tot = ctypes.c_int64(0)
    _check(lib().sg_gather(plan.handle, ctypes.c_void_p(comm_ptr), int(gather_values), _ptr(plan.row_ptr),
                           _ptr(local_col), _ptr(local_val), _ptr(rp), n_global + 1, _ptr(col), _ptr(val), cap,
                           ctypes.byref(tot), _stream()), "sg_gather")
    return rp, col, val, int(tot.value)


class profile:
    """Context manager: per-launch CUDA-event timing of every libsg kernel launched inside.
    After exit (the stream synchronised), .records is a list of (kernel_name, ms)."""

    def __init__(self):
        self.records = []

    def __enter__(self):
        lib().sg_profile_reset()
        lib().sg_profile_enable(1)
        self.launches0 = int(lib().sg_launch_count())
        return self

    def __exit__(self, *exc):
        torch.cuda.synchronize()
        L = lib()
        L.sg_profile_enable(0)
        n = int(L.sg_profile_count())
        names = ctypes.create_string_buffer(32 * max(n, 1))
        import numpy as np
        ms = np.zeros(max(n, 1), dtype=np.float64)
        n = int(L.sg_profile_read(names, ms.ctypes.data_as(ctypes.c_void_p), n))
        raw = names.raw
        self.records = [(raw[32 * i:32 * i + 32].split(b"\0")[0].decode(), float(ms[i])) for i in range(n)]
        self.launches = int(L.sg_launch_count()) - self.launches0
        L.sg_profile_reset()
        return False

    def by_kernel(self):
        out = {}
        for name, t in self.records:
            c, s = out.get(name, (0, 0.0))
            out[name] = (c + 1, s + t)
        return out


def launch_count() -> int:
    return int(lib().sg_launch_count())


class SymC:
    """C assembled in NCCL symmetric windows (NEXT #3; include/sg.h sg_sym_c_*). Collective over the
    communicator: every rank creates it with the same (n_rows, nnz_cap, dtype)."""

    def __init__(self, comm_ptr: int, n_rows: int, nnz_cap: int, dtype=torch.float64):
        _require_cuda()
        self.n, self.cap, self.dtype = int(n_rows), int(nnz_cap), dtype
        h = ctypes.c_void_p()
        _check(lib().sg_sym_c_create(ctypes.c_void_p(comm_ptr), self.n, self.cap,
                                     0 if dtype == torch.float64 else 1, ctypes.byref(h)), "sg_sym_c_create")
        self.handle = h
        rp, col, val = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_void_p()
        _check(lib().sg_sym_c_buffers(h, ctypes.byref(rp), ctypes.byref(col), ctypes.byref(val)), "sg_sym_c_buffers")
        self._ptrs = (rp.value, col.value, val.value)
        self.offset = None
        self.total = None

    def layout(self, plan: "Plan"):
        off, tot = ctypes.c_int64(0), ctypes.c_int64(0)
        _check(lib().sg_sym_c_layout(self.handle, plan.handle, ctypes.byref(off), ctypes.byref(tot), _stream()),
               "sg_sym_c_layout")
        self.offset, self.total = int(off.value), int(tot.value)
        return self.offset, self.total

    def numeric_into(self, plan: "Plan", A: "DeviceCSR", B: "DeviceCSR"):
        """sg_numeric writing this rank's rows straight into its window at the layout offset."""
        vs = 8 if self.dtype == torch.float64 else 4
        _check(lib().sg_numeric(plan.handle, ctypes.byref(A.view()), ctypes.byref(B.view()),
                                ctypes.c_void_p(self._ptrs[1] + 4 * self.offset),
                                ctypes.c_void_p(self._ptrs[2] + vs * self.offset), _stream()), "sg_numeric")

    def assemble(self, plan: "Plan"):
        _check(lib().sg_sym_c_assemble(self.handle, plan.handle, _ptr(plan.row_ptr), _stream()), "sg_sym_c_assemble")

    def tensors(self):
        """(row_ptr, col, val) of the assembled C as host-owned copies (the windows stay with the SymC)."""
        import numpy as np
        L = lib()
        out = []
        for ptr, n, dt in ((self._ptrs[0], self.n + 1, torch.int64), (self._ptrs[1], self.total, torch.int32),
                           (self._ptrs[2], self.total, self.dtype)):
            t = torch.empty(n, dtype=dt, device="cuda")
            nbytes = n * t.element_size()
            if nbytes:
                _check(L.sg_copy_device(ctypes.c_void_p(t.data_ptr()), ctypes.c_void_p(ptr), nbytes, _stream()),
                       "sg_copy_device")
            out.append(t)
        return tuple(out)

    def destroy(self):
        if self.handle:
            lib().sg_sym_c_destroy(self.handle)
            self.handle = None


# ---- NEXT #4: the HH-CPU four-block variant (PAPER Alg. 3, Section V-A) ----------

def sg_hh_filter(M: DeviceCSR, t: int, high: bool) -> DeviceCSR:
    """Phase I: the rows of M whose class is `high` (more than t non-zeros); others emptied."""
    _require_cuda()
    dev = M.row_ptr.device
    rp = torch.empty(M.nrows + 1, dtype=torch.int64, device=dev)
    col = torch.empty(max(M.nnz, 1), dtype=torch.int32, device=dev)
    val = torch.empty(max(M.nnz, 1), dtype=M.val.dtype, device=dev)
    nz = ctypes.c_int64(0)
    _check(lib().sg_hh_filter(ctypes.byref(M.view()), int(t), int(bool(high)), _ptr(rp), _ptr(col), _ptr(val),
                              ctypes.byref(nz), _stream()), "sg_hh_filter")
    return DeviceCSR(M.nrows, M.ncols, rp, col[: nz.value], val[: nz.value])


def sg_hh_add(P: DeviceCSR, Q: DeviceCSR, thr: int | None = None) -> DeviceCSR:
    """Phase IV: P + Q (same shape) as the product [P Q] * [I; I] on the hot path (equal columns added,
    union sorted, structural zeros kept)."""
    _require_cuda()
    dev = P.row_ptr.device
    n = P.nrows
    rp = torch.empty(n + 1, dtype=torch.int64, device=dev)
    col = torch.empty(max(P.nnz + Q.nnz, 1), dtype=torch.int32, device=dev)
    val = torch.empty(max(P.nnz + Q.nnz, 1), dtype=P.val.dtype, device=dev)
    _check(lib().sg_hh_hstack(ctypes.byref(P.view()), ctypes.byref(Q.view()), _ptr(rp), _ptr(col), _ptr(val), _stream()),
           "sg_hh_hstack")
    PQ = DeviceCSR(n, P.ncols + Q.ncols, rp, col[: P.nnz + Q.nnz], val[: P.nnz + Q.nnz])
    p = P.ncols
    irp = torch.empty(2 * p + 1, dtype=torch.int64, device=dev)
    icol = torch.empty(max(2 * p, 1), dtype=torch.int32, device=dev)
    ival = torch.empty(max(2 * p, 1), dtype=P.val.dtype, device=dev)
    _check(lib().sg_hh_identity2(p, 0 if P.val.dtype == torch.float64 else 1, _ptr(irp), _ptr(icol), _ptr(ival),
                                 _stream()), "sg_hh_identity2")
    I2 = DeviceCSR(2 * p, p, irp, icol[: 2 * p], ival[: 2 * p])
    C, _ = spgemm(PQ, I2, thr=thr if thr is not None else SG_CAP_L_MAX)
    return C


def spgemm_hh(A: DeviceCSR, B: DeviceCSR, t: int, sample_frac: float = 0.01, seed: int = 1):
    """HH-CPU (Alg. 3) at density threshold t: Phase I splits A and B into high / low dense rows, Phases
    II-III compute A_X B_Y for X, Y in {H, L} on the hot path, Phase IV adds them. Returns (C, info)."""
    AH, AL = sg_hh_filter(A, t, True), sg_hh_filter(A, t, False)
    BH, BL = (AH, AL) if B is A else (sg_hh_filter(B, t, True), sg_hh_filter(B, t, False))
    info = {"t": int(t), "blocks": {}}
    sums = []
    for xa, AX in (("H", AH), ("L", AL)):
        parts = []
        for yb, BY in (("H", BH), ("L", BL)):
            Cxy, inf = spgemm(AX, BY, sample_frac, seed) if AX.nnz and BY.nnz else (None, None)
            if Cxy is None:
                Cxy = DeviceCSR(A.nrows, B.ncols, torch.zeros(A.nrows + 1, dtype=torch.int64, device=A.row_ptr.device),
                                torch.empty(0, dtype=torch.int32, device=A.row_ptr.device),
                                torch.empty(0, dtype=A.val.dtype, device=A.row_ptr.device))
            info["blocks"][xa + yb] = Cxy.nnz
            parts.append(Cxy)
        sums.append(sg_hh_add(parts[0], parts[1]))
    return sg_hh_add(sums[0], sums[1]), info


def sg_hh_sample(A: DeviceCSR, seed: int, f: float | None = None):
    """Phase I Sample (L285-L287, reading R20): the principal sub-matrix A[S, S], |S| ~ f n (f = 1/sqrt(n)
    by default). Returns (rows S, A' as DeviceCSR, positions of A' entries in A)."""
    _require_cuda()
    import math
    n = A.nrows
    f = 1.0 / max(1.0, math.sqrt(n)) if f is None else f
    dev = A.row_ptr.device
    rows = torch.empty(max(n, 1), dtype=torch.int64, device=dev)
    rp = torch.empty(n + 1, dtype=torch.int64, device=dev)
    col = torch.empty(max(A.nnz, 1), dtype=torch.int32, device=dev)
    pos = torch.empty(max(A.nnz, 1), dtype=torch.int64, device=dev)
    val = torch.empty(max(A.nnz, 1), dtype=A.val.dtype, device=dev)
    sn, nz = ctypes.c_int64(0), ctypes.c_int64(0)
    _check(lib().sg_hh_sample(ctypes.byref(A.view()), seed, f, _ptr(rows), _ptr(rp), _ptr(col), _ptr(pos), _ptr(val),
                              ctypes.byref(sn), ctypes.byref(nz), _stream()), "sg_hh_sample")
    s_, m = int(sn.value), int(nz.value)
    return rows[:s_], DeviceCSR(s_, s_, rp[: s_ + 1], col[:m], val[:m]), pos[:m]


def hh_threshold(A: DeviceCSR, seed: int = 1, f: float | None = None, reps: int = 3):
    """Sample -> Identify -> Extrapolate for HH-CPU (Section V-A): A' = sg_hh_sample(A); Identify = a descent
    over thresholds t' on the measured time of spgemm_hh(A', A', t') (the paper's "gradient descent based
    approach", L289: doubling steps from the median row density while the time drops, then one refining
    step of sqrt(2) each way); Extrapolate t_A = t_s^2 (L291). Returns (t_A, info)."""
    import math
    _, As, _ = sg_hh_sample(A, seed, f)
    dens = torch.diff(As.row_ptr).float()
    cache = {}

    def T(t):
        t = int(max(0, t))
        if t not in cache:
            ms = []
            for _ in range(reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                spgemm_hh(As, As, t, sample_frac=0.05, seed=seed)
                e1.record()
                torch.cuda.synchronize()
                ms.append(e0.elapsed_time(e1))
            cache[t] = sorted(ms)[len(ms) // 2]
        return cache[t]

    t = max(1, int(dens[dens > 0].median().item()) if bool((dens > 0).any()) else 1)
    best = t
    for step in (2.0, 0.5):  # walk up, then down, while the time keeps dropping
        cur = best
        while True:
            nxt = int(round(cur * step))
            if nxt == cur or nxt < 0 or nxt > 1 << 20 or T(nxt) >= T(cur):
                break
            cur = nxt
        if T(cur) < T(best):
            best = cur
    for nxt in (int(round(best * math.sqrt(2))), int(round(best / math.sqrt(2)))):
        if T(nxt) < T(best):
            best = nxt
    return best * best, {"t_s": best, "sample_rows": As.nrows, "sample_nnz": As.nnz,
                         "curve": {str(k): v for k, v in sorted(cache.items())}}


def set_option(key: int, value: int) -> None:
    """sg_set_option: process-wide library options (SG_OPT_VALIDATE 0/1, SG_OPT_DENSE_LOG2 -1 or 0..62)."""
    _check(lib().sg_set_option(int(key), int(value)), "sg_set_option")


def get_option(key: int) -> int:
    return int(lib().sg_get_option(int(key)))


def sg_gather_layout(layouts):
    """Host-only assembly arithmetic of sg_gather: layouts = [(row_begin, row_end, nnz)] in rank
    order -> (begin[nranks], off[nranks+1], n, total). Raises SgError(SHAPE) if not contiguous."""
    import numpy as np
    lay = np.ascontiguousarray(np.asarray(layouts, dtype=np.int64).reshape(-1))
    G = lay.shape[0] // 3
    begin = np.zeros(G, dtype=np.int64)
    off = np.zeros(G + 1, dtype=np.int64)
    n, tot = ctypes.c_int64(0), ctypes.c_int64(0)
    _check(lib().sg_gather_layout(lay.ctypes.data_as(ctypes.c_void_p), G, begin.ctypes.data_as(ctypes.c_void_p),
                                  off.ctypes.data_as(ctypes.c_void_p), ctypes.byref(n), ctypes.byref(tot)),
           "sg_gather_layout")
    return begin, off, int(n.value), int(tot.value)


def spgemm(A: DeviceCSR, B: DeviceCSR, sample_frac: float = 0.01, seed: int = 1, cm: CostModel | None = None,
           thr: int | None = None):
    """The one-call API: sampled threshold (unless thr is given), symbolic, numeric.
    Returns (C as DeviceCSR, info dict)."""
    rep = None
    if thr is None:
        try:
            thr, rep = sg_sample_threshold(A, B, sample_frac, seed, cm)
        except SgError as e:
            if e.code != 5:  # SG_ERR_EMPTY_SAMPLE: a small or very sparse input; Identify over every row
                raise
            try:
                thr, rep = sg_sample_threshold(A, B, 1.0, seed, cm)
            except SgError as e2:
                if e2.code != 5:
                    raise
                thr = 0  # no row has any product: every row is EMPTY, the threshold is moot
    plan = sg_symbolic(A, B, thr)
    col, val = sg_numeric(plan, A, B)
    C = DeviceCSR(A.nrows, B.ncols, plan.row_ptr, col, val)
    info = {"thr": thr, "sample": rep, "nnz": plan.nnz}
    plan.destroy()
    return C, info


def spgemm_to_host(A: DeviceCSR, B: DeviceCSR, sink, blocks: int = 8, sample_frac: float = 0.01, seed: int = 1,
                   cm: CostModel | None = None, thr: int | None = None, inflight: int = 3):
    """Row-blocked SpGEMM whose result streams to the host while the next block computes.

    Rows are cut into `blocks` work-balanced blocks (sg_partition, Alg. 2's split); block g+1's
    symbolic + numeric run on the current stream while block g's C crosses PCIe on a copy stream, so
    the D2H of the result overlaps the compute. For each block, sink(g, row_begin, row_end, row_ptr,
    col, val) is called with the copy stream as the current stream: it enqueues its device->host copies
    (non_blocking) there; row_ptr is the block's LOCAL prefix (add the returned offset of the block).
    At most `inflight` blocks' C stay on the device (the host waits for older copies first).
    Returns info with the per-block C offsets."""
    _require_cuda()
    comp = torch.cuda.current_stream()
    copy = torch.cuda.Stream(device=A.row_ptr.device)
    rep = None
    if thr is None:
        thr, rep = sg_sample_threshold(A, B, sample_frac, seed, cm)
    cuts, W = sg_partition(A, B, blocks)
    done, offs = [], [0]
    for g in range(blocks):
        if g >= inflight:
            done[g - inflight].synchronize()  # bounds the device memory held by in-flight blocks
        r0, r1 = cuts[g], cuts[g + 1]
        plan = sg_symbolic(A, B, thr, r0, r1)
        col, val = sg_numeric(plan, A, B)
        rp = plan.row_ptr
        ready = torch.cuda.Event()
        ready.record(comp)
        copy.wait_event(ready)
        with torch.cuda.stream(copy):
            sink(g, r0, r1, rp, col, val)
            ev = torch.cuda.Event()
            ev.record(copy)
        for t in (rp, col, val):
            t.record_stream(copy)  # the caching allocator keeps them until the copy stream is past them
        done.append(ev)
        offs.append(offs[-1] + plan.nnz)
        plan.destroy()
        del rp, col, val
    comp.wait_stream(copy)
    return {"thr": thr, "sample": rep, "nnz": offs[-1], "cuts": cuts, "offsets": offs, "W": W}

