#!/usr/bin/env python
"""bench.py — SpGEMM GFLOP/s of the sampled-threshold Gustavson path on 1..8 B200.

One STEP is one pass of the whole hot path over the workload:
  sg_sample_threshold (Sample -> Identify -> Extrapolate)
  sg_partition        (work-prefix row cuts, Alg. 2 l.1-4 L215-L218)
  sg_symbolic         (row work, binning, exact u_i, C.row_ptr)
  sg_numeric          (light + heavy accumulators, sorted CSR out)
  sg_gather           (N > 1: global row_ptr assembly over NCCL, Alg. 2 l.7 L224)
value = 2 * W_total / time (W = sum_i w_i multiply-adds, BASELINE metric), time = device time of
K steps between barriers + synchronisation, max over ranks (CUDA events).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl sglib|reference]

Under torchrun (N > 1) every rank computes identical cuts and thresholds from the same inputs and
seed (no runtime communication for partitioning) and runs its row block; the only
collective is the row_ptr assembly.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
os.environ.setdefault("PYTORCH_CUDA_ALLOC_CONF", "expandable_segments:True")

METRIC = "SpGEMM GFLOP/s at 1/2/4/8 B200; sampled-vs-best threshold gap (%)"
WORKLOADS = {
    "C1": "uniform-random 1000x1000 ~8 nnz/row, C=A*A, fp64",
    "C2": "Erdos-Renyi 2^18 rows, 16 nnz/row, C=A*A, fp64",
    "C3": "R-MAT scale 20, edge factor 16 (a=0.57,b=c=0.19), permuted, C=A*A, fp64",
    "R18": "R-MAT scale 18, edge factor 16, permuted, C=A*A, fp64",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="sglib", choices=["sglib", "reference"])
    ap.add_argument("--config", default="C3")
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--split", default="cost", choices=["cost", "flops"],
                    help="N > 1: cost-weighted split (sg_partition_cost, DESIGN.md §7.7) or Alg. 2's flops split")
    ap.add_argument("--sample-frac", type=float, default=0.01)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-blocks", type=int, default=8, help="row blocks of the e2e path (D2H overlaps compute)")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-gap", action="store_true")
    ap.add_argument("--cpu-budget-s", type=float, default=15.0)
    ap.add_argument("--profile-out", default="")
    ap.add_argument("--no-profile", action="store_true",
                    help="time the K steps without per-launch CUDA events (launch-bound small configs); the kernel "
                         "shares and the roofline then come from a separate profiled pass of the same K steps")
    return ap.parse_args()


# ------------------------------------------------------------------------------------------------
# clocks during the timed region (nvidia-smi every 200 ms)
# ------------------------------------------------------------------------------------------------
class Clocks:
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "--query-gpu=" + self.Q, "--format=csv,noheader,nounits",
                                       "-lms", "200"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None
        time.sleep(0.25)

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = []
        with open(self.f.name) as fh:
            for line in fh:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) < 9 or not parts[0].isdigit() or int(parts[0]) != self.idx:
                    continue
                rows.append(parts)
        os.unlink(self.f.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = sorted(float(r[1]) for r in rows if r[1].replace(".", "").isdigit())
        mx = max(float(r[2]) for r in rows if r[2].replace(".", "").isdigit())
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in rows for k in range(4) if r[5 + k].lower() == "active"})
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(rows), "power_w_max": max(float(r[3]) for r in rows if r[3].replace(".", "").isdigit())}


# ------------------------------------------------------------------------------------------------
# helpers
# ------------------------------------------------------------------------------------------------
def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def smem_peaks():
    """Measured shared-memory atomic throughputs (Gop/s, whole GPU) from tools/microbench on a B200."""
    f = os.path.join(ROOT, "profiles", "r01_microbench_accumulator_primitives.txt")
    out = {}
    try:
        for line in open(f):
            parts = line.split()
            if len(parts) >= 5 and parts[4] == "Gop/s":
                out[parts[0]] = float(parts[3])
    except OSError:
        return None
    return out


def csr_bytes(nrows, nnz, vbytes):
    return 8 * (nrows + 1) + (4 + vbytes) * nnz


def cpu_baseline(H, budget_s: float, seed: int):
    """The oracle (plain std::map Gustavson) as it stands, on a bounded Bernoulli row sample of
    the same workload, on the host cores."""
    import numpy as np
    import oracle
    w = oracle.row_work(H, H)
    W = int(w.sum())
    # size the sample for ~budget_s of CPU work from a short probe
    f = 0.001
    rows = oracle.sample_rows(H.nrows, seed + 7919, f)
    t0 = time.perf_counter()
    oracle.spgemm(H, H, rows=rows)
    tp = max(time.perf_counter() - t0, 1e-3)
    f = min(1.0, f * max(1.0, budget_s / tp))
    rows = oracle.sample_rows(H.nrows, seed + 7919, f)
    Ws = int(w[rows].sum())
    t0 = time.perf_counter()
    R = oracle.spgemm(H, H, rows=rows)
    t = time.perf_counter() - t0
    return {"value": 2.0 * Ws / t / 1e9, "unit": "GFLOP/s", "cores": oracle.threads(), "kind": "oracle",
            "sample": f"Bernoulli({f:.4f}) row sample (seed {seed + 7919}) of the same matrix: {len(rows)} rows, "
                      f"{Ws} of {W} multiply-adds, {R.nnz} C entries; std::map Gustavson, OpenMP dynamic",
            "seconds": t}


def reference_arm(args, rank, world):
    """--impl reference: the oracle timed on host cores on this arm's config/metric (rank 0 only)."""
    if rank != 0:
        return
    import sginputs as gen
    import oracle
    H = gen.config(args.config, seed=args.seed, dtype=args.dtype)
    w = oracle.row_work(H, H)
    W = int(w.sum())
    steps, warm = args.steps, args.warmup
    # each step: the oracle on a bounded Bernoulli row sample (all steps together ~ a few minutes)
    per_step_budget = max(2.0, min(20.0, 120.0 / max(steps + warm, 1)))
    f = 0.001
    rows = oracle.sample_rows(H.nrows, args.seed, f)
    t0 = time.perf_counter()
    oracle.spgemm(H, H, rows=rows)
    tp = max(time.perf_counter() - t0, 1e-3)
    f = min(1.0, f * max(1.0, per_step_budget / tp))
    times, works = [], []
    for s in range(warm + steps):
        rows = oracle.sample_rows(H.nrows, args.seed + 1 + s, f)
        t0 = time.perf_counter()
        oracle.spgemm(H, H, rows=rows)
        t = time.perf_counter() - t0
        if s >= warm:
            times.append(t)
            works.append(int(w[rows].sum()))
    T = sum(times)
    value = 2.0 * sum(works) / T / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world,
        "steps": steps, "warmup": warm, "ms_per_step": 1e3 * T / steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
        "config": {"workload": WORKLOADS.get(args.config, args.config), "config_id": args.config, "W": W},
        "cpu_baseline": {"value": value, "unit": "GFLOP/s", "cores": oracle.threads(), "kind": "oracle",
                         "sample": f"each step a Bernoulli({f:.4f}) row sample of the workload ({W} multiply-adds "
                                   f"in full); value = 2*sum(sampled w)/sum(step times)"},
        "e2e": {"value": value, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------------------------
# the GPU arm
# ------------------------------------------------------------------------------------------------
def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        reference_arm(args, rank, world)
        return

    import numpy as np
    import torch
    import torch.distributed as dist
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    comm = None
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
        dist.barrier()
        comm = dist.group.WORLD._get_backend(dev)._comm_ptr()
    sg.load(build_if_missing=False)

    H = gen.config(args.config, seed=args.seed, dtype=args.dtype)
    A = sg.DeviceCSR.from_host(H, device=dev)
    vbytes = 8 if args.dtype == "f64" else 4
    stream = torch.cuda.current_stream()

    W_all = sg.sg_partition(A, A, 1)[1]  # the workload's W (a constant of the matrix)
    cbuf = {}  # C buffers reused across steps (same nnz every step; allocation kept out of the loop)

    def step(Ad, with_values=False):
        thr, rep = sg.sg_sample_threshold(Ad, Ad, args.sample_frac, args.seed)
        if world > 1 and args.split == "cost":
            comp = [rep["U_est_L"], rep["W_est_L"], rep["U_est_H"], rep["W_est_H"]]
            cuts, _cost = sg.sg_partition_cost(Ad, Ad, world, thr, comp)
            W = W_all
        else:
            cuts, W = sg.sg_partition(Ad, Ad, world)
        plan = sg.sg_symbolic(Ad, Ad, thr, cuts[rank], cuts[rank + 1])
        if cbuf.get("nnz") != plan.nnz:
            cbuf.clear()
            torch.cuda.empty_cache()
            cbuf["nnz"] = plan.nnz
            cbuf["col"] = torch.empty(plan.nnz, dtype=torch.int32, device=dev)
            cbuf["val"] = torch.empty(plan.nnz, dtype=plan.dtype, device=dev)
        col, val = sg.sg_numeric(plan, Ad, Ad, out=(cbuf["col"], cbuf["val"]))
        gathered = None
        if world > 1:
            gathered = sg.sg_gather(plan, comm, n_global=Ad.nrows)
        return thr, rep, cuts, W, plan, col, val, gathered

    # warm-up (also the run whose outputs describe the workload)
    for _ in range(max(args.warmup, 1)):
        col = val = None
        thr, rep, cuts, W, plan, col, val, _g = step(A)
        info = plan.info()
        cls = plan.classes()
        wrow = plan.work()
        rp_local = plan.row_ptr
        plan.destroy()
        del col, val
    torch.cuda.synchronize()
    nnz_local = int(rp_local[-1].item())
    u = (rp_local[1:] - rp_local[:-1])
    nnzC_heavy = int(u[cls == 2].sum().item())
    nnzC_light = nnz_local - nnzC_heavy
    a_rows = (A.row_ptr[1:] - A.row_ptr[:-1])[cuts[rank]:cuts[rank + 1]]
    nnzA_heavy = int(a_rows[cls == 2].sum().item())
    nnzA_light = int(a_rows[cls == 1].sum().item())
    nheavy = int((cls == 2).sum().item())
    # heavy rows split between the dense-window kernel (w >= 2^dense_log2) and the rank kernel
    dmask = (cls == 2) & (wrow >= (1 << min(int(info["dense_log2"]), 62)))
    ndense = int(dmask.sum().item())
    nnzC_dense = int(u[dmask].sum().item())
    nnzA_dense = int(a_rows[dmask].sum().item())
    W_heavy = int(wrow[cls == 2].sum().item())
    W_dense = int(wrow[dmask].sum().item())
    # rank rows (heavy, below the dense cut): <= 64 k entries on the warp-tile kernel (k_num_tile), the rest
    # on the CTA rank kernel (k_num_heavy); SG_OPT_VARIANT bit 3 puts them all on k_num_heavy
    tmask = (cls == 2) & ~dmask & (a_rows <= 64)
    if sg.get_option(sg.SG_OPT_VARIANT) & 8:
        tmask = torch.zeros_like(tmask)
    ntile = int(tmask.sum().item())
    nnzC_tile = int(u[tmask].sum().item())
    nnzA_tile = int(a_rows[tmask].sum().item())
    W_tile = int(wrow[tmask].sum().item())
    del cls, u, a_rows, wrow, dmask, tmask
    nnzC_total = nnz_local
    if world > 1:
        t = torch.tensor([nnz_local], device=dev, dtype=torch.int64)
        dist.all_reduce(t)
        nnzC_total = int(t.item())

    # ---- timed region: K steps, device time, max over ranks ----
    cvd = [x for x in os.environ.get("CUDA_VISIBLE_DEVICES", "").split(",") if x.strip()]
    clocks = Clocks(int(cvd[local]) if len(cvd) > local and cvd[local].strip().isdigit() else local)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    l0 = sg.launch_count()

    def timed_steps():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        out = None
        for _ in range(args.steps):
            out = step(A)
            out[4].destroy()
            out = out[:4]
        e1.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        return e0, e1, out

    if args.no_profile:
        e0, e1, (thr, rep, cuts, W) = timed_steps()
        launches = sg.launch_count() - l0
        with sg.profile() as prof:  # kernel shares / roofline from a second, profiled pass
            timed_steps()
    else:
        with sg.profile() as prof:
            e0, e1, (thr, rep, cuts, W) = timed_steps()
        launches = sg.launch_count() - l0
    ck = clocks.stop()
    ms = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([ms], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_per_step = ms / args.steps
    value = 2.0 * W / (ms_per_step / 1e3) / 1e9   # whole-job: every rank's rows together = W

    # ---- roofline of the dominant kernel (algorithmic bytes per launch / mean launch time) ----
    bk = prof.by_kernel()
    hbm, peak_kind = peaks()
    Bbytes = csr_bytes(H.nrows, H.nnz, vbytes)
    alg = {
        # compulsory bytes of one launch: its A rows, B once, its C entries
        "k_num_heavy": 12 * (nnzA_heavy - nnzA_dense - nnzA_tile) + 8 * (nheavy - ndense - ntile) + Bbytes
                       + (4 + vbytes) * (nnzC_heavy - nnzC_dense - nnzC_tile),
        "k_num_tile": 12 * nnzA_tile + 8 * ntile + Bbytes + (4 + vbytes) * nnzC_tile,
        "k_num_dense": 12 * nnzA_dense + 8 * ndense + Bbytes + (4 + vbytes) * nnzC_dense,
        "k_sym_heavy": 4 * nnzA_heavy + 8 * nheavy + 8 * (H.nrows + 1) + 4 * H.nnz,
    }
    dom = max(bk.items(), key=lambda kv: kv[1][1])[0] if bk else None
    roof = None
    share = {k: v[1] / max(ms, 1e-9) for k, v in bk.items()}
    if dom in alg:
        cnt, tot = bk[dom]
        per_launch_ms = tot / cnt
        achieved = alg[dom] / (per_launch_ms / 1e3) / 1e9
        traffic = None
        tf = os.path.join(ROOT, "profiles", "ncu_traffic.json")
        if os.path.exists(tf):
            try:
                traffic = json.load(open(tf)).get(f"{args.config}:{args.dtype}:{dom}")
            except Exception:
                traffic = None
        roof = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": hbm, "unit": "GB/s",
                "frac": achieved / hbm, "traffic": traffic, "peak_kind": peak_kind,
                "alg_bytes_per_launch": alg[dom], "launch_ms": per_launch_ms, "launches": cnt}
    # ---- the on-chip bound of the heavy kernels: every product ends in one shared-memory atomic (fp64 CAS add
    # in the numeric kernels, a 32-bit OR in the symbolic / rank pass 1); peak = our microbenchmark of that
    # atomic at random addresses on this B200 (profiles/r01_microbench_accumulator_primitives.txt) ----
    roof_smem = None
    mb = smem_peaks()
    if mb and bk:
        ops = {"k_num_dense": (W_dense, "smem_cas_f64_16K"), "k_num_heavy": (W_heavy - W_dense - W_tile, "smem_cas_f64_16K"),
               "k_num_tile": (W_tile, "smem_cas_f64_16K"),
               "k_sym_heavy": (W_heavy, "smem_or32_16K")}
        roof_smem = {}
        for k, (nprod, prim) in ops.items():
            if k in bk and prim in mb:
                cnt, tot = bk[k]
                # per STEP (a kernel may launch several times a step: the symbolic runs as a 1024-thread
                # part for the rows with w >= 2^20 and a small-CTA part, plus the sampler's pass)
                rate = nprod / (tot / args.steps / 1e3) / 1e9
                roof_smem[k] = {"bound": "smem_atomic", "achieved": rate, "peak": mb[prim], "unit": "Gop/s",
                                "frac": rate / mb[prim], "op": prim, "ops_per_step": nprod, "launches_per_step": cnt / args.steps}
    step_alg_bytes = 2 * csr_bytes(H.nrows, H.nnz, vbytes) + csr_bytes(H.nrows, nnzC_total, vbytes)
    compulsory = {"bytes_per_step": step_alg_bytes,
                  "GBps": step_alg_bytes / (ms_per_step / 1e3) / 1e9,
                  "frac_of_hbm": step_alg_bytes / (ms_per_step / 1e3) / 1e9 / hbm}

    # ---- e2e: host CSR in (pinned), C out to pinned host buffers, through the public API ----
    e2e = None
    cbuf.clear()
    torch.cuda.empty_cache()
    if not args.no_e2e and rank == 0 and world == 1:
        e2e = run_e2e(args, sg, H, nnzC_total, vbytes, dev, torch)

    # ---- threshold gap (sampled vs exhaustive, model mode; outside the timed region) ----
    gap = None
    if not args.no_gap and rank == 0:
        ts, Jts = sg.sg_exhaustive_threshold(A, A)
        Jc = sg.sg_cost_curve(A, A, [thr, ts])
        w = sg.sg_row_work(A, A).to(torch.float64)
        Wf = float(w.sum().item())
        r = lambda t: 100.0 * float(w[w > t].sum().item()) / Wf
        gap = {"thr_s": thr, "thr_star": ts, "sample_frac": args.sample_frac, "dr_pp": abs(r(thr) - r(ts)),
               "delta_rel": abs(thr - ts) / max(ts, 1), "dJ": Jc[0] / Jc[1] - 1.0 if Jc[1] else 0.0,
               "r_s": r(thr), "r_star": r(ts)}

    cpu = None
    if not args.no_cpu and rank == 0 and world == 1:
        cpu = cpu_baseline(H, args.cpu_budget_s, args.seed)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": WORKLOADS.get(args.config, args.config), "config_id": args.config,
                       "n": H.nrows, "nnz_A": H.nnz, "W": W, "nnz_C": nnzC_total, "sample_frac": args.sample_frac,
                       "thr": thr, "seed": args.seed, "parallelism": f"rows{world}", "split": args.split if world > 1 else "none",
                       "l2": "inputs larger than L2 (A=B %.0f MB > 126 MB; C %.1f GB written per step)"
                             % (Bbytes / 1e6, csr_bytes(H.nrows, nnzC_total, vbytes) / 1e9)},
            "roofline": roof, "roofline_smem": roof_smem, "compulsory": compulsory, "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": launches, "clocks": ck, "threshold_gap": gap,
            "kernel_share": {k: round(v, 4) for k, v in sorted(share.items(), key=lambda kv: -kv[1])},
            "plan": {k: info[k] for k in ("n_empty", "n_light", "n_heavy", "n_ranges", "n_dense", "dense_log2")},
        }
        print(json.dumps(line), flush=True)
        if args.profile_out:
            with open(args.profile_out, "w") as f:
                json.dump({"by_kernel": bk, "ms": ms, "steps": args.steps}, f, indent=1)
    if world > 1:
        dist.destroy_process_group()


def run_e2e(args, sg, H, nnzC, vbytes, dev, torch):
    """End to end through the public API: pinned host CSR -> H2D -> spgemm() (sample, symbolic,
    numeric) -> D2H of all of C. When C does not fit the host RAM next to everything else (C3:
    116 GB of a 196 GB host), every byte of C still crosses PCIe each step, streamed through a
    fixed pinned ring (the host keeps the last chunk only); the JSON says which."""
    import psutil
    vt = torch.float64 if vbytes == 8 else torch.float32
    need = nnzC * (4 + vbytes) + 8 * (H.nrows + 1)
    avail = psutil.virtual_memory().available
    keep_all = need * 2 + 32e9 < avail
    hrp = torch.from_numpy(H.row_ptr).pin_memory()
    hcol = torch.from_numpy(H.col).pin_memory()
    hval = torch.from_numpy(H.val).pin_memory()
    h2d = hrp.numel() * 8 + hcol.numel() * 4 + hval.numel() * vbytes
    d2h = (H.nrows + 1) * 8 + nnzC * (4 + vbytes)
    if keep_all:
        o_rp = torch.empty(H.nrows + 1, dtype=torch.int64, pin_memory=True)
        o_col = torch.empty(nnzC, dtype=torch.int32, pin_memory=True)
        o_val = torch.empty(nnzC, dtype=vt, pin_memory=True)
    else:
        ring = torch.empty(1 << 30, dtype=torch.uint8, pin_memory=True)  # 1 GiB pinned ring
    stream = torch.cuda.current_stream()

    def d2h_stream(t):
        b = t.view(torch.uint8) if t.dtype != torch.uint8 else t
        n = b.numel()
        for off in range(0, n, ring.numel()):
            m = min(ring.numel(), n - off)
            ring[:m].copy_(b[off:off + m], non_blocking=True)   # stream-ordered: chunks never overlap

    def one():
        A = sg.DeviceCSR(H.nrows, H.ncols, hrp.to(dev, non_blocking=True), hcol.to(dev, non_blocking=True),
                         hval.to(dev, non_blocking=True))
        if args.e2e_blocks <= 1:
            C, info = sg.spgemm(A, A, args.sample_frac, args.seed)
            if keep_all:
                o_rp.copy_(C.row_ptr, non_blocking=True)
                o_col.copy_(C.col, non_blocking=True)
                o_val.copy_(C.val, non_blocking=True)
            else:
                d2h_stream(C.row_ptr)
                d2h_stream(C.col)
                d2h_stream(C.val)
            return info
        # row blocks: block g+1 computes while block g's C crosses PCIe (spgemm_to_host)
        offs = {}

        def sink(g, r0, r1, rp, col, val):
            if keep_all:
                o_rp[r0:r1].copy_(rp[:-1], non_blocking=True)  # local prefixes; block offsets added on the host
                o = offs.setdefault("o", 0)
                o_col[o:o + col.numel()].copy_(col, non_blocking=True)
                o_val[o:o + val.numel()].copy_(val, non_blocking=True)
                offs["o"] = o + col.numel()
            else:
                d2h_stream(rp)
                d2h_stream(col)
                d2h_stream(val)

        return sg.spgemm_to_host(A, A, sink, blocks=args.e2e_blocks, sample_frac=args.sample_frac, seed=args.seed)

    one()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.e2e_steps):
        one()
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.e2e_steps
    W = int(np.sum(oracle_free_row_work(sg, H, dev, torch)))
    return {"value": 2.0 * W / (ms / 1e3) / 1e9, "unit": "GFLOP/s", "h2d_bytes_per_step": int(h2d),
            "d2h_bytes_per_step": int(d2h), "ms_per_step": ms, "steps": args.e2e_steps,
            "path": ("pinned host CSR -> spgemm() (sample, symbolic, numeric) -> " if args.e2e_blocks <= 1 else
                     "pinned host CSR -> spgemm_to_host(%d row blocks; block g+1 computes while block g's C is copied "
                     "D2H on a second stream) -> " % args.e2e_blocks) +
                    ("pinned host C (all of it)" if keep_all else
                     "all of C streamed D2H through a 1 GiB pinned ring (C %.0f GB > host RAM budget)" % (need / 1e9))}


def oracle_free_row_work(sg, H, dev, torch):
    A = sg.DeviceCSR.from_host(H, device=dev)
    return sg.sg_row_work(A, A).cpu().numpy()


import numpy as np  # noqa: E402  (used by run_e2e)

if __name__ == "__main__":
    main()
