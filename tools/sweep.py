"""Config 5: threshold sweep — measured exhaustive search vs the sampled threshold, plus the
calibration of the cost model (the paper's "offline relation").

For each matrix (ER 2^18 = C2 and R-MAT 18 by default):
  1. T(t): device time of sg_symbolic + sg_numeric at every t of a geometric grid (median of reps)
     and per-class kernel times -> least-squares fit of the light / heavy cost constants.
  2. the exhaustive model threshold thr* (sg_exhaustive_threshold) and, for f in {1,2,5,10} % and
     20 sampler seeds, the sampled thr_s (sg_sample_threshold) with its gaps: dr (pp of work share,
     DESIGN.md R2), delta_rel, dJ, and the measured time gap dT = T(thr_s) / min_t T(t) - 1 (PAPER
     Table I "Time Difference") plus the sampling overhead t_sample / (t_sample + T(thr_s)).

  python tools/sweep.py [--configs C2,R18] [--seeds 20] [--out profiles/r01_sweep.json] [--fit]
"""
import argparse
import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def grid(cap=4096):
    ts = {0}
    k = 0
    while True:
        t = int(round(16 * 2 ** (k / 4)))
        if t > cap:
            break
        ts.add(t)
        k += 1
    ts.add(cap)
    return sorted(ts)


def product_only(sg, A, t):
    """symbolic + numeric at threshold t; C is dropped at once (C3's C is 116 GB: never two alive)."""
    plan = sg.sg_symbolic(A, A, t)
    col, val = sg.sg_numeric(plan, A, A)
    plan.destroy()
    del col, val


def timed(fn, reps):
    import torch
    out = []
    for _ in range(reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        r = fn()
        e1.record()
        torch.cuda.synchronize()
        out.append((e0.elapsed_time(e1), r))
    out.sort(key=lambda x: x[0])
    return out[len(out) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C2,R18")
    ap.add_argument("--seeds", type=int, default=20)
    ap.add_argument("--fracs", default="0.01,0.02,0.05,0.1")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default="gpurun_out/sweep.json")
    a = ap.parse_args()
    import numpy as np
    import torch
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg

    report = {"cost_model": sg.sg_default_cost_model().as_dict(), "configs": {}}
    for name in a.configs.split(","):
        H = gen.config(name)
        A = sg.DeviceCSR.from_host(H)
        cm = sg.sg_default_cost_model(H.ncols)  # the model calls with cm=None use for this B (R's floor from p)
        tf = max(1, int(cm.tiles_fixed))
        w = sg.sg_row_work(A, A).cpu().numpy()
        W = float(w.sum())
        r = lambda t: 100.0 * float(w[w > t].sum()) / W
        rows = []
        # ---- measured T(t) and per-class stats for calibration ----
        for t in grid():
            def run():
                with sg.profile() as prof:
                    plan = sg.sg_symbolic(A, A, t)
                    col, val = sg.sg_numeric(plan, A, A)
                u = (plan.row_ptr[1:] - plan.row_ptr[:-1]).cpu().numpy()
                plan.destroy()
                del col, val
                return prof.by_kernel(), u
            _, (bk, u) = timed(run, 1)                      # per-class split (profiled run)
            ms = timed(lambda: product_only(sg, A, t), a.reps)[0]  # T(t) without profiling events
            light = (w > 0) & (w <= t)
            heavy = w > t
            arow = np.diff(H.row_ptr)
            # light path: k_sym_light, k_num_light (hash) and k_num_light_sort (sorted warp path);
            # heavy path: k_sym_heavy, the rank kernels k_num_heavy / k_num_tile and k_num_dense
            kl = sum(v[1] for k, v in bk.items() if k.startswith(("k_sym_light", "k_num_light")))
            kh = sum(v[1] for k, v in bk.items() if k in ("k_sym_heavy", "k_num_heavy", "k_num_tile", "k_num_dense"))
            rows.append({"t": t, "ms": ms, "ms_light": kl, "ms_heavy": kh, "r": r(t),
                         "L": [int(light.sum()), int(w[light].sum()), int(u[light].sum())],
                         "H": [int(heavy.sum()), int(w[heavy].sum()), int(u[heavy].sum()),
                               int(arow[heavy].sum()),
                               int((arow[heavy] * np.maximum(tf, np.ceil(u[heavy] / max(cm.capu, 1)))).sum())]})
            print(f"{name} t={t:5d} T={ms:8.3f} ms  light {kl:7.3f}  heavy {kh:7.3f}  r={r(t):6.2f}%", flush=True)
        Tbest = min(x["ms"] for x in rows)
        t_meas = min(rows, key=lambda x: x["ms"])["t"]
        thr_star, J_star = sg.sg_exhaustive_threshold(A, A, cm)
        T_at = lambda t: timed(lambda: product_only(sg, A, t), a.reps)[0]
        T_star = T_at(thr_star)
        samples = {}
        for f in [float(x) for x in a.fracs.split(",")]:
            res = []
            for seed in range(a.seeds):
                ts_ms, (thr_s, rep) = timed(lambda: sg.sg_sample_threshold(A, A, f, seed, cm), 1)
                Jc = sg.sg_cost_curve(A, A, [thr_s, thr_star], cm)
                res.append({"seed": seed, "thr_s": thr_s, "dr_pp": abs(r(thr_s) - r(thr_star)),
                            "delta_rel": abs(thr_s - thr_star) / max(thr_star, 1),
                            "dJ": Jc[0] / Jc[1] - 1.0, "t_sample_ms": ts_ms})
            # measured time at each distinct sampled threshold
            tcache = {}
            for x in res:
                if x["thr_s"] not in tcache:
                    tcache[x["thr_s"]] = T_at(x["thr_s"])
                x["T_ms"] = tcache[x["thr_s"]]
                x["dT"] = x["T_ms"] / Tbest - 1.0
                x["overhead"] = x["t_sample_ms"] / (x["t_sample_ms"] + x["T_ms"])
            agg = {k: {"mean": float(np.mean([x[k] for x in res])), "max": float(np.max([x[k] for x in res]))}
                   for k in ("dr_pp", "delta_rel", "dJ", "dT", "overhead")}
            samples[str(f)] = {"agg": agg, "runs": res}
            print(f"{name} f={f:.2f}: " + "  ".join(f"{k} mean {v['mean']:.4f} max {v['max']:.4f}" for k, v in agg.items()),
                  flush=True)
        report["configs"][name] = {"n": H.nrows, "W": W, "tiles_fixed": tf, "grid": rows, "T_best_ms": Tbest, "t_best_measured": t_meas,
                                   "thr_star_model": thr_star, "J_star": J_star, "T_at_thr_star_ms": T_star,
                                   "r_at_t_best_measured": r(t_meas), "r_at_thr_star": r(thr_star),
                                   "samples": samples}
        del A
        torch.cuda.empty_cache()
    # ---- least-squares calibration of the cost constants from the grid (ps per unit) ----
    fit = {}
    try:
        XL, yL, XH, yH = [], [], [], []
        for name, c in report["configs"].items():
            for x in c["grid"]:
                nL, wL, uL = x["L"]
                nH, wH, uH, aH, aR = x["H"]
                if nL:
                    XL.append([nL, wL, uL]); yL.append(x["ms_light"] * 1e9)   # ms -> ps
                if nH:
                    XH.append([nH, wH, aR, uH]); yH.append(x["ms_heavy"] * 1e9)
        from scipy.optimize import nnls
        cL, _ = nnls(np.array(XL, float), np.array(yL, float))
        cH, _ = nnls(np.array(XH, float), np.array(yH, float))
        # SM-time: a kernel's wall time is shared by 148 SMs; per-row SM cost = fitted wall ps x 148
        fit = {"kappa_L": cL[0] * 148, "lambda_L": cL[1] * 148, "rho_L": cL[2] * 148,
               "kappa_H": cH[0] * 148, "lambda_H": cH[1] * 148, "tau_H": cH[2] * 148, "mu_H": cH[3] * 148}
        print("fit (ps of SM time per unit):", {k: round(v, 1) for k, v in fit.items()})
    except Exception as e:  # noqa: BLE001
        fit = {"error": str(e)}
    report["fit"] = fit
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(report, f, indent=1)


if __name__ == "__main__":
    main()
