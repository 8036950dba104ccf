"""The paper's sampling experiments on the synthetic configs (PAPER Figs. 4, 6,
7, 9 and the coarse->fine Identify of §III-A), measured on one B200:

  size     : total time (sampling overhead + SpGEMM at the sampled threshold) vs sample size, from
             sqrt(n)/4 to n/4 rows ("near-concave", interior optimum)
  random   : a PREDETERMINED sample (the first f*n rows) vs a uniformly random one (PAPER L250,
             Fig. 7) - run on the un-permuted R-MAT (--unperm), where low row ids are the hubs
  measured : the paper's measured Identify on the sample: time the heavy/light
             kernels on the sampled sub-matrix A_S (B intact) at candidate thresholds, a coarse pass
             over every 8th point of the geometric grid then a fine pass over +-8 points around the
             coarse best; the fastest is the threshold (identity extrapolation, L236)

Every threshold is scored against the measured exhaustive curve T(t) of the full matrix (the
paper's ground truth, L186, L242): dT = T(thr)/min_t T(t) - 1, and dr = |r(thr) - r(t_best)| in
work-share percentage points (R2).

  python tools/sample_study.py --config R18 [--unperm] [--seeds 10] [--out gpurun_out/study.json]
"""
import argparse
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def grid(cap=4096):
    ts, k = {0}, 0
    while True:
        t = int(round(32 * 2 ** (k / 8)))
        if t > cap:
            break
        ts.add(t)
        k += 1
    ts.add(cap)
    return sorted(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="R18")
    ap.add_argument("--unperm", action="store_true", help="un-permuted R-MAT of the config's scale")
    ap.add_argument("--seeds", type=int, default=10)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import numpy as np
    import torch
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg

    if a.unperm:
        scale = {"R18": 18, "C3": 20, "rmat16": 16}[a.config]
        H = gen.rmat(scale, permute=False)
        name = f"rmat{scale}_unperm"
    else:
        H = gen.config(a.config)
        name = a.config
    A = sg.DeviceCSR.from_host(H)
    n = H.nrows
    cm = sg.sg_default_cost_model()
    w = sg.sg_row_work(A, A).cpu().numpy()
    W = float(w.sum())

    def r(t):
        return 100.0 * float(w[w > t].sum()) / W

    def ev_time(fn, reps):
        ts = []
        for _ in range(reps):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            out = fn()
            e1.record()
            torch.cuda.synchronize()
            ts.append((e0.elapsed_time(e1), out))
        ts.sort(key=lambda x: x[0])
        return ts[len(ts) // 2]

    def spgemm_at(M, t):
        plan = sg.sg_symbolic(M, A, t)
        col, val = sg.sg_numeric(plan, M, A)
        plan.destroy()
        del col, val

    Tcache = {}

    def T(t):
        if t not in Tcache:
            Tcache[t] = ev_time(lambda: spgemm_at(A, t), a.reps)[0]
        return Tcache[t]

    # ---- ground truth: the measured exhaustive curve on the full matrix ----
    G = grid(cm.cap_L)
    curve = [(t, T(t)) for t in G]
    t_best, T_best = min(curve, key=lambda x: x[1])
    thr_star, _ = sg.sg_exhaustive_threshold(A, A, cm)
    print(f"{name}: n={n} W={W:.3e} measured best t={t_best} T={T_best:.3f} ms; model thr*={thr_star} "
          f"T={T(thr_star):.3f} ms", flush=True)

    def score(thr, t_identify_ms):
        Tt = T(thr)
        return {"thr": int(thr), "T_ms": Tt, "dT": Tt / T_best - 1.0, "dr_pp": abs(r(thr) - r(t_best)),
                "t_identify_ms": t_identify_ms, "total_ms": t_identify_ms + Tt,
                "overhead": t_identify_ms / (t_identify_ms + Tt)}

    def agg(runs):
        keys = ("dT", "dr_pp", "t_identify_ms", "total_ms", "overhead")
        return {k: {"mean": float(np.mean([x[k] for x in runs])), "max": float(np.max([x[k] for x in runs]))}
                for k in keys}

    report = {"config": name, "n": n, "W": W, "grid": curve, "t_best": t_best, "T_best_ms": T_best,
              "thr_star_model": thr_star, "cost_model": cm.as_dict()}

    # ---- size: total time vs sample size (PAPER Figs. 4, 6, 9) ----
    sq = math.sqrt(n)
    sizes = [("sqrt(n)/4", sq / 4), ("sqrt(n)/2", sq / 2), ("sqrt(n)", sq), ("2sqrt(n)", 2 * sq),
             ("4sqrt(n)", 4 * sq), ("n/200", n / 200), ("n/100", n / 100), ("n/50", n / 50), ("n/20", n / 20),
             ("n/10", n / 10), ("n/4", n / 4)]
    report["size"] = {}
    for label, m in sizes:
        f = min(1.0, m / n)
        runs = []
        for seed in range(a.seeds):
            try:
                ms, (thr, _) = ev_time(lambda: sg.sg_sample_threshold(A, A, f, seed, cm), 1)
            except sg.SgError:
                continue
            runs.append(dict(score(thr, ms), seed=seed))
        if runs:
            report["size"][label] = {"f": f, "agg": agg(runs), "runs": runs}
            g = report["size"][label]["agg"]
            print(f"size {label:10s} f={f:.5f}: total {g['total_ms']['mean']:.3f} ms  dT {g['dT']['mean']:.4f} "
                  f"dr {g['dr_pp']['mean']:.3f} pp  overhead {g['overhead']['mean']:.4f}", flush=True)

    # ---- random vs predetermined (Fig. 7) ----
    report["random"] = {}
    for f in (0.01, 0.05, 0.1):
        first = torch.arange(max(int(f * n), 1), dtype=torch.int64, device="cuda")
        ms, (thr_p, _) = ev_time(lambda: sg.sg_threshold_on_rows(A, A, first, cm), 1)
        pre = score(thr_p, ms)
        rnd = []
        for seed in range(a.seeds):
            ms, (thr, _) = ev_time(lambda: sg.sg_sample_threshold(A, A, f, seed, cm), 1)
            rnd.append(dict(score(thr, ms), seed=seed))
        J = sg.sg_cost_curve(A, A, [thr_p, thr_star] + [x["thr"] for x in rnd], cm)
        pre["dJ"] = J[0] / J[1] - 1.0
        for i, x in enumerate(rnd):
            x["dJ"] = J[2 + i] / J[1] - 1.0
        report["random"][str(f)] = {"predetermined": pre, "random_agg": agg(rnd),
                                    "random_dJ_max": max(x["dJ"] for x in rnd), "random": rnd}
        print(f"random f={f}: predetermined thr={thr_p} dT {pre['dT']:.4f} dr {pre['dr_pp']:.3f} dJ {pre['dJ']:.4f} | "
              f"random dT mean {np.mean([x['dT'] for x in rnd]):.4f} dr mean {np.mean([x['dr_pp'] for x in rnd]):.3f} "
              f"dJ max {max(x['dJ'] for x in rnd):.4f}", flush=True)

    # ---- measured Identify on the sample: coarse (every 8th grid point) -> fine (+-8) ----
    rp = A.row_ptr
    lens = rp[1:] - rp[:-1]
    report["measured"] = {}
    for f in (0.01, 0.05):
        runs = []
        for seed in range(min(a.seeds, 5)):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            S = sg.sg_sample_rows(n, f, seed)
            # A_S: the sampled rows of A as a CSR (B intact) - plumbing for the experiment, torch ops
            ls = lens[S]
            srp = torch.zeros(S.numel() + 1, dtype=torch.int64, device="cuda")
            srp[1:] = torch.cumsum(ls, 0)
            idx = torch.repeat_interleave(rp[S], ls) + (torch.arange(int(srp[-1]), device="cuda")
                                                         - torch.repeat_interleave(srp[:-1], ls))
            AS = sg.DeviceCSR(int(S.numel()), A.ncols, srp, A.col[idx].contiguous(), A.val[idx].contiguous())
            timed = {}

            def TS(t):
                if t not in timed:
                    timed[t] = ev_time(lambda: spgemm_at(AS, t), 1)[0]
                return timed[t]

            coarse = G[::8] + ([G[-1]] if (len(G) - 1) % 8 else [])
            tc = min(coarse, key=TS)
            k = G.index(tc)
            fine = G[max(0, k - 8): k + 9]
            thr = min(fine, key=TS)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1)
            runs.append(dict(score(thr, ms), seed=seed, evaluations=len(timed)))
            del AS
        report["measured"][str(f)] = {"agg": agg(runs), "runs": runs}
        g = report["measured"][str(f)]["agg"]
        print(f"measured f={f}: dT {g['dT']['mean']:.4f} (max {g['dT']['max']:.4f}) dr {g['dr_pp']['mean']:.3f} pp "
              f"overhead {g['overhead']['mean']:.4f}", flush=True)

    out = a.out or os.path.join(ROOT, "gpurun_out", f"sample_study_{name}.json")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    json.dump(report, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
