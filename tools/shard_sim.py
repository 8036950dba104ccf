"""Row-shard balance of the multi-GPU split, measured on ONE B200.

Each rank's work is independent given a replicated B (C_i depends only on A_i and B), so the time a
G-GPU run spends in symbolic + numeric is max_g T(shard g), where T(shard g) is the time of rank g's
rows on a whole B200. This tool times every shard alone on the one GPU, for the flops split of Alg. 2
(sg_partition) and the cost-weighted split (sg_partition_cost, R19), and
reports per-shard times, the imbalance max/mean, and the projected G-GPU makespan (compute only: the
sampling step, the B broadcast and the NCCL assembly are not included). Not a multi-GPU measurement.

  python tools/shard_sim.py --config C3 [--unperm] --G 8 [--reps 2] [--out profiles/...json]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--unperm", action="store_true", help="R-MAT without the label permutation (hubs at low ids)")
    ap.add_argument("--G", type=int, nargs="+", default=[8])
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--sample-frac", type=float, default=0.01)
    ap.add_argument("--kinds", nargs="+", default=["flops", "cost"])
    ap.add_argument("--seed", type=int, default=1, help="matrix seed")
    ap.add_argument("--cm-json", default="", help="cost model for the cost split (tools/fit_partition_model.py output)")
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import torch
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg
    if a.unperm:
        scale = {"C3": 20, "R18": 18, "C4": 22}[a.config]
        H = gen.rmat(scale, 16, seed=a.seed, permute=False)
    else:
        H = gen.config(a.config, seed=a.seed)
    A = sg.DeviceCSR.from_host(H)
    cm = sg.sg_default_cost_model()
    pcm = None  # sg_partition_cost's default: the partition model fitted to measured shard times
    if a.cm_json:
        pcm = sg.sg_default_cost_model()
        for k, v in json.load(open(a.cm_json))["model"].items():
            setattr(pcm, k, int(v))
    thr, rep = sg.sg_sample_threshold(A, A, a.sample_frac, 1, cm)
    comp = [rep["U_est_L"], rep["W_est_L"], rep["U_est_H"], rep["W_est_H"]]
    _, W = sg.sg_partition(A, A, 1)
    w = sg.sg_row_work(A, A).cpu()
    out = {"config": a.config, "unperm": a.unperm, "seed": a.seed, "n": H.nrows, "W": W, "thr": thr, "comp": comp, "splits": {}}

    def shard_ms(r0, r1):
        best = None
        for _ in range(a.reps):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan = sg.sg_symbolic(A, A, thr, r0, r1)
            col = torch.empty(plan.nnz, dtype=torch.int32, device="cuda")
            val = torch.empty(plan.nnz, dtype=plan.dtype, device="cuda")
            sg.sg_numeric(plan, A, A, out=(col, val))
            e1.record()
            torch.cuda.synchronize()
            t = e0.elapsed_time(e1)
            plan.destroy()
            del col, val
            best = t if best is None else min(best, t)
        return best

    for G in a.G:
        for kind in a.kinds:
            if kind == "flops":
                cuts, _ = sg.sg_partition(A, A, G)
            else:
                cuts, _ = sg.sg_partition_cost(A, A, G, thr, comp, pcm)
            ts, ws = [], []
            for g in range(G):
                ts.append(shard_ms(cuts[g], cuts[g + 1]))
                ws.append(int(w[cuts[g]:cuts[g + 1]].sum().item()))
            mx, mean = max(ts), sum(ts) / G
            rec = {"cuts": cuts, "shard_ms": ts, "shard_W": ws, "max_ms": mx, "mean_ms": mean,
                   "imbalance": mx / mean, "projected_GFLOPs": 2 * W / (mx / 1e3) / 1e9}
            out["splits"][f"G{G}_{kind}"] = rec
            print(f"G={G} {kind:5s}: max {mx:7.2f} ms  mean {mean:7.2f}  imbalance {mx / mean:.3f}  "
                  f"projected {rec['projected_GFLOPs']:.0f} GFLOP/s  shards " + " ".join(f"{t:.1f}" for t in ts), flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
