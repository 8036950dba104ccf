"""Where a bench step's time goes: host wall time of each public call of the step (synchronised after
each call, so a call's host syncs and launch gaps are inside its own number), next to the device time
of its kernels (sg.profile). One B200.

  python tools/step_breakdown.py --config C2 --reps 20
"""
import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--dtype", default="f64")
    a = ap.parse_args()
    import torch
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg
    H = gen.config(a.config, dtype=a.dtype)
    A = sg.DeviceCSR.from_host(H)
    names = ["sample_threshold", "partition", "symbolic", "numeric", "destroy"]
    tot = {k: 0.0 for k in names}
    whole = 0.0
    for r in range(a.reps + 3):
        torch.cuda.synchronize()
        t = {}
        w0 = time.perf_counter()
        t0 = time.perf_counter()
        thr, rep = sg.sg_sample_threshold(A, A, 0.01, 1)
        torch.cuda.synchronize(); t["sample_threshold"] = time.perf_counter() - t0; t0 = time.perf_counter()
        cuts, W = sg.sg_partition(A, A, 1)
        torch.cuda.synchronize(); t["partition"] = time.perf_counter() - t0; t0 = time.perf_counter()
        plan = sg.sg_symbolic(A, A, thr, cuts[0], cuts[1])
        torch.cuda.synchronize(); t["symbolic"] = time.perf_counter() - t0; t0 = time.perf_counter()
        col, val = sg.sg_numeric(plan, A, A)
        torch.cuda.synchronize(); t["numeric"] = time.perf_counter() - t0; t0 = time.perf_counter()
        plan.destroy()
        del col, val
        torch.cuda.synchronize(); t["destroy"] = time.perf_counter() - t0
        if r >= 3:
            whole += time.perf_counter() - w0
            for k in names:
                tot[k] += t[k]
    with sg.profile() as prof:
        thr, rep = sg.sg_sample_threshold(A, A, 0.01, 1)
        cuts, W = sg.sg_partition(A, A, 1)
        plan = sg.sg_symbolic(A, A, thr, cuts[0], cuts[1])
        col, val = sg.sg_numeric(plan, A, A)
        plan.destroy()
    bk = prof.by_kernel()
    print(f"{a.config}: wall per step {whole / a.reps * 1e3:.3f} ms | " +
          "  ".join(f"{k} {tot[k] / a.reps * 1e3:.3f}" for k in names))
    print(f"kernels (one step): {sum(v[1] for v in bk.values()):.3f} ms in {sum(v[0] for v in bk.values())} launches | " +
          "  ".join(f"{k}={v[1]:.3f}/{v[0]}" for k, v in sorted(bk.items(), key=lambda kv: -kv[1][1])[:12]))


if __name__ == "__main__":
    main()
