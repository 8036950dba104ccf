"""Profiling driver: one sampled-threshold symbolic + numeric pass over a ROW SUBSET of a config,
so that ncu can replay the heavy kernels of a large workload (C3) without backing up the whole C.
Heavy rows are spread uniformly by the R-MAT label permutation, so a prefix of the rows is
representative.

  python tools/prof_rows.py --config C3 --frac 0.0625 [--reps 2]
"""
import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--frac", type=float, default=0.0625)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--thr", type=int, default=-1)
    a = ap.parse_args()
    import torch
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg
    H = gen.config(a.config)
    A = sg.DeviceCSR.from_host(H)
    thr = a.thr if a.thr >= 0 else sg.sg_sample_threshold(A, A, 0.01, 1)[0]
    re = int(H.nrows * a.frac)
    for r in range(a.reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        with sg.profile() as prof:
            plan = sg.sg_symbolic(A, A, thr, 0, re)
            col, val = sg.sg_numeric(plan, A, A)
        t = time.perf_counter() - t0
        bk = prof.by_kernel()
        print(f"rep {r}: rows [0,{re}) thr={thr} nnz={plan.nnz} wall {t*1e3:.1f} ms  " +
              "  ".join(f"{k}={v[1]:.2f}ms" for k, v in sorted(bk.items(), key=lambda kv: -kv[1][1])[:5]), flush=True)
        plan.destroy()
        del col, val


if __name__ == "__main__":
    main()
