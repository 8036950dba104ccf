"""One sampled-threshold symbolic + numeric pass over a whole config (for ncu captures of the light
kernels on small configs).  python tools/prof_config.py --config C2 [--reps 2]"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--reps", type=int, default=2)
    a = ap.parse_args()
    import torch
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg
    H = gen.config(a.config)
    A = sg.DeviceCSR.from_host(H)
    thr = sg.sg_sample_threshold(A, A, 0.01, 1)[0]
    for r in range(a.reps):
        with sg.profile() as prof:
            plan = sg.sg_symbolic(A, A, thr)
            col, val = sg.sg_numeric(plan, A, A)
        info = plan.info()
        print(f"rep {r}: thr {thr} nnz {plan.nnz} bins {info['light_bins']} heavy {info['n_heavy']} | " +
              "  ".join(f"{k}={v[1]:.3f}" for k, v in sorted(prof.by_kernel().items(), key=lambda kv: -kv[1][1])[:6]),
              flush=True)
        plan.destroy()


if __name__ == "__main__":
    main()
