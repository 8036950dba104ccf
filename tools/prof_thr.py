"""Per-kernel times of one symbolic + numeric pass at given thresholds (profiling helper).
  python tools/prof_thr.py --config R18 [--unperm] --thr 128,4096"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="R18")
    ap.add_argument("--unperm", action="store_true")
    ap.add_argument("--thr", default="128,4096")
    a = ap.parse_args()
    import torch
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg
    H = gen.rmat({"R18": 18, "C3": 20, "rmat16": 16}[a.config], permute=False) if a.unperm else gen.config(a.config)
    A = sg.DeviceCSR.from_host(H)
    for t in [int(x) for x in a.thr.split(",")]:
        for rep in range(2):
            with sg.profile() as prof:
                plan = sg.sg_symbolic(A, A, t)
                col, val = sg.sg_numeric(plan, A, A)
            torch.cuda.synchronize()
            info = plan.info()
            plan.destroy()
            del col, val
        bk = prof.by_kernel()
        tot = sum(v[1] for v in bk.values())
        print(f"t={t}: {tot:.2f} ms  " + "  ".join(f"{k}={v[1]:.2f}" for k, v in sorted(bk.items(), key=lambda kv: -kv[1][1])[:6])
              + f" | light {info['n_light']} sorted {info['n_light_sorted']} bins {info['light_bins']}", flush=True)


if __name__ == "__main__":
    main()
