"""A/B of kernel variants (sg_set_option(SG_OPT_VARIANT / SG_OPT_DENSE_LOG2)) on one config, one B200.

For every (variant, dense_log2) setting: symbolic + numeric of rows [0, frac*n) at the sampled
threshold, `reps` times; prints the per-kernel CUDA-event times of the last rep and a digest of C
(sum of columns, sum of values, xor-hash of (row, col)) so that the settings can be checked against
each other for the same result.

  python tools/ab_variant.py --config C3 --frac 1.0 --settings 0:-1,1:-1 --reps 2
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
    ap.add_argument("--frac", type=float, default=1.0)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--thr", type=int, default=-1)
    ap.add_argument("--settings", default="0:-1,1:-1", help="variant:dense_log2 pairs")
    ap.add_argument("--dtype", default="f64")
    a = ap.parse_args()
    import torch
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg
    H = gen.config(a.config, dtype=a.dtype)
    A = sg.DeviceCSR.from_host(H)
    thr = a.thr if a.thr >= 0 else sg.sg_sample_threshold(A, A, 0.01, 1)[0]
    re = int(H.nrows * a.frac)
    for st in a.settings.split(","):
        var, dl = (int(x) for x in st.split(":"))
        sg.set_option(sg.SG_OPT_VARIANT, var)
        sg.set_option(sg.SG_OPT_DENSE_LOG2, dl)
        for r in range(a.reps):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            with sg.profile() as prof:
                plan = sg.sg_symbolic(A, A, thr, 0, re)
                col, val = sg.sg_numeric(plan, A, A)
            t = time.perf_counter() - t0
            info = plan.info()
            if r + 1 < a.reps:  # C3's C is 116 GB: never two alive
                plan.destroy()
                del col, val
        bk = prof.by_kernel()
        tot = sum(v[1] for v in bk.values())
        rows = torch.repeat_interleave(torch.arange(re, device=col.device, dtype=torch.int64),
                                       torch.diff(plan.row_ptr)) if plan.nnz < 2**31 else None
        step = 1 << 29  # chunked: C3's C has 9.7e9 entries
        dig = {"nnz": plan.nnz,
               "colsum": sum(int(col[i:i + step].sum(dtype=torch.int64)) for i in range(0, col.numel(), step)),
               "valsum": sum(float(val[i:i + step].double().sum()) for i in range(0, val.numel(), step))}
        if rows is not None:
            dig["hash"] = int(((rows * 1000003 + col.long()) * 0x9E3779B1 % (2**61 - 1)).sum())
        print(f"variant={var} dense_log2={dl} (n_dense {info['n_dense']}) rows [0,{re}) thr={thr} wall {t*1e3:.1f} ms "
              f"kernels {tot:.2f} ms | " + "  ".join(f"{k}={v[1]:.2f}" for k, v in sorted(bk.items(), key=lambda kv: -kv[1][1])[:6])
              + f" | {dig}", flush=True)
        plan.destroy()
        del col, val
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
