"""Driver for compute-sanitizer (memcheck / racecheck / synccheck): every kernel path of the hot path
on small seeded inputs, each compared with the oracle so that a silent corruption also fails.

  compute-sanitizer --tool racecheck --kernel-name regex:k_ python tools/sanitize_run.py [--scale 12]
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=12)
    a = ap.parse_args()
    import torch
    import oracle
    import sginputs as gen
    import paper_conf_icpp_hardhikbrks17_b200 as sg
    from _util import compare_rows
    cases = [  # (label, matrix, thr, dense_log2, variant)
        ("light+rank", gen.rmat(a.scale), 256, 62, 0),
        ("light (sorted warp path) + rank (warp-tile)", gen.rmat(a.scale), 256, 62, 32),
        ("light (hash path) + rank (CTA)", gen.rmat(a.scale), 256, 62, 8 | 16),
        ("rank only", gen.rmat(a.scale), 0, 62, 0),
        ("rank only, warp-tile forced", gen.rmat(a.scale, mode="signed"), 0, 62, 32),
        ("dense2 only", gen.rmat(a.scale, mode="signed"), 0, 0, 0),
        ("dense (round-1) only", gen.rmat(a.scale, mode="signed"), 0, 0, 1),
        ("mixed default", gen.rmat(a.scale + 2), -1, -1, 0),
        ("sorted light (unpermuted)", gen.rmat(a.scale + 1, permute=False, mode="zeros"), 4096, -1, 0),
        ("fp32", gen.rmat(a.scale, dtype="f32"), 64, 8, 0),
    ]
    cases.append(("no tile pointers, warp-tile + CTA rank + dense2", gen.rmat(a.scale, mode="signed"), 0, 10, 32 | 128))
    ok = True
    for label, A, thr, dl, var in cases:
        sg.set_option(sg.SG_OPT_DENSE_LOG2, dl)
        sg.set_option(sg.SG_OPT_VARIANT, var & 127)
        sg.set_option(sg.SG_OPT_TP_MAX_BYTES, 0 if var & 128 else -1)
        dA = sg.DeviceCSR.from_host(A)
        t = thr if thr >= 0 else sg.sg_sample_threshold(dA, dA, 0.05, 3)[0]
        plan = sg.sg_symbolic(dA, dA, t)
        col, val = sg.sg_numeric(plan, dA, dA)
        torch.cuda.synchronize()
        R = oracle.spgemm(A, A, with_absmag=True)
        rp = plan.row_ptr.cpu().numpy()
        try:
            assert np.array_equal(rp, R.row_ptr)
            exact = bool(np.all(A.val == np.round(A.val)))  # integer-valued inputs: sums exact, values bit-exact
            compare_rows(rp, col.cpu().numpy(), val.cpu().numpy(), R, A.dtype, exact_values=exact)
            print(f"{label}: OK (nnz {plan.nnz}, info {plan.info()['n_heavy']} heavy / {plan.info()['n_dense']} dense)", flush=True)
        except AssertionError as e:
            ok = False
            print(f"{label}: FAILED {e}", flush=True)
        plan.destroy()
    sg.set_option(sg.SG_OPT_DENSE_LOG2, -1)
    sg.set_option(sg.SG_OPT_VARIANT, 0)
    sg.set_option(sg.SG_OPT_TP_MAX_BYTES, -1)
    print("ALL OK" if ok else "SOME FAILED")


if __name__ == "__main__":
    main()
