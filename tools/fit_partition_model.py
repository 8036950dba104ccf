"""Calibrates a cost model for the cost-weighted multi-GPU split (reading R19, §7.7) from
measured shard times — the paper's "offline relation" fitted to what a GPU
actually spends on a block of rows, instead of to the light/heavy threshold sweep (§4).

Input: tools/shard_sim.py JSON files (cuts, measured shard ms, thr, the sample's compression).
Each shard's time is modeled as the sum over its rows of the sg_cost_model path costs (c_L or c_H at
thr, u estimated from the sample's per-class compression); the 8 constants are fitted by
non-negative least squares (relative residuals), for each candidate capu, and the best is printed as
an sg_cost_model (ps of SM time; 148 SMs).

  python tools/fit_partition_model.py gpurun_out/fit_*.json [--out profiles/...json]
"""
import argparse
import json
import os
import sys

import numpy as np
from scipy.optimize import nnls

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

NSM = 148


def matrix(rec):
    import sginputs as gen
    if rec.get("unperm"):
        scale = {"C3": 20, "R18": 18, "C4": 22}[rec["config"]]
        return gen.rmat(scale, 16, seed=rec.get("seed", 1), permute=False)
    return gen.config(rec["config"], seed=rec.get("seed", 1))


def row_features(H, thr, comp, capu):
    """Per-row feature matrix (n x 8) so that cost = F @ [kL, lL, sL, rL, kH, lH, tH, mH]."""
    lenB = np.diff(H.row_ptr)
    a = lenB.copy()  # A = B (A*A)
    prod = lenB[H.col]
    w = np.zeros(H.nrows, dtype=np.int64)
    nz = a > 0
    w[nz] = np.add.reduceat(prod, H.row_ptr[:-1][nz])
    light = (w > 0) & (w <= thr)
    heavy = w > thr
    UL, WL, UH, WH = comp
    uh = w.astype(np.float64)
    if WL > 0:
        uh[light] = np.minimum(w[light], np.ceil(w[light] * UL / WL))
    if WH > 0:
        uh[heavy] = np.minimum(w[heavy], np.ceil(w[heavy] * UH / WH))
    F = np.zeros((H.nrows, 8))
    lg = np.ceil(np.log2(np.maximum(uh, 2)))
    F[light, 0] = 1
    F[light, 1] = w[light]
    F[light, 2] = uh[light] * lg[light]
    F[light, 3] = uh[light]
    R = np.ones(H.nrows) if capu == 0 else np.maximum(1, np.ceil(uh / capu))
    F[heavy, 4] = 1
    F[heavy, 5] = w[heavy]
    F[heavy, 6] = a[heavy] * R[heavy]
    F[heavy, 7] = uh[heavy]
    return F


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("files", nargs="+")
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    recs = [json.load(open(f)) for f in args.files]
    best = None
    for capu in (0, 4096, 12288, 65536):
        X, y = [], []
        for rec in recs:
            H = matrix(rec)
            F = row_features(H, rec["thr"], rec["comp"], capu)
            P = np.vstack([np.zeros(8), np.cumsum(F, axis=0)])
            for k, sp in rec["splits"].items():
                c = sp["cuts"]
                for g in range(len(c) - 1):
                    # + a per-shard constant (launches, host syncs): paid by every shard alike, so it does
                    # not move the cuts and is not part of the per-row model
                    X.append(np.concatenate([P[c[g + 1]] - P[c[g]], [1.0]]))
                    y.append(sp["shard_ms"][g] * 1e9 * NSM)  # ps of SM time
        X, y = np.array(X), np.array(y)
        sc = np.maximum(X.max(axis=0), 1e-30)
        Xr = (X / sc) / y[:, None]  # relative residuals: minimise sum (pred/y - 1)^2
        coef, _ = nnls(Xr, np.ones(len(y)))
        coef = coef / sc
        pred = X @ coef
        shard_const_ms = coef[8] / 1e9 / NSM
        coef = coef[:8]
        err = np.abs(pred / y - 1)
        res = {"capu": capu, "coef": coef.tolist(), "mean_rel_err": float(err.mean()), "max_rel_err": float(err.max()),
               "n_shards": int(len(y)), "shard_const_ms": float(shard_const_ms)}
        print(f"capu {capu:6d}: mean rel err {err.mean():.4f} max {err.max():.4f}  shard const {shard_const_ms:.2f} ms  coef " +
              " ".join(f"{x:.4g}" for x in coef), flush=True)
        if best is None or res["mean_rel_err"] < best["mean_rel_err"]:
            best = res
    names = ["kappa_L", "lambda_L", "sigma_L", "rho_L", "kappa_H", "lambda_H", "tau_H", "mu_H"]
    model = {n: int(round(v)) for n, v in zip(names, best["coef"])}
    model.update({"tiles_fixed": 1, "capu": best["capu"], "cap_L": 4096})
    print("partition model:", json.dumps(model))
    if args.out:
        json.dump({"model": model, "fit": best, "files": args.files}, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
