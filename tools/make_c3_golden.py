"""Writes tests/golden/c3_structure_moments.npz: the oracle's structure digest of C = A*A for
config C3 (R-MAT scale 20, edge factor 16, seed 1), for the -m gpu parity test
test_c3_structure_vs_oracle_digest. Calls ONLY oracle/ (and the seeded input generator sginputs/).

C3's C has 9.69e9 entries (116 GB), more than this host holds, so the oracle reports per row
(u_i, sum c, sum c^2, sum c^3) over the columns of C_i (oracle.moments, the std::map Gustavson of
PAPER L74 / Alg. 2 l.5-6 L222-L223), and this script stores them summed over blocks of 256 rows
(mod 2^64) plus every row's u_i. About 20-40 min on 8 host cores.

  python tools/make_c3_golden.py [--config C3] [--block 256]
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--block", type=int, default=256)
    ap.add_argument("--chunk", type=int, default=16384)
    a = ap.parse_args()
    import oracle
    import sginputs as gen
    A = gen.config(a.config)
    n = A.nrows
    t0 = time.time()
    # heaviest rows first within the run so that the OpenMP dynamic schedule balances
    m = np.zeros((n, 4), dtype=np.uint64)
    for c0 in range(0, n, a.chunk):
        rows = np.arange(c0, min(n, c0 + a.chunk), dtype=np.int64)
        m[c0:c0 + len(rows)] = oracle.moments(A, A, rows)
        if (c0 // a.chunk) % 8 == 0:
            print(f"rows {c0 + len(rows)}/{n}  {time.time() - t0:.0f} s", flush=True)
    nb = (n + a.block - 1) // a.block
    pad = np.zeros((nb * a.block - n, 4), dtype=np.uint64)
    blocks = np.concatenate([m, pad]).reshape(nb, a.block, 4).sum(axis=1, dtype=np.uint64)
    out = os.path.join(ROOT, "tests", "golden", f"{a.config.lower()}_structure_moments.npz")
    np.savez_compressed(out, block_moments=blocks, u=m[:, 0].astype(np.int64), block=np.int64(a.block))
    meta = {
        "_source": "oracle.moments (std::map Gustavson, PAPER L74, Alg. 2 l.5-6 L222-L223) over every row of "
                   f"{a.config} = sginputs.config('{a.config}') (seed 1), written by tools/make_c3_golden.py; "
                   "per block of `block` rows: sums mod 2^64 of (u_i, sum c, sum c^2, sum c^3); u = every row's nnz.",
        "config": a.config, "nrows": int(n), "nnz_C": int(m[:, 0].sum()), "block": a.block,
        "oracle_threads": oracle.threads(), "seconds": round(time.time() - t0, 1),
    }
    json.dump(meta, open(out.replace(".npz", ".json"), "w"), indent=1)
    print(json.dumps(meta))


if __name__ == "__main__":
    main()
