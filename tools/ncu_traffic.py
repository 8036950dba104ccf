"""Per-launch DRAM traffic of the heavy kernels from an ncu CSV (metrics dram__bytes_read.sum,
dram__bytes_write.sum, gpu__time_duration.sum; --print-units base) -> profiles/ncu_traffic.json,
the file bench.py reads for roofline.traffic.

  python tools/ncu_traffic.py gpurun_out/traffic.csv --key C3:f64 [--out profiles/ncu_traffic.json]
"""
import argparse
import csv
import json
import os
import re
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def parse(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    per = defaultdict(dict)  # (launch id, kernel) -> metric -> value
    for r in csv.DictReader(lines[start:]):
        k = re.sub(r"^void ", "", r["Kernel Name"]).split("<")[0].split("(")[0].split("::")[-1]
        v = float(r["Metric Value"].replace(",", ""))
        v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
              "nsecond": 1, "ns": 1, "usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6}.get(r.get("Metric Unit", ""), 1)
        per[(int(r["ID"]), k)][r["Metric Name"]] = v
    return per


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csv")
    ap.add_argument("--key", required=True, help="config:dtype, e.g. C3:f64")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "ncu_traffic.json"))
    a = ap.parse_args()
    per = parse(a.csv)
    agg = defaultdict(list)
    for (_, k), m in sorted(per.items()):
        if "dram__bytes_read.sum" in m:
            agg[k].append((m["dram__bytes_read.sum"] + m.get("dram__bytes_write.sum", 0.0),
                           m.get("gpu__time_duration.sum", 0.0)))
    d = json.load(open(a.out)) if os.path.exists(a.out) else {}
    for k, xs in agg.items():
        d[f"{a.key}:{k}"] = sum(x[0] for x in xs) / len(xs)
        d[f"{a.key}:{k}:ncu_ns"] = sum(x[1] for x in xs) / len(xs)
        print(f"{k}: {len(xs)} launch(es), {d[f'{a.key}:{k}'] / 1e9:.3f} GB DRAM per launch, "
              f"{d[f'{a.key}:{k}:ncu_ns'] / 1e6:.2f} ms under ncu")
    d["_source"] = "ncu --replay-mode application --metrics dram__bytes_read.sum,dram__bytes_write.sum," \
                   "gpu__time_duration.sum on the bench command (bytes per launch)"
    json.dump(d, open(a.out, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
