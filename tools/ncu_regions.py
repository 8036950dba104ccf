"""Stall-reason breakdown of an ncu report's SASS source page over instruction-index regions.
  python tools/ncu_regions.py rep.ncu-rep [a:b ...]"""
import csv, subprocess, sys

rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
r = list(csv.reader(out.splitlines()))
h = r[1]
rows = r[2:]
reasons = [x for x in h if x.startswith("stall_") and "Not Issued" not in x]
regions = [tuple(map(int, a.split(":"))) for a in sys.argv[2:]] or [(0, len(rows))]
for a, b in regions:
    tot = {k: sum(int(x[h.index(k)] or 0) for x in rows[a:b] if len(x) > h.index(k)) for k in reasons}
    s = sum(tot.values())
    print(f"[{a},{b}) samples {s}: " + " ".join(f"{k[6:]}={v}" for k, v in sorted(tot.items(), key=lambda kv: -kv[1]) if v > 0.02 * s))
