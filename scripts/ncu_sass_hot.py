"""Per-instruction execution counts of a kernel's SASS from an ncu report, normalised per unit.
python scripts/ncu_sass_hot.py rep units [min_ratio]"""
import csv
import io
import subprocess
import sys
from collections import Counter

rep, units = sys.argv[1], float(sys.argv[2])
lo = float(sys.argv[3]) if len(sys.argv) > 3 else 0.9
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
data = rows[2:]
ia, isrc = hdr.index("Instructions Executed"), hdr.index("Source")
iss = hdr.index("Warp Stall Sampling (All Samples)")
tot = 0
per = []
for r in data:
    c = int(r[ia]) if r[ia].isdigit() else 0
    tot += c
    per.append((c / units, int(r[iss]) if r[iss].isdigit() else 0, r[isrc].strip()))
print(f"total per unit {tot / units:.1f}")
hot = [p for p in per if p[0] >= lo]
print(f"instructions executed >= {lo}/unit: {len(hot)}  sum/unit {sum(p[0] for p in hot):.1f}")
ops = Counter(p[2].split()[0] if not p[2].startswith('@') else p[2].split()[1] for p in hot)
print(ops.most_common(30))
if "-v" in sys.argv:
    for p in per:
        if p[0] >= lo:
            print(f"{p[0]:6.2f} {p[1]:6d} {p[2][:80]}")
