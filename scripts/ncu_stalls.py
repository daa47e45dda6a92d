"""Top stalled SASS instructions of an ncu report with their dominant stall reasons.
python scripts/ncu_stalls.py rep [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
# the first kernel of the report only (a report of several launches repeats the header)
data = []
for r in rows[2:]:
    if len(r) < len(hdr) or r == hdr:
        break
    data.append(r)
isrc = hdr.index("Source")
scols = [i for i, c in enumerate(hdr) if c.startswith("stall_") and "Not Issued" not in c]
tot_by = {hdr[i]: 0 for i in scols}
lines = []
for idx, r in enumerate(data):
    vals = {hdr[i]: int(r[i]) if r[i].isdigit() else 0 for i in scols}
    for k, v in vals.items():
        tot_by[k] += v
    s = sum(vals.values())
    lines.append((s, idx, r[isrc].strip()[:60], sorted(vals.items(), key=lambda kv: -kv[1])[:2]))
T = sum(tot_by.values())
print("stall totals:", ", ".join(f"{k[6:]}={100*v/T:.1f}%" for k, v in sorted(tot_by.items(), key=lambda kv: -kv[1]) if v))
for s, idx, src, tops in sorted(lines, reverse=True)[:top]:
    print(f"{100*s/T:5.1f}% #{idx:5d} {src:60s} {tops[0][0][6:]}:{tops[0][1]} {tops[1][0][6:]}:{tops[1][1]}")
