"""Instructions executed and stall samples per CUDA source line of the first kernel in an ncu
report (needs -lineinfo and --import-source on), normalised per unit.
python scripts/ncu_lines.py rep units [top] [--by-stall]"""
import csv
import io
import subprocess
import sys

rep, units = sys.argv[1], float(sys.argv[2])
top = int(sys.argv[3]) if len(sys.argv) > 3 else 60
by_stall = "--by-stall" in sys.argv
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = []
fname, hdr = "?", None
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] in ("File Path", "File Name"):
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or not r[0].isdigit():
        continue
    ie = hdr.index("Instructions Executed")
    ws = hdr.index("Warp Stall Sampling (All Samples)")
    try:
        n = int(r[ie])
    except ValueError:
        continue
    if n:
        rows.append((n / units, int(r[ws]) if r[ws].isdigit() else 0, f"{fname}:{r[0]}", r[1].strip()))
tot = sum(x[0] for x in rows)
stot = sum(x[1] for x in rows) or 1
print(f"total instructions per unit {tot:.1f}")
for n, s, loc, src in sorted(rows, key=lambda x: x[1] if by_stall else x[0], reverse=True)[:top]:
    print(f"{n:7.2f} {100 * s / stot:5.1f}% {loc:22s} {src[:90]}")
