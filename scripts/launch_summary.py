"""Per-kernel share of an ncu launch list (--metrics gpu__time_duration.sum --csv).
python scripts/launch_summary.py launches.csv [header line ...]"""
import csv
import io
import sys
from collections import defaultdict

path = sys.argv[1]
lines = [ln for ln in open(path) if ln.startswith('"')]
rows = list(csv.reader(io.StringIO("".join(lines))))
hdr = rows[0]
ik, iv, iu = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
tot, cnt = defaultdict(float), defaultdict(int)
for r in rows[1:]:
    scale = {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}.get(r[iu], 1e-6)
    name = r[ik].split("(")[0][:90]
    tot[name] += float(r[iv].replace(",", "")) * scale
    cnt[name] += 1
allt = sum(tot.values())
for h in sys.argv[2:]:
    print(h)
for name, t in sorted(tot.items(), key=lambda kv: -kv[1]):
    print(f"{100 * t / allt:6.2f}%  {t:10.3f} ms  x {cnt[name]:3d}  {name}")
