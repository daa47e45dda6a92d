"""DRAM bytes (read + write) of the first kernel in an ncu --set full report, as the JSON that
bench.py reads for roofline.traffic.  python scripts/ncu_dram.py rep kernel_label source_note out.json"""
import csv
import io
import json
import subprocess
import sys

rep, label, note, out = sys.argv[1:5]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, first = rows[0], rows[1], rows[2]


def val(name):
    i = hdr.index(name)
    v = float(first[i].replace(",", ""))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(units[i], 1)
    return int(round(v * scale))


rd, wr = val("dram__bytes_read.sum"), val("dram__bytes_write.sum")
json.dump({"kernel": label, "source": note, "dram_bytes_read": rd, "dram_bytes_write": wr,
           "dram_bytes_per_launch": rd + wr}, open(out, "w"), indent=1)
print(open(out).read())
