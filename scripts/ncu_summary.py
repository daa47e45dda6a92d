"""Summarise an ncu report (details page) into a few lines: python scripts/ncu_summary.py rep [evals]"""
import csv
import io
import subprocess
import sys

KEYS = ["Duration", "Elapsed Cycles", "SM Frequency", "DRAM Throughput", "Compute (SM) Throughput",
        "L1/TEX Cache Throughput", "L2 Cache Throughput", "Executed Ipc Active", "Issue Slots Busy",
        "Issued Instructions", "Registers Per Thread", "Achieved Active Warps Per SM",
        "Achieved Occupancy", "Warp Cycles Per Issued Instruction", "Eligible Warps Per Scheduler",
        "No Eligible", "Memory Throughput", "Mem Busy", "Max Bandwidth", "L1/TEX Hit Rate",
        "L2 Hit Rate", "Grid Size", "Block Limit Registers", "Block Limit Shared Mem",
        "Dynamic Shared Memory Per Block"]


def main():
    rep = sys.argv[1]
    evals = float(sys.argv[2]) if len(sys.argv) > 2 else None
    out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[0]
    iname, iunit, ival = hdr.index("Metric Name"), hdr.index("Metric Unit"), hdr.index("Metric Value")
    ik = hdr.index("Kernel Name")
    seen = set()
    for r in rows[1:]:
        if len(r) <= ival:
            continue
        k = (r[ik][:60], r[iname])
        if r[iname] in KEYS and k not in seen:
            seen.add(k)
            print(f"{r[iname]:40s} {r[ival]:>20s} {r[iunit]}")
            if r[iname] == "Issued Instructions" and evals:
                print(f"{'  -> warp instructions per eval':40s} {float(r[ival].replace(',', '')) / evals:>20.1f}")


if __name__ == "__main__":
    main()
