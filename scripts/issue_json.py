"""profiles/sa_kernel_issue.json from an `ncu --page raw --metrics sass__inst_executed_per_opcode`
CSV of the headline SA launch: executed warp instructions per evaluation, total and per opcode.
python scripts/issue_json.py profiles/r2_sa_opcodes.csv EVALS_PER_LAUNCH > profiles/sa_kernel_issue.json"""
import csv
import json
import re
import sys


def main():
    path, evals = sys.argv[1], int(sys.argv[2])
    rows = [r for r in csv.reader(open(path)) if len(r) > 11 and r[0].isdigit()]
    # several launches of the same kernel (e.g. the bench step's four instances): averaged
    kname = rows[0][4]
    total, ops = 0, {}
    for r in rows:
        cell = r[11]
        total += int(cell.split()[0])
        for m in re.finditer(r"([A-Z0-9_.]+): (\d+)", cell):
            ops[m.group(1)] = ops.get(m.group(1), 0) + int(m.group(2))
    total /= len(rows)
    ops = {k: v / len(rows) for k, v in ops.items()}
    top = sorted(ops.items(), key=lambda kv: -kv[1])[:16]
    print(json.dumps({
        "kernel": kname.replace("void ", "").replace("(anonymous namespace)", "").replace("unnamed>::", ""),
        "executed_warp_instructions": total,
        "evals_per_launch": evals,
        "launches_averaged": len(rows),
        "warp_instr_per_eval": total / evals,
        "source": f"ncu --set full --clock-control none, sass__inst_executed_per_opcode ({path})",
        "per_opcode_per_eval": {k: round(v / evals, 2) for k, v in top},
    }, indent=1))


if __name__ == "__main__":
    main()
