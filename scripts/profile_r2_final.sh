#!/bin/bash
# Round-2 final evidence on the GPU box: the default bench line, per-row measurements, the ncu launch
# list of one bench step, the SA kernel's ncu summary and opcode mix (scripts/prof_sa.sh), ncu
# summaries of the batched evaluators, and the SA occupancy sweep (CTAs per SM).
set -x
mkdir -p gpurun_out
S=scripts
CDD_BENCH_WATCHDOG=800 python bench.py > gpurun_out/r2f_bench_full.json 2> gpurun_out/r2f_bench_full.err
python $S/row_bench.py > gpurun_out/r2f_rows.jsonl 2> gpurun_out/r2f_rows.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2f_launches.csv \
    python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-quality > /dev/null 2>&1
python $S/launch_summary.py gpurun_out/r2f_launches.csv > gpurun_out/r2f_launches_summary.txt 2>&1
LINES=60 bash $S/prof_sa.sh
cd gpurun_out
N="ncu --set full --clock-control none --import-source on"
$N -k regex:eval2 -s 1 -c 1 -o p_ev python ../$S/eval_sweep.py --reps 2 1000 > /dev/null 2>&1
$N -k regex:eval2 -s 1 -c 1 -o p_evu python ../$S/eval_sweep.py --problem ucddcp --reps 2 1000 > /dev/null 2>&1
{ python ../$S/ncu_summary.py p_ev.ncu-rep 1048576; echo; python ../$S/ncu_stalls.py p_ev.ncu-rep 25; echo; python ../$S/ncu_lines.py p_ev.ncu-rep 1048576 40; } > r2f_ncu_eval2_cdd_full.txt 2>&1
{ python ../$S/ncu_summary.py p_evu.ncu-rep 1048576; echo; python ../$S/ncu_stalls.py p_evu.ncu-rep 25; echo; python ../$S/ncu_lines.py p_evu.ncu-rep 1048576 40; } > r2f_ncu_eval2_ucddcp_full.txt 2>&1
rm -f *.ncu-rep
cd ..
for k in 3 4 5; do
  echo -n "ctas_per_sm=$k warps_per_sm=$((4 * k)) "
  CDD_SA_OCC=$k python bench.py --steps 2 --warmup 2 --no-quality --no-configs --no-eval --no-cpu-baseline --no-e2e 2>/dev/null |
    python -c "import json,sys;d=json.loads(sys.stdin.read().strip().splitlines()[-1]);print('evals_per_s', round(d['value']), 'kernel_ms', round(d['roofline']['kernel_ms_avg'], 2))"
done > gpurun_out/r2f_sa_occupancy.txt 2>&1
ls -la gpurun_out
