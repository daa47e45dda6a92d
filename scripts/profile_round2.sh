#!/bin/bash
# Round 2 evidence on the GPU box (gpurun): the bench line, per-row measurements, the ncu launch list
# of a bench step, ncu --set full captures (summarised here, reports removed) of the headline SA
# kernel, the batched evaluators, the group DPSO kernel and both schedule kernels, the SA
# instruction mix per opcode, and the SA occupancy sweep.
set -x
mkdir -p gpurun_out
S=scripts
python bench.py --steps 3 --warmup 3 > gpurun_out/r2_bench_full.json 2> gpurun_out/r2_bench_full.err
python $S/row_bench.py > gpurun_out/r2_rows.jsonl 2> gpurun_out/r2_rows.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_launches.csv \
    python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-quality > /dev/null 2>&1
cd gpurun_out
N="ncu --set full --clock-control none --import-source on"
$N -k regex:sa_group -c 1 -o p_sa python ../bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-eval --no-configs --no-quality > /dev/null 2>&1
$N -k regex:eval2 -s 1 -c 1 -o p_ev python ../$S/eval_sweep.py --reps 2 1000 > /dev/null 2>&1
$N -k regex:eval2 -s 1 -c 1 -o p_evu python ../$S/eval_sweep.py --problem ucddcp --reps 2 1000 > /dev/null 2>&1
$N -k regex:dpsog_iter -c 1 -o p_dp python ../$S/dpso_time.py 500 > /dev/null 2>&1
$N -k regex:schedule -s 1 -c 1 -o p_sch python ../$S/row_bench.py F1 > /dev/null 2>&1
$N --kernel-name-base demangled -k "regex:schedule_kernel<.bool.1" -s 1 -c 1 -o p_schu python ../$S/row_bench.py F1 > /dev/null 2>&1
{ python ../$S/ncu_summary.py p_sa.ncu-rep 327745536; echo; python ../$S/ncu_stalls.py p_sa.ncu-rep 25; echo; python ../$S/ncu_lines.py p_sa.ncu-rep 327745536 40; } > r2_ncu_sa_full.txt 2>&1
{ python ../$S/ncu_summary.py p_ev.ncu-rep 1048576; echo; python ../$S/ncu_stalls.py p_ev.ncu-rep 25; echo; python ../$S/ncu_lines.py p_ev.ncu-rep 1048576 40; } > r2_ncu_eval2_cdd_full.txt 2>&1
{ python ../$S/ncu_summary.py p_evu.ncu-rep 1048576; echo; python ../$S/ncu_stalls.py p_evu.ncu-rep 25; echo; python ../$S/ncu_lines.py p_evu.ncu-rep 1048576 40; } > r2_ncu_eval2_ucddcp_full.txt 2>&1
{ python ../$S/ncu_summary.py p_dp.ncu-rep 1638400; echo; python ../$S/ncu_stalls.py p_dp.ncu-rep 25; echo; python ../$S/ncu_lines.py p_dp.ncu-rep 1638400 40 --by-stall; } > r2_ncu_dpso_group_n500.txt 2>&1
{ python ../$S/ncu_summary.py p_sch.ncu-rep 131072; echo; python ../$S/ncu_stalls.py p_sch.ncu-rep 25; echo; python ../$S/ncu_lines.py p_sch.ncu-rep 131072 40; } > r2_ncu_schedule_full.txt 2>&1
{ python ../$S/ncu_summary.py p_schu.ncu-rep 131072; echo; python ../$S/ncu_stalls.py p_schu.ncu-rep 25; echo; python ../$S/ncu_lines.py p_schu.ncu-rep 131072 40; } > r2_ncu_schedule_ucddcp_full.txt 2>&1
python ../$S/ncu_dram.py p_sa.ncu-rep "sa_group_kernel<8,128> (CDD, byte rows)" "profiles/r2_ncu_sa_full.txt (ncu --set full, bench config 5 launch)" r2_sa_dram.json > /dev/null 2>&1
python ../$S/ncu_dram.py p_ev.ncu-rep "eval2_kernel<16,64> (CDD n=1000)" "profiles/r2_ncu_eval2_cdd_full.txt (ncu --set full, eval_sweep n=1000, 2^20 rows)" r2_eval_dram.json > /dev/null 2>&1
ncu -i p_sa.ncu-rep --page raw --csv --metrics sass__inst_executed_per_opcode --print-metric-instances details > r2_sa_opcodes.csv 2>&1
rm -f *.ncu-rep
python ../$S/issue_json.py r2_sa_opcodes.csv 327745536 > r2_sa_issue.json 2>&1
python ../$S/launch_summary.py r2_launches.csv > r2_launches_summary.txt 2>&1
cd ..
bash $S/occ_sweep.sh > gpurun_out/r2_sa_occupancy.txt 2>&1
cd gpurun_out
ls -la
