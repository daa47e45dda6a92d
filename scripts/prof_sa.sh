# ncu of the headline SA kernel: --set full of the first launch of a bench step (h = 0.2: summary,
# stalls, per-line counts), the opcode mix averaged over the step's four launches (h = 0.2 .. 0.8)
mkdir -p gpurun_out; cd gpurun_out
N="ncu --set full --clock-control none --import-source on"
B="../bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-eval --no-configs --no-quality"
$N -k regex:sa_group -c 1 -o p_sa python $B > /dev/null 2>&1
ncu --clock-control none --metrics sass__inst_executed_per_opcode -k regex:sa_group -c 4 -o p_sa4 python $B > /dev/null 2>&1
{ python ../scripts/ncu_summary.py p_sa.ncu-rep 327745536; echo; python ../scripts/ncu_stalls.py p_sa.ncu-rep 25; echo; python ../scripts/ncu_lines.py p_sa.ncu-rep 327745536 ${LINES:-40}; } > sa_full.txt 2>&1
ncu -i p_sa4.ncu-rep --page raw --csv --metrics sass__inst_executed_per_opcode --print-metric-instances details > sa_opcodes.csv 2>&1
python ../scripts/issue_json.py sa_opcodes.csv 327745536 > sa_issue.json 2>&1
python ../scripts/ncu_dram.py p_sa.ncu-rep "sa_group_kernel<8,128> (CDD, 4-bit weights + sub-block summaries)" "profiles/r2_ncu_sa_full.txt (ncu --set full, bench config 5 launch)" sa_dram.json > /dev/null 2>&1
rm -f p_sa.ncu-rep p_sa4.ncu-rep
cat sa_issue.json | head -8
