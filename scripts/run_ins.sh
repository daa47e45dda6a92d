mkdir -p gpurun_out
cd gpurun_out
N="ncu --set full --clock-control none --import-source on --kernel-name-base demangled"
$N -k "regex:sa_group_kernel<.int.8, .int.128, .bool.0, .bool.0, .int.1>" -c 1 -o p_ins python ../scripts/row_bench.py S4 > ncu_ins.log 2>&1
{ python ../scripts/ncu_summary.py p_ins.ncu-rep 65601536; echo; python ../scripts/ncu_stalls.py p_ins.ncu-rep 25; echo; python ../scripts/ncu_lines.py p_ins.ncu-rep 65601536 50; } > r2_ncu_sa_insert_full.txt 2>&1
$N -k "regex:schedule_kernel<.bool.1" -s 1 -c 1 -o p_schu python ../scripts/row_bench.py F1 > ncu_schu.log 2>&1
{ python ../scripts/ncu_summary.py p_schu.ncu-rep 131072; echo; python ../scripts/ncu_stalls.py p_schu.ncu-rep 25; echo; python ../scripts/ncu_lines.py p_schu.ncu-rep 131072 40; } > r2_ncu_schedule_ucddcp_full.txt 2>&1
rm -f *.ncu-rep
