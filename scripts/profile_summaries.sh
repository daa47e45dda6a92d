#!/bin/bash
# On the GPU box after scripts/profile_round.sh: summaries of the ncu reports into gpurun_out/*.txt
# and the DRAM-bytes JSON, then the reports are removed (gpurun copies back at most 64 MiB).
cd gpurun_out
S=../scripts
{ python $S/ncu_summary.py prof_sa_full.ncu-rep 327680000; echo; python $S/ncu_stalls.py prof_sa_full.ncu-rep 25 2>/dev/null; echo; python $S/ncu_lines.py prof_sa_full.ncu-rep 327680000 40; } > sum_sa.txt 2>&1
{ python $S/ncu_summary.py prof_eval_full.ncu-rep 1048576; echo; python $S/ncu_stalls.py prof_eval_full.ncu-rep 25 2>/dev/null; echo; python $S/ncu_lines.py prof_eval_full.ncu-rep 1048576 40; } > sum_eval.txt 2>&1
{ python $S/ncu_summary.py prof_eval_ucd_full.ncu-rep 1048576; echo; python $S/ncu_stalls.py prof_eval_ucd_full.ncu-rep 25 2>/dev/null; echo; python $S/ncu_lines.py prof_eval_ucd_full.ncu-rep 1048576 40; } > sum_eval_ucd.txt 2>&1
python $S/ncu_dram.py prof_sa_full.ncu-rep "sa_group_kernel<8,128> (CDD)" "profiles/r1b_ncu_sa_full.txt (ncu --set full, bench config 5 launch)" sa_dram.json > /dev/null 2>&1
python $S/ncu_dram.py prof_eval_full.ncu-rep "eval2_kernel<16,64> (CDD n=1000)" "profiles/r1b_ncu_eval2_cdd_full.txt (ncu --set full, eval_sweep n=1000, 2^20 rows)" eval_dram.json > /dev/null 2>&1
rm -f *.ncu-rep
ls -la
