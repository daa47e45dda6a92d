#!/bin/bash
# Runs on the GPU box (gpurun): bench line, per-row measurements, launch list, and full ncu
# captures of the top kernels (SA group kernel, CDD and UCDDCP batched evaluation, DPSO iteration).
set -x
mkdir -p gpurun_out
python bench.py --steps 3 --warmup 3 > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
python scripts/row_bench.py > gpurun_out/rows.jsonl 2> gpurun_out/rows.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:sa_group -c 1 -o gpurun_out/prof_sa_full \
    python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-eval --no-configs > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:eval2 -s 1 -c 1 -o gpurun_out/prof_eval_full \
    python scripts/eval_sweep.py --reps 2 1000 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:eval2 -s 1 -c 1 -o gpurun_out/prof_eval_ucd_full \
    python scripts/eval_sweep.py --problem ucddcp --reps 2 1000 > /dev/null 2>&1
ls -la gpurun_out
