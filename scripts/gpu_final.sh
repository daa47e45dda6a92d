# final state: every -m gpu test, smoke, the default bench line and the per-row measurements
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
CDD_BENCH_WATCHDOG=800 timeout 900 python bench.py > gpurun_out/r2f_bench_full.json 2> gpurun_out/r2f_bench_full.err; echo "bench rc=$?"
python -c "import json; d=json.load(open('gpurun_out/r2f_bench_full.json')); print(d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks'])"
timeout 900 python scripts/row_bench.py > gpurun_out/r2f_rows.jsonl 2> gpurun_out/r2f_rows.err; echo "rows rc=$?"
cut -c1-170 gpurun_out/r2f_rows.jsonl
