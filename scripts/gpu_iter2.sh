# GPU iteration: SA/DPSO/sync parity tests, the default bench line, per-row measurements
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sa.py tests/test_gpu_sync.py tests/test_gpu_dpso.py tests/test_gpu_sa_init.py -x -q > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_iter.log
CDD_BENCH_WATCHDOG=600 timeout 700 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; tail -3 gpurun_out/bench.err
python -c "import json; d=json.load(open('gpurun_out/bench.json')); print(d['value'], d['roofline']['frac'], d['cpu_baseline']['cores'], d['e2e']['value'])"
timeout 600 python scripts/row_bench.py > gpurun_out/rows.jsonl 2> gpurun_out/rows.err; echo "rows rc=$?"
cut -c1-160 gpurun_out/rows.jsonl
