# quick GPU iteration: selected tests + per-row measurements
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_eval.py tests/test_gpu_sync.py tests/test_gpu_dist.py -x -q > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_iter.log
timeout 600 python scripts/row_bench.py > gpurun_out/rows.jsonl 2> gpurun_out/rows.err; echo "rows rc=$?"
cut -c1-250 gpurun_out/rows.jsonl
