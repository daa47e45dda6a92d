mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sa.py -x -q > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_iter.log
for i in 1 2; do python bench.py --steps 3 --warmup 2 --no-quality --no-configs --no-eval --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys;d=json.loads(sys.stdin.read().strip().splitlines()[-1]);print('evals_per_s', round(d['value']), 'kernel_ms', round(d['roofline']['kernel_ms_avg'], 2))"; done
