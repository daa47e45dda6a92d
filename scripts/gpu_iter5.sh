mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sa.py -x -q -k "nibble or insert or move" > gpurun_out/pytest_ins.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_ins.log
timeout 600 python -m pytest tests/test_gpu_sync.py -x -q 2>&1 | tail -2
python scripts/row_bench.py S4 2>/dev/null | cut -c1-200
