mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_eval.py -x -q > gpurun_out/pytest_eval.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_eval.log
timeout 300 python scripts/eval_sweep.py --problem ucddcp 50 100 200 500 1000 > gpurun_out/ucd_new.jsonl
CDD_EVAL2_NO_UCD=1 timeout 300 python scripts/eval_sweep.py --problem ucddcp 50 100 200 500 1000 > gpurun_out/ucd_old.jsonl
timeout 300 python scripts/eval_sweep.py 1000 > gpurun_out/cdd_1000.jsonl
cat gpurun_out/ucd_new.jsonl gpurun_out/ucd_old.jsonl gpurun_out/cdd_1000.jsonl
