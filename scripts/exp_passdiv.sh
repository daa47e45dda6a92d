# timing experiment: SA kernel with 1/4 of the quad pass (exp/libcdd_pd4.so, wrong results) vs the
# product library, at 12 and 16 warps per SM
mkdir -p gpurun_out
for lib in "" exp/libcdd_pd4.so; do
 for k in 3 4; do
  echo -n "lib=${lib:-product} ctas_per_sm=$k "
  CDD_LIB=${lib:+$PWD/$lib} CDD_SA_OCC=$k python bench.py --steps 2 --warmup 2 --no-quality --no-configs --no-eval --no-cpu-baseline --no-e2e 2>/dev/null |
    python -c "import json,sys;d=json.loads(sys.stdin.read().strip().splitlines()[-1]);print('evals_per_s', round(d['value']), 'kernel_ms', round(d['roofline']['kernel_ms_avg'], 2))"
 done
done
timeout 600 python -m pytest tests/test_gpu_eval.py -x -q -k "ucddcp or UCD or ucd" 2>&1 | tail -2
python scripts/row_bench.py A6 2>/dev/null | cut -c1-200
