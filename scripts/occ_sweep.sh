#!/bin/bash
# Headline SA throughput against the resident CTAs per SM (CDD_SA_OCC=k caps them; 4 warps each)
for k in 1 2 3 4; do
  echo -n "ctas_per_sm=$k warps_per_sm=$((4 * k)) "
  CDD_SA_OCC=$k python bench.py --steps 2 --warmup 3 --no-quality --no-configs --no-eval --no-cpu-baseline --no-e2e 2>/dev/null |
    python -c "import json,sys;d=json.loads(sys.stdin.read().strip().splitlines()[-1]);print('evals_per_s', round(d['value']), 'kernel_ms', round(d['roofline']['kernel_ms_avg'], 2))"
done
