# UCDDCP batched-eval layout sweep (CDD_EVAL2_UCD_GE=G:E overrides the automatic choice)
for ge in 8:16 16:16 8:32 16:32 32:32 16:64; do echo "GE=$ge"; CDD_EVAL2_UCD_GE=$ge timeout 300 python scripts/eval_sweep.py --problem ucddcp 100 200 500 1000 2>&1 | cut -c1-150; done
