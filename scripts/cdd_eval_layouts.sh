# CDD batched-eval layout sweep (CDD_EVAL2_GE=G:E overrides the automatic choice when G*E >= n)
for ge in 0:0 4:32 8:16 16:16 8:32 16:32 8:64 16:64; do echo "GE=$ge"; CDD_EVAL2_GE=$ge timeout 300 python scripts/eval_sweep.py --reps 5 100 128 200 256 300 500 2>&1 | cut -c1-150; done
