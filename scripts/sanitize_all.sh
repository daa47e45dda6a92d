#!/bin/bash
# compute-sanitizer over every kernel family (scripts/sanitize.py); summary in gpurun_out/sanitizer.txt
mkdir -p gpurun_out
out=gpurun_out/sanitizer.txt
echo "compute-sanitizer --tool {memcheck,racecheck,synccheck,initcheck} --error-exitcode 9 python scripts/sanitize.py" > $out
for t in memcheck racecheck synccheck initcheck; do
  echo "== $t" >> $out
  timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool $t --error-exitcode 9 python scripts/sanitize.py 2>&1 | grep -E "sanitize run ok|SUMMARY|Invalid|Race|hazard|Error|error" | head -20 >> $out
  echo "rc=${PIPESTATUS[0]}" >> $out
done
cat $out
