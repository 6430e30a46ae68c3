#!/bin/bash
# compute-sanitizer over every product kernel (tools/sanitize_cases.py); logs -> gpurun_out/sanitize_*.txt
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  for sub in select radix merge knn; do
    timeout 900 $CS --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_cases.py $sub \
      > gpurun_out/sanitize_${tool}_${sub}.txt 2>&1
    echo "$tool $sub rc=$?" | tee -a gpurun_out/sanitize_summary.txt
  done
done
