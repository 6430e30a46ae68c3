#!/bin/bash
for d in U T; do for k in 32 256 1024; do
  printf "C2 %-2s k=%-4d " $d $k; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 4 --inner 20 | tail -1
done; done
timeout 120 python tools/run_knn.py --reps 3 | tail -1
timeout 1500 python -m pytest tests -m gpu -x -q -k "not slow" 2>&1 | tail -3
