#!/bin/bash
# C2 (Q=1024, N=65536) k x distribution sweep of ksel_select (default algo), CUDA-event timing
for d in U G DG SA SD T; do for k in 1 8 32 128 256 1024; do
  printf "C2 %-2s k=%-4d " $d $k; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 5 | tail -1
done; done
