#!/bin/bash
# C3 shape (Q=16384, N=2^20) per distribution and k
for d in U G DG SA SD T; do for k in 32 256 1024; do
  printf "C3 %-2s k=%-4d " $d $k; timeout 120 python tools/run_select.py --Q 16384 --N 1048576 --k $k --dist $d --reps 3 | tail -1
done; done
