#!/bin/bash
for d in U DG SD T; do for k in 1 32 128 256 1024; do
  printf "C2 %-2s k=%-4d " $d $k; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 4 --inner 20 | tail -1
done; done
