#!/bin/bash
# C2 k x distribution sweep: pool kernel (algo 2) vs cluster radix (algo 3)
for d in U DG SD T; do for k in 1 32 256 1024; do for a in 2 3; do
  printf "C2 %-2s k=%-4d algo=%d " $d $k $a; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 6 --algo $a | tail -1
done; done; done
for N in 4096 16384 32768; do for a in 2 3; do printf "Q=4096 N=%d k=256 algo=%d " $N $a; timeout 60 python tools/run_select.py --Q 4096 --N $N --k 256 --reps 6 --algo $a | tail -1; done; done
