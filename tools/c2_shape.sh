#!/bin/bash
# fixed-cost vs streaming: ksel_select time over N, Q and warps per row
for k in 1 256; do
 for N in 16384 65536 262144; do printf "Q=1024 N=%-7d k=%-4d " $N $k; timeout 60 python tools/run_select.py --Q 1024 --N $N --k $k --reps 8 | tail -1; done
 printf "Q=4096 N=65536 k=%-4d " $k; timeout 60 python tools/run_select.py --Q 4096 --N 65536 --k $k --reps 8 | tail -1
 for w in 1 2 4 8; do printf "C2 k=%-4d wpr=%d " $k $w; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --reps 8 --wpr $w --algo 2 | tail -1; done
done
