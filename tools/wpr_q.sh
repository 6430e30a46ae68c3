#!/bin/bash
for k in 32 128 256 512; do for w in 1 2 4; do
  printf "C2 U k=%-4d wpr=%d " $k $w; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --reps 4 --inner 20 --algo 2 --wpr $w | tail -1
done; printf "C2 U k=%-4d auto  " $k; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --reps 4 --inner 20 | tail -1; done
