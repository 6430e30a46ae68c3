#!/bin/bash
for d in U T SD; do for k in 128 256 512 1024; do for w in 1 2 4 8; do
  printf "C2 %-2s k=%-4d wpr=%d " $d $k $w; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 5 --algo 2 --wpr $w | tail -1
done; done; done
