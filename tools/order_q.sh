#!/bin/bash
for d in SD SA U T; do for k in 1 32 256 1024; do
  printf "C2 %-2s k=%-4d " $d $k; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 4 --inner 20 | tail -1
done; done
for d in U SD; do printf "C3 %s k=256 " $d; timeout 120 python tools/run_select.py --Q 16384 --N 1048576 --k 256 --dist $d --reps 3 | tail -1; done
timeout 900 python -m pytest tests/test_ksel_gpu.py -q -x 2>&1 | tail -1
