#!/bin/bash
for d in U T SD; do printf "C3 %s k=1024 " $d; timeout 120 python tools/run_select.py --Q 16384 --N 1048576 --k 1024 --dist $d --reps 3 | tail -1; done
for d in U T SD; do printf "C2 %s k=1024 " $d; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k 1024 --dist $d --reps 4 --inner 20 | tail -1; done
