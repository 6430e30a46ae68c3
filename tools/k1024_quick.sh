#!/bin/bash
for k in 256 1024; do printf "C3 U k=%-4d " $k; timeout 120 python tools/run_select.py --Q 16384 --N 1048576 --k $k --reps 3 | tail -1; done
tools/c2_quick.sh
