#!/bin/bash
# Quick timing sweep (CUDA events) of ksel_select on the GPU box.
# usage: tools/perf_sweep.sh [algo...]   (default: 2)
algos=${@:-2}
for a in $algos; do
  for d in U SA SD T; do for k in 1 32 256 1024; do
    echo "== C2 algo=$a $d k=$k"; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 3 --algo $a | tail -1
  done; done
  echo "== C3 algo=$a U k=256"; timeout 120 python tools/run_select.py --Q 16384 --N 1048576 --k 256 --dist U --reps 3 --algo $a | tail -1
done
