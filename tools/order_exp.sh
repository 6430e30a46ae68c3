#!/bin/bash
# chunk-order experiment: same box, same binary, KSEL_ORDER = 0/1/2
for rep in 1 2; do for o in 0 1 2; do
  echo "== order=$o C3 U"; KSEL_ORDER=$o timeout 120 python tools/run_select.py --Q 16384 --N 1048576 --k 256 --dist U --reps 3 --algo 2 | tail -1
done; done
for o in 0 1 2; do for d in U SD; do
  echo "== order=$o C2 $d k=256"; KSEL_ORDER=$o timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k 256 --dist $d --reps 3 --algo 2 | tail -1
done; done
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv
