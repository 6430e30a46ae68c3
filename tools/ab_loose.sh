#!/bin/bash
for rep in 1 2; do for L in 0 1; do for d in U T; do for k in 1 256; do
  echo "== loose=$L $d k=$k"; KSEL_LOOSE=$L timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 3 --algo 2 | tail -1
done; done; done; done
for L in 0 1; do echo "== loose=$L C3"; KSEL_LOOSE=$L timeout 120 python tools/run_select.py --Q 16384 --N 1048576 --k 256 --dist U --reps 3 --algo 2 | tail -1; done
