#!/bin/bash
for w in 1 2 4 8; do for k in 32 256 1024; do
  echo "== wpr=$w k=$k"; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist U --reps 3 --algo 2 --wpr $w | tail -1
done; done
