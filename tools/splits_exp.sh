#!/bin/bash
for s in 0 9 13 18; do echo "== k=1024 splits $s"; KSEL_KNN_SPLITS=$s timeout 120 python tools/run_knn.py --reps 3 --k 1024 | tail -1; done
for s in 0 13 18; do echo "== k=100 splits $s"; KSEL_KNN_SPLITS=$s timeout 120 python tools/run_knn.py --reps 3 | tail -1; done
