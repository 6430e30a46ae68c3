#!/bin/bash
echo "== EW4"; timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== EW8"; KSEL_KNN_EW=8 timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== EW8 k=1024"; KSEL_KNN_EW=8 timeout 120 python tools/run_knn.py --reps 3 --k 1024 | tail -1
echo "== EW8 prof"; KSEL_KNN_EW=8 timeout 300 python tools/knn_prof.py | tail -12
