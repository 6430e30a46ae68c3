#!/bin/bash
export KSEL_KNN_PAIR=1
timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== pipeline only 3-pass pair"; KSEL_KNN_MODE=2 timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== no-read 3-pass pair"; KSEL_KNN_MODE=4 timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== no-read 1-pass pair"; KSEL_KNN_MODE=4 KSEL_KNN_PASSES=1 timeout 120 python tools/run_knn.py --reps 4 | tail -1
