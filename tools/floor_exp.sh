#!/bin/bash
# where is the fused kNN kernel's floor?  MODE 4 = MMA pipeline, no TMEM reads; MODE 2 = + reads
for m in 4 2; do for p in 1 3; do
 echo "== mode $m passes $p"; KSEL_KNN_MODE=$m KSEL_KNN_PASSES=$p timeout 300 python tools/run_knn.py --reps 4 | tail -2
done; done
echo "== mode 2 passes 3 EW8"; KSEL_KNN_MODE=2 KSEL_KNN_EW=8 timeout 300 python tools/run_knn.py --reps 4 | tail -2
echo "== prof"; timeout 300 python tools/knn_prof.py
echo "== prof passes 1"; KSEL_KNN_PASSES=1 timeout 300 python tools/knn_prof.py
