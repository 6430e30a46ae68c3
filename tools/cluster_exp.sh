#!/bin/bash
# kNN cluster-multicast experiment: C4 timing per cluster size, bit-identity vs cs=1, pipeline-only floors
mkdir -p gpurun_out
for c in 1 2 4; do
  echo "== cluster $c"; KSEL_KNN_CLUSTER=$c timeout 300 python tools/run_knn.py --reps 5 --save gpurun_out/knn_c$c.npz
done
for c in 2 4; do
python - <<PY
import numpy as np
a=np.load("gpurun_out/knn_c1.npz"); b=np.load("gpurun_out/knn_c$c.npz")
print("cluster $c identical:", np.array_equal(a["i"],b["i"]) and np.array_equal(a["v"].view(np.uint32),b["v"].view(np.uint32)))
PY
done
for c in 2 4; do
echo "== cluster $c passes=1 pipeline only"; KSEL_KNN_CLUSTER=$c KSEL_KNN_MODE=2 KSEL_KNN_PASSES=1 timeout 300 python tools/run_knn.py --reps 4
echo "== cluster $c passes=3 pipeline only"; KSEL_KNN_CLUSTER=$c KSEL_KNN_MODE=2 timeout 300 python tools/run_knn.py --reps 4
done
echo "== cluster 2 passes=1 full (inexact)"; KSEL_KNN_PASSES=1 timeout 300 python tools/run_knn.py --reps 4
echo "== k=1024"; timeout 300 python tools/run_knn.py --reps 3 --k 1024
timeout 900 python -m pytest tests/test_knn_gpu.py -q -x 2>&1 | tail -5
