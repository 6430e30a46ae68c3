#!/bin/bash
for q in 1 2; do
echo "== qpc $q"; KSEL_KNN_QPC=$q timeout 120 python tools/run_knn.py --reps 4 --save gpurun_out/knn_ns$q.npz | tail -1
echo "== qpc $q pipeline-only"; KSEL_KNN_QPC=$q KSEL_KNN_MODE=2 timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== qpc $q no-read 1-pass"; KSEL_KNN_QPC=$q KSEL_KNN_MODE=4 KSEL_KNN_PASSES=1 timeout 120 python tools/run_knn.py --reps 4 | tail -1
done
python - <<PY
import numpy as np
a=np.load("gpurun_out/knn_q1.npz") if False else np.load("gpurun_out/knn_ns1.npz"); b=np.load("gpurun_out/knn_ns2.npz")
print("identical:", np.array_equal(a["i"],b["i"]) and np.array_equal(a["v"].view(np.uint32),b["v"].view(np.uint32)))
PY
