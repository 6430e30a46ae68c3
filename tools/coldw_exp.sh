#!/bin/bash
for c in 1000 500 300 200 125; do
  echo "== coldw $c"; KSEL_KNN_COLDW=$c timeout 300 python tools/run_knn.py --reps 5 --save gpurun_out/knn_w$c.npz | tail -2
done
for c in 500 300 200 125; do
python - <<PY
import numpy as np
a=np.load("gpurun_out/knn_w1000.npz"); b=np.load("gpurun_out/knn_w$c.npz")
print("coldw $c identical:", np.array_equal(a["i"],b["i"]) and np.array_equal(a["v"].view(np.uint32),b["v"].view(np.uint32)))
PY
done
for c in 300; do echo "== k=1024 coldw $c"; KSEL_KNN_COLDW=$c timeout 300 python tools/run_knn.py --reps 3 --k 1024 | tail -1; done
echo "== k=1024 coldw 1000"; timeout 300 python tools/run_knn.py --reps 3 --k 1024 | tail -1
