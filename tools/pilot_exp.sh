#!/bin/bash
# kNN pilot-launch experiment: C4 timing per pilot stride + bit-identity vs no pilot
mkdir -p gpurun_out
for p in 0 8 16 32 64; do
  echo "== pilot $p"; KSEL_KNN_PILOT=$p timeout 300 python tools/run_knn.py --reps 6 --save gpurun_out/knn_p$p.npz
done
for p in 8 16 32 64; do
python - <<PY
import numpy as np
a=np.load("gpurun_out/knn_p0.npz"); b=np.load("gpurun_out/knn_p$p.npz")
print("pilot $p identical:", np.array_equal(a["i"],b["i"]) and np.array_equal(a["v"].view(np.uint32),b["v"].view(np.uint32)))
PY
done
echo "== passes=1 pipeline only"; KSEL_KNN_MODE=2 KSEL_KNN_PASSES=1 timeout 300 python tools/run_knn.py --reps 4
echo "== passes=3 pipeline only"; KSEL_KNN_MODE=2 timeout 300 python tools/run_knn.py --reps 4
echo "== passes=1 full (inexact)"; KSEL_KNN_PASSES=1 KSEL_KNN_PILOT=16 timeout 300 python tools/run_knn.py --reps 4
echo "== k=1024 pilot 0/16"; timeout 300 python tools/run_knn.py --reps 3 --k 1024; KSEL_KNN_PILOT=16 timeout 300 python tools/run_knn.py --reps 3 --k 1024
timeout 900 python -m pytest tests/test_knn_gpu.py -q -x -k "pilot" 2>&1 | tail -5
