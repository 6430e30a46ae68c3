#!/bin/bash
# two query tiles per CTA (BN = 128): timing, bit-identity vs QPC=1, parity
KSEL_KNN_QPC=1 timeout 120 python tools/run_knn.py --reps 4 --save gpurun_out/knn_q1.npz | tail -1
KSEL_KNN_QPC=2 timeout 120 python tools/run_knn.py --reps 4 --save gpurun_out/knn_q2.npz | tail -1
python - <<PY
import numpy as np
a=np.load("gpurun_out/knn_q1.npz"); b=np.load("gpurun_out/knn_q2.npz")
print("qpc identical:", np.array_equal(a["i"],b["i"]) and np.array_equal(a["v"].view(np.uint32),b["v"].view(np.uint32)))
PY
echo "== qpc2 pipeline-only"; KSEL_KNN_QPC=2 KSEL_KNN_MODE=2 timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== qpc2 no-read 1-pass"; KSEL_KNN_QPC=2 KSEL_KNN_MODE=4 KSEL_KNN_PASSES=1 timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== qpc2 k=1024"; KSEL_KNN_QPC=2 timeout 120 python tools/run_knn.py --reps 3 --k 1024 | tail -1
echo "== qpc2 knn-S"; KSEL_KNN_QPC=2 timeout 120 python tools/run_knn.py --reps 3 --kind knn-S | tail -1
KSEL_KNN_QPC=2 timeout 900 python -m pytest tests/test_knn_gpu.py -q -x 2>&1 | tail -3
