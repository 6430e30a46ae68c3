#!/bin/bash
# CTA-pair (cta_group::2) kNN: sanity, parity, timing
export KSEL_KNN_PAIR=1
timeout 120 python tools/knn_check.py; echo "check rc=$?"
timeout 120 python tools/run_knn.py --reps 5 --save gpurun_out/knn_pair.npz | tail -2; echo "run rc=$?"
KSEL_KNN_PAIR=0 timeout 120 python tools/run_knn.py --reps 5 --save gpurun_out/knn_nopair.npz | tail -2
python - <<PY
import numpy as np
a=np.load("gpurun_out/knn_nopair.npz"); b=np.load("gpurun_out/knn_pair.npz")
print("pair identical:", np.array_equal(a["i"],b["i"]) and np.array_equal(a["v"].view(np.uint32),b["v"].view(np.uint32)))
PY
echo "== pipeline only 3-pass pair"; KSEL_KNN_MODE=2 timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== pipeline only 1-pass pair"; KSEL_KNN_MODE=2 KSEL_KNN_PASSES=1 timeout 120 python tools/run_knn.py --reps 4 | tail -1
echo "== k=1024 pair"; timeout 120 python tools/run_knn.py --reps 3 --k 1024 | tail -1
timeout 900 python -m pytest tests/test_knn_gpu.py -x -q 2>&1 | tail -3
