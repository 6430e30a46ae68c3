timeout 600 python -m pytest tests/test_knn_gpu.py -m gpu -x -q 2>&1 | tail -2
KSEL_KNN_EW=8 timeout 600 python -m pytest tests/test_knn_gpu.py -m gpu -x -q 2>&1 | tail -2
for ew in 4 8; do for cap in 0 256 384 512 768; do
  echo "EW=$ew cap=$cap $(KSEL_KNN_EW=$ew KSEL_KNN_SOFTCAP=$cap python tools/run_knn.py --reps 3 | tail -1)"
done; done
