# the kNN / distributed / P2P GPU test files on one box
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_knn_gpu.py tests/test_dist_gpu.py tests/test_p2p_gpu.py -q -m gpu --durations=8 > gpurun_out/pytest_knnall.log 2>&1; echo "pytest=$?"
