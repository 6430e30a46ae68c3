cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --error-exitcode 9 --print-limit 50 python tools/sanitize_cases.py knn > gpurun_out/sanitize_racecheck_knn.txt 2>&1; echo "racecheck knn rc=$?"
timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool synccheck --error-exitcode 9 python tools/sanitize_cases.py knn > gpurun_out/sanitize_synccheck_knn.txt 2>&1; echo "synccheck knn rc=$?"
timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize_cases.py knn > gpurun_out/sanitize_memcheck_knn.txt 2>&1; echo "memcheck knn rc=$?"
timeout 900 python -m pytest tests/test_knn_gpu.py tests/test_p2p_gpu.py tests/test_dist_gpu.py -q -m gpu > gpurun_out/pytest_knn.log 2>&1; echo "pytest=$?"
for k in 100 1024; do timeout 300 python tools/run_knn.py --k $k --reps 3; done > gpurun_out/knn_time.txt 2>&1
