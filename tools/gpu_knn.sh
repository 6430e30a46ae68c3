cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_knn_gpu.py -x -q -m "gpu and not slow" > gpurun_out/pytest_knn.log 2>&1; echo "pytest=$?"
for lib in libksel_A.so libksel.so; do for k in 100 1024; do echo "== $lib k=$k"; KSEL_AB_LIB=$lib timeout 300 python tools/run_knn.py --k $k --reps 3; done; done > gpurun_out/knn_time.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"knn|ksel" --csv --log-file gpurun_out/knn_launches.csv python tools/run_knn.py --reps 2 > /dev/null 2>&1; echo "ncu=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"knn|ksel" --csv --log-file gpurun_out/knn_launches_k1024.csv python tools/run_knn.py --reps 2 --k 1024 > /dev/null 2>&1; echo "ncu=$?"
