# A/B of the kNN path on one box: tests of the current library, then both libraries timed
# alternately at k = 100 and 1024, then the ncu launch list of the current one.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_knn_gpu.py -x -q -m "gpu" > gpurun_out/pytest_knn.log 2>&1; echo "pytest=$?"
for k in 100 1024; do for lib in libksel_A.so libksel.so libksel_A.so libksel.so; do echo "== $lib k=$k"; KSEL_AB_LIB=$lib timeout 300 python tools/run_knn.py --k $k --reps 3; done; done > gpurun_out/knn_time.txt 2>&1
for k in 100 1024; do
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"knn|ksel" --csv --log-file gpurun_out/knn_launches_k$k.csv python tools/run_knn.py --reps 2 --k $k > /dev/null 2>&1; echo "ncu=$?"
done
