cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python tools/knn_counters.py > gpurun_out/knn_ctr.txt 2>&1; echo "ctr=$?"
for lib in libksel_A.so libksel.so; do echo "== $lib"; KSEL_AB_LIB=$lib timeout 300 python tools/run_knn.py --reps 3; done > gpurun_out/knn_ab.txt 2>&1
