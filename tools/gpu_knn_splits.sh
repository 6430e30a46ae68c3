cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for k in 100 1024; do for S in 0 2 3 4 6 8 12 16; do echo "== k=$k S=$S"; KSEL_KNN_SPLITS=$S timeout 300 python tools/run_knn.py --k $k --reps 2 | tail -1; done; done > gpurun_out/knn_splits.txt 2>&1
