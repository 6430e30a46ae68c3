# ncu --set full capture of the main kNN filter launch + SASS-level hot spots and the raw SASS listing
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:knn_fused -s 1 -c 1 -o gpurun_out/knn_sass python tools/run_knn.py --reps 1 --k 100 > gpurun_out/knn_sass.log 2>&1; echo "ncu=$?"
python tools/ncu_sass_hot.py gpurun_out/knn_sass.ncu-rep 40 > gpurun_out/knn_sass_hot.txt 2>&1
ncu -i gpurun_out/knn_sass.ncu-rep --page source --csv --print-source sass > gpurun_out/knn_sass_full.csv 2>/dev/null
rm -f gpurun_out/knn_sass.ncu-rep
