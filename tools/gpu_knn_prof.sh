cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:knn_fused -s 1 -c 1 -o gpurun_out/knn_prof python tools/run_knn.py --reps 2 > gpurun_out/knn_prof.log 2>&1; echo "ncu=$?"
ncu -i gpurun_out/knn_prof.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/knn_src.csv 2>/dev/null
ncu -i gpurun_out/knn_prof.ncu-rep --page raw --csv > gpurun_out/knn_raw.csv 2>/dev/null
rm -f gpurun_out/knn_prof.ncu-rep
