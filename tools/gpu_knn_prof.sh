# ncu --set full capture of the main knn_fused launch (the 2nd fused launch: after the speculative pre-pass)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
K=${1:-100}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:knn_fused -s 1 -c 1 -o gpurun_out/knn_prof python tools/run_knn.py --reps 1 --k $K > gpurun_out/knn_prof.log 2>&1; echo "ncu=$?"
python tools/ncu_summary.py gpurun_out/knn_prof.ncu-rep > gpurun_out/knn_prof_summary.txt 2>&1
python tools/ncu_src_lines.py gpurun_out/knn_prof.ncu-rep 60 > gpurun_out/knn_prof_src.txt 2>&1
rm -f gpurun_out/knn_prof.ncu-rep
