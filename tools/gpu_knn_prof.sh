# ncu --set full captures of the fused kNN launches: the speculative pre-pass (launch 0) and
# the main pass (launch 1), with per-source-line summaries
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
K=${1:-100}
for s in 0 1; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:knn_fused -s $s -c 1 -o gpurun_out/knn_prof$s python tools/run_knn.py --reps 1 --k $K > gpurun_out/knn_prof$s.log 2>&1; echo "ncu=$?"
python tools/ncu_summary.py gpurun_out/knn_prof$s.ncu-rep > gpurun_out/knn_prof${s}_summary.txt 2>&1
python tools/ncu_src_lines.py gpurun_out/knn_prof$s.ncu-rep 50 > gpurun_out/knn_prof${s}_src.txt 2>&1
rm -f gpurun_out/knn_prof$s.ncu-rep
done
