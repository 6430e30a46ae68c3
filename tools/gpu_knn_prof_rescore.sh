# ncu --set full capture of the kNN rescore kernel (k = $1) with per-source-line summary
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
K=${1:-1024}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:knn_rescore -s 0 -c 1 -o gpurun_out/knn_rs python tools/run_knn.py --reps 1 --k $K > gpurun_out/knn_rs.log 2>&1; echo "ncu=$?"
python tools/ncu_summary.py gpurun_out/knn_rs.ncu-rep > gpurun_out/knn_rs_summary.txt 2>&1
python tools/ncu_src_lines.py gpurun_out/knn_rs.ncu-rep 50 > gpurun_out/knn_rs_src.txt 2>&1
rm -f gpurun_out/knn_rs.ncu-rep
