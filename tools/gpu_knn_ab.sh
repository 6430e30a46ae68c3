# A/B of the kNN path on one box: the kNN GPU tests of the current library, then variants
# timed alternately at k = 100 and 1024 (VARIANTS: "label|env assignments" separated by ';'
# -- env may set KSEL_AB_LIB=libksel_A.so), then the ncu launch list of the current one.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_knn_gpu.py -x -q -m "gpu" > gpurun_out/pytest_knn.log 2>&1; echo "pytest=$?"
VARIANTS=${VARIANTS:-"A|KSEL_AB_LIB=libksel_A.so;B|"}
for k in 100 1024; do for rep in 1 2; do
  IFS=';' read -ra VS <<< "$VARIANTS"
  for v in "${VS[@]}"; do lab=${v%%|*}; envs=${v#*|}; echo "== $lab k=$k"; env $envs timeout 300 python tools/run_knn.py --k $k --reps 3 2>&1 | grep -v "rep 0"; done
done; done > gpurun_out/knn_time.txt 2>&1
for k in 100 1024; do
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"knn|ksel" --csv --log-file gpurun_out/knn_launches_k$k.csv python tools/run_knn.py --reps 2 --k $k > /dev/null 2>&1; echo "ncu=$?"
done
