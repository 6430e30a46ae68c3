cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python tools/c2_phases.py U,G,T,SD 1,8,32,128,256,1024 > gpurun_out/c2_phases.txt 2>&1; echo "phases=$?"
CS=/usr/local/cuda/bin/compute-sanitizer
for sub in select radix knn merge; do
  timeout 900 $CS --tool racecheck --error-exitcode 9 --print-limit 50 python tools/sanitize_cases.py $sub > gpurun_out/sanitize_racecheck_${sub}.txt 2>&1; echo "racecheck $sub rc=$?"
done
