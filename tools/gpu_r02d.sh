cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for cfg in "U 256" "T 256" "U 1024" "U 32"; do set -- $cfg
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ksel_pool -s 3 -c 1 -o gpurun_out/c2_${1}_k$2 \
  python tools/run_select.py --Q 1024 --N 65536 --k $2 --dist $1 --reps 4 > gpurun_out/c2_ncu_${1}_$2.log 2>&1; echo "ncu $cfg rc=$?"
ncu -i gpurun_out/c2_${1}_k$2.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/c2_src_${1}_k$2.csv 2>/dev/null
done
