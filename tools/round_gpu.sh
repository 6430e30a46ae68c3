#!/bin/bash
# One GPU-box evidence pass: smoke, bench (N=1: C3 headline + sweep; C4 kNN), reference arm,
# ncu launch lists and full captures of the bench kernels, N1 split rows.
#   usage: tools/round_gpu.sh <tag> [skip_tests]
tag=${1:-r02}
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
(nproc; lscpu | grep -E "Model name|Socket"; free -g; nvidia-smi -L) > gpurun_out/box_$tag.txt 2>&1
timeout 600 python __graft_entry__.py smoke > gpurun_out/smoke_$tag.log 2>&1; echo "smoke=$?"
if [ -z "$2" ]; then
timeout 2400 python -m pytest tests -m gpu -q -rA > gpurun_out/pytest_$tag.log 2>&1; echo "pytest=$?"
fi
timeout 900 python bench.py > gpurun_out/bench_$tag.json 2> gpurun_out/bench_$tag.err; echo "bench=$?"
timeout 900 python bench.py --config c4 > gpurun_out/bench_c4_$tag.json 2> gpurun_out/bench_c4_$tag.err; echo "bench_c4=$?"
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$tag.json 2>&1; echo "bench_ref=$?"
for cfg in "1 67108864 256 U" "4 16777216 256 U" "1 67108864 32 U"; do set -- $cfg
  printf "N1 Q=%s N=%s k=%s %s " $1 $2 $3 $4; timeout 120 python tools/run_select.py --Q $1 --N $2 --k $3 --dist $4 --reps 3 --inner 10 | tail -1
done > gpurun_out/n1_$tag.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"ksel|knn" --csv \
   --log-file gpurun_out/launches_$tag.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/bench_ncu_$tag.log 2>&1; echo "ncu_launches=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"knn|ksel" --csv \
   --log-file gpurun_out/launches_c4_$tag.csv python bench.py --config c4 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4_ncu_$tag.log 2>&1; echo "ncu_launches_c4=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ksel_pool -s 3 -c 1 \
   -o gpurun_out/prof_bench_$tag python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep > gpurun_out/ncu_full_$tag.log 2>&1; echo "ncu_full=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:knn_fused -s 3 -c 1 \
   -o gpurun_out/prof_bench_c4_$tag python bench.py --config c4 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_c4_$tag.log 2>&1; echo "ncu_full_c4=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ksel_pool -s 2 -c 1 \
   -o gpurun_out/prof_c2_$tag python tools/run_select.py --Q 1024 --N 65536 --k 256 --dist U --reps 3 > gpurun_out/ncu_c2_$tag.log 2>&1; echo "ncu_c2=$?"
for r in prof_bench_$tag prof_bench_c4_$tag prof_c2_$tag; do
  python tools/ncu_summary.py gpurun_out/$r.ncu-rep --json gpurun_out/${r}_summary.json > gpurun_out/${r}_summary.txt 2>&1
  python tools/ncu_src_lines.py gpurun_out/$r.ncu-rep 30 > gpurun_out/${r}_src.txt 2>&1
  rm -f gpurun_out/$r.ncu-rep
done
