#!/bin/bash
# One GPU-box pass: full gpu tests, smoke, bench (N=1, c3 and c4), ncu launch lists + full
# captures of the bench kernels.   usage: tools/round_gpu.sh <tag> [skip_tests]
tag=${1:-r01}
mkdir -p gpurun_out
(nproc; free -g; nvidia-smi -L; nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv) > gpurun_out/box_$tag.txt 2>&1
timeout 600 python __graft_entry__.py smoke > gpurun_out/smoke_$tag.log 2>&1; echo "smoke=$?"
if [ -z "$2" ]; then
timeout 2400 python -m pytest tests -m gpu -q -rA > gpurun_out/pytest_$tag.log 2>&1; echo "pytest=$?"
fi
timeout 900 python bench.py > gpurun_out/bench_$tag.json 2> gpurun_out/bench_$tag.err; echo "bench=$?"
timeout 900 python bench.py --config c4 > gpurun_out/bench_c4_$tag.json 2> gpurun_out/bench_c4_$tag.err; echo "bench_c4=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:ksel --csv \
   --log-file gpurun_out/launches_$tag.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_ncu_$tag.log 2>&1; echo "ncu_launches=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"knn|ksel" --csv \
   --log-file gpurun_out/launches_c4_$tag.csv python bench.py --config c4 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_c4_ncu_$tag.log 2>&1; echo "ncu_launches_c4=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ksel_pool -s 3 -c 1 \
   -o gpurun_out/prof_bench_$tag python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_$tag.log 2>&1; echo "ncu_full=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:knn_fused -s 3 -c 1 \
   -o gpurun_out/prof_bench_c4_$tag python bench.py --config c4 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_c4_$tag.log 2>&1; echo "ncu_full_c4=$?"
