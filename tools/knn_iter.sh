#!/bin/bash
# kNN iteration on the GPU box: parity tests, timing, epilogue counters.
# usage: tools/knn_iter.sh <tag> [extra pytest -k expr]
tag=${1:-x}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_knn_gpu.py -m gpu -x -q ${2:+-k "$2"} > gpurun_out/knn_pytest_$tag.log 2>&1; echo "pytest=$?"
tail -3 gpurun_out/knn_pytest_$tag.log
timeout 300 python tools/run_knn.py --reps 4 > gpurun_out/knn_time_$tag.txt 2>&1; echo "time=$?"; cat gpurun_out/knn_time_$tag.txt
timeout 300 python tools/run_knn.py --reps 3 --kind knn-S > gpurun_out/knn_timeS_$tag.txt 2>&1; cat gpurun_out/knn_timeS_$tag.txt
timeout 300 python tools/knn_prof.py > gpurun_out/knn_prof_$tag.txt 2>&1; echo "prof=$?"; head -12 gpurun_out/knn_prof_$tag.txt
