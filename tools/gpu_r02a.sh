cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
tag=r02a
(nproc; lscpu | grep -E "Model name|Socket"; nvidia-smi -L) > gpurun_out/box_$tag.txt 2>&1
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke_$tag.log 2>&1; echo "smoke=$?"
timeout 1500 python -m pytest tests -m gpu -x -q -rf > gpurun_out/pytest_$tag.log 2>&1; echo "pytest=$?"
timeout 900 python bench.py > gpurun_out/bench_$tag.json 2> gpurun_out/bench_$tag.err; echo "bench=$?"
timeout 1200 bash tools/sanitize.sh; echo "sanitize=$?"
