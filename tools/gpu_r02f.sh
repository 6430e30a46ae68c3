cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_ksel_gpu.py -x -q -m gpu -k "k_sweep_all or special or unaligned or config2_full or fuzz_shapes" > gpurun_out/pytest_block.log 2>&1; echo "pytest=$?"
for d in U G DG T SD SA; do for k in 1 32 256 1024; do
  printf "C2 %-2s k=%-4d blk " $d $k; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 3 --inner 20 --algo 4 | tail -1
done; done > gpurun_out/c2_block.txt 2>&1
