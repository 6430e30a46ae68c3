cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for a in 0; do for d in U T SD; do for k in 1 32 256 1024; do
  printf "C2 %-2s k=%-4d algo=%d " $d $k $a; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 3 --inner 20 --algo $a | tail -1
done; done; done > gpurun_out/c2_h.txt 2>&1
timeout 300 python tools/run_select.py --Q 16384 --N 1048576 --k 256 --dist U --reps 3 > gpurun_out/c3_h.txt 2>&1
timeout 300 python tools/run_select.py --Q 16384 --N 1048576 --k 1024 --dist U --reps 3 >> gpurun_out/c3_h.txt 2>&1
