cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for d in U G T SD; do for k in 32 256 1024; do for w in 1 2 4; do
  printf "C2 %-2s k=%-4d wpr=%d " $d $k $w; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 3 --inner 20 --algo 2 --wpr $w | tail -1
done; done; done > gpurun_out/c2_wpr.txt 2>&1
