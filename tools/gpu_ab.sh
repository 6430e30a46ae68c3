cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python tools/ab_select.py "$1" ${2:-3} > gpurun_out/ab.txt 2>&1; echo "ab=$?"
