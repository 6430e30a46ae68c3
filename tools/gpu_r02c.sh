cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python tools/c2_phases.py U,G,T,SD 1,8,32,128,256,1024 > gpurun_out/c2_phases.txt 2>&1; echo "phases=$?"
