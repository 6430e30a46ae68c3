cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for c in 1 2 4; do KSEL_BENCH_CHUNKS=$c timeout 900 python bench.py --knn-sharded on --no-sweep --no-e2e --no-cpu-baseline --steps 3 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('chunks', $c, d['knn_row_sharded']['ms_per_step'])"; done > gpurun_out/knnsh_chunks.txt 2>&1
for c in 1 2 4; do KSEL_BENCH_CHUNKS=$c timeout 300 python -c "
import sys,torch; sys.path.insert(0,'.')
import paper_conf_ipps_tang0emg15_b200 as K, synth
ref=synth.knn_points('knn-U',41,0,1000000,128,device='cuda'); qry=synth.knn_points('knn-U',42,0,10000,128,device='cuda')
for k in (100,1024):
  ws=torch.empty(K.knn_search_workspace(1000000,10000//$c,128,k),dtype=torch.uint8,device='cuda')
  for rep in range(2):
    e0,e1=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True); torch.cuda.synchronize(); e0.record()
    for i in range($c): K.knn_search(ref, qry[i*(10000//$c):(i+1)*(10000//$c)].contiguous(), k, workspace=ws)
    e1.record(); torch.cuda.synchronize()
  print('chunks $c k',k, e0.elapsed_time(e1))
"; done >> gpurun_out/knnsh_chunks.txt 2>&1
