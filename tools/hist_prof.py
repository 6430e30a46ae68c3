"""One ksel_select launch config for profiling: python tools/hist_prof.py Q N k dist algo [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402

Q, N, k, dist, algo = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4], int(sys.argv[5])
reps = int(sys.argv[6]) if len(sys.argv) > 6 else 2
x = synth.rows(dist, synth.seed_for(2, dist), 0, Q, N, device="cuda")
for _ in range(reps):
    K.ksel_select(x, k, algo=algo)
torch.cuda.synchronize()
