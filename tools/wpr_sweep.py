"""Pool-kernel launch-shape sweep: per-launch ms of ksel_select(algo=2, warps_per_row=W).
usage: python tools/wpr_sweep.py "Q,N,k,dist;..." "0,1,2,4,8" """
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402

wprs = [int(w) for w in sys.argv[2].split(",")]
print("%-24s" % "config" + "".join("%9s" % ("w=%d" % w) for w in wprs))
for cfg in sys.argv[1].split(";"):
    Q, N, k, dist = cfg.split(",")
    Q, N, k = int(Q), int(N), int(k)
    x = synth.rows(dist, synth.seed_for(2, dist), 0, Q, N, device="cuda")
    row = []
    for w in wprs:
        for _ in range(3):
            K.ksel_select(x, k, algo=2, warps_per_row=w)
        torch.cuda.synchronize()
        K.timing_collect()
        K.timing_enable(True)
        for _ in range(10):
            K.ksel_select(x, k, algo=2, warps_per_row=w)
        torch.cuda.synchronize()
        K.timing_enable(False)
        ms, n = K.timing_collect()
        row.append(ms / n)
    print("%-24s" % cfg + "".join("%9.4f" % v for v in row), flush=True)
    del x
