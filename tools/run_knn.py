"""Time knn_search on a synthetic workload (CUDA events); optional ncu target.

    python tools/run_knn.py --N 1000000 --Q 10000 --D 128 --k 100 --kind knn-U --reps 3
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--N", type=int, default=1000000)
ap.add_argument("--Q", type=int, default=10000)
ap.add_argument("--D", type=int, default=128)
ap.add_argument("--k", type=int, default=100)
ap.add_argument("--kind", default="knn-U")
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--save", default="")
a = ap.parse_args()
ref = synth.knn_points(a.kind, 41, 0, a.N, a.D, device="cuda")
qry = synth.knn_points(a.kind, 42, 0, a.Q, a.D, device="cuda")
ws = torch.full((K.knn_search_workspace(a.N, a.Q, a.D, a.k),), 255, dtype=torch.uint8, device="cuda")
ov = torch.empty((a.Q, a.k), dtype=torch.float32, device="cuda")
oi = torch.empty((a.Q, a.k), dtype=torch.int32, device="cuda")
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
flops = 2.0 * a.N * a.Q * a.D
for r in range(a.reps):
    torch.cuda.synchronize()
    K.timing_collect()
    K.timing_enable(True)
    e0.record()
    K.knn_search(ref, qry, a.k, out_dist=ov, out_idx=oi, workspace=ws)
    e1.record()
    torch.cuda.synchronize()
    K.timing_enable(False)
    kms, kn = K.timing_collect()
    ms = e0.elapsed_time(e1)
    print("rep %d: %.3f ms (filter kernel %.3f ms)  %.1f TFLOP/s (1-pass algorithmic, call)  %.0f queries/s"
          % (r, ms, kms, flops / ms / 1e9, a.Q / ms * 1e3), flush=True)
if a.save:
    import numpy as np
    np.savez(a.save, v=ov.cpu().numpy(), i=oi.cpu().numpy())
