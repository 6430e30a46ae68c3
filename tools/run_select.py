"""Run ksel_select on a synthetic workload a few times (for ncu / quick timing).

    python tools/run_select.py --Q 1024 --N 65536 --k 256 --dist U --reps 5
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--Q", type=int, default=1024)
ap.add_argument("--N", type=int, default=65536)
ap.add_argument("--k", type=int, default=256)
ap.add_argument("--dist", default="U")
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--algo", type=int, default=0)
ap.add_argument("--wpr", type=int, default=0)
ap.add_argument("--nosplit", action="store_true", help="force one CTA per row (no split rows)")
ap.add_argument("--inner", type=int, default=1, help="calls per timed region (hides host launch latency)")
a = ap.parse_args()
x = synth.rows(a.dist, synth.seed_for(2, a.dist), 0, a.Q, a.N, device="cuda")
v = torch.empty((a.Q, a.k), dtype=torch.float32, device="cuda")
i = torch.empty((a.Q, a.k), dtype=torch.int32, device="cuda")
need = K.ksel_select_workspace(a.Q, a.N, a.k)
ws = torch.empty(max(need, 1), dtype=torch.uint8, device="cuda")
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for r in range(a.reps):
    torch.cuda.synchronize()
    e0.record()
    for _ in range(a.inner):
        K.ksel_select(x, a.k, v, i, algo=a.algo, warps_per_row=a.wpr, workspace=ws, split_rows=not a.nosplit)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.inner
    gbs = a.Q * (4.0 * a.N + 8 * a.k) / (ms / 1e3) / 1e9
    print("rep %d: %.4f ms  %.1f GB/s  %.3g rows/s" % (r, ms, gbs, a.Q / (ms / 1e3)), flush=True)
