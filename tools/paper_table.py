"""Table I on B200: the paper's per-thread variants (ksel_select_paper) vs ksel_select.

    python tools/paper_table.py [--Q 8192] [--N 32768] [--ks 32,256,1024]

Q = 2^13 queries, N = 2^15 uniform values (Table I); the
variants read the query-contiguous matrix, ksel_select the row-major one.
Prints one line per (variant, k): ms and the speedup of the paper's optimisations.
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--Q", type=int, default=8192)
ap.add_argument("--N", type=int, default=32768)
ap.add_argument("--ks", default="32,256,1024")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--max-ms", type=float, default=20000.0, help="skip repeats of variants slower than this")
a = ap.parse_args()
x = synth.rows("U", 11, 0, a.Q, a.N, device="cuda")
xt = x.t().contiguous()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def timed(fn):
    best = None
    for r in range(a.reps):
        torch.cuda.synchronize()
        e0.record()
        out = fn()
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        best = ms if best is None else min(best, ms)
        if ms > a.max_ms:
            break
    return best, out


QN = {0: "Insertion", 1: "Heap", 2: "Merge", 3: "Merge aligned"}
K.ksel_select(x, 32)  # load the kernels outside the timed calls
torch.cuda.synchronize()
for k in [int(s) for s in a.ks.split(",")]:
    ms_ref, (rv, ri) = timed(lambda: K.ksel_select(x, k))
    print("k=%-5d %-28s %10.3f ms" % (k, "ksel_select (B200 design)", ms_ref), flush=True)
    for queue in (0, 1, 2, 3):
        base = None
        for buf, G, name in ((0, 0, ""), (3, 0, " buf"), (0, 4, " hp"), (3, 4, " buf+hp")):
            ws = torch.empty(K._lib.ksel_select_paper_workspace(a.Q, a.N, k, queue, buf, G, 8, 16),
                             dtype=torch.uint8, device="cuda")
            ms, (gv, gi) = timed(lambda: K.ksel_select_paper(xt, k, queue=queue, buffer=buf, hp_G=G, m=8, bsize=16,
                                                              workspace=ws))
            same = torch.equal(gi, ri)
            base = base or ms
            print("k=%-5d %-28s %10.3f ms  x%6.2f vs plain  x%8.1f vs ksel_select  %s"
                  % (k, QN[queue] + name, ms, base / ms, ms / ms_ref, "exact" if same else "MISMATCH"), flush=True)
