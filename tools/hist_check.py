"""Histogram select (algo 4, experiments library: build with KSEL_BUILD_EXPERIMENTS=1, run
with KSEL_EXPERIMENTS_LIB=1) vs the pool kernel (algo 2): bitwise agreement on ragged
shapes and every synthetic distribution, then per-launch times of both.
usage: python tools/hist_check.py [quick]   (HC_SHAPES="QxN,..." HC_ALLK=1 select the timing grid)"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402

bad = 0
for dist in synth.DISTS:
    for (Q, N) in ((7, 1), (5, 33), (300, 1000), (64, 4099), (40, 65537), (20, 131072)):
        for k in (1, 7, 32, 100, 256, 600, 1024):
            if k > N:
                continue
            x = synth.rows(dist, synth.seed_for(2, dist), 0, Q, N, device="cuda")
            for off in (0, 1):  # misaligned row starts too
                xx = x.view(-1)[off:off + Q * N - (Q * N if off and False else 0)] if off == 0 else None
                if off:
                    buf = torch.empty(Q * N + 1, device="cuda")
                    buf[1:] = x.view(-1)
                    xx = buf[1:].view(Q, N)
                else:
                    xx = x
                a = K.ksel_select(xx, k, algo=2)
                b = K.ksel_select(xx, k, algo=4)
                torch.cuda.synchronize()
                if not (torch.equal(a[0].view(torch.int32), b[0].view(torch.int32)) and torch.equal(a[1], b[1])):
                    bad += 1
                    print("MISMATCH", dist, Q, N, k, off, flush=True)
print("parity mismatches:", bad, flush=True)
if len(sys.argv) > 1:
    sys.exit(0)
print("%-22s %9s %9s %6s" % ("config", "pool ms", "hist ms", "h/p"))
for dist in synth.DISTS:
    for k in ((1, 8, 32, 128, 256, 1024) if os.environ.get('HC_ALLK') else (32, 256, 1024)):
        for (Q, N) in [tuple(map(int, c.split('x'))) for c in os.environ.get('HC_SHAPES', '1024x65536,1024x131072,8192x4096').split(',')]:
            x = synth.rows(dist, synth.seed_for(2, dist), 0, Q, N, device="cuda")
            r = {}
            for algo in (2, 4):
                for _ in range(3):
                    K.ksel_select(x, k, algo=algo)
                torch.cuda.synchronize()
                K.timing_collect()
                K.timing_enable(True)
                for _ in range(10):
                    K.ksel_select(x, k, algo=algo)
                torch.cuda.synchronize()
                K.timing_enable(False)
                ms, n = K.timing_collect()
                r[algo] = ms / n
            print("%-22s %9.4f %9.4f %6.3f" % ("%s Q%d N%d k%d" % (dist, Q, N, k), r[2], r[4], r[4] / r[2]),
                  flush=True)
            del x
