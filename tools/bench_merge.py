"""Time ksel_merge for (Q, S, k): per-list cost of the merge kernel."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402

for Q, S, k in [(5, 60, 256), (1, 64, 256), (1000, 60, 256), (5, 60, 32), (5, 8, 256), (148, 8, 256)]:
    v = torch.rand(S, Q, k, device="cuda").sort(dim=2).values.contiguous()
    i = torch.arange(S * Q * k, dtype=torch.int32, device="cuda").reshape(S, Q, k)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for r in range(3):
        torch.cuda.synchronize()
        e0.record()
        K.ksel_merge(v, i, k)
        e1.record()
        torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    print("Q=%d S=%d k=%d: %.3f ms  (%.2f us per list per warp)" % (Q, S, k, ms, ms * 1e3 / S), flush=True)
