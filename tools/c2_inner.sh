#!/bin/bash
# C2 with 20 back-to-back calls per timed region (host launch latency hidden, as in bench.py)
for d in U DG SD T; do for k in 1 8 32 128 256 1024; do
  printf "C2 %-2s k=%-4d " $d $k; timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 4 --inner 20 | tail -1
done; done
python - <<'PY'
import torch, sys
sys.path.insert(0, ".")
import synth
x = synth.rows("U", 1, 0, 1024, 65536, device="cuda")
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for name, fn in (("torch.amin", lambda: torch.amin(x, dim=1)), ("torch.topk k=256", lambda: torch.topk(x, 256, dim=1, largest=False, sorted=True))):
    fn(); torch.cuda.synchronize()
    e0.record()
    for _ in range(20): fn()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 20
    print("%s: %.4f ms  %.1f GB/s" % (name, ms, 1024 * 65536 * 4 / ms / 1e6))
PY
