"""KSEL_KNN_MODE=3: per-warp epilogue cycle counters of the fused kNN kernel."""
import os
import sys

os.environ["KSEL_KNN_MODE"] = "3"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402

N, Q, D, k = [int(x) for x in (sys.argv[1:5] if len(sys.argv) > 4 else (1000000, 10000, 128, 100))]
ref = synth.knn_points("knn-U", 41, 0, N, D, device="cuda")
qry = synth.knn_points("knn-U", 42, 0, Q, D, device="cuda")
ws = torch.zeros(K.knn_search_workspace(N, Q, D, k), dtype=torch.uint8, device="cuda")
for rep in range(2):
    K.knn_search(ref, qry, k, workspace=ws)
    torch.cuda.synchronize()
# the counters sit at the end of the workspace (layout: ... qthr | prof); S as in knn_geometry
CS = int(os.environ.get('KSEL_KNN_CLUSTER', '1'))
QT = (Q + 127) // 128
QT = (QT + CS - 1) // CS * CS if QT >= CS else QT
NT = (N + 255) // 256
best, best_cost = 1, 1e30
for s_ in range(1, min(NT, 64) + 1):
    ctas = QT * s_
    waves = ctas / 148.0
    cost = ((ctas + 147) // 148) / waves + (2.0 - waves if waves < 2.0 else 0.0) + 0.01 * s_ * (max(k, 32) / 128.0 if max(k, 32) > 128 else 1.0)
    if cost < best_cost:
        best, best_cost = s_, cost
S = best
raw = ws.cpu().numpy()
EW = 8 if os.environ.get('KSEL_KNN_EW') == '8' else 4
sz = QT * S * 8 * 16 * 8
szp = (sz + 255) // 256 * 256
arr = raw[raw.size - szp: raw.size - szp + sz].view(np.uint64)[:QT * S * EW * 16].reshape(QT * S, EW, 16)[:, :, :9]
print("S =", S)
names = ["narrow", "wait_accf", "chunks", "rare", "n_rare", "n_narrow", "final", "total", "appends"]
tot = arr.reshape(-1, 9).astype(np.float64)
print("CTAs x warps:", tot.shape[0])
for i, nm in enumerate(names):
    print("%-10s mean %.3g  max %.3g" % (nm, tot[:, i].mean(), tot[:, i].max()))
split = np.arange(arr.shape[0]) // QT
for s in range(split.max() + 1):
    m = arr[split == s].reshape(-1, 9).astype(np.float64).mean(axis=0)
    print("split %d: " % s + "  ".join("%s %.3g" % (nm, v) for nm, v in zip(names, m)))
