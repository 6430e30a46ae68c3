"""Quick knn_distances / knn_search check against the oracle (debug helper)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402

for kind, N, Q, D in [("knn-S", 700, 200, 128), ("knn-U", 700, 200, 128), ("knn-U", 1000, 130, 64),
                      ("knn-U", 513, 77, 3), ("knn-S", 300, 260, 256)]:
    ref = synth.knn_points(kind, 1, 0, N, D)
    qry = synth.knn_points(kind, 2, 0, Q, D)
    dg = K.knn_distances(ref.cuda(), qry.cuda())
    torch.cuda.synchronize()
    do = oracle.knn_dist(ref.numpy(), qry.numpy())
    dg = dg.cpu().numpy()
    err = np.abs(dg.astype(np.float64) - do)
    rel = err / np.maximum(do, 1e-30)
    print(kind, N, Q, D, "max abs err %.3g  max rel %.3g  exact frac %.4f" % (err.max(), rel[do > 1e-3].max(), (dg == do).mean()), flush=True)
    if err.max() > 1:
        bad = np.argwhere(err > 1)[:5]
        print("  bad:", [(int(a), int(b), float(dg[a, b]), float(do[a, b])) for a, b in bad])
for kind, N, Q, D, k in [("knn-S", 5000, 300, 128, 100), ("knn-U", 5000, 300, 128, 100), ("knn-U", 20000, 200, 128, 1024)]:
    ref = synth.knn_points(kind, 3, 0, N, D)
    qry = synth.knn_points(kind, 4, 0, Q, D)
    gv, gi = K.knn_search(ref.cuda(), qry.cuda(), k)
    torch.cuda.synchronize()
    ov, oi = oracle.knn(ref.numpy(), qry.numpy(), k)
    gi = gi.cpu().numpy(); gv = gv.cpu().numpy()
    same = (gi == oi).mean()
    print(kind, N, Q, D, k, "idx agreement %.4f" % same, "max val diff %.3g" % np.abs(gv - ov).max(), flush=True)
