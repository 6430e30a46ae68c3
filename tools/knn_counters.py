"""Epilogue event counters of the fused kNN filter (experiments build, KSEL_EXPERIMENTS_LIB=1):
chunks scanned (32 columns x 32 queries), rare chunks, appends, narrowings, pairs kept."""
import ctypes
import os
import sys

os.environ["KSEL_EXPERIMENTS_LIB"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402

N, Q, D = 1000000, 10000, 128
ref = synth.knn_points("knn-U", 41, 0, N, D, device="cuda")
qry = synth.knn_points("knn-U", 42, 0, Q, D, device="cuda")
buf = (ctypes.c_ulonglong * 8)()
for k in (100, 1024):
    K.knn_search(ref, qry, k)
    torch.cuda.synchronize()
    K._lib.ksel_knn_counters(buf)
    K.knn_search(ref, qry, k)
    torch.cuda.synchronize()
    K._lib.ksel_knn_counters(buf)
    c = list(buf)
    print("k=%d chunks %d rare %d (%.1f%%) appends %d (%.0f/query) narrowings %d kept/narrowing %.0f failures %d"
          % (k, c[0], c[1], 100.0 * c[1] / max(1, c[0]), c[2], c[2] / Q, c[3], c[4] / max(1, c[3]), c[5]))
