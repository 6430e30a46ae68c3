"""Small launches of every product kernel, for compute-sanitizer (memcheck, racecheck,
synccheck, initcheck): ksel_pool_kernel (R = 1 and 32; 1, 2 and 8 warps per row; the
3-stage and the 6-stage ring; unaligned rows), ksel_radix_kernel (a cluster of 8 CTAs),
ksel_stream_kernel, the split-row path, ksel_merge_kernel (plain and pointer-table with
ready flags), knn_prep/knn_fused/ksel_merge_pools (k <= 128 and k = 1000), knn_graph.
Each result is checked against torch's stable sort so a run that passes the sanitizer
also computed the right answer.

    compute-sanitizer --tool memcheck python tools/sanitize_cases.py [subset]
"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_tang0emg15_b200 as K  # noqa: E402
import synth  # noqa: E402


def ref_topk(x, k):
    v, i = torch.sort(x, dim=1, stable=True)
    return v[:, :k], i[:, :k].int()


def check_select(x, k, **kw):
    v, i = K.ksel_select(x, k, **kw)
    rv, ri = ref_topk(x, k)
    torch.cuda.synchronize()
    assert torch.equal(i, ri), ("select", x.shape, k, kw)


def select_cases():
    for dist in ("U", "T", "SD"):
        x = synth.rows(dist, 5, 0, 6, 20000, device="cuda")
        for k in (20, 1000):
            for wpr in (1, 2, 8):
                check_select(x, k, warps_per_row=wpr, algo=K.ALGO_POOL)  # few rows: 6-stage ring
    x = synth.rows("U", 6, 0, 400, 4099, device="cuda")  # many rows: 3-stage ring, unaligned rows
    for k in (7, 256):
        check_select(x, k, warps_per_row=1, algo=K.ALGO_POOL)
        check_select(x[:, 1:].contiguous(), k, warps_per_row=2, algo=K.ALGO_POOL)
    print("select ok", flush=True)


def radix_stream_split_cases():
    x = synth.rows("U", 7, 0, 3, 65536, device="cuda")  # cluster of 8 CTAs per row
    for k in (32, 1024):
        check_select(x, k, algo=K.ALGO_RADIX)
        check_select(x, k, algo=K.ALGO_QUEUE)
    y = synth.rows("G", 8, 0, 2, 1 << 20, device="cuda")  # split rows (N1)
    check_select(y, 100)
    print("radix/stream/split ok", flush=True)


def merge_cases():
    S, Q, kin = 3, 50, 64
    x = synth.rows("T", 9, 0, Q, S * 512, device="cuda")
    vs, is_ = [], []
    for s in range(S):
        v, i = K.ksel_select(x[:, s * 512:(s + 1) * 512].contiguous(), kin)
        vs.append(v)
        is_.append(i + s * 512)
    mv, mi = K.ksel_merge(torch.stack(vs), torch.stack(is_), 100)
    rv, ri = ref_topk(x, 100)
    torch.cuda.synchronize()
    assert torch.equal(mi, ri)
    flags = torch.zeros(S, dtype=torch.int32, device="cuda")
    for s in range(S):
        K.flag_signal(flags.data_ptr() + 4 * s, 1)
    ov = torch.empty((Q, 100), dtype=torch.float32, device="cuda")
    oi = torch.empty((Q, 100), dtype=torch.int32, device="cuda")
    K.flag_wait([flags.data_ptr() + 4 * s for s in range(S)], 1)
    K.ksel_merge_lists([v.data_ptr() for v in vs], [i.data_ptr() for i in is_], Q, kin, 100, ov, oi,
                       ready_ptrs=[flags.data_ptr() + 4 * s for s in range(S)], epoch=1)
    torch.cuda.synchronize()
    assert torch.equal(oi, ri)
    print("merge ok", flush=True)


def knn_cases():
    for kind, N, Q, D, k in (("knn-S", 3000, 300, 128, 50), ("knn-U", 2500, 130, 64, 1000),
                             ("knn-U", 700, 40, 17, 7)):
        ref = synth.knn_points(kind, 1, 0, N, D, device="cuda")
        qry = synth.knn_points(kind, 2, 0, Q, D, device="cuda")
        v, i = K.knn_search(ref, qry, k)
        d = torch.cdist(qry.double(), ref.double()) ** 2
        rv, ri = torch.sort(d, dim=1, stable=True)
        torch.cuda.synchronize()
        if kind == "knn-S":
            assert torch.equal(i.long(), ri[:, :k])
        assert torch.allclose(v.double(), rv[:, :k], rtol=1e-4, atol=1e-3)
    x = synth.knn_points("knn-S", 3, 0, 900, 32, device="cuda")
    gv, gi = K.knn_graph(x, 5)
    torch.cuda.synchronize()
    print("knn ok", flush=True)


CASES = {"select": select_cases, "radix": radix_stream_split_cases, "merge": merge_cases, "knn": knn_cases}

if __name__ == "__main__":
    names = sys.argv[1:] or list(CASES)
    for n in names:
        CASES[n]()
    print("ALL OK", flush=True)
