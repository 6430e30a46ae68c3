"""GPU tests of the collective-free row-sharded k-NN exchange.

* ksel_merge_lists (pointer tables, optional ready flags) == oracle.merge (the
  divide-and-merge definition), bit for bit, and == ksel_merge;
* the ready-flag wait really orders the merge after a producer on another stream
  (the merged result is again checked against oracle.merge);
* KnnP2P with 2 and 3 processes on ONE GPU: the exchange buffers are mapped across
  processes with CUDA IPC (the same mechanism as NVLink peer mappings on a
  multi-GPU box), several epochs (double buffering, consumed flags); every rank's
  slice is checked against oracle.knn (bit-exact) and is bit-identical to the
  unsharded knn_search.
"""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def K():
    import paper_conf_ipps_tang0emg15_b200 as k
    assert torch.cuda.is_available()
    return k


def _lists(K, S, Q, kin, seed):
    W = max(512, 2 * kin)
    x = synth.rows("T", seed, 0, Q, S * W, device="cuda")  # ties across lists
    vs, is_ = [], []
    for s in range(S):
        v, i = K.ksel_select(x[:, s * W:(s + 1) * W].contiguous(), kin)
        vs.append(v)
        is_.append(i + s * W)
    return vs, is_


@pytest.mark.parametrize("S,kin,k", [(2, 32, 32), (3, 100, 64), (8, 256, 256), (5, 1024, 1000)])
def test_merge_lists_equals_merge(K, oracle_mod, S, kin, k):
    Q = 300
    vs, is_ = _lists(K, S, Q, kin, 7 + S)
    ev, ei = K.ksel_merge(torch.stack(vs), torch.stack(is_), k)
    # the oracle's merge of the same lists (concatenate, stable sort by (value, index), truncate)
    xv, xi = oracle_mod.merge(torch.stack(vs).cpu().numpy(), torch.stack(is_).cpu().numpy(), k)
    assert np.array_equal(ei.cpu().numpy(), xi)
    assert np.array_equal(ev.cpu().numpy().view(np.uint32), xv.view(np.uint32))
    ov = torch.empty((Q, k), dtype=torch.float32, device="cuda")
    oi = torch.empty((Q, k), dtype=torch.int32, device="cuda")
    K.ksel_merge_lists([v.data_ptr() for v in vs], [i.data_ptr() for i in is_], Q, kin, k, ov, oi)
    torch.cuda.synchronize()
    assert torch.equal(oi, ei) and torch.equal(ov.view(torch.int32), ev.view(torch.int32))
    # query slice through offset pointers, with (already set) ready flags
    flags = torch.zeros(S, dtype=torch.int32, device="cuda")
    for s in range(S):
        K.flag_signal(flags.data_ptr() + 4 * s, 5)
    q0, q1 = 77, 201
    ov2 = torch.empty((q1 - q0, k), dtype=torch.float32, device="cuda")
    oi2 = torch.empty((q1 - q0, k), dtype=torch.int32, device="cuda")
    K.ksel_merge_lists([v.data_ptr() + q0 * kin * 4 for v in vs], [i.data_ptr() + q0 * kin * 4 for i in is_],
                       q1 - q0, kin, k, ov2, oi2, ready_ptrs=[flags.data_ptr() + 4 * s for s in range(S)], epoch=5)
    torch.cuda.synchronize()
    assert torch.equal(oi2, ei[q0:q1]) and torch.equal(ov2.view(torch.int32), ev[q0:q1].view(torch.int32))


def test_merge_lists_waits_for_ready_flags(K, oracle_mod):
    # the producer fills list 1 on another stream after a long busy kernel and only then
    # signals; the merge (launched first) must wait for the flag and see the new data
    S, Q, kin, k = 2, 256, 64, 64
    vs, is_ = _lists(K, S, Q, kin, 3)
    torch.cuda.synchronize()
    xv, xi = oracle_mod.merge(torch.stack(vs).cpu().numpy(), torch.stack(is_).cpu().numpy(), k)
    ev, ei = torch.from_numpy(xv).cuda(), torch.from_numpy(xi).cuda()
    target_v, target_i = vs[1].clone(), is_[1].clone()
    vs[1].fill_(float("inf"))
    is_[1].fill_(-1)
    flags = torch.zeros(S, dtype=torch.int32, device="cuda")
    K.flag_signal(flags.data_ptr(), 1)
    torch.cuda._sleep(100)  # load every kernel of the concurrent part first (lazy loading)
    target_v.copy_(target_v)
    torch.cuda.synchronize()
    ov = torch.empty((Q, k), dtype=torch.float32, device="cuda")
    oi = torch.empty((Q, k), dtype=torch.int32, device="cuda")
    cons = torch.cuda.Stream()
    prod = torch.cuda.Stream()
    with torch.cuda.stream(cons):
        K.ksel_merge_lists([v.data_ptr() for v in vs], [i.data_ptr() for i in is_], Q, kin, k, ov, oi,
                           ready_ptrs=[flags.data_ptr(), flags.data_ptr() + 4], epoch=1)
    with torch.cuda.stream(prod):
        torch.cuda._sleep(20_000_000)  # ~10 ms of spinning before the producer writes
        vs[1].copy_(target_v)
        is_[1].copy_(target_i)
        K.flag_signal(flags.data_ptr() + 4, 1)
    torch.cuda.synchronize()
    assert torch.equal(oi, ei) and torch.equal(ov.view(torch.int32), ev.view(torch.int32))


def test_flag_wait_orders_stream(K):
    flag = torch.zeros(1, dtype=torch.int32, device="cuda")
    out = torch.zeros(1, dtype=torch.int32, device="cuda")
    K.flag_wait([flag.data_ptr()], 0)  # load every kernel of the concurrent part first (lazy loading)
    K.flag_signal(out.data_ptr(), 0)
    out.add_(flag)
    torch.cuda._sleep(100)
    torch.cuda.synchronize()
    a, b = torch.cuda.Stream(), torch.cuda.Stream()
    with torch.cuda.stream(a):
        K.flag_wait([flag.data_ptr()], 3)
        out.add_(flag)  # runs after the wait: sees 3
    with torch.cuda.stream(b):
        torch.cuda._sleep(10_000_000)
        K.flag_signal(flag.data_ptr(), 3)
    torch.cuda.synchronize()
    assert int(out.item()) == 3


def test_p2p_api_validation(K):
    import ctypes
    lib = K._lib
    assert lib.ksel_flag_signal(None, 1, None) == 1
    assert lib.ksel_flag_wait(None, 1, 1, None) == 1
    arr = (ctypes.c_void_p * 1)(None)
    assert lib.ksel_merge_lists(arr, arr, 1, 10, 4, 4, None, None, None, 0, None) == 1


_P2P_SCRIPT = r"""
import os, sys, numpy as np, torch, torch.distributed as tdist
root, out, rank, world, port = sys.argv[1], sys.argv[2], int(sys.argv[3]), int(sys.argv[4]), sys.argv[5]
sys.path.insert(0, root)
import paper_conf_ipps_tang0emg15_b200 as K, synth
from paper_conf_ipps_tang0emg15_b200 import dist
torch.cuda.set_device(0)
tdist.init_process_group("gloo", init_method="tcp://127.0.0.1:" + port, rank=rank, world_size=world)
N, Q, D, k = 20000, 1000, 128, 100
p2p = dist.KnnP2P(Q, k, N, chunks=3)
r0, r1 = dist.shard_range(N, world, rank)
for ep in range(4):
    kind = "knn-S" if ep % 2 else "knn-U"
    ref = synth.knn_points(kind, 70 + ep, 0, N, D, device="cuda")
    qry = synth.knn_points(kind, 80 + ep, 0, Q, D, device="cuda")
    mv, mi, qids = p2p(ref[r0:r1].contiguous(), qry)
    torch.cuda.synchronize()
    np.save(out + "/v_%d_%d.npy" % (ep, rank), mv.cpu().numpy())
    np.save(out + "/i_%d_%d.npy" % (ep, rank), mi.cpu().numpy())
    np.save(out + "/q_%d_%d.npy" % (ep, rank), qids.numpy())
p2p.check()
p2p.close()
tdist.destroy_process_group()
"""


@pytest.mark.parametrize("world", [2, 3])
def test_knn_p2p_processes_on_one_gpu(K, oracle_mod, tmp_path, world):
    from test_knn_gpu import check_knn
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = str(s.getsockname()[1])
    s.close()
    procs = [subprocess.Popen([sys.executable, "-c", _P2P_SCRIPT, ROOT, str(tmp_path), str(r), str(world), port],
                              env=dict(os.environ, CUDA_MODULE_LOADING="EAGER" if world == 3 else "LAZY"))
             for r in range(world)]
    try:
        for p in procs:
            assert p.wait(timeout=240) == 0
    finally:
        for p in procs:
            if p.poll() is None:
                p.kill()
    from paper_conf_ipps_tang0emg15_b200 import dist
    N, Q, D, k = 20000, 1000, 128, 100
    for ep in range(4):
        kind = "knn-S" if ep % 2 else "knn-U"
        ref = synth.knn_points(kind, 70 + ep, 0, N, D, device="cuda")
        qry = synth.knn_points(kind, 80 + ep, 0, Q, D, device="cuda")
        ev, ei = K.knn_search(ref, qry, k)
        ev, ei = ev.cpu().numpy(), ei.cpu().numpy()
        qids = np.concatenate([np.load(tmp_path / ("q_%d_%d.npy" % (ep, r))) for r in range(world)])
        gv = np.concatenate([np.load(tmp_path / ("v_%d_%d.npy" % (ep, r))) for r in range(world)])
        gi = np.concatenate([np.load(tmp_path / ("i_%d_%d.npy" % (ep, r))) for r in range(world)])
        assert sorted(qids.tolist()) == list(range(Q))  # every query merged by exactly one rank
        order = np.argsort(qids)
        gv, gi = gv[order], gi[order]
        # against the oracle (all Q queries), and bit-identical to the unsharded knn_search
        check_knn(oracle_mod, ref.cpu(), qry.cpu(), k, gv, gi)
        assert np.array_equal(gi, ei), ep
        assert np.array_equal(gv.view(np.uint32), ev.view(np.uint32)), ep


def test_flag_wait_timeout_reports_without_killing_the_context(K):
    # a wait whose flag never arrives gives up after the timeout, records
    # KSEL_ERR_TIMEOUT in the library's status word and leaves the context usable
    flag = torch.zeros(1, dtype=torch.int32, device="cuda")
    K.device_status_clear()
    K.set_flag_timeout(0.05)
    try:
        K.flag_wait([flag.data_ptr()], 7)  # nobody ever signals 7
        vs = [torch.full((4, 8), 1.0, device="cuda"), torch.full((4, 8), 2.0, device="cuda")]
        ids = [torch.arange(32, dtype=torch.int32, device="cuda").view(4, 8),
               torch.arange(32, 64, dtype=torch.int32, device="cuda").view(4, 8)]
        ov = torch.empty((4, 8), dtype=torch.float32, device="cuda")
        oi = torch.empty((4, 8), dtype=torch.int32, device="cuda")
        K.ksel_merge_lists([v.data_ptr() for v in vs], [i.data_ptr() for i in ids], 4, 8, 8, ov, oi,
                           ready_ptrs=[flag.data_ptr(), flag.data_ptr()], epoch=9)
        torch.cuda.synchronize()
        assert K.device_status() == 5
    finally:
        K.set_flag_timeout(600.0)
        K.device_status_clear()
    assert K.device_status() == 0
    x = torch.rand(8, 1000, device="cuda")  # the context still works
    v, i = K.ksel_select(x, 5)
    torch.cuda.synchronize()
    assert torch.equal(i.long(), torch.sort(x, dim=1, stable=True).indices[:, :5])
