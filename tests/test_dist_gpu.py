"""Row-sharded k-NN through the real CUDA kernels in several processes.

dist.knn_search_sharded with the library's knn_search writing straight into the
all-gather send buffer and ksel_merge_lists reading the gathered [g][2][qc][k]
buffer in place, pipelined over query chunks, world sizes 2 and 3 -- the processes
share the one GPU of the test box and exchange through gloo (NCCL refuses two
ranks on one device; under torchrun on a multi-GPU box bench.py runs the same
function over NCCL).  Every rank's slices are checked bit for bit against the
oracle (oracle.knn) and against the unsharded knn_search.
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

_SCRIPT = r"""
import os, sys, numpy as np, torch, torch.distributed as tdist
root, out, rank, world, port, chunks = sys.argv[1], sys.argv[2], int(sys.argv[3]), int(sys.argv[4]), sys.argv[5], int(sys.argv[6])
sys.path.insert(0, root)
import paper_conf_ipps_tang0emg15_b200 as K, synth
from paper_conf_ipps_tang0emg15_b200 import dist
torch.cuda.set_device(0)
tdist.init_process_group("gloo", init_method="tcp://127.0.0.1:" + port, rank=rank, world_size=world)
N, Q, D, k = 30011, 1500, 128, 64
for kind in ("knn-U", "knn-S"):
    ref = synth.knn_points(kind, 31, 0, N, D, device="cuda")
    qry = synth.knn_points(kind, 32, 0, Q, D, device="cuda")
    r0, r1 = dist.shard_range(N, world, rank)
    v, i, qids = dist.knn_search_sharded(ref[r0:r1].contiguous(), qry, k, N, chunks=chunks)
    torch.cuda.synchronize()
    np.save(out + "/v_%s_%d.npy" % (kind, rank), v.cpu().numpy())
    np.save(out + "/i_%s_%d.npy" % (kind, rank), i.cpu().numpy())
    np.save(out + "/q_%s_%d.npy" % (kind, rank), qids.numpy())
tdist.barrier()
tdist.destroy_process_group()
"""


@pytest.mark.parametrize("world,chunks", [(2, 3), (3, 1)])
def test_row_sharded_knn_real_kernels(oracle_mod, tmp_path, world, chunks):
    import paper_conf_ipps_tang0emg15_b200 as K
    from test_knn_gpu import check_knn
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = str(s.getsockname()[1])
    s.close()
    procs = [subprocess.Popen([sys.executable, "-c", _SCRIPT, ROOT, str(tmp_path), str(r), str(world), port,
                               str(chunks)]) for r in range(world)]
    try:
        for p in procs:
            assert p.wait(timeout=300) == 0
    finally:
        for p in procs:
            if p.poll() is None:
                p.kill()
    N, Q, D, k = 30011, 1500, 128, 64
    for kind in ("knn-U", "knn-S"):
        ref = synth.knn_points(kind, 31, 0, N, D)
        qry = synth.knn_points(kind, 32, 0, Q, D)
        qids = np.concatenate([np.load(tmp_path / ("q_%s_%d.npy" % (kind, r))) for r in range(world)])
        gv = np.concatenate([np.load(tmp_path / ("v_%s_%d.npy" % (kind, r))) for r in range(world)])
        gi = np.concatenate([np.load(tmp_path / ("i_%s_%d.npy" % (kind, r))) for r in range(world)])
        assert sorted(qids.tolist()) == list(range(Q))
        order = np.argsort(qids)
        check_knn(oracle_mod, ref, qry, k, gv[order], gi[order])
        ev, ei = K.knn_search(ref.cuda(), qry.cuda(), k)
        assert np.array_equal(gi[order], ei.cpu().numpy())
