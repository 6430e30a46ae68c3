"""Multi-process (world_size 2 and 3, gloo, CPU) tests of the sharding logic.

The local kernels are replaced by CPU stand-ins built on the oracle (test
infrastructure) so that the host-side plumbing of the multi-GPU paths --
partitioning, global index offsets, the query-chunk pipeline, the in-place
[2][qc][k] send / [g][2][qc][k] receive buffers, the async all-gathers and the
per-rank query slices of the merge -- is checked end to end against the
unsharded oracle result, bit for bit.  tests/test_dist_gpu.py runs the same
function with the CUDA kernels (several processes sharing one GPU); bench.py
runs it with NCCL under torchrun.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as tdist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _cpu_knn(ref, query, k, idx_offset, out_v, out_i):
    import oracle
    v, i = oracle.knn(ref.numpy(), query.numpy(), k, idx_offset=idx_offset)
    out_v.copy_(torch.from_numpy(v))
    out_i.copy_(torch.from_numpy(i))


def _cpu_merge(vals, idxs, k, out_v, out_i):
    import oracle
    v, i = oracle.merge(torch.stack(vals).numpy(), torch.stack(idxs).numpy(), k)
    out_v.copy_(torch.from_numpy(v))
    out_i.copy_(torch.from_numpy(i))


def _worker(rank, world, port, kind, N, Q, D, k, chunks, out_dir):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    import synth
    from paper_conf_ipps_tang0emg15_b200 import dist as kd
    ref = synth.knn_points(kind, 11, 0, N, D)
    qry = synth.knn_points(kind, 12, 0, Q, D)
    r0, r1 = kd.shard_range(N, world, rank)
    v, i, qids = kd.knn_search_sharded(ref[r0:r1].contiguous(), qry, k, N, chunks=chunks, local_knn=_cpu_knn,
                                       merge=_cpu_merge)
    np.save(os.path.join(out_dir, "v%d.npy" % rank), v.numpy())
    np.save(os.path.join(out_dir, "i%d.npy" % rank), i.numpy())
    np.save(os.path.join(out_dir, "q%d.npy" % rank), qids.numpy())
    tdist.barrier()
    tdist.destroy_process_group()


@pytest.mark.parametrize("world,chunks", [(2, 1), (2, 3), (3, 4)])
@pytest.mark.parametrize("kind", ["knn-S", "knn-U"])
def test_row_sharded_knn_equals_unsharded(tmp_path, oracle_mod, world, chunks, kind):
    N, Q, D, k = 1003, 37, 16, 25
    mp.start_processes(_worker, args=(world, _free_port(), kind, N, Q, D, k, chunks, str(tmp_path)),
                       nprocs=world, join=True, start_method="spawn")
    import synth
    ref = synth.knn_points(kind, 11, 0, N, D).numpy()
    qry = synth.knn_points(kind, 12, 0, Q, D).numpy()
    ev, ei = oracle_mod.knn(ref, qry, k)
    seen = []
    for r in range(world):
        qids = np.load(tmp_path / ("q%d.npy" % r))
        v = np.load(tmp_path / ("v%d.npy" % r))
        i = np.load(tmp_path / ("i%d.npy" % r))
        assert np.array_equal(i, ei[qids])
        assert np.array_equal(v.view(np.uint32), ev[qids].view(np.uint32))
        seen += qids.tolist()
    assert sorted(seen) == list(range(Q))  # every query merged by exactly one rank


def test_chunk_ranges_partition():
    from paper_conf_ipps_tang0emg15_b200 import dist as kd
    for Q in (1, 5, 37, 10000):
        for c in (1, 3, 4, 8, 100):
            spans = kd.chunk_ranges(Q, c)
            assert spans[0][0] == 0 and spans[-1][1] == Q and len(spans) == min(c, Q)
            assert all(spans[j][1] == spans[j + 1][0] for j in range(len(spans) - 1))


def test_query_rows_partition():
    from paper_conf_ipps_tang0emg15_b200 import dist as kd
    for Q in (1, 7, 16384, 16385):
        for world in (1, 2, 3, 8):
            spans = [kd.query_rows(Q, world, r) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == Q
            assert all(spans[r][1] == spans[r + 1][0] for r in range(world - 1))
            assert max(b - a for a, b in spans) - min(b - a for a, b in spans) <= 1


def test_p2p_layout_regions_disjoint():
    from paper_conf_ipps_tang0emg15_b200 import dist
    for Q, k, world in [(1, 1, 1), (1000, 100, 8), (10000, 1024, 64), (7, 3, 5)]:
        L = dist.p2p_layout(Q, k, world)
        spans = [(L["ready"](b, c), 4) for b in range(2) for c in range(dist.P2P_MAX_CHUNKS)]
        spans += [(L["consumed"](s), 4) for s in range(world)]
        spans += [(L["val"](b), Q * k * 4) for b in range(2)] + [(L["idx"](b), Q * k * 4) for b in range(2)]
        spans.sort()
        for (a, n), (b_, _) in zip(spans, spans[1:]):
            assert a + n <= b_
        assert spans[-1][0] + spans[-1][1] <= L["bytes"]
        assert all(off % 4 == 0 for off, _ in spans)
    with pytest.raises(ValueError):
        dist.p2p_layout(10, 10, 65)
