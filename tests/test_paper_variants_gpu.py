"""GPU parity of the paper's own per-thread designs (SURVEY.md 8(f) N4 ablation):
every queue (insertion, heap, Merge Queue, aligned Merge Queue) x Buffered Search
mode x Hierarchical Partition group size must return exactly the oracle's top-k
(the input is query-contiguous: dist_t = dist.T)."""
import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def K():
    import paper_conf_ipps_tang0emg15_b200 as k
    assert torch.cuda.is_available()
    return k


def _check(K, oracle_mod, x_cpu, k, **kw):
    xt = x_cpu.t().contiguous().cuda()
    gv, gi = K.ksel_select_paper(xt, k, **kw)
    torch.cuda.synchronize()
    ev, ei = oracle_mod.select(x_cpu.numpy(), k)
    gi, gv = gi.cpu().numpy(), gv.cpu().numpy()
    assert np.array_equal(gi, ei), kw
    assert np.array_equal(gv.view(np.uint32), ev.view(np.uint32)), kw


@pytest.mark.parametrize("queue", [0, 1, 2, 3])
@pytest.mark.parametrize("buffer", [0, 1, 2, 3])
@pytest.mark.parametrize("G", [0, 2, 4, 6])
def test_paper_variant_vs_oracle(K, oracle_mod, queue, buffer, G):
    x = synth.rows("U", 5, 0, 150, 2000)
    for k in (1, 7, 32, 100):
        _check(K, oracle_mod, x, k, queue=queue, buffer=buffer, hp_G=G, m=8, bsize=8)


@pytest.mark.parametrize("queue", [0, 1, 2, 3])
@pytest.mark.parametrize("dist", ["T", "X", "SD", "SA"])
def test_paper_variant_distributions(K, oracle_mod, queue, dist):
    # ties decided by index, -0.0 / NaN bits, sorted rows (worst / best case insertions)
    x = synth.rows(dist, 6, 0, 70, 1500)
    for G in (0, 4):
        for k in (3, 64, 256):
            _check(K, oracle_mod, x, k, queue=queue, buffer=3, hp_G=G, m=8, bsize=16)


def test_paper_variant_large_k_and_levels(K, oracle_mod):
    x = synth.rows("G", 8, 0, 40, 5000)
    for queue in (0, 1, 2, 3):
        for G, m in ((0, 8), (4, 8), (8, 16), (3, 4)):
            _check(K, oracle_mod, x, 1024, queue=queue, buffer=3, hp_G=G, m=m, bsize=32)
            _check(K, oracle_mod, x, 1000, queue=queue, buffer=2, hp_G=G, m=m, bsize=32)


def test_paper_variant_invalid(K):
    xt = torch.zeros((100, 10), device="cuda")
    with pytest.raises(K.KselError):
        K.ksel_select_paper(xt, 10, m=6)
    with pytest.raises(K.KselError):
        K.ksel_select_paper(xt, 10, hp_G=1)
    with pytest.raises(K.KselError):
        K.ksel_select_paper(xt, 101)
