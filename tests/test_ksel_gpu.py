"""GPU parity of ksel_select / ksel_merge / ksel_select_host against the oracle.

Every comparison is BIT-EXACT: values compared as uint32 bit patterns and
indices as int32 (north star: "ksel_select must be bit-exact in values and
indices on identical generated inputs").  Inputs come from synth/ (the same
bits on both sides); no expected value is produced by the CUDA path.
"""
import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu

KS = [1, 2, 3, 8, 31, 32, 33, 100, 128, 255, 256, 257, 512, 1000, 1024]


@pytest.fixture(scope="module")
def K():
    import paper_conf_ipps_tang0emg15_b200 as k
    assert torch.cuda.is_available(), "GPU test run without a GPU"
    return k


def _bits(a):
    return np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)


def assert_same(ev, ei, gv, gi, ctx=""):
    gv = gv.cpu().numpy() if torch.is_tensor(gv) else gv
    gi = gi.cpu().numpy() if torch.is_tensor(gi) else gi
    bad_i = np.nonzero((gi != ei).any(axis=1) | (_bits(gv) != _bits(ev)).any(axis=1))[0]
    if bad_i.size:
        r = bad_i[0]
        j = np.nonzero((gi[r] != ei[r]) | (_bits(gv[r]) != _bits(ev[r])))[0][0]
        raise AssertionError("%s: %d bad rows; row %d first diff at %d: gpu (%r,%d) oracle (%r,%d)"
                             % (ctx, bad_i.size, r, j, gv[r][j], gi[r][j], ev[r][j], ei[r][j]))


def _check_select(K, oracle_mod, x_cpu, k, ctx, algo=0, wpr=0):
    x = x_cpu.cuda()
    gv, gi = K.ksel_select(x, k, algo=algo, warps_per_row=wpr)
    torch.cuda.synchronize()
    ev, ei = oracle_mod.select(x_cpu.numpy(), k)
    assert_same(ev, ei, gv, gi, ctx)


def test_config1(K, oracle_mod):
    # configs[0]: Q=16 rows, N=4096 uniform fp32 distances, k=32
    x = synth.rows("U", synth.seed_for(1, "U"), 0, 16, 4096)
    _check_select(K, oracle_mod, x, 32, "C1")


@pytest.mark.parametrize("algo", [1, 2, 3])
@pytest.mark.parametrize("dist", synth.DISTS)
def test_k_sweep_all_distributions(K, oracle_mod, dist, algo):
    # every kernel variant: 1 = bitonic queue per flush, 2 = pool + radix narrowing,
    # 3 = cluster radix select (row in registers)
    x = synth.rows(dist, synth.seed_for(7, dist), 0, 48, 5003)  # ragged N (N % 4 != 0)
    for k in KS:
        _check_select(K, oracle_mod, x, k, "%s k=%d algo=%d" % (dist, k, algo), algo=algo)


@pytest.mark.parametrize("N", [1, 2, 3, 5, 31, 1000, 1023, 1024, 1025, 4095, 4096, 9999, 65536])
def test_edge_lengths(K, oracle_mod, N):
    for dist in ("U", "T", "X"):
        x = synth.rows(dist, 99, 0, 9, N)
        for k in sorted({1, min(N, 2), min(N, 3), min(N, 32), min(N, 33), min(N, 257), min(N, 1024), min(N, 1024)}):
            _check_select(K, oracle_mod, x, k, "%s N=%d k=%d" % (dist, N, k))


@pytest.mark.parametrize("Q", [1, 2, 5, 16, 150, 600, 2000])
def test_row_counts_and_warps_per_row(K, oracle_mod, Q):
    # small Q selects several warps per row (shared threshold + in-CTA merge)
    x = synth.rows("G", 31, 0, Q, 40000)
    for k in (1, 32, 100, 256, 1024):
        _check_select(K, oracle_mod, x, k, "Q=%d k=%d" % (Q, k))


@pytest.mark.parametrize("algo", [1, 2])
@pytest.mark.parametrize("wpr", [1, 2, 4, 8])
def test_forced_warps_per_row(K, oracle_mod, wpr, algo):
    for dist in ("U", "SD", "T", "X"):
        x = synth.rows(dist, 41, 0, 13, 30011)
        for k in (1, 33, 256, 1000):
            _check_select(K, oracle_mod, x, k, "%s wpr=%d algo=%d k=%d" % (dist, wpr, algo, k), algo, wpr)


@pytest.mark.parametrize("N", [1, 3, 31, 1025, 8191, 8192, 8193, 16385, 24576 + 7, 40000, 57343, 65535, 65536])
def test_radix_cluster_sizes(K, oracle_mod, N):
    # KSEL_ALGO_RADIX: clusters of 1..8 CTAs (8192 values each), ragged and aligned rows,
    # ties cut inside a CTA and across CTAs (T), specials (X), sorted rows
    for dist in ("U", "T", "X", "SD", "DG"):
        x = synth.rows(dist, 123, 0, 5, N)
        for k in sorted({1, min(N, 2), min(N, 33), min(N, 256), min(N, 1000), min(N, 1024)}):
            _check_select(K, oracle_mod, x, k, "radix %s N=%d k=%d" % (dist, N, k), algo=3)


def test_radix_all_equal_and_unsupported(K, oracle_mod):
    x = torch.full((3, 65536), 7.0)
    x[1, 1000:] = -0.0
    x[2, ::3] = float("nan")
    for k in (1, 100, 1024):
        _check_select(K, oracle_mod, x, k, "radix equal k=%d" % k, algo=3)
    with pytest.raises(K.KselError):
        K.ksel_select(torch.zeros((2, 65537), device="cuda"), 10, algo=3)


@pytest.mark.parametrize("k", [1, 32, 256, 1024])
@pytest.mark.parametrize("dist", ["U", "DG", "SD", "T"])
def test_radix_config2_full_size(K, oracle_mod, dist, k):
    x = synth.rows(dist, synth.seed_for(2, dist), 0, 1024, 65536, device="cuda")
    gv, gi = K.ksel_select(x, k, algo=3)
    torch.cuda.synchronize()
    ev, ei = oracle_mod.select(x.cpu().numpy(), k)
    assert_same(ev, ei, gv, gi, "C2 radix %s k=%d" % (dist, k))


def test_unaligned_base_pointer(K, oracle_mod):
    # row starts that are not 16-byte aligned, including the base pointer itself
    big = synth.rows("U", 5, 0, 1, 7 * 4099 + 3)[0]
    for off in (1, 2, 3):
        x_cpu = big[off:off + 7 * 4099].reshape(7, 4099).contiguous()
        xg = big.cuda()[off:off + 7 * 4099].view(7, 4099)
        assert xg.data_ptr() % 16 != 0
        for k in (1, 64, 300):
            for algo in (0, 3):
                gv, gi = K.ksel_select(xg, k, algo=algo)
                ev, ei = oracle_mod.select(x_cpu.numpy(), k)
                assert_same(ev, ei, gv, gi, "off=%d k=%d algo=%d" % (off, k, algo))


def test_special_rows(K, oracle_mod):
    N = 3000
    rows = [np.full(N, 0.25, np.float32), np.arange(N, dtype=np.float32),
            np.arange(N, dtype=np.float32)[::-1].copy(),
            np.where(np.arange(N) % 2 == 0, -0.0, 0.0).astype(np.float32),
            np.full(N, np.nan, np.float32), np.full(N, np.inf, np.float32),
            np.concatenate([np.full(N - 5, np.nan), [np.inf, -np.inf, 1e-45, -1e-45, -0.0]]).astype(np.float32)]
    x = torch.from_numpy(np.stack(rows))
    for k in (1, 5, 6, 32, 100, 1024):
        _check_select(K, oracle_mod, x, k, "special k=%d" % k)
        _check_select(K, oracle_mod, x, k, "special radix k=%d" % k, algo=3)


@pytest.mark.parametrize("k", [1, 8, 32, 128, 256, 1024])
@pytest.mark.parametrize("dist", ["U", "G", "DG", "SA", "SD", "T"])
def test_config2_full_size(K, oracle_mod, dist, k):
    # configs[1]: Q=1024, N=65536, the k sweep, all distributions -- all rows, with the
    # launch bench.py times (auto) and the streaming kernel variants forced
    x = synth.rows(dist, synth.seed_for(2, dist), 0, 1024, 65536, device="cuda")
    ev, ei = oracle_mod.select(x.cpu().numpy(), k)
    for algo in (0, 1, 2):
        gv, gi = K.ksel_select(x, k, algo=algo)
        torch.cuda.synchronize()
        assert_same(ev, ei, gv, gi, "C2 %s k=%d algo=%d" % (dist, k, algo))


@pytest.mark.slow
def test_config3_full_size_sampled_rows(K, oracle_mod):
    # configs[2] at one GPU, exactly the launch bench.py times: Q=16384, N=2^20,
    # k=256; the oracle checks a fixed sample (first 32 rows of each 2048 block)
    Q, N, k = 16384, 1 << 20, 256
    seed = synth.seed_for(3, "U")
    x = synth.rows("U", seed, 0, Q, N, device="cuda")
    gv, gi = K.ksel_select(x, k)
    torch.cuda.synchronize()
    sample = [b * 2048 + t for b in range(Q // 2048) for t in range(32)]
    del x
    xs = synth.row_subset("U", seed, sample, N)
    ev, ei = oracle_mod.select(xs.numpy(), k)
    assert_same(ev, ei, gv[sample].cpu().numpy(), gi[sample].cpu().numpy(), "C3 sample")


@pytest.mark.slow
@pytest.mark.parametrize("dist,k", [("T", 256), ("T", 1024), ("SD", 256), ("G", 1024), ("DG", 256), ("U", 1024)])
def test_config3_rows_other_distributions(K, oracle_mod, dist, k):
    # configs[2] row shape (N=2^20) with the kernel configuration the Q=16384 bench launch
    # uses (one warp per row, 3-stage ring: any Q > 1776 rows), on 2048 rows; heavy ties
    # exercise the strict pre-filter past the bound's index
    Q, N = 2048, 1 << 20
    seed = synth.seed_for(3, dist)
    x = synth.rows(dist, seed, 0, Q, N, device="cuda")
    gv, gi = K.ksel_select(x, k)
    torch.cuda.synchronize()
    sample = list(range(24)) + list(range(100, Q, 53))
    del x
    xs = synth.row_subset(dist, seed, sample, N)
    ev, ei = oracle_mod.select(xs.numpy(), k)
    assert_same(ev, ei, gv[sample].cpu().numpy(), gi[sample].cpu().numpy(), "C3-shape %s k=%d" % (dist, k))


# ---- split rows (few long rows over the whole GPU) ----------------

@pytest.mark.parametrize("Q,N", [(1, (1 << 18) + 13), (3, 1 << 20), (7, 3 * (1 << 19) + 1), (40, 1 << 18)])
@pytest.mark.parametrize("dist", ["U", "SA", "SD", "T", "X"])
def test_split_rows_vs_oracle(K, oracle_mod, Q, N, dist):
    # Q below the SM count: ksel_select cuts rows into segments (one CTA each, row-global
    # indices) and merges the S lists; ragged N makes unaligned segment heads and a short
    # last segment
    assert K.ksel_select_workspace(Q, N, 100) > 0
    x_cpu = synth.rows(dist, 41, 0, Q, N)
    x = x_cpu.cuda()
    for k in (1, 100, 256, 1024):
        gv, gi = K.ksel_select(x, k)
        dv, di = K.ksel_select(x, k, split_rows=False)
        torch.cuda.synchronize()
        ev, ei = oracle_mod.select(x_cpu.numpy(), k)
        assert_same(ev, ei, gv, gi, "split Q=%d N=%d %s k=%d" % (Q, N, dist, k))
        assert_same(ev, ei, dv, di, "direct Q=%d N=%d %s k=%d" % (Q, N, dist, k))


@pytest.mark.slow
def test_split_rows_single_long_row(K, oracle_mod):
    # one row of 2^24 over every SM (148 segments), then the second-level selection over
    # 148*k candidates with ties mapped back to row indices
    N = 1 << 24
    for dist in ("G", "T"):
        x = synth.rows(dist, 42, 0, 1, N, device="cuda")
        assert K.ksel_select_workspace(1, N, 64) > 0
        for k in (64, 1000):
            gv, gi = K.ksel_select(x, k)
            torch.cuda.synchronize()
            ev, ei = oracle_mod.select(x.cpu().numpy(), k)
            assert_same(ev, ei, gv, gi, "one row %s k=%d" % (dist, k))


def test_split_rows_shared_bound_edge_cases(K, oracle_mod):
    # the segments of a row share a row-wide bound: segments that end up with fewer than k
    # pairs below it pad with (NaN, -1), which the second level must never select; the
    # bound is not shared while it is NaN (rows with fewer than k non-NaN values)
    N = (1 << 20) + 7
    rng = np.random.default_rng(77)
    rows = []
    a = np.full(N, np.nan, dtype=np.float32)  # 50 finite values, the rest NaN (k > 50 below)
    a[rng.choice(N, 50, replace=False)] = rng.random(50, dtype=np.float32)
    rows.append(a)
    b = np.arange(N, dtype=np.float32)  # ascending: every later segment runs short
    rows.append(b)
    c = np.full(N, 2.0, dtype=np.float32)  # ties everywhere + a few smaller values late
    c[-100:] = 1.0
    rows.append(c)
    d = rng.random(N, dtype=np.float32)  # NaNs mixed into random values
    d[rng.choice(N, N // 3, replace=False)] = np.nan
    rows.append(d)
    x_cpu = torch.from_numpy(np.stack(rows))
    x = x_cpu.cuda()
    for k in (1, 64, 100, 1024):
        gv, gi = K.ksel_select(x, k)
        torch.cuda.synchronize()
        ev, ei = oracle_mod.select(x_cpu.numpy(), k)
        assert_same(ev, ei, gv, gi, "split shared-bound edge k=%d" % k)
        assert int(gi.min()) >= 0


def test_split_rows_workspace_errors(K):
    x = torch.rand(2, 1 << 20, device="cuda")
    v = torch.empty(2, 10, device="cuda")
    i = torch.empty(2, 10, dtype=torch.int32, device="cuda")
    need = K.ksel_select_workspace(2, 1 << 20, 10)
    assert need > 0
    small = torch.empty(need - 256, dtype=torch.uint8, device="cuda")
    st = K._lib.ksel_select_ex(x.data_ptr(), 2, 1 << 20, 10, v.data_ptr(), i.data_ptr(), small.data_ptr(),
                               small.numel(), K._stream(x.device))
    assert st == 1
    # enough rows for every SM: no workspace, ksel_select_ex == ksel_select
    assert K.ksel_select_workspace(4096, 1 << 16, 10) == 0


# ---- ksel_merge -----------------------------------------------------------

@pytest.mark.parametrize("S", [1, 2, 3, 8])
@pytest.mark.parametrize("dist", ["U", "T", "X"])
def test_sharded_select_then_merge_equals_full(K, oracle_mod, S, dist):
    # the row-sharded path on one GPU: per-shard ksel_select with global
    # indices, concatenate like an all-gather, ksel_merge == unsharded result
    Q, N = 64, 12000
    x = synth.rows(dist, 77, 0, Q, N)
    xg = x.cuda()
    bounds = np.linspace(0, N, S + 1).astype(int)
    for k in (1, 32, 100, 256, 1000):
        if any(bounds[s + 1] - bounds[s] < k for s in range(S)):
            continue
        vals, idxs = [], []
        for s in range(S):
            v, i = K.ksel_select(xg[:, bounds[s]:bounds[s + 1]].contiguous(), k)
            vals.append(v)
            idxs.append(i + int(bounds[s]))
        mv, mi = K.ksel_merge(torch.stack(vals).contiguous(), torch.stack(idxs).contiguous(), k)
        ev, ei = oracle_mod.select(x.numpy(), k)
        assert_same(ev, ei, mv, mi, "merge S=%d %s k=%d" % (S, dist, k))


def test_merge_vs_oracle_merge_unsorted_and_long_lists(K, oracle_mod):
    rng = np.random.default_rng(5)
    for (S, Q, kin, k) in [(2, 33, 4, 8), (4, 100, 100, 100), (3, 7, 1024, 64), (8, 50, 300, 1024), (5, 9, 37, 3)]:
        v = rng.integers(0, 50, size=(S, Q, kin)).astype(np.float32)
        i = rng.permutation(S * Q * kin).astype(np.int32).reshape(S, Q, kin)
        # sorted lists (the contract) ...
        order = np.lexsort((i, v), axis=-1)
        vs = np.take_along_axis(v, order, -1)
        is_ = np.take_along_axis(i, order, -1)
        ev, ei = oracle_mod.merge(vs, is_, k)
        gv, gi = K.ksel_merge(torch.from_numpy(vs).cuda(), torch.from_numpy(is_).cuda(), k)
        assert_same(ev, ei, gv, gi, "merge sorted %r" % ((S, Q, kin, k),))
        # ... and unsorted lists are handled exactly too
        ev, ei = oracle_mod.merge(v, i, k)
        gv, gi = K.ksel_merge(torch.from_numpy(v).cuda(), torch.from_numpy(i).cuda(), k)
        assert_same(ev, ei, gv, gi, "merge unsorted %r" % ((S, Q, kin, k),))


def test_merge_keeps_special_bits(K, oracle_mod):
    v = np.array([[[-0.0, 1.0, np.nan]], [[0.0, 2.0, float.fromhex("0x1.8p+0")]]], np.float32)
    v[0, 0, 2] = np.frombuffer(np.uint32(0x7fc00123).tobytes(), np.float32)[0]
    i = np.array([[[3, 4, 5]], [[1, 6, 7]]], np.int32)
    order = np.lexsort((i, v), axis=-1)
    vs, is_ = np.take_along_axis(v, order, -1), np.take_along_axis(i, order, -1)
    ev, ei = oracle_mod.merge(vs, is_, 6)
    gv, gi = K.ksel_merge(torch.from_numpy(vs).cuda(), torch.from_numpy(is_).cuda(), 6)
    assert_same(ev, ei, gv, gi, "merge special")


# ---- host (end-to-end) entry point ------------------------------------------

def test_select_host_pipeline(K, oracle_mod):
    Q, N, k = 300, 70000, 100
    x = synth.rows("DG", 55, 0, Q, N).pin_memory()
    ws = torch.empty(K.ksel_select_host_workspace(N, k) // 8, dtype=torch.uint8, device="cuda")  # force many blocks
    gv, gi = K.ksel_select_host(x, k, workspace=ws)
    ev, ei = oracle_mod.select(x.numpy(), k)
    assert_same(ev, ei, gv.numpy(), gi.numpy(), "host pipeline")


def test_launch_count_increments(K):
    x = torch.rand(4, 100, device="cuda")
    c0 = K.launch_count()
    K.ksel_select(x, 3)
    assert K.launch_count() == c0 + 1


@pytest.mark.parametrize("dist", synth.DISTS)
def test_synth_same_bits_on_gpu_and_cpu(dist):
    # the oracle may regenerate rows on the host: the generator must be device-independent
    a = synth.rows(dist, 123, 5000, 6, 7777, device="cuda").cpu()
    b = synth.rows(dist, 123, 5000, 6, 7777)
    assert torch.equal(a.view(torch.int32), b.view(torch.int32))
    for kind in ("knn-U", "knn-S"):
        p = synth.knn_points(kind, 9, 100, 50, 128, device="cuda").cpu()
        q = synth.knn_points(kind, 9, 100, 50, 128)
        assert torch.equal(p.view(torch.int32), q.view(torch.int32))


@pytest.mark.parametrize("seed", range(6))
def test_fuzz_shapes_all_algorithms(K, oracle_mod, seed):
    # random row counts / lengths / k / distributions / alignment, every kernel variant
    rng = np.random.default_rng(1000 + seed)
    for case in range(10):
        N = int(np.exp(rng.uniform(0, np.log(70000))))
        Q = int(max(1, min(300, 4_000_000 // max(N, 1), int(np.exp(rng.uniform(0, np.log(300)))))))
        k = int(rng.integers(1, min(N, 1024) + 1))
        dist = str(rng.choice(synth.DISTS))
        off = int(rng.integers(0, 4))
        big = synth.rows(dist, 7000 + seed * 10 + case, 0, 1, Q * N + off)[0]
        x_cpu = big[off:off + Q * N].reshape(Q, N).contiguous()
        xg = big.cuda()[off:off + Q * N].view(Q, N)
        ev, ei = oracle_mod.select(x_cpu.numpy(), k)
        algos = [0, 1, 2] + ([3] if N <= 65536 else [])
        for algo in algos:
            gv, gi = K.ksel_select(xg, k, algo=algo)
            torch.cuda.synchronize()
            assert_same(ev, ei, gv, gi, "fuzz seed=%d case=%d Q=%d N=%d k=%d %s off=%d algo=%d"
                        % (seed, case, Q, N, k, dist, off, algo))


@pytest.mark.parametrize("seed", range(3))
def test_fuzz_split_rows(K, oracle_mod, seed):
    # few long rows (the split-row path: segments per SM + a second selection)
    rng = np.random.default_rng(2000 + seed)
    for case in range(4):
        Q = int(rng.integers(1, 24))
        N = int(rng.integers(70000, 4_000_000 // Q + 70001))
        k = int(rng.integers(1, 1025))
        dist = str(rng.choice(synth.DISTS))
        x_cpu = synth.rows(dist, 8000 + seed * 10 + case, 0, Q, N)
        gv, gi = K.ksel_select(x_cpu.cuda(), k)
        torch.cuda.synchronize()
        ev, ei = oracle_mod.select(x_cpu.numpy(), k)
        assert_same(ev, ei, gv, gi, "split fuzz seed=%d case=%d Q=%d N=%d k=%d %s" % (seed, case, Q, N, k, dist))


@pytest.mark.parametrize("seed", range(3))
def test_fuzz_merge(K, oracle_mod, seed):
    # random list counts / lengths / k, lists from selections of random column blocks
    rng = np.random.default_rng(3000 + seed)
    for case in range(5):
        S = int(rng.integers(1, 9))
        kin = int(rng.integers(1, 1025))
        k = int(rng.integers(1, min(S * kin, 1024) + 1))
        Q = int(rng.integers(1, 200))
        W = max(kin, 64)
        dist = str(rng.choice(synth.DISTS))
        x = synth.rows(dist, 9000 + seed * 10 + case, 0, Q, S * W, device="cuda")
        vs, is_ = [], []
        for s in range(S):
            v, i = K.ksel_select(x[:, s * W:(s + 1) * W].contiguous(), kin)
            vs.append(v)
            is_.append(i + s * W)
        cv, ci = torch.stack(vs), torch.stack(is_)
        gv, gi = K.ksel_merge(cv, ci, k)
        torch.cuda.synchronize()
        ev, ei = oracle_mod.merge(cv.cpu().numpy(), ci.cpu().numpy(), k)  # top-k of the union of the lists
        assert_same(ev, ei, gv, gi, "merge fuzz seed=%d case=%d S=%d kin=%d k=%d Q=%d %s" % (seed, case, S, kin, k, Q, dist))


@pytest.mark.parametrize("seed", range(2))
def test_fuzz_select_host(K, oracle_mod, seed):
    # the host-buffer entry (double-buffered H2D / select / D2H): pinned and pageable
    # inputs, workspaces from one block to many
    rng = np.random.default_rng(4000 + seed)
    for case in range(4):
        N = int(rng.integers(1, 200000))
        Q = int(rng.integers(1, max(2, 3_000_000 // N)))
        k = int(rng.integers(1, min(N, 1024) + 1))
        dist = str(rng.choice(synth.DISTS))
        x = synth.rows(dist, 4100 + seed * 10 + case, 0, Q, N)
        if case % 2 == 0:
            x = x.pin_memory()
        need = K.ksel_select_host_workspace(N, k)
        ws = torch.empty(max(need // int(rng.integers(1, 9)), need // 8 + 1), dtype=torch.uint8, device="cuda")
        if ws.numel() < need // 8:
            ws = torch.empty(need, dtype=torch.uint8, device="cuda")
        gv, gi = K.ksel_select_host(x, k, workspace=ws)
        ev, ei = oracle_mod.select(x.numpy(), k)
        assert_same(ev, ei, gv.numpy(), gi.numpy(), "host fuzz seed=%d case=%d Q=%d N=%d k=%d %s" % (seed, case, Q, N, k, dist))


_ORDER_CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import paper_conf_ipps_tang0emg15_b200 as K, synth
out = {}
for dist in ("U", "T", "SA", "SD", "X"):
    x = synth.rows(dist, 61, 0, 300, 20011, device="cuda")
    for k in (1, 100, 1024):
        for wpr in (0, 1, 4):
            v, i = K.ksel_select(x, k, algo=2, warps_per_row=wpr)
            out["%s_%d_%d_v" % (dist, k, wpr)] = v.cpu().numpy()
            out["%s_%d_%d_i" % (dist, k, wpr)] = i.cpu().numpy()
np.savez(sys.argv[2], **out)
"""


@pytest.mark.parametrize("order", ["0", "1", "2", "3", "3-nospec"])
def test_chunk_visit_orders_bit_exact(oracle_mod, order, tmp_path):
    # the chunk visit order (KSEL_ORDER, read once per process; default 3) and the speculative
    # starting bound (KSEL_SPEC=0: off) change only which candidates are admitted when, never
    # the result
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    f = str(tmp_path / "res.npz")
    env = dict(os.environ, KSEL_ORDER=order[0])
    if order.endswith("nospec"):
        env["KSEL_SPEC"] = "0"
    subprocess.run([sys.executable, "-c", _ORDER_CHILD, root, f], env=env, check=True, timeout=600)
    res = np.load(f)
    for dist in ("U", "T", "SA", "SD", "X"):
        x = synth.rows(dist, 61, 0, 300, 20011).numpy()
        for k in (1, 100, 1024):
            ev, ei = oracle_mod.select(x, k)
            for wpr in (0, 1, 4):
                assert_same(ev, ei, res["%s_%d_%d_v" % (dist, k, wpr)], res["%s_%d_%d_i" % (dist, k, wpr)],
                            "KSEL_ORDER=%s %s k=%d wpr=%d" % (order, dist, k, wpr))


@pytest.mark.parametrize("seed", range(4))
def test_fuzz_clustered_ties_many_narrowings(K, oracle_mod, seed):
    # rows long enough for many mid-stream narrowings (which stop early at a valid, not
    # exact, bound) with values drawn from a few hundred levels -- tie runs of random length
    # straddle every rank a narrowing may stop at -- plus -0.0/+0.0, +-Inf and NaN sprinkled in
    rng = np.random.default_rng(7000 + seed)
    for case in range(3):
        Q = int(rng.integers(3, 40))
        N = int(rng.integers(60000, 260000))
        levels = np.sort(rng.standard_normal(int(rng.integers(20, 400))).astype(np.float32))
        x = levels[rng.integers(0, levels.size, size=(Q, N))]
        specials = np.array([0.0, -0.0, np.inf, -np.inf, np.nan], dtype=np.float32)
        mask = rng.random((Q, N)) < 0.002
        x[mask] = specials[rng.integers(0, specials.size, size=int(mask.sum()))]
        x_cpu = torch.from_numpy(np.ascontiguousarray(x))
        xg = x_cpu.cuda()
        for k in (int(rng.integers(1, 64)), int(rng.integers(64, 600)), int(rng.integers(600, 1025))):
            ev, ei = oracle_mod.select(x, k)
            for algo, wpr in ((0, 0), (2, 1), (2, 2), (2, 8)):
                gv, gi = K.ksel_select(xg, k, algo=algo, warps_per_row=wpr)
                torch.cuda.synchronize()
                assert_same(ev, ei, gv, gi, "clustered seed=%d case=%d Q=%d N=%d k=%d algo=%d wpr=%d"
                            % (seed, case, Q, N, k, algo, wpr))


@pytest.mark.parametrize("k", [32, 256, 1000])
@pytest.mark.parametrize("wpr", [1, 2])
def test_speculative_bound_failure_restreams(K, oracle_mod, k, wpr):
    """The pool kernel's speculative starting bound (the j-th of the sampled chunks) assumes the
    sample is representative.  Here every warp's sampled chunks (its first and last chunks:
    visit order 3) hold the row's smallest values, so the j-th sampled key has fewer than k of
    the warp's keys below it: the verification at the end of the share fails, the share is
    streamed again from the rigorous bound -- and the result must still be the oracle's."""
    Q, N = 24, 65536
    x = synth.rows("U", synth.seed_for(21, "U"), 0, Q, N) * 0.5 + 0.5  # U[0.5, 1)
    small = synth.rows("U", synth.seed_for(22, "U"), 0, Q, N) * 1e-3    # U[0, 1e-3)
    nch = N // 512
    L = (k + 511) // 512 + 1
    for w in range(wpr):
        c0, c1 = nch * w // wpr, nch * (w + 1) // wpr
        for c in [c0] + list(range(c1 - L, c1)):
            x[:, c * 512:(c + 1) * 512] = small[:, c * 512:(c + 1) * 512]
    _check_select(K, oracle_mod, x.contiguous(), k, "spec-fail k=%d wpr=%d" % (k, wpr), algo=2, wpr=wpr)
