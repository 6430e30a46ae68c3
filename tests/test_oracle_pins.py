"""Pins for the CPU oracle (oracle/) against things other than itself.

Each test checks the oracle against something the paper or mathematics fixes
(SURVEY.md 8(c) "What pins each part"):

* brute-force rank counting, exhaustive over a tiny alphabet containing every
  special value (reading R1-R5), written independently of the oracle's sort;
* a library routine: numpy's stable argsort (NaNs last, -0.0 == +0.0);
* the north-star invariants (sorted, selected <= excluded, distinct in-range
  indices, bit-exact values, k=1 argmin, k=N full sort) and special rows;
* the paper's worked examples (tests/golden/, each citing PAPER.md lines);
* for the distance: exact integer arithmetic, torch.cdist in float64,
  geometric special cases.

A plausible oracle bug -- a flipped comparison, ties by higher index, NaN
first, -0.0 < +0.0, a dropped term or wrong sign in the distance, transposed
ref/query -- fails at least one of these.
"""
import itertools
import math
import random
import struct

import numpy as np
import pytest
import torch

import synth
from conftest import read_golden

ALPHABET = [0.0, 1.0, 2.0, -0.0, math.inf, math.nan]


def _bits(a):
    return np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)


def _brute_rank_select(row, k):
    """Rank counting: rank(j) = #{i : (v_i, i) precedes (v_j, j)}; slot = rank.

    The value order is written here independently: NaN after everything, all
    NaNs equal, otherwise Python float comparison (-0.0 == 0.0)."""
    def before(a, i, b, j):
        an, bn = math.isnan(a), math.isnan(b)
        if an and bn:
            return i < j
        if an:
            return False
        if bn:
            return True
        if a != b:
            return a < b
        return i < j

    n = len(row)
    vals = [None] * k
    idxs = [None] * k
    for j in range(n):
        r = sum(1 for i in range(n) if i != j and before(row[i], i, row[j], j))
        if r < k:
            vals[r] = row[j]
            idxs[r] = j
    return vals, idxs


@pytest.mark.parametrize("L", [1, 2, 3, 4, 5, 6])
def test_exhaustive_rank_counting(oracle_mod, L):
    rows = np.array(list(itertools.product(ALPHABET, repeat=L)), dtype=np.float32)
    for k in range(1, L + 1):
        ov, oi = oracle_mod.select(rows, k)
        for q in range(rows.shape[0]):
            ev, ei = _brute_rank_select([float(x) for x in rows[q]], k)
            assert list(oi[q]) == ei, (rows[q], k)
            assert list(_bits(ov[q])) == list(_bits(np.array(ev, np.float32))), (rows[q], k)


def test_random_len7_rank_counting(oracle_mod):
    rng = random.Random(7)
    rows = np.array([[rng.choice(ALPHABET) for _ in range(7)] for _ in range(3000)], np.float32)
    for k in (1, 3, 7):
        ov, oi = oracle_mod.select(rows, k)
        for q in range(rows.shape[0]):
            ev, ei = _brute_rank_select([float(x) for x in rows[q]], k)
            assert list(oi[q]) == ei


def test_survey_special_row_matches_numpy_and_torch(oracle_mod):
    # [NaN, 1, -0, +0, Inf, -Inf, NaN, -0, 1] -> [5,2,3,7,1,8,4,0,6]
    row = np.array([[math.nan, 1, -0.0, 0.0, math.inf, -math.inf, math.nan, -0.0, 1]], np.float32)
    expect = [5, 2, 3, 7, 1, 8, 4, 0, 6]
    assert list(np.argsort(row[0], kind="stable")) == expect
    assert torch.sort(torch.from_numpy(row[0]), stable=True).indices.tolist() == expect
    ov, oi = oracle_mod.select(row, 9)
    assert list(oi[0]) == expect
    assert list(_bits(ov[0])) == list(_bits(row[0][expect]))


@pytest.mark.parametrize("dist", synth.DISTS)
def test_numpy_stable_argsort(oracle_mod, dist):
    x = synth.rows(dist, synth.seed_for(0, dist), 0, 24, 1531).numpy()
    for k in (1, 2, 31, 32, 33, 256, 1000, 1531):
        ov, oi = oracle_mod.select(x, k)
        ref = np.argsort(x, axis=1, kind="stable")[:, :k]
        assert np.array_equal(oi, ref.astype(np.int32)), (dist, k)
        assert np.array_equal(_bits(ov), _bits(np.take_along_axis(x, ref, axis=1)))


@pytest.mark.parametrize("dist", ["U", "G", "DG", "T", "SD"])
def test_invariants(oracle_mod, dist):
    Q, N = 16, 4096
    x = synth.rows(dist, synth.seed_for(1, dist), 0, Q, N).numpy()
    for k in (1, 7, 32, 100, 1024):
        ov, oi = oracle_mod.select(x, k)
        for q in range(Q):
            idx = oi[q]
            assert len(set(idx.tolist())) == k
            assert idx.min() >= 0 and idx.max() < N
            assert np.array_equal(_bits(ov[q]), _bits(x[q][idx]))
            # sorted by (value, index)
            for t in range(k - 1):
                assert ov[q][t] < ov[q][t + 1] or (ov[q][t] == ov[q][t + 1] and idx[t] < idx[t + 1])
            # every output value <= every excluded value; ties at the k-th value
            # are resolved by index (no excluded equal value has a smaller index)
            mask = np.ones(N, bool)
            mask[idx] = False
            assert ov[q].max() <= x[q][mask].min()
            kth = ov[q][-1]
            excluded_ties = np.nonzero(mask & (x[q] == kth))[0]
            if excluded_ties.size:
                assert excluded_ties.min() > idx[ov[q] == kth].max()
        if k == 1:
            assert np.array_equal(oi[:, 0], np.argmin(x, axis=1).astype(np.int32))


def test_k_equals_n_is_full_sort(oracle_mod):
    x = synth.rows("T", 3, 0, 8, 300).numpy()
    ov, oi = oracle_mod.select(x, 300)
    assert np.array_equal(oi, np.argsort(x, axis=1, kind="stable").astype(np.int32))


def test_special_rows(oracle_mod):
    N, k = 1000, 37
    same = np.full((1, N), 0.25, np.float32)
    asc = np.arange(N, dtype=np.float32)[None]
    desc = asc[:, ::-1].copy()
    assert list(oracle_mod.select(same, k)[1][0]) == list(range(k))
    assert list(oracle_mod.select(asc, k)[1][0]) == list(range(k))
    assert list(oracle_mod.select(desc, k)[1][0]) == list(range(N - 1, N - 1 - k, -1))
    # permuting a row permutes the indices and keeps the value multiset
    x = synth.rows("U", 11, 0, 1, N).numpy()
    perm = np.random.default_rng(0).permutation(N)
    v1, i1 = oracle_mod.select(x, k)
    v2, i2 = oracle_mod.select(x[:, perm], k)
    assert np.array_equal(_bits(v1), _bits(v2))
    assert np.array_equal(perm[i2[0]], i1[0])


def test_denormals_and_signed_zero_bits(oracle_mod):
    tiny = struct.unpack("<f", struct.pack("<I", 1))[0]
    row = np.array([[tiny, -0.0, 0.0, -tiny, 2 * tiny]], np.float32)
    ov, oi = oracle_mod.select(row, 5)
    assert list(oi[0]) == [3, 1, 2, 0, 4]
    assert list(_bits(ov[0])) == [0x80000001, 0x80000000, 0, 1, 2]


# ---- paper worked examples (tests/golden) ---------------------------------

def test_golden_fig1b_merge_queue(oracle_mod):
    g = dict(read_golden("fig1b_merge_queue.txt"))
    row = np.array([[float(t) for t in g["row"].split()]], np.float32)
    ov, oi = oracle_mod.select(row, int(g["k"]))
    assert [float(v) for v in ov[0]] == [float(t) for t in g["expect_val"].split()]
    assert list(oi[0]) == [int(t) for t in g["expect_idx"].split()]


def test_golden_fig2_bitonic_merge(oracle_mod):
    entries = read_golden("fig2_bitonic_merge.txt")
    lists = [[tuple(p.split(":")) for p in v.split()] for key, v in entries if key == "list"]
    g = dict(entries)
    vals = np.array([[[float(a) for a, _ in L]] for L in lists], np.float32)
    idxs = np.array([[[int(b) for _, b in L]] for L in lists], np.int32)
    ov, oi = oracle_mod.merge(vals, idxs, int(g["k"]))
    assert [float(v) for v in ov[0]] == [float(t) for t in g["expect_val"].split()]
    assert list(oi[0]) == [int(t) for t in g["expect_idx"].split()]


def test_golden_fig3_buffered_search(oracle_mod):
    for key, v in read_golden("fig3_buffered_search.txt"):
        head, lst, buf, pos = [p.split() for p in v.split("|")]
        row = np.array([[float(t) for t in lst]], np.float32)
        c = sum(1 for t in lst if float(t) < float(head[0]))
        assert c == len(buf)
        ov, oi = oracle_mod.select(row, c)
        assert [float(x) for x in ov[0]] == [float(t) for t in buf]
        assert list(oi[0]) == [int(t) for t in pos]


def test_golden_fig4_hierarchical_partition(oracle_mod):
    entries = read_golden("fig4_hierarchical_partition.txt")
    g = dict(entries)
    k = int(g["k"])
    for key, v in entries:
        if key != "row":
            continue
        row = np.array([[float(t) for t in v.split()]], np.float32)
        assert sorted(row[0].tolist()) == list(range(16))
        ov, oi = oracle_mod.select(row, k)
        assert [float(x) for x in ov[0]] == [float(t) for t in g["expect_val"].split()]
        assert list(oi[0]) == [int(np.nonzero(row[0] == float(t))[0][0]) for t in g["expect_val"].split()]


# ---- merge ------------------------------------------------------------------

def test_merge_of_column_shards_equals_full_select(oracle_mod):
    # divide-and-merge: per-shard top-k with global indices,
    # merged, equals the unsharded top-k -- on tie-heavy rows too.
    for dist in ("T", "U", "X"):
        x = synth.rows(dist, 21, 0, 12, 1200).numpy()
        k = 50
        for S in (2, 3, 4):
            bounds = np.linspace(0, 1200, S + 1).astype(int)
            vals, idxs = [], []
            for s in range(S):
                v, i = oracle_mod.select(x[:, bounds[s]:bounds[s + 1]], k)
                vals.append(v)
                idxs.append(i + bounds[s])
            mv, mi = oracle_mod.merge(np.stack(vals), np.stack(idxs), k)
            fv, fi = oracle_mod.select(x, k)
            assert np.array_equal(mi, fi)
            assert np.array_equal(_bits(mv), _bits(fv))


def test_merge_brute_force(oracle_mod):
    rng = random.Random(3)
    for _ in range(200):
        S, kin = rng.randint(1, 4), rng.randint(1, 6)
        pool = [rng.choice(ALPHABET) for _ in range(S * kin)]
        ids = rng.sample(range(1000), S * kin)
        lists = []
        for s in range(S):
            L = sorted(zip(pool[s * kin:(s + 1) * kin], ids[s * kin:(s + 1) * kin]),
                       key=lambda p: (math.isnan(p[0]), 0.0 if math.isnan(p[0]) else p[0], p[1]))
            lists.append(L)
        k = rng.randint(1, S * kin)
        vals = np.array([[[a for a, _ in L]] for L in lists], np.float32)
        idxs = np.array([[[b for _, b in L]] for L in lists], np.int32)
        ov, oi = oracle_mod.merge(vals, idxs, k)
        allp = sorted(zip(pool, ids), key=lambda p: (math.isnan(p[0]), 0.0 if math.isnan(p[0]) else p[0], p[1]))
        assert list(oi[0]) == [b for _, b in allp[:k]]


# ---- k-NN distance ------------------------------------------------------------

def test_knn_dist_exact_on_integers(oracle_mod):
    # Integer data in [0,255], D = 128: the exact squared distance is an integer
    # < 2^24, computed here with Python ints (no rounding anywhere).
    ref = synth.knn_points("knn-S", 5, 0, 40, 128).numpy()
    qry = synth.knn_points("knn-S", 6, 0, 7, 128).numpy()
    d = oracle_mod.knn_dist(ref, qry)
    R = ref.astype(np.int64)
    Qm = qry.astype(np.int64)
    for q in range(7):
        for r in range(40):
            exact = int(sum((int(a) - int(b)) ** 2 for a, b in zip(Qm[q], R[r])))
            assert d[q, r] == exact


def test_knn_dist_vs_cdist_float64(oracle_mod):
    ref = synth.knn_points("knn-U", 7, 0, 300, 128)
    qry = synth.knn_points("knn-U", 8, 0, 9, 128)
    d = oracle_mod.knn_dist(ref.numpy(), qry.numpy())
    c = torch.cdist(qry.double(), ref.double()) ** 2
    rel = np.abs(d.astype(np.float64) - c.numpy()) / c.numpy()
    assert rel.max() < 2e-7  # one fp32 rounding of a double value (plus cdist's sqrt^2)


def test_knn_geometry(oracle_mod):
    D = 16
    eye = np.eye(D, dtype=np.float32)
    d = oracle_mod.knn_dist(eye, eye)
    assert np.array_equal(d, 2.0 * (1 - np.eye(D, dtype=np.float32)))
    # asymmetric roles: ref (N x D) vs query (Q x D) are not transposed
    ref = np.array([[0, 0, 0], [3, 4, 0]], np.float32)
    qry = np.array([[0, 0, 12]], np.float32)
    assert oracle_mod.knn_dist(ref, qry).tolist() == [[144.0, 169.0]]


def test_knn_self_match_first(oracle_mod):
    ref = synth.knn_points("knn-U", 9, 0, 500, 32).numpy()
    qry = ref[[17, 250, 499]]
    dv, di = oracle_mod.knn(ref, qry, 5, idx_offset=1000)
    assert list(di[:, 0]) == [1017, 1250, 1499]
    assert list(dv[:, 0]) == [0.0, 0.0, 0.0]
    assert np.all(np.diff(dv, axis=1) >= 0)


def test_knn_graph_brute_force_integers(oracle_mod):
    """k-NN graph (QMS [9]): exact Python integer distances,
    self excluded, ties (duplicate points) by lower index."""
    rng = random.Random(11)
    for trial in range(40):
        N, D = rng.randint(2, 9), rng.randint(1, 4)
        pts = [[rng.randint(0, 3) for _ in range(D)] for _ in range(N)]
        k = rng.randint(1, N - 1)
        ov, oi = oracle_mod.knn_graph(np.array(pts, np.float32), k)
        for i in range(N):
            pairs = sorted((sum((a - b) ** 2 for a, b in zip(pts[i], pts[j])), j) for j in range(N) if j != i)[:k]
            assert oi[i].tolist() == [j for _, j in pairs], (trial, i)
            assert ov[i].tolist() == [float(d) for d, _ in pairs], (trial, i)


def test_knn_graph_equals_knn_without_self(oracle_mod):
    x = synth.knn_points("knn-U", 21, 0, 60, 16).numpy()
    ov, oi = oracle_mod.knn_graph(x, 7)
    for i in (0, 17, 59):
        rest = np.delete(x, i, axis=0)
        rv, ri = oracle_mod.knn(rest, x[i:i + 1], 7)
        ri = ri[0] + (ri[0] >= i)  # back to indices of x
        assert np.array_equal(oi[i], ri) and np.array_equal(ov[i].view(np.uint32), rv[0].view(np.uint32))
        assert i not in oi[i].tolist()
