"""Multi-GPU drivers (one process per GPU, torch.distributed for the plumbing).

Two modes:

* ``ksel_select`` shards by queries: rows are independent ("the k-selection for
  different queries can be embarrassingly parallelized"), rank r
  owns rows [r*Q/g, (r+1)*Q/g) -- no collective at all (:func:`query_rows`).
* ``knn_search`` shards the reference set by rows: rank r holds references
  [r*N/g, (r+1)*N/g), computes the per-query top-k of its shard with global
  indices (idx_offset), the candidates are exchanged with one NCCL
  all-gather over NVLink and ``ksel_merge`` (divide-and-merge)
  produces the exact global top-k.  Each rank merges only its own slice of
  queries, so the merge work also scales with g (:func:`knn_search_sharded`).

Exactness: each shard's lexicographic (value, index) order is the global one
(indices are offset monotonically), every global top-k element is in its
shard's top-k, so the merge of the shard lists is the global top-k --
bit-identical to the unsharded result.

The local kernels and the collective are parameters so that the host-side
logic (partitioning, offsets, packing, slicing) can be exercised with gloo on
CPU in tests; the defaults are the CUDA library and NCCL.
"""
from __future__ import annotations

import torch
import torch.distributed as tdist


def shard_range(n: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous block [a, b) of n items owned by `rank` out of `world`."""
    return n * rank // world, n * (rank + 1) // world


def query_rows(Q: int, world: int, rank: int) -> tuple[int, int]:
    """Rows of a query-sharded ksel_select owned by this rank (no communication)."""
    return shard_range(Q, world, rank)


def _default_knn(ref, query, k, idx_offset):
    from . import knn_search
    return knn_search(ref, query, k, idx_offset=idx_offset)


def _default_merge(cand_val, cand_idx, k):
    from . import ksel_merge
    return ksel_merge(cand_val, cand_idx, k)


def _all_gather(out: torch.Tensor, inp: torch.Tensor, group=None):
    """all_gather_into_tensor, with a list fallback for backends without it."""
    try:
        tdist.all_gather_into_tensor(out, inp, group=group)
    except (RuntimeError, AttributeError, NotImplementedError):
        world = tdist.get_world_size(group)
        parts = list(out.chunk(world, dim=0))
        tdist.all_gather(parts, inp, group=group)


def knn_search_sharded(ref_shard: torch.Tensor, query: torch.Tensor, k: int, n_total: int, group=None,
                       local_knn=None, merge=None):
    """Row-sharded k-NN: local top-k with global indices, all-gather, merge.

    ``ref_shard`` holds this rank's references (rows shard_range(n_total, g, r)),
    ``query`` all Q queries (replicated).  Returns (values, indices, (q0, q1)):
    the exact global top-k of queries [q0, q1) -- this rank's slice.
    """
    world = tdist.get_world_size(group)
    rank = tdist.get_rank(group)
    local_knn = local_knn or _default_knn
    merge = merge or _default_merge
    r0, r1 = shard_range(n_total, world, rank)
    assert ref_shard.shape[0] == r1 - r0, "ref_shard must hold rows [%d, %d)" % (r0, r1)
    Q = query.shape[0]
    v, i = local_knn(ref_shard, query, k, r0)
    # one collective: (value bits, index) packed as int32 pairs
    packed = torch.stack([v.contiguous().view(torch.int32), i.contiguous()], dim=-1)  # [Q, k, 2]
    flat = torch.empty((world * Q,) + tuple(packed.shape[1:]), dtype=packed.dtype, device=packed.device)
    _all_gather(flat, packed, group)
    gathered = flat.view((world,) + tuple(packed.shape))
    q0, q1 = shard_range(Q, world, rank)
    cand = gathered[:, q0:q1]
    cand_val = cand[..., 0].contiguous().view(torch.float32)  # [world, q1-q0, k]
    cand_idx = cand[..., 1].contiguous()
    mv, mi = merge(cand_val, cand_idx, k)
    return mv, mi, (q0, q1)
