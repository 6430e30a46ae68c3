"""Multi-GPU drivers (one process per GPU, torch.distributed for the plumbing).

Two modes:

* ``ksel_select`` shards by queries: rows are independent ("the k-selection for
  different queries can be embarrassingly parallelized"), rank r
  owns rows [r*Q/g, (r+1)*Q/g) -- no collective at all (:func:`query_rows`).
* ``knn_search`` shards the reference set by rows: rank r holds references
  [r*N/g, (r+1)*N/g), computes the per-query top-k of its shard with global
  indices (idx_offset), the candidates are exchanged with NCCL all-gathers over
  NVLink -- one per query chunk, overlapping the next chunk's search -- and the
  merge (divide-and-merge) reads the gathered lists in place and
  produces the exact global top-k.  Each rank merges only its own slice of every
  chunk, so the merge work also scales with g (:func:`knn_search_sharded`).

Exactness: each shard's lexicographic (value, index) order is the global one
(indices are offset monotonically), every global top-k element is in its
shard's top-k, so the merge of the shard lists is the global top-k --
bit-identical to the unsharded result.

The local kernels are parameters so that the host-side logic (partitioning,
offsets, chunking, the in-place buffers, slicing) can be exercised with gloo on
CPU in tests; the defaults are the CUDA library (and NCCL under torchrun).
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


def _default_knn(ref, query, k, idx_offset, out_val, out_idx):
    from . import knn_search
    knn_search(ref, query, k, idx_offset=idx_offset, out_dist=out_val, out_idx=out_idx)


def _default_merge(vals, idxs, k, out_val, out_idx):
    """Top-k of the union of the lists vals[s] / idxs[s] ([nq, kin] views, possibly inside
    one gathered buffer): ksel_merge_lists reads them in place through a pointer table."""
    from . import ksel_merge_lists
    nq, kin = vals[0].shape
    ksel_merge_lists([v.data_ptr() for v in vals], [i.data_ptr() for i in idxs], nq, kin, k, out_val, out_idx)


def _all_gather(out: torch.Tensor, inp: torch.Tensor, group=None, async_op=False):
    """all_gather_into_tensor, with a list fallback for backends without it."""
    try:
        return tdist.all_gather_into_tensor(out, inp, group=group, async_op=async_op)
    except (RuntimeError, AttributeError, NotImplementedError):
        world = tdist.get_world_size(group)
        parts = list(out.chunk(world, dim=0))
        return tdist.all_gather(parts, inp, group=group, async_op=async_op)


def auto_chunks(Q: int) -> int:
    """Query chunks of the exchange pipeline.  Every extra knn_search call pays a cold
    start (first-wave CTAs without a published bound) and a reference prologue; measured
    on one B200 at configs[4]'s per-rank shape (10^6 references, Q = 10^4, k = 1024):
    1 / 2 / 4 chunks = 18.4 / 23.6 / 36.8 ms per step against an all-gather of ~1 ms at
    8 GPUs -- so the pipeline is used only for large query batches (>= 20000 per chunk)."""
    return max(1, min(4, Q // 20000))


def chunk_ranges(Q: int, chunks: int) -> list:
    """Contiguous query chunks [a, b) of the exchange pipeline."""
    c = max(1, min(int(chunks), Q))
    return [shard_range(Q, c, i) for i in range(c)]


def knn_search_sharded(ref_shard: torch.Tensor, query: torch.Tensor, k: int, n_total: int, group=None,
                       chunks: int | None = None, local_knn=None, merge=None):
    """Row-sharded k-NN: local top-k with global indices, all-gather, merge -- pipelined
    over query chunks.

    ``ref_shard`` holds this rank's references (rows shard_range(n_total, g, r)),
    ``query`` all Q queries (replicated).  Queries go in ``chunks`` contiguous chunks; for
    chunk c the local search writes its (value bits, index) lists straight into one
    [2][qc][k] send buffer, ONE all-gather (async, NCCL over NVLink) moves them into a
    [g][2][qc][k] receive buffer while the search of chunk c + 1 runs, and this rank then
    merges its slice of chunk c's queries reading the g lists in place (pointer tables:
    no stacking, no copies).  Returns (values, indices, qids): the exact global top-k of
    the queries qids (this rank's slice of every chunk, ascending).
    """
    world = tdist.get_world_size(group)
    rank = tdist.get_rank(group)
    local_knn = local_knn or _default_knn
    merge = merge or _default_merge
    r0, r1 = shard_range(n_total, world, rank)
    assert ref_shard.shape[0] == r1 - r0, "ref_shard must hold rows [%d, %d)" % (r0, r1)
    Q = query.shape[0]
    dev = query.device
    spans = chunk_ranges(Q, auto_chunks(Q) if chunks is None else chunks)
    slices = [(qa + shard_range(qb - qa, world, rank)[0], qa + shard_range(qb - qa, world, rank)[1])
              for qa, qb in spans]
    qids = torch.cat([torch.arange(a, b, dtype=torch.int64) for a, b in slices])
    out_v = torch.empty((qids.numel(), k), dtype=torch.float32, device=dev)
    out_i = torch.empty((qids.numel(), k), dtype=torch.int32, device=dev)
    pending = []  # (work, recv, slice in the chunk, output row offset)

    def finish(item):
        work, recv, (s0, s1), off = item
        if work is not None:
            work.wait()
        if s1 > s0:
            vals = [recv[s, 0, s0:s1].view(torch.float32) for s in range(world)]
            idxs = [recv[s, 1, s0:s1] for s in range(world)]
            merge(vals, idxs, k, out_v[off:off + s1 - s0], out_i[off:off + s1 - s0])

    off = 0
    for (qa, qb), (sa, sb) in zip(spans, slices):
        qc = qb - qa
        send = torch.empty((2, qc, k), dtype=torch.int32, device=dev)
        local_knn(ref_shard, query[qa:qb], k, r0, send[0].view(torch.float32), send[1])
        recv = torch.empty((world, 2, qc, k), dtype=torch.int32, device=dev)
        work = _all_gather(recv.view(-1), send.view(-1), group, async_op=True)
        # the previous chunk's exchange overlapped this chunk's search: merge it now
        if pending:
            finish(pending.pop())
        pending.append((work, recv, (sa - qa, sb - qa), off))
        off += sb - sa
    while pending:
        finish(pending.pop())
    return out_v, out_i, qids


# ---------------------------------------------------------------------------
# Collective-free exchange: the merge reads peers' lists
# ---------------------------------------------------------------------------

_P2P_HDR = 512  # bytes: ready[2][8] u32 at 0, consumed[world <= 64] u32 at 64
P2P_MAX_CHUNKS = 8


def p2p_layout(Q: int, k: int, world: int) -> dict:
    """Byte offsets inside each rank's exchange buffer.

    ``ready(b, c)``: u32 epoch flag of query chunk c of double buffer b (written by
    the owner); ``consumed(s)``: u32 epoch flag written by rank s once it merged the
    owner's lists; ``val(b)`` / ``idx(b)``: the owner's [Q][k] fp32 / int32 top-k lists.
    """
    if not 1 <= world <= 64:
        raise ValueError("world size must be in [1, 64]")
    lst = Q * k * 4
    return {
        "ready": lambda b, c=0: 4 * (b * P2P_MAX_CHUNKS + c),
        "consumed": lambda s: 64 + 4 * s,
        "val": lambda b: _P2P_HDR + b * 2 * lst,
        "idx": lambda b: _P2P_HDR + b * 2 * lst + lst,
        "bytes": _P2P_HDR + 4 * lst,
    }


class KnnP2P:
    """Row-sharded k-NN whose exchange is the merge reading peers' memory.

    One exportable buffer per rank (``ipc_alloc``) holds two epochs of its
    [Q][k] candidate lists plus flags; handles are exchanged once over the
    process group and mapped with CUDA IPC (NVLink / NVSwitch peer memory; on a
    single GPU, several processes share it the same way).  Per call (epoch e,
    buffer b = e % 2), all stream-ordered on the current stream, no host sync,
    pipelined over ``chunks`` query chunks:

    1. (e >= 2) wait until every rank consumed epoch e - 2 of this buffer;
    2. for each chunk c: ``knn_search`` of the local shard (global indices) for
       chunk c's queries straight into buffer b, then signal ready[b][c] = e + 1;
       after chunk c's search, ``ksel_merge_lists`` of chunk c - 1 -- this rank's
       slice of it, read in place from the peers' buffers, each list waited for
       (ready >= e + 1) -- so the peers' chunk c - 1 is normally complete while
       the next search is queued behind the merge;
    3. signal consumed[rank] = e + 1 in every peer's buffer.

    Same result as :func:`knn_search_sharded` (bit-identical to unsharded).
    """

    def __init__(self, Q: int, k: int, n_total: int, group=None, local_knn=None, chunks: int | None = None):
        from . import ipc_alloc, ipc_open
        self.group = group
        self.world = tdist.get_world_size(group)
        self.rank = tdist.get_rank(group)
        self.Q, self.k, self.n_total = Q, k, n_total
        self.lay = p2p_layout(Q, k, self.world)
        self.local_knn = local_knn
        self.base, handle = ipc_alloc(self.lay["bytes"])
        torch.cuda.synchronize()
        handles = [None] * self.world
        tdist.all_gather_object(handles, handle, group=group)
        self.peer = [self.base if s == self.rank else ipc_open(handles[s]) for s in range(self.world)]
        tdist.barrier(group=group)
        self.chunks = max(1, min(int(auto_chunks(Q) if chunks is None else chunks), P2P_MAX_CHUNKS, Q))
        self.epoch = 0
        self.warm = False

    def _warm_up(self, D: int, device):
        # Load every kernel the exchange uses before any cross-process wait is pending:
        # with CUDA lazy loading, a module load may otherwise queue behind a spinning wait.
        from . import flag_signal, flag_wait, knn_search, ksel_merge_lists
        k = self.k
        ref = torch.zeros((max(k, 32), D), dtype=torch.float32, device=device)
        v, i = knn_search(ref, ref[:1].contiguous(), k)
        scratch = torch.zeros(1, dtype=torch.int32, device=device)
        flag_signal(scratch.data_ptr(), 0)
        flag_wait([scratch.data_ptr()], 0)
        mv = torch.empty((1, k), dtype=torch.float32, device=device)
        mi = torch.empty((1, k), dtype=torch.int32, device=device)
        ksel_merge_lists([v.data_ptr()], [i.data_ptr()], 1, k, k, mv, mi, ready_ptrs=[scratch.data_ptr()], epoch=0)
        torch.cuda.synchronize()
        tdist.barrier(group=self.group)
        self.warm = True

    def __call__(self, ref_shard: torch.Tensor, query: torch.Tensor):
        from . import device_bytes, flag_signal, flag_wait, ksel_merge_lists
        L, e, Q, k = self.lay, self.epoch, self.Q, self.k
        b = e & 1
        r0, r1 = shard_range(self.n_total, self.world, self.rank)
        assert ref_shard.shape[0] == r1 - r0 and query.shape[0] == Q
        if not self.warm:
            self._warm_up(query.shape[1], query.device)
        if e >= 2:  # buffer b was last filled at epoch e - 2: all ranks must be done reading it
            flag_wait([self.base + L["consumed"](s) for s in range(self.world)], e - 1)
        own = device_bytes(self.base, L["bytes"])
        ov = own[L["val"](b): L["val"](b) + Q * k * 4].view(torch.float32).view(Q, k)
        oi = own[L["idx"](b): L["idx"](b) + Q * k * 4].view(torch.int32).view(Q, k)
        spans = chunk_ranges(Q, self.chunks)
        slices = [(qa + shard_range(qb - qa, self.world, self.rank)[0],
                   qa + shard_range(qb - qa, self.world, self.rank)[1]) for qa, qb in spans]
        qids = torch.cat([torch.arange(a_, b_, dtype=torch.int64) for a_, b_ in slices])
        mv = torch.empty((qids.numel(), k), dtype=torch.float32, device=query.device)
        mi = torch.empty((qids.numel(), k), dtype=torch.int32, device=query.device)
        offs = [0]
        for a_, b_ in slices:
            offs.append(offs[-1] + b_ - a_)

        def merge(c):
            s0, s1 = slices[c]
            if s1 > s0:
                ksel_merge_lists([p + L["val"](b) + s0 * k * 4 for p in self.peer],
                                 [p + L["idx"](b) + s0 * k * 4 for p in self.peer], s1 - s0, k, k,
                                 mv[offs[c]:offs[c + 1]], mi[offs[c]:offs[c + 1]],
                                 ready_ptrs=[p + L["ready"](b, c) for p in self.peer], epoch=e + 1)

        for c, (qa, qb) in enumerate(spans):
            if self.local_knn is None:  # the library writes straight into the exchange buffer
                from . import knn_search
                knn_search(ref_shard, query[qa:qb], k, idx_offset=r0, out_dist=ov[qa:qb], out_idx=oi[qa:qb])
            else:
                v, i = self.local_knn(ref_shard, query[qa:qb], k, r0)
                ov[qa:qb].copy_(v)
                oi[qa:qb].copy_(i)
            flag_signal(self.base + L["ready"](b, c), e + 1)
            if c > 0:
                merge(c - 1)
        merge(len(spans) - 1)
        for p in self.peer:
            flag_signal(p + L["consumed"](self.rank), e + 1)
        self.epoch += 1
        return mv, mi, qids

    def check(self):
        """Synchronise and raise if a device-side flag wait of the exchange timed out
        (a peer that never signalled: the results of that step are invalid)."""
        from . import KselError, device_status
        torch.cuda.synchronize()
        st = device_status()
        if st:
            raise KselError("KnnP2P exchange", st)

    def close(self):
        from . import ipc_close, ipc_free
        torch.cuda.synchronize()
        tdist.barrier(group=self.group)
        for s, p in enumerate(self.peer):
            if s != self.rank:
                ipc_close(p)
        tdist.barrier(group=self.group)
        ipc_free(self.base)
