"""Multi-GPU dispatch for GANNS search (one process per GPU,
torch.distributed: NCCL over NVLink on B200s, gloo in the CPU tests).

Two modes -- the paper itself is single-GPU; its Remarks note
that independent work units parallelise directly.

* Replicated graph, query data-parallel: every rank holds the same graph (the
  build is deterministic, so each rank builds it locally -- no broadcast), rank r
  searches its slice [r*nq/W, (r+1)*nq/W) of the batch.  No data-path collective
  is needed for throughput; :func:`search_replicated` all-gathers the slices
  when the caller wants the whole result on every rank.

* Sharded base set (BASELINE configs[4], DEEP100M-shaped): the rows are split
  into shards, each with its own graph; a rank holds one or more shards, searches
  ALL queries on each, turns local ids into global ids, and one
  all_gather_into_tensor of the stacked [S, nq, k] (id, dist) lists is followed by
  the K6 merge (ganns_merge_topk): the k smallest (dist, global id) over all shards.

The per-shard search / merge functions are injected, so the same orchestration
runs the sm_100a kernels on GPUs and is exercised on CPU by the gloo tests.
"""
from __future__ import annotations

from typing import Callable, Tuple

import torch
import torch.distributed as dist

SearchFn = Callable[[torch.Tensor], Tuple[torch.Tensor, torch.Tensor]]
MergeFn = Callable[[torch.Tensor, torch.Tensor], Tuple[torch.Tensor, torch.Tensor]]


def _world(group=None) -> Tuple[int, int]:
    if dist.is_available() and dist.is_initialized():
        return dist.get_rank(group), dist.get_world_size(group)
    return 0, 1


def query_slice(nq: int, rank: int, world: int) -> Tuple[int, int]:
    """Contiguous slice [floor(r*nq/W), floor((r+1)*nq/W)) of the query batch."""
    return nq * rank // world, nq * (rank + 1) // world


def shard_bounds(n: int, rank: int, world: int) -> Tuple[int, int]:
    """Rows of the base set owned by `rank` (contiguous, sizes differ by <= 1)."""
    return n * rank // world, n * (rank + 1) // world


def _all_gather_rows(x: torch.Tensor, counts, group=None) -> torch.Tensor:
    """Gather variable-length row blocks (padded to the largest) in rank order."""
    _, world = _world(group)
    m = max(counts)
    pad = x.new_zeros((m,) + tuple(x.shape[1:]))
    pad[: x.shape[0]] = x
    outs = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(outs, pad, group=group)
    return torch.cat([o[:c] for o, c in zip(outs, counts)], 0)


def search_replicated(search_fn: SearchFn, queries: torch.Tensor, gather: bool = True,
                      group=None):
    """Rank r searches its slice of `queries` with `search_fn` (the local replica).
    Returns (ids, dists) for the whole batch when `gather`, else for the slice."""
    rank, world = _world(group)
    nq = queries.shape[0]
    lo, hi = query_slice(nq, rank, world)
    ids, dists = search_fn(queries[lo:hi])
    if not gather or world == 1:
        return ids, dists
    counts = [query_slice(nq, r, world)[1] - query_slice(nq, r, world)[0] for r in range(world)]
    return _all_gather_rows(ids, counts, group), _all_gather_rows(dists, counts, group)


class ShardedIndex:
    """The shards of a base set held by this rank; `search` returns the global top-k.

    shards: [(global_offset, search_fn)] -- this rank's shards (every rank holds
    the same number of shards; shard s lives on rank s % W in the bench, any
    placement works).  search_fn(queries) -> (local ids, dists) [nq, k] of that
    shard (ids in [0, shard size), -1 = empty); offset_fn(ids, offset) makes them
    global in place; merge_fn(ids [S, nq, k], dists [S, nq, k]) -> global
    (ids, dists) [nq, k].  streams (optional, one per concurrent shard search):
    shard j's search + offset run on streams[j % len(streams)] so consecutive
    shard searches overlap on the device; the exchange waits for all of them.

    The one exchange step is an all_gather_into_tensor of the stacked per-shard
    lists ([S_local, nq, k] ids and dists per rank) -- 800 KB per shard at 10K
    queries, k = 10 -- followed by the K6 merge on every rank.
    """

    def __init__(self, shards, merge_fn: MergeFn,
                 offset_fn: Callable[[torch.Tensor, int], torch.Tensor], group=None,
                 streams=None):
        self.rank, self.world = _world(group)
        self.group = group
        self.shards = list(shards)
        if not self.shards:
            raise ValueError("a rank must hold at least one shard")
        self.merge_fn = merge_fn
        self.offset_fn = offset_fn
        self.streams = list(streams) if streams else None

    def local(self, queries: torch.Tensor):
        """Every local shard searched, ids made global: stacked [S_local, nq, k]."""
        if self.streams is None:
            outs = []
            for off, fn in self.shards:
                ids, dists = fn(queries)
                outs.append((self.offset_fn(ids, off), dists))
        else:
            cur = torch.cuda.current_stream()
            ev0 = torch.cuda.Event()
            ev0.record(cur)
            outs = [None] * len(self.shards)
            for j, (off, fn) in enumerate(self.shards):
                st = self.streams[j % len(self.streams)]
                st.wait_event(ev0)
                with torch.cuda.stream(st):
                    ids, dists = fn(queries)
                    outs[j] = (self.offset_fn(ids, off), dists)
            for st in self.streams:
                ev = torch.cuda.Event()
                ev.record(st)
                cur.wait_event(ev)
        return torch.stack([o[0] for o in outs]), torch.stack([o[1] for o in outs])

    def search(self, queries: torch.Tensor):
        ids, dists = self.local(queries)
        if self.world > 1:
            gi = ids.new_empty((self.world * ids.shape[0],) + tuple(ids.shape[1:]))
            gd = dists.new_empty((self.world * dists.shape[0],) + tuple(dists.shape[1:]))
            dist.all_gather_into_tensor(gi, ids.contiguous(), group=self.group)
            dist.all_gather_into_tensor(gd, dists.contiguous(), group=self.group)
            ids, dists = gi, gd
        return self.merge_fn(ids, dists)


def gpu_sharded_index(shards, k: int, l: int, e: int = 0, group=None,
                      streams=None) -> ShardedIndex:
    """ShardedIndex wired to the sm_100a kernels: shards = [(global_offset, graph,
    points_shard)]; K1 search on each local shard graph, in-place id offset, K6
    merge (all through libganns.so)."""
    from . import search, offset_ids, merge_topk

    def _fn(graph, pts):
        return lambda q: search(graph, pts, q, k, l, e=e)

    return ShardedIndex([(off, _fn(gr, pts)) for off, gr, pts in shards],
                        lambda i, d: merge_topk(i, d), lambda ids, off: offset_ids(ids, off),
                        group=group, streams=streams)


def gpu_replicated_search(graph, points: torch.Tensor, queries: torch.Tensor, k: int, l: int,
                          e: int = 0, gather: bool = True, group=None):
    """search_replicated wired to the K1 kernel on this rank's replica."""
    from . import search
    return search_replicated(lambda q: search(graph, points, q, k, l, e=e), queries,
                             gather=gather, group=group)


def _comm(t: torch.Tensor, group=None) -> torch.Tensor:
    """gloo collectives run on host tensors (NCCL on device tensors)."""
    if t.is_cuda and dist.get_backend(group) == "gloo":
        return t.cpu()
    return t


def _gather_blocks(blocks, counts, group=None):
    """All-gather per-rank row blocks (tuples of tensors with `counts[r]` rows on rank
    r) in rank order; every tensor comes back on the device of the local block."""
    dev = blocks[0].device
    out = []
    for t in blocks:
        out.append(_all_gather_rows(_comm(t, group), counts, group).to(dev))
    return out


def build_distributed(builder, group=None):
    """Algorithm 2 over the ranks of `group` (NEXT-2; the paper's Remarks,
    P:299: each working unit builds local graphs and runs its share of a round's
    searches).  `builder` is one rank's replica of the staged construction
    (StagedBuild on a GPU; the tests also drive a CPU one):

      Phase 1  rank r builds groups [r*G/W, (r+1)*G/W) (a group touches only its
               own rows), then the rows (build form + N') are all-gathered so every
               replica holds every local graph;
      Phase 2  round i: rank r searches its contiguous share of P_i
               (query_slice), the new forward rows F [|P_i|, d_min] are all-gathered
               in vertex order, and every rank applies the same round (rows of P_i,
               E, GatherScatter, merges) -- one exchange per round.

    The replicas stay bit-identical to a one-GPU build with the same parameters.
    Returns builder.finish()."""
    rank, world = _world(group)
    S, G, d_min, d_max = builder.info()
    # ---- Phase 1
    gb = [query_slice(G, r, world) for r in range(world)]
    builder.phase1(*gb[rank])
    if world > 1:
        vb = [builder.group_rows(*gb[r]) for r in range(world)]
        counts = [b - a for a, b in vb]
        rows = _gather_blocks(builder.export_rows(*vb[rank]), counts, group)
        off = 0
        for r in range(world):
            if r != rank and counts[r] > 0:
                builder.import_rows(vb[r][0], vb[r][1],
                                    tuple(t[off:off + counts[r]].contiguous() for t in rows))
            off += counts[r]
    # ---- Phase 2, one exchange per round
    for i in range(1, G):
        lo, hi = builder.group_rows(i, i + 1)
        sl = [query_slice(hi - lo, r, world) for r in range(world)]
        a, b = sl[rank]
        f = builder.round_search(i, lo + a, lo + b)
        if world > 1:
            f = _gather_blocks(f, [y - x for x, y in sl], group)
        builder.round_apply(i, *f)
    return builder.finish()


def max_over_ranks(value: float, device=None, group=None) -> float:
    """Max of a per-rank scalar (timings are reported as the max over ranks)."""
    rank, world = _world(group)
    if world == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
