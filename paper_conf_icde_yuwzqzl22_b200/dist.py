"""Multi-GPU dispatch for GANNS search (one process per GPU,
torch.distributed: NCCL over NVLink on B200s, gloo in the CPU tests).

Two modes -- the paper itself is single-GPU; its Remarks note
that independent work units parallelise directly.

* Replicated graph, query data-parallel: every rank holds the same graph (the
  build is deterministic, so each rank builds it locally -- no broadcast), rank r
  searches its slice [r*nq/W, (r+1)*nq/W) of the batch.  No data-path collective
  is needed for throughput; :func:`search_replicated` all-gathers the slices
  when the caller wants the whole result on every rank.

* Sharded base set (BASELINE configs[4], DEEP100M-shaped): rank r holds rows
  [r*n/W, (r+1)*n/W) and its own graph over them; every rank searches ALL
  queries on its shard, turns local ids into global ids, and one all-gather of
  the [nq, k] (id, dist) lists is followed by the K6 merge (ganns_merge_topk):
  the k smallest (dist, global id) over all shards.

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
    """One shard of a base set split across ranks; `search` returns the global top-k.

    search_fn(queries) -> (local ids, dists) of this rank's shard (ids in
    [0, shard size), -1 = empty); offset_fn(ids, offset) makes them global in
    place; merge_fn(ids[W,nq,k], dists[W,nq,k]) -> global (ids, dists) [nq, k].
    """

    def __init__(self, n_total: int, search_fn: SearchFn, merge_fn: MergeFn,
                 offset_fn: Callable[[torch.Tensor, int], torch.Tensor], group=None):
        self.rank, self.world = _world(group)
        self.group = group
        self.lo, self.hi = shard_bounds(n_total, self.rank, self.world)
        self.search_fn = search_fn
        self.merge_fn = merge_fn
        self.offset_fn = offset_fn

    def search(self, queries: torch.Tensor):
        ids, dists = self.search_fn(queries)
        ids = self.offset_fn(ids, self.lo)
        if self.world == 1:
            return self.merge_fn(ids[None], dists[None])
        # the one exchange step: all-gather of every shard's [nq, k] lists
        gi = [torch.empty_like(ids) for _ in range(self.world)]
        gd = [torch.empty_like(dists) for _ in range(self.world)]
        dist.all_gather(gi, ids.contiguous(), group=self.group)
        dist.all_gather(gd, dists.contiguous(), group=self.group)
        return self.merge_fn(torch.stack(gi), torch.stack(gd))


def gpu_sharded_index(graph, points_shard: torch.Tensor, n_total: int, k: int, l: int,
                      e: int = 0, group=None) -> ShardedIndex:
    """ShardedIndex wired to the sm_100a kernels: K1 search on the local shard graph,
    in-place id offset, K6 merge (all through libganns.so)."""
    from . import search, offset_ids, merge_topk

    def _search(q):
        return search(graph, points_shard, q, k, l, e=e)

    return ShardedIndex(n_total, _search, lambda i, d: merge_topk(i, d),
                        lambda ids, off: offset_ids(ids, off), group=group)


def gpu_replicated_search(graph, points: torch.Tensor, queries: torch.Tensor, k: int, l: int,
                          e: int = 0, gather: bool = True, group=None):
    """search_replicated wired to the K1 kernel on this rank's replica."""
    from . import search
    return search_replicated(lambda q: search(graph, points, q, k, l, e=e), queries,
                             gather=gather, group=group)


def max_over_ranks(value: float, device=None, group=None) -> float:
    """Max of a per-rank scalar (timings are reported as the max over ranks)."""
    rank, world = _world(group)
    if world == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
