"""Multi-GPU plumbing (D and the
query set partitioned across GPU-equipped nodes).

Queries are independent (one query per unit of work), so the path
shards by query: every rank holds the same D + index and searches its own
contiguous query-id range.  The only exchange is the per-rank result count,
all-gathered (8 bytes per rank) so every rank knows where its slice starts in
the global (query_id, entry_id)-ordered result: concatenation in rank order
of contiguous query-id ranges is the canonical global order.

torch.distributed is used for the plumbing only (NCCL on GPUs, gloo on CPU
for the tests); the search itself is libdts.
"""
from __future__ import annotations

import numpy as np


def shard_bounds(nq: int, world: int, weights=None):
    """Contiguous query-id ranges [b[r], b[r+1]) for each rank.  With weights
    (e.g. per-query candidate estimates) the split balances their prefix sum;
    every rank computes the same split, no communication."""
    if world <= 0:
        raise ValueError("world must be positive")
    if weights is None:
        return [int(nq * r // world) for r in range(world + 1)]
    w = np.asarray(weights, dtype=np.float64)
    if w.shape[0] != nq:
        raise ValueError("weights must have one entry per query")
    c = np.concatenate([[0.0], np.cumsum(np.maximum(w, 0.0))])
    total = c[-1]
    if total <= 0:
        return shard_bounds(nq, world)
    b = [0]
    for r in range(1, world):
        b.append(int(np.searchsorted(c, total * r / world, side="left")))
    b.append(nq)
    for r in range(1, world + 1):           # keep monotone
        b[r] = max(b[r], b[r - 1])
    return b


def global_offset(count: int, rank: int, world: int, group=None, device=None):
    """All-gather the per-rank result counts; returns (offset of this rank's
    slice in the global result, global total, list of counts)."""
    import torch
    import torch.distributed as dist
    if world == 1:
        return 0, int(count), [int(count)]
    if device is None:
        device = torch.device("cuda", torch.cuda.current_device()) \
            if dist.get_backend(group) == "nccl" else torch.device("cpu")
    t = torch.tensor([int(count)], dtype=torch.int64, device=device)
    out = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(out, t, group=group)
    counts = [int(x.item()) for x in out]
    return int(sum(counts[:rank])), int(sum(counts)), counts


def search_sharded(search_fn, Q, d: float, rank: int, world: int, group=None, weights=None):
    """Strong-scaling helper: search this rank's contiguous shard of Q with
    `search_fn(Q_shard, d, query_id_base)` (e.g. a bound libdts search) and
    place it in the global order.  Returns (local results, offset, total)."""
    b = shard_bounds(len(Q), world, weights)
    lo, hi = b[rank], b[rank + 1]
    res = search_fn(Q[lo:hi], d, lo)
    off, total, _ = global_offset(len(res), rank, world, group=group)
    return res, off, total
