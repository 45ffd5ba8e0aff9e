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


def _comm_device(group=None):
    import torch
    import torch.distributed as dist
    if dist.get_backend(group) == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def block_split(nblocks: int, world: int):
    """Equal split of `nblocks` cost blocks over ranks (block indices)."""
    return [nblocks * r // world for r in range(world + 1)]


def balanced_query_bounds(idx, Q_dev, d: float, rank: int, world: int, group=None,
                          block: int = 256, stream=None, costs_fn=None, stride: int = 8):
    """Query-id bounds [b[r], b[r+1]) of every rank, balanced by the
    candidate counts of the search (dts_query_costs_device, SURVEY.md
    §8(a4)/(e)).  Each rank costs an equal share of Q's blocks of `block`
    queries (so the estimate itself is sharded); the per-block sums are
    all-gathered (8 bytes per block) and every rank cuts the same prefix
    sum at total * r / world.  The counts are estimated from every
    `stride`-th query (dts_query_costs_sampled_device; 32 of each block of
    256 by default: exact counting cost a rank 0.10 ms on its 1/8 of C4,
    more than half its search).  Returns the bounds list (query ids,
    multiples of `block` except the last) on every rank.  costs_fn(lo, hi)
    replaces the library call (CPU tests of the exchange)."""
    import torch
    import torch.distributed as dist

    nq = int(Q_dev.shape[0])
    nb = (nq + block - 1) // block
    if world == 1:
        return [0, nq]
    eb = block_split(nb, world)
    lo, hi = eb[rank] * block, min(nq, eb[rank + 1] * block)
    if costs_fn is None:
        import paper_conf_ipps_gowanlockc15_b200 as dts
        mine = dts.query_costs_device(idx, Q_dev[lo:hi], d, block=block, stream=stream,
                                      stride=stride)
    else:
        mine = costs_fn(lo, hi)
    width = max(eb[r + 1] - eb[r] for r in range(world))
    cdev = _comm_device(group)
    pad = torch.zeros(width, dtype=torch.int64, device=cdev)
    pad[:mine.numel()] = mine.to(cdev)
    parts = [torch.zeros_like(pad) for _ in range(world)]
    dist.all_gather(parts, pad, group=group)
    costs = np.concatenate([parts[r][:eb[r + 1] - eb[r]].cpu().numpy() for r in range(world)])
    bb = shard_bounds(nb, world, weights=costs)
    return [min(nq, x * block) for x in bb]


def search_strong(idx, Q_dev, d: float, rank: int, world: int, group=None, block: int = 256,
                  stream=None, bounds=None, time_kernels: bool = False):
    """One strong-scaling search step: the one query set
    Q_dev (resident on every rank, as is the index) is split into contiguous
    query-id ranges balanced by candidate counts (or by `bounds` if given),
    this rank searches its range with global query ids, and the per-rank
    result counts are all-gathered (the only exchange of the search).
    Returns (DeviceResults, search stats, (lo, hi), offset of this rank's
    slice in the global canonical result, global total)."""
    import paper_conf_ipps_gowanlockc15_b200 as dts
    if bounds is None:
        bounds = balanced_query_bounds(idx, Q_dev, d, rank, world, group, block, stream)
    lo, hi = bounds[rank], bounds[rank + 1]
    res, st = dts.search_device(idx, Q_dev[lo:hi], d, query_id_base=lo, stream=stream,
                                time_kernels=time_kernels)
    off, total, _ = global_offset(res.count, rank, world, group=group,
                                  device=_comm_device(group) if world > 1 else None)
    return res, st, (lo, hi), off, total


# --------------------------------------------------------------------------
# Fallback when D exceeds one GPU's HBM: shard D by
# t_start range.  Rank r holds the entries with t_start in [T_r, T_{r+1});
# each entry lives on exactly one rank, so per-rank results are disjoint and
# their union is exact.  A query is routed to every rank whose entries it can
# overlap strictly in time: q.t_end > T_r and q.t_start < T_{r+1} + maxdur_r.
# Ranks report global entry ids (index built with entry_ids) and global query
# ids (search with query_ids); rank 0 concatenates and restores canonical
# order with one device sort (dts_canonicalize_device).

def temporal_partition(D, world: int):
    """Split D's rows by t_start quantiles.  Returns (T, rows, maxdur):
    boundaries T[0..world] (T[0] = -inf, T[world] = +inf), the row indices of
    each rank (ascending), and each rank's max segment duration."""
    D = np.asarray(D).reshape(-1, 8)
    t0 = D[:, 0]
    srt = np.sort(t0)
    T = [-np.inf]
    for r in range(1, world):
        T.append(float(srt[min(len(srt) - 1, (len(srt) * r) // world)]) if len(srt) else 0.0)
    T.append(np.inf)
    T = np.array(T)
    owner = np.searchsorted(T, t0, side="right") - 1
    rows = [np.flatnonzero(owner == r).astype(np.int64) for r in range(world)]
    maxdur = [float((D[rr, 4] - D[rr, 0]).max()) if rr.size else 0.0 for rr in rows]
    return T, rows, maxdur


def route_queries(Q, T, maxdur, rank: int):
    """Rows of Q that can strictly overlap an entry of `rank` in time (with a
    relative 1e-9 slack against rounding of t_start + duration)."""
    Q = np.asarray(Q).reshape(-1, 8)
    lo, hi = T[rank], T[rank + 1]
    slack = 1e-9 * (np.abs(hi) + maxdur[rank] + 1.0) if np.isfinite(hi) else 0.0
    ok = (Q[:, 4] > lo) & (Q[:, 0] < hi + maxdur[rank] + slack)
    return np.flatnonzero(ok).astype(np.int64)


def gather_to_root(local, rank: int, world: int, group=None):
    """Variable-length uint8 tensors to rank 0: the sizes are all-gathered
    (8 bytes per rank), then every rank sends exactly its bytes to rank 0
    (point to point), so no rank holds more than its own slice except the
    root.  Returns the concatenation in rank order on rank 0, None elsewhere."""
    import torch
    import torch.distributed as dist
    n = torch.tensor([local.numel()], dtype=torch.int64, device=local.device)
    sizes = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(sizes, n, group=group)
    sizes = [int(s.item()) for s in sizes]
    if rank != 0:
        if sizes[rank]:
            dist.send(local.contiguous(), dst=0, group=group)
        return None
    parts = [local]
    for r in range(1, world):
        buf = torch.empty(sizes[r], dtype=torch.uint8, device=local.device)
        if sizes[r]:
            dist.recv(buf, src=r, group=group)
        parts.append(buf)
    return torch.cat(parts)


def search_temporal_sharded(D, Q, d: float, rank: int, world: int, group=None,
                            method: str = "grid", device=None):
    """Temporal-range sharding of D over `world` GPUs (one rank each; device
    defaults to the rank's current CUDA device, i.e. LOCAL_RANK under a
    one-process-per-GPU launch).  Returns the canonical global results
    (numpy) on rank 0, None elsewhere."""
    import torch

    import paper_conf_ipps_gowanlockc15_b200 as dts
    if device is None:
        device = torch.cuda.current_device()
    T, rows, maxdur = temporal_partition(D, world)
    dev = torch.device("cuda", device)
    mine = rows[rank]
    Dd = torch.from_numpy(np.ascontiguousarray(np.asarray(D)[mine])).to(dev)
    ids = torch.from_numpy(mine.astype(np.int32)).to(dev)
    qrows = route_queries(Q, T, maxdur, rank)
    Qd = torch.from_numpy(np.ascontiguousarray(np.asarray(Q)[qrows])).to(dev)
    qids = torch.from_numpy(qrows.astype(np.int32)).to(dev)
    idx = dts.build_index_device(Dd, device=device, method=method, entry_ids=ids)
    res, _ = dts.search_device(idx, Qd, d, query_ids=qids)
    local = res.tensor().clone()
    res.free()
    idx.free()
    if _comm_device(group).type == "cpu":
        local = local.cpu()
    allres = gather_to_root(local, rank, world, group)
    if allres is None:
        return None
    allres = allres.to(dev)
    dts.canonicalize_device(allres)
    return allres.cpu().numpy().view(dts.RESULT_DTYPE)
