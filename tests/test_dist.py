"""Multi-process (gloo, world_size 2, CPU) checks of the query-sharding
plumbing of paper_conf_ipps_gowanlockc15_b200.dist: every
rank searches a contiguous query-id range, the per-rank result counts are
all-gathered, and rank-order concatenation at the gathered offsets equals
the unsharded canonical result.  The per-rank search here is the oracle
(there is no GPU in the CPU suite); on GPUs it is libdts."""
import os
import socket

import numpy as np
import pytest

import synth


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir, weighted):
    import torch.distributed as dist

    import oracle
    from paper_conf_ipps_gowanlockc15_b200 import dist as dts_dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    c = synth.make_config("C0")
    weights = (np.arange(c.Q.shape[0]) % 7 + 1.0) if weighted else None

    def local_search(Qs, d, base):
        r = oracle.search(c.D, Qs, d)
        r["query_id"] += np.uint32(base)
        return r

    res, off, total = dts_dist.search_sharded(local_search, c.Q, c.d, rank, world,
                                              weights=weights)
    np.save(os.path.join(out_dir, f"r{rank}.npy"), res)
    with open(os.path.join(out_dir, f"r{rank}.txt"), "w") as f:
        f.write(f"{off} {total}")
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("weighted", [False, True])
def test_sharded_search_matches_unsharded(tmp_path, weighted):
    import torch.multiprocessing as mp

    import oracle
    world = 2
    port = _free_port()
    mp.spawn(_worker, args=(world, port, str(tmp_path), weighted), nprocs=world, join=True)
    c = synth.make_config("C0")
    full = oracle.search(c.D, c.Q, c.d)
    out = np.empty(full.shape[0], dtype=full.dtype)
    seen = 0
    for r in range(world):
        part = np.load(tmp_path / f"r{r}.npy")
        off, total = map(int, open(tmp_path / f"r{r}.txt").read().split())
        assert total == full.shape[0]
        out[off:off + part.shape[0]] = part
        seen += part.shape[0]
    assert seen == full.shape[0]
    assert out.tobytes() == full.tobytes()


def test_shard_bounds():
    from paper_conf_ipps_gowanlockc15_b200 import dist as dts_dist
    assert dts_dist.shard_bounds(10, 3) == [0, 3, 6, 10]
    b = dts_dist.shard_bounds(8, 2, weights=[1, 1, 1, 1, 1, 1, 10, 10])
    assert b[0] == 0 and b[-1] == 8 and 0 < b[1] < 8
    assert b[1] == 7          # first prefix (16 of 26) reaching half the weight
    assert dts_dist.shard_bounds(0, 4) == [0, 0, 0, 0, 0]


def _temporal_worker(rank, world, port, out_dir):
    import torch.distributed as dist

    import oracle
    from paper_conf_ipps_gowanlockc15_b200 import dist as dts_dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import torch
    c = synth.make_config("C0")
    T, rows, maxdur = dts_dist.temporal_partition(c.D, world)
    mine = rows[rank]
    qrows = dts_dist.route_queries(c.Q, T, maxdur, rank)
    # the per-rank search (libdts on GPUs) is the oracle here, ids mapped back
    r = oracle.search(c.D[mine], c.Q[qrows], c.d)
    r["entry_id"] = mine[r["entry_id"]].astype(np.uint32)
    r["query_id"] = qrows[r["query_id"]].astype(np.uint32)
    local = torch.from_numpy(r.view(np.uint8).copy())
    allres = dts_dist.gather_to_root(local, rank, world)
    if rank == 0:
        np.save(os.path.join(out_dir, "all.npy"), allres.numpy())
    dist.barrier()
    dist.destroy_process_group()


def test_temporal_sharding_of_D_is_exact(tmp_path):
    """Each entry on exactly one rank, queries routed by time: the union of
    the per-rank results is exactly the unsharded result (no duplicates)."""
    import torch.multiprocessing as mp

    import oracle
    world = 2
    mp.spawn(_temporal_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world,
             join=True)
    c = synth.make_config("C0")
    full = oracle.search(c.D, c.Q, c.d)
    got = np.load(tmp_path / "all.npy").view(full.dtype)
    keys = got["query_id"].astype(np.int64) * 2**32 + got["entry_id"]
    order = np.argsort(keys, kind="stable")
    assert np.unique(keys).size == keys.size                  # disjoint per rank
    assert got[order].tobytes() == full.tobytes()


def test_temporal_partition_properties():
    from paper_conf_ipps_gowanlockc15_b200 import dist as dts_dist
    c = synth.make_config("C0")
    for world in (1, 2, 3, 5):
        T, rows, maxdur = dts_dist.temporal_partition(c.D, world)
        allrows = np.sort(np.concatenate(rows))
        assert np.array_equal(allrows, np.arange(c.D.shape[0]))      # a partition
        for r in range(world):
            t0 = c.D[rows[r], 0]
            assert np.all(t0 >= T[r]) and np.all(t0 < T[r + 1])


def _balance_worker(rank, world, port, out_dir):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_gowanlockc15_b200 import dist as dts_dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    nq, block = 1000, 16
    # skewed per-query costs: the first fifth of the queries is 20x heavier
    per = np.where(np.arange(nq) < nq // 5, 20, 1).astype(np.int64)

    def costs_fn(lo, hi):
        # blocks of `block` queries, as dts_query_costs_device(block=16) returns
        p = per[lo:hi]
        nb = (p.size + block - 1) // block
        p = np.pad(p, (0, nb * block - p.size))
        return torch.from_numpy(p.reshape(nb, block).sum(1))

    Q = torch.zeros((nq, 8), dtype=torch.float64)
    b = dts_dist.balanced_query_bounds(None, Q, 0.1, rank, world, block=block, costs_fn=costs_fn)
    with open(os.path.join(out_dir, f"b{rank}.txt"), "w") as f:
        f.write(" ".join(map(str, b)))
    dist.barrier()
    dist.destroy_process_group()


def test_balanced_bounds_exchange(tmp_path):
    """Strong-scaling split: each rank costs an equal share
    of the query blocks, the per-block costs are all-gathered, and every rank
    computes the same balanced contiguous bounds (block-aligned), which put
    about half of the total cost on each rank."""
    import torch.multiprocessing as mp
    world = 2
    mp.spawn(_balance_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    bs = [list(map(int, open(tmp_path / f"b{r}.txt").read().split())) for r in range(world)]
    assert bs[0] == bs[1]
    b = bs[0]
    assert b[0] == 0 and b[-1] == 1000 and b[1] % 16 == 0
    per = np.where(np.arange(1000) < 200, 20, 1)
    half = per.sum() / 2
    assert abs(per[:b[1]].sum() - half) <= 16 * 20      # within one block of the cut
    assert b[1] < 500                                    # far from the equal-count split
