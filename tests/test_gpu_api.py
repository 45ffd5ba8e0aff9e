"""GPU tests of the C ABI's contract beyond the result set: duplicate-free
output with crowded hash blocks under coarse cells, non-distinct caller
entry ids, concurrent searches on two streams, the per-query candidate costs
(dts_query_costs_device), and the multi-rank paths (strong query sharding
and temporal sharding of D) running libdts in two processes on one GPU."""
import os
import socket
import threading

import numpy as np
import pytest

import synth
import dts_parity as parity

pytestmark = pytest.mark.gpu

THREADS = max(1, min(32, os.cpu_count() or 1))


@pytest.fixture(scope="module")
def dts():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_gowanlockc15_b200 as m
    m.load()
    return m


def test_crowded_block_with_long_segment_no_duplicates(dts, oracle_mod):
    """A block of 8 cells with > 65,535 entries is returned whole by a row
    probe.  One spatially long segment makes the cells coarse and every
    stencil several rows tall; the x-cells per row are a multiple of 8, so a
    block never straddles two rows and no entry comes back twice (canonical,
    duplicate-free output, reading c7)."""
    D, Q = synth.crowded(5)
    D = np.concatenate([D, [[0.0, 0.05, 0.5, 0.5, 1.0, 0.95, 0.52, 0.5]]])
    for d in (0.01, 0.05):
        idx = dts.build_index(D)
        inf = idx.info()
        assert inf["grid"][0] % 8 == 0
        got = dts.search(idx, Q, d)
        idx.free()
        parity.assert_canonical(got)          # strictly increasing keys: no duplicates
        ora = oracle_mod.search(D, Q, d, threads=THREADS)
        info = parity.compare(got, ora, D, Q, d, oracle_mod)
        assert info["common"] > 100000


def test_non_distinct_entry_ids(dts, oracle_mod):
    """Caller entry ids need not be distinct (e.g. a per-trajectory segment
    number): every result is still reported once, with its interval, and no
    stage slot is left unwritten (staged ranks break ties by slot)."""
    c = synth.make_config("C2", scale=0.004)
    ids = (np.arange(c.D.shape[0]) // 3).astype(np.uint32)
    d = 2.0
    idx = dts.build_index(c.D, entry_ids=ids)
    got = dts.search(idx, c.Q, d)
    idx.free()
    ora = oracle_mod.search(c.D, c.Q, d, threads=THREADS)
    ora["entry_id"] = ids[ora["entry_id"]]
    assert got.shape == ora.shape

    def canon(a):
        return np.sort(a, order=["query_id", "entry_id", "t_start", "t_end"])
    g, o = canon(got), canon(ora)
    assert np.array_equal(g["query_id"], o["query_id"])
    assert np.array_equal(g["entry_id"], o["entry_id"])
    span = float(c.D[:, 4].max() - c.D[:, 0].min())
    assert np.max(np.abs(g["t_start"] - o["t_start"])) / span < 1e-9
    assert np.max(np.abs(g["t_end"] - o["t_end"])) / span < 1e-9
    # non-decreasing (query, entry id) order
    k = got["query_id"].astype(np.uint64) << np.uint64(32) | got["entry_id"].astype(np.uint64)
    assert np.all(k[1:] >= k[:-1])


def test_concurrent_searches_two_streams(dts):
    """An index is immutable after build: two host threads searching it at
    once, each on its own stream, get the bytes of sequential searches."""
    import torch
    c = synth.make_config("C2", scale=0.02)
    idx = dts.build_index(c.D)
    Qa, Qb = c.Q, np.ascontiguousarray(c.Q[::-1])
    ref_a = dts.search(idx, Qa, 2.0).tobytes()
    ref_b = dts.search(idx, Qb, 0.5).tobytes()
    Qa_d, Qb_d = torch.from_numpy(Qa).cuda(), torch.from_numpy(Qb).cuda()
    out = {}
    errs = []

    def run(name, Qh, Qd, d):
        try:
            s = torch.cuda.Stream()
            for k in range(4):
                if k % 2 == 0:
                    out[(name, k)] = dts.search(idx, Qh, d, stream=s).tobytes()
                else:
                    with torch.cuda.stream(s):
                        res, _ = dts.search_device(idx, Qd, d, stream=s)
                        out[(name, k)] = res.numpy().tobytes()
                        res.free()
        except Exception as e:          # surfaced below
            errs.append(e)

    ta = threading.Thread(target=run, args=("a", Qa, Qa_d, 2.0))
    tb = threading.Thread(target=run, args=("b", Qb, Qb_d, 0.5))
    ta.start(); tb.start(); ta.join(); tb.join()
    assert not errs, errs
    for k in range(4):
        assert out[("a", k)] == ref_a, k
        assert out[("b", k)] == ref_b, k
    idx.free()


def test_deferred_phase_times(dts):
    """time_kernels="defer": the call returns without reading its phase
    events; dts_search_read_times reads them afterwards (the same numbers a
    time_kernels=1 call reports, to within event resolution), and rejects a
    slot that was never recorded."""
    import torch
    c = synth.make_config("C2", scale=0.05)
    idx = dts.build_index(c.D)
    Qd = torch.from_numpy(c.Q).cuda()
    res0, st0 = dts.search_device(idx, Qd, c.d, time_kernels=True)
    ref = res0.numpy().tobytes()
    res0.free()
    slots = []
    for _ in range(3):
        res, st = dts.search_device(idx, Qd, c.d, time_kernels="defer")
        assert res.numpy().tobytes() == ref
        assert st["ms_count"] == 0.0 and st["timer_slot"] != 0xFFFFFFFF
        slots.append(st)
        res.free()
    assert len({s["timer_slot"] for s in slots}) == 3
    for st in slots:
        t = dts.read_times(st)
        assert t["ms_count"] > 0.0 and t["ms_prep"] > 0.0 and t["ms_scan"] > 0.0
        assert t["candidates"] == st0["candidates"]
    # pass 1's two events only
    res, st = dts.search_device(idx, Qd, c.d, time_kernels="pass1")
    res.free()
    t = dts.read_times(st)
    assert t["ms_count"] > 0.0 and t["ms_prep"] == 0.0 and t["ms_scan"] == 0.0
    _, st_off = dts.search_device(idx, Qd, c.d)
    assert st_off["timer_slot"] == 0xFFFFFFFF
    with pytest.raises(dts.DTSError):
        dts.read_times(st_off)
    idx.free()


def test_query_costs_match_candidates(dts):
    """dts_query_costs_device sums, per block of queries, exactly the
    candidate pairs the search refines (its `candidates` statistic)."""
    import torch
    for name, scale, d in (("C1", 0.2, 0.005), ("C2", 0.01, 2.0), ("C3", 0.02, 5.0)):
        c = synth.make_config(name, scale=scale)
        for method in ("grid", "subbin", "temporal"):
            idx = dts.build_index_device(torch.from_numpy(c.D).cuda(), method=method)
            Qd = torch.from_numpy(c.Q).cuda()
            res, st = dts.search_device(idx, Qd, d)
            per = dts.query_costs_device(idx, Qd, d, block=1)
            blk = dts.query_costs_device(idx, Qd, d, block=100)
            assert int(per.sum()) == st["candidates"], (name, method)
            assert blk.numel() == (c.Q.shape[0] + 99) // 100
            ref = torch.nn.functional.pad(per, (0, blk.numel() * 100 - per.numel()))
            assert torch.equal(ref.view(-1, 100).sum(1), blk)
            # sub-ranges: the costs of rows [a, b) alone
            a, b = c.Q.shape[0] // 3, c.Q.shape[0] // 2
            assert torch.equal(dts.query_costs_device(idx, Qd[a:b], d), per[a:b])
            # sampled estimate (every 4th query counted 4 times): per block it
            # is exactly 4 x the sum of the sampled queries' exact costs
            smp = dts.query_costs_device(idx, Qd, d, block=100, stride=4)
            keep = torch.zeros_like(per)
            keep[::4] = per[::4] * 4
            ref4 = torch.nn.functional.pad(keep, (0, blk.numel() * 100 - keep.numel()))
            assert torch.equal(ref4.view(-1, 100).sum(1), smp)
            assert torch.equal(dts.query_costs_device(idx, Qd, d, block=100, stride=1), blk)
            res.free()
            idx.free()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_worker(rank, world, port, out_dir):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_gowanlockc15_b200 as dts
    from paper_conf_ipps_gowanlockc15_b200 import dist as dts_dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    c = synth.make_config("C2", scale=0.01)
    d = 2.0
    idx = dts.build_index_device(torch.from_numpy(c.D).cuda())
    Qd = torch.from_numpy(c.Q).cuda()
    res, st, (lo, hi), off, total = dts_dist.search_strong(idx, Qd, d, rank, world, block=64)
    np.save(os.path.join(out_dir, f"strong{rank}.npy"), res.numpy())
    with open(os.path.join(out_dir, f"strong{rank}.txt"), "w") as f:
        f.write(f"{lo} {hi} {off} {total}")
    res.free()
    idx.free()
    tmp = dts_dist.search_temporal_sharded(c.D, c.Q, d, rank, world)
    if rank == 0:
        np.save(os.path.join(out_dir, "temporal.npy"), tmp)
    dist.barrier()
    dist.destroy_process_group()


def test_multirank_libdts_on_one_gpu(dts, tmp_path):
    """Two ranks (gloo) running libdts on the same GPU: the strong query
    sharding (balanced by dts_query_costs_device, counts all-gathered) placed
    at the gathered offsets, and the temporal sharding of D gathered on rank 0,
    both give the unsharded search's bytes."""
    import torch.multiprocessing as mp
    world = 2
    mp.spawn(_rank_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    c = synth.make_config("C2", scale=0.01)
    idx = dts.build_index(c.D)
    ref = dts.search(idx, c.Q, 2.0)
    idx.free()
    out = np.empty(ref.shape[0], dtype=ref.dtype)
    prev_hi = 0
    for r in range(world):
        part = np.load(tmp_path / f"strong{r}.npy")
        lo, hi, off, total = map(int, open(tmp_path / f"strong{r}.txt").read().split())
        assert lo == prev_hi and total == ref.shape[0]
        prev_hi = hi
        out[off:off + part.shape[0]] = part
    assert prev_hi == c.Q.shape[0]
    assert out.tobytes() == ref.tobytes()
    assert np.load(tmp_path / "temporal.npy").tobytes() == ref.tobytes()


def test_search_count_and_stream(dts, oracle_mod):
    """Count-only search (per-query counts, total) and the streamed search
    (canonical chunks through a callback) agree with the materialised
    search byte for byte; a query with more results than a chunk is a chunk
    of its own; the callback can stop the search."""
    import torch
    c = synth.make_config("C2", scale=0.01)
    idx = dts.build_index(c.D, entry_traj=c.etraj)
    for d, excl in ((2.0, False), (8.0, False), (2.0, True)):
        kw = dict(query_traj=c.qtraj, exclude_same_trajectory=True) if excl else {}
        ref, _ = dts.search_ex(idx, c.Q, d, **kw)
        total, counts, st = dts.search_count(idx, c.Q, d, **kw)
        assert total == ref.shape[0] == int(counts.sum())
        assert np.array_equal(counts, np.bincount(ref["query_id"], minlength=c.Q.shape[0]))
        chunks = []
        st = dts.search_stream(idx, c.Q, d, lambda ch: chunks.append(ch.copy()),
                               chunk_results=max(1, int(counts.max()) // 2),
                               query_id_base=0, **kw)
        got = np.concatenate(chunks)
        assert got.tobytes() == ref.tobytes()
        assert st["results"] == ref.shape[0]
        assert max(ch.shape[0] for ch in chunks) <= max(int(counts.max()), int(counts.max()) // 2)
    # device count, and an early stop after the first chunk
    idd = dts.build_index_device(torch.from_numpy(c.D).cuda())
    total_d, counts_d, _ = dts.search_count_device(idd, torch.from_numpy(c.Q).cuda(), 2.0)
    ref = dts.search(idx, c.Q, 2.0)
    assert total_d == ref.shape[0]
    assert np.array_equal(counts_d.cpu().numpy().astype(np.uint32),
                          np.bincount(ref["query_id"], minlength=c.Q.shape[0]))
    seen = []
    dts.search_stream(idx, c.Q, 2.0, lambda ch: seen.append(ch.shape[0]) or True, chunk_results=50)
    assert len(seen) == 1
    # oracle parity of the streamed output on a sample
    qs = np.arange(0, c.Q.shape[0], 23)
    parity.compare(parity.restrict(ref, qs), oracle_mod.search_queries(c.D, c.Q, qs, 2.0),
                   c.D, c.Q, 2.0, oracle_mod)
    idx.free()
    idd.free()


@pytest.mark.parametrize("budget_mb", [70, 66])
def test_mem_budget_temporal_shards(dts, oracle_mod, budget_mb):
    """An index over the device budget (mem_budget_bytes) keeps D in temporal
    shards on the host and indexes them one at a time at search time
    (SURVEY.md §8(e) fallback): same bytes as the resident index for the
    plain, trajectory-excluding, count-only and streamed searches."""
    c = synth.make_config("C2", scale=0.01)
    ref_idx = dts.build_index(c.D, entry_traj=c.etraj)
    idx = dts.build_index(c.D, entry_traj=c.etraj, mem_budget_bytes=budget_mb << 20)
    inf = idx.info()
    assert inf["shards"] >= 2, inf
    assert ref_idx.info()["shards"] == 0
    for d in (0.5, 2.0, 8.0):
        ref = dts.search(ref_idx, c.Q, d, query_id_base=3)
        got = dts.search(idx, c.Q, d, query_id_base=3)
        assert got.tobytes() == ref.tobytes(), d
    kw = dict(query_traj=c.qtraj, exclude_same_trajectory=True)
    ref, _ = dts.search_ex(ref_idx, c.Q, 2.0, **kw)
    got, _ = dts.search_ex(idx, c.Q, 2.0, **kw)
    assert got.tobytes() == ref.tobytes()
    total, counts, _ = dts.search_count(idx, c.Q, 2.0)
    rt, rc, _ = dts.search_count(ref_idx, c.Q, 2.0)
    assert total == rt and np.array_equal(counts, rc)
    chunks = []
    dts.search_stream(idx, c.Q, 2.0, lambda ch: chunks.append(ch.copy()), chunk_results=5000)
    assert np.concatenate(chunks).tobytes() == dts.search(ref_idx, c.Q, 2.0).tobytes()
    qs = np.arange(0, c.Q.shape[0], 29)
    parity.compare(parity.restrict(dts.search(idx, c.Q, 2.0), qs),
                   oracle_mod.search_queries(c.D, c.Q, qs, 2.0), c.D, c.Q, 2.0, oracle_mod)
    idx.free()
    ref_idx.free()


def test_host_results_over_1gb(dts, oracle_mod):
    """A host search whose results exceed 1 GB lands in huge-page backed
    pageable memory through the staged, multi-threaded copy: the bytes equal
    the device search's, and sampled queries match the oracle."""
    import torch
    g = np.random.default_rng(11)
    n, nq = 20000, 2400                       # 4.8e7 results, 1.15 GB
    D = np.zeros((n, 8))
    D[:, 4] = 1.0
    D[:, 1:4] = g.uniform(0, 0.01, (n, 3))
    D[:, 5:8] = D[:, 1:4] + g.uniform(-1e-3, 1e-3, (n, 3))
    Q = np.zeros((nq, 8))
    Q[:, 4] = 1.0
    Q[:, 1:4] = g.uniform(0, 0.01, (nq, 3))
    Q[:, 5:8] = Q[:, 1:4]
    d = 0.1                                   # every pair, the whole time
    idx = dts.build_index(D)
    host = dts.search(idx, Q, d)
    assert host.shape[0] == n * nq and host.nbytes > (1 << 30)
    dev, _ = dts.search_device(idx, torch.from_numpy(Q).cuda(), d)
    assert dev.count == host.shape[0]
    assert np.array_equal(dev.numpy().view(np.uint8), host.view(np.uint8))
    dev.free()
    for q in (0, 777, nq - 1):
        got = host[host["query_id"] == q].copy()
        got["query_id"] = 0
        info = parity.compare(got, oracle_mod.search(D, Q[q:q + 1], d), D, Q[q:q + 1], d,
                              oracle_mod)
        assert info["common"] == n
    idx.free()
