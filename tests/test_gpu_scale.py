"""GPU parity at the BASELINE.json full sizes and on the paper-replica shapes
(P:L127-P:L141), sampled: the CUDA path (through the C ABI, in the launch
configuration bench.py times) against the oracle on sampled queries, each
brute-forced against all of D.  Rule: tests/dts_parity.py."""
import os
import subprocess
import sys

import numpy as np
import pytest

import synth
import dts_parity as parity

pytestmark = pytest.mark.gpu

THREADS = max(1, min(64, os.cpu_count() or 1))
REPO = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def dts():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_gowanlockc15_b200 as m
    m.load()
    return m


def _device_search(dts, D, Q, d_list, **params):
    import torch
    Dd = torch.from_numpy(D).cuda()
    Qd = torch.from_numpy(Q).cuda()
    idx = dts.build_index_device(Dd, **params)
    out = []
    for d in d_list:
        res, st = dts.search_device(idx, Qd, d)
        out.append((res.numpy(), st))
        res.free()
    idx.free()
    return out


def c4_stratified_sample(c, n_uniform=4000, n_centre=1000, seed=123):
    """Query rows of C4: n_uniform uniform + n_centre whose midpoint lies
    within 0.7 of a disk centre at its time (the dense galaxy centres, where
    candidates per query are highest): disk 1 at the origin, disk 2 at
    (12 - 0.06 t, 4 - 0.02 t, 0) (synth.galaxy)."""
    Q = c.Q
    t = Q[:, 0]
    mid = 0.5 * (Q[:, 1:4] + Q[:, 5:8])
    c2 = np.stack([12.0 - 0.06 * t, 4.0 - 0.02 * t, np.zeros_like(t)], axis=1)
    r = np.minimum(np.linalg.norm(mid, axis=1), np.linalg.norm(mid - c2, axis=1))
    g = synth.rng(seed)
    centre = np.flatnonzero(r < 0.7)
    assert centre.size >= n_centre
    a = g.choice(centre, size=n_centre, replace=False)
    rest = np.setdiff1d(np.arange(Q.shape[0]), a)
    b = g.choice(rest, size=n_uniform, replace=False)
    return np.sort(np.concatenate([a, b]))


def test_c4_full_size_stratified(dts, oracle_mod):
    """configs[4] at full size (20.1 M entries, 1 M queries), bench launch
    configuration, at the headline d and at d = 0.02 (real hits beyond the
    self pairs): 5,000 sampled queries, 1,000 of them in the disk centres."""
    c = synth.make_config("C4")
    qs = c4_stratified_sample(c)
    for (got, st), d in zip(_device_search(dts, c.D, c.Q, (c.d, 0.02)), (c.d, 0.02)):
        parity.assert_canonical(got)
        assert np.unique(got["query_id"]).size == c.Q.shape[0]     # every self pair
        ora = oracle_mod.search_queries(c.D, c.Q, qs, d, threads=THREADS)
        info = parity.compare(parity.restrict(got, qs), ora, c.D, c.Q, d, oracle_mod)
        assert info["common"] >= qs.size
        if d == 0.02:
            assert info["common"] > 1.2 * qs.size        # hits beyond the self pairs


@pytest.mark.parametrize("name,dlist,nsample", [
    ("C2", (0.09, 2.0, 8.0), 300),
    ("C3", (5.0, 50.0), 400),
    ("C1", (0.005, 0.02), 400),
])
def test_configs_full_size_sampled(dts, oracle_mod, name, dlist, nsample):
    """configs[1..3] at full size: sampled queries, several d (C2 at d = 8 is
    the candidate-heavy, output-heavy point: hundreds of results per query)."""
    c = synth.make_config(name)
    g = synth.rng(31)
    qs = np.sort(g.choice(c.Q.shape[0], size=nsample, replace=False))
    for (got, st), d in zip(_device_search(dts, c.D, c.Q, dlist), dlist):
        parity.assert_canonical(got)
        ora = oracle_mod.search_queries(c.D, c.Q, qs, d, threads=THREADS)
        parity.compare(parity.restrict(got, qs), ora, c.D, c.Q, d, oracle_mod)


@pytest.mark.parametrize("name,d,nsample", [
    ("S1", 20.0, 200),        # 997,500 entries, 39,900 queries
    ("S2", 0.01, 120),        # 25,165,824 entries, 50,880 queries
    ("S3", 0.05, 150),        # 12,582,912 entries, 50,880 queries
])
def test_paper_replicas_sampled(dts, oracle_mod, name, d, nsample):
    """The paper's three scenarios at their exact sizes,
    grid and subbin (GPUSpatioTemporal) methods: sampled queries vs the oracle,
    and the two methods return the same bytes."""
    c = synth.make_config(name)
    g = synth.rng(41)
    qs = np.sort(g.choice(c.Q.shape[0], size=nsample, replace=False))
    (grid, _), = _device_search(dts, c.D, c.Q, (d,))
    (sub, _), = _device_search(dts, c.D, c.Q, (d,), method="subbin")
    assert sub.tobytes() == grid.tobytes()
    ora = oracle_mod.search_queries(c.D, c.Q, qs, d, threads=THREADS)
    parity.compare(parity.restrict(grid, qs), ora, c.D, c.Q, d, oracle_mod)


def _run_sub(code, env):
    out = subprocess.run([sys.executable, "-c", code], env={**os.environ, **env},
                         capture_output=True, timeout=900)
    assert out.returncode == 0, out.stderr.decode()[-3000:]
    return out.stdout


def test_sorted_query_path_forced(dts, oracle_mod):
    """The grid method sorts queries (by the key's top 9 bits, one counting
    pass) only from 2^18 queries (DTS_QSORT_MIN); forcing the sorted path on small sets (adversarial sets,
    C2 at several d) gives the same bytes as the unsorted path and matches
    the oracle."""
    code = ("import sys; sys.path[:0] = [%r, %r]; import numpy as np, synth, "
            "paper_conf_ipps_gowanlockc15_b200 as m\n"
            "out = []\n"
            "for seed in range(40):\n"
            "    D, Q = synth.adversarial(7000 + seed, 60, 60)\n"
            "    i = m.build_index(D); out.append(m.search(i, Q, [0.0, 0.03, 0.1, 0.3][seed %% 4]).tobytes())\n"
            "c = synth.make_config('C2', scale=0.02)\n"
            "i = m.build_index(c.D)\n"
            "for d in (0.09, 2.0, 8.0): out.append(m.search(i, c.Q, d).tobytes())\n"
            "sys.stdout.buffer.write(b''.join(len(o).to_bytes(8, 'little') + o for o in out))"
            % (REPO, os.path.join(REPO, "tests")))

    def split(buf):
        parts, k = [], 0
        while k < len(buf):
            n = int.from_bytes(buf[k:k + 8], "little")
            parts.append(buf[k + 8:k + 8 + n])
            k += 8 + n
        return parts
    sorted_out = split(_run_sub(code, {"DTS_QSORT_MIN": "0"}))
    plain_out = split(_run_sub(code, {"DTS_QSORT_MIN": "1000000000"}))
    # the multi-pass radix sort of the key's top bits (DTS_QSORT_DROP) instead
    # of the one-pass counting sort of the bin bits
    multi_out = split(_run_sub(code, {"DTS_QSORT_MIN": "0", "DTS_QSORT_DROP": "4"}))
    assert len(sorted_out) == 43
    assert sorted_out == plain_out
    assert multi_out == plain_out
    for seed in range(40):
        D, Q = synth.adversarial(7000 + seed, 60, 60)
        d = [0.0, 0.03, 0.1, 0.3][seed % 4]
        got = np.frombuffer(sorted_out[seed], dtype=dts.RESULT_DTYPE)
        parity.compare(got, oracle_mod.search(D, Q, d), D, Q, d, oracle_mod)
    c = synth.make_config("C2", scale=0.02)
    g = synth.rng(5)
    qs = np.sort(g.choice(c.Q.shape[0], size=120, replace=False))
    for k, d in enumerate((0.09, 2.0, 8.0)):
        got = np.frombuffer(sorted_out[40 + k], dtype=dts.RESULT_DTYPE)
        parity.compare(parity.restrict(got, qs),
                       oracle_mod.search_queries(c.D, c.Q, qs, d, threads=THREADS),
                       c.D, c.Q, d, oracle_mod)
