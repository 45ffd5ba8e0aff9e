"""GPU parity: the CUDA path (through the C ABI) against the oracle on the
same seeded inputs.  Rule: tests/parity.py (pair set outside the 1e-9*d tie
band identical, endpoints within 1e-9 normalised time, canonical order)."""
import os

import numpy as np
import pytest

import synth
import dts_parity as parity

pytestmark = pytest.mark.gpu

THREADS = max(1, min(32, os.cpu_count() or 1))
REPO = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def dts():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_gowanlockc15_b200 as m
    m.load()
    return m


def run_and_compare(dts, oracle_mod, D, Q, d, **params):
    idx = dts.build_index(D, **params)
    got = dts.search(idx, Q, d)
    ora = oracle_mod.search(D, Q, d, threads=THREADS)
    info = parity.compare(got, ora, D, Q, d, oracle_mod)
    idx.free()
    return got, info


# ------------------------------------------------------------------ C0
@pytest.mark.parametrize("d", [0.0, 0.01, 0.05, 0.2])
def test_c0_exhaustive(dts, oracle_mod, d):
    c = synth.make_config("C0")
    got, info = run_and_compare(dts, oracle_mod, c.D, c.Q, d)
    if d >= 0.05:
        assert info["common"] > 0


def test_c0_headline_has_hits_and_crossings(dts, oracle_mod):
    c = synth.make_config("C0")
    got, info = run_and_compare(dts, oracle_mod, c.D, c.Q, c.d)
    assert info["common"] >= 20


# ------------------------------------------------ random / adversarial sets
def test_random_adversarial_sets(dts, oracle_mod):
    total = 0
    for seed in range(300):
        D, Q = synth.adversarial(1000 + seed, 50, 50)
        d = [0.0, 0.03, 0.1, 0.3][seed % 4]
        _, info = run_and_compare(dts, oracle_mod, D, Q, d)
        total += info["common"]
    assert total > 1000


def test_paper_example_on_gpu(dts):
    import json
    ex = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_example.json")))
    idx = dts.build_index(np.array(ex["D"]))
    got = dts.search(idx, np.array(ex["Q"]), ex["d"])
    assert got.shape[0] == 2
    for r, e in zip(got, ex["expected"]):
        assert (int(r["query_id"]), int(r["entry_id"])) == tuple(e[:2])
        assert abs(r["t_start"] - e[2]) < 1e-12 and abs(r["t_end"] - e[3]) < 1e-12


def test_golden_pairs_on_gpu(dts):
    import json
    spec = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "pairs.json")))
    for p in spec["pairs"]:
        idx = dts.build_index(np.array([p["l"]]))
        got = dts.search(idx, np.array([p["q"]]), p["d"])
        if p["expected"] is None:
            assert got.shape[0] == 0, p["id"]
        elif not p["tie_band"]:
            assert got.shape[0] == 1, p["id"]
            assert abs(got[0]["t_start"] - p["expected"][0]) < 1e-12, p["id"]
            assert abs(got[0]["t_end"] - p["expected"][1]) < 1e-12, p["id"]


# ------------------------------------------------ index invariance, determinism
def test_index_parameter_invariance_and_determinism(dts, oracle_mod):
    c = synth.make_config("C2", scale=0.02)
    d = 0.5
    ref = None
    for params in ({}, {"temporal_bins": 7}, {"temporal_bins": 5000}, {"cells_per_dim": 3},
                   {"d_hint": 2.0}, {"d_hint": 0.01, "temporal_bins": 1}):
        idx = dts.build_index(c.D, **params)
        for _ in range(2):
            got = dts.search(idx, c.Q, d)
            if ref is None:
                ref = got
                parity.compare(got, oracle_mod.search(c.D, c.Q, d, threads=THREADS), c.D, c.Q, d,
                               oracle_mod)
            assert got.tobytes() == ref.tobytes(), params
        idx.free()


def test_index_layout_variants_invariant(dts, oracle_mod, monkeypatch):
    """Same result bytes whatever digit plan the build's radix sort takes
    (8-bit only, or 9-bit digits where they save a pass), whichever grid
    source (sampled + fused keys pass, or exact bounds first), hash load,
    gather shape, pass-1 occupancy, query order and queries per warp tile the
    index and search use: they only change the layout and the schedule."""
    c = synth.make_config("C1", scale=0.1)
    ref = None
    for env in ({"DTS_RADIX9": "0"}, {"DTS_RADIX9": "1"}, {"DTS_HASH_SLOTS": "1.2"},
                {"DTS_FUSED_KEYS": "0"}, {"DTS_OS_SHAPE": "0"}, {"DTS_GATHER": "4"},
                {"DTS_GATHER": "1"}, {"DTS_TILE_OCC": "6"}, {"DTS_TILE_OCC": "8"},
                {"DTS_QSORT_MIN": "0"}, {"DTS_QSORT_MIN": "0", "DTS_QSORT_DROP": "0"},
                {"DTS_TILE_FILL": "0"}, {"DTS_TILE_Q": "1"}, {"DTS_TILE_Q": "3"}):
        # the toggles are read once per process: run each in a subprocess
        import subprocess
        import sys
        code = ("import sys; sys.path[:0] = [%r, %r]; import numpy as np, synth, "
                "paper_conf_ipps_gowanlockc15_b200 as m; c = synth.make_config('C1', scale=0.1); "
                "i = m.build_index(c.D); r = m.search(i, c.Q, c.d); "
                "sys.stdout.buffer.write(r.tobytes())" % (REPO, os.path.join(REPO, "tests")))
        out = subprocess.run([sys.executable, "-c", code], env={**os.environ, **env},
                             capture_output=True, timeout=600)
        assert out.returncode == 0, out.stderr.decode()[-2000:]
        if ref is None:
            ref = out.stdout
            got = np.frombuffer(ref, dtype=dts.RESULT_DTYPE)
            parity.compare(got, oracle_mod.search(c.D, c.Q, c.d, threads=THREADS), c.D, c.Q,
                           c.d, oracle_mod)
        assert out.stdout == ref, env


def test_crowded_cells(dts, oracle_mod):
    """Blocks of 8 cells holding more than a warp's worth of entries (the
    insert's warp path) and more than 65,535 (one run per block): parity with
    the oracle, and the same bytes with a denser hash table, the exact-bounds
    grid and sorted queries."""
    import subprocess
    import sys
    D, Q = synth.crowded(5)
    d = 0.01
    got, info = run_and_compare(dts, oracle_mod, D, Q, d)
    assert info["common"] > 200000
    code = ("import sys; sys.path[:0] = [%r, %r]; import synth, "
            "paper_conf_ipps_gowanlockc15_b200 as m; D, Q = synth.crowded(5); "
            "i = m.build_index(D); r = m.search(i, Q, %r); "
            "sys.stdout.buffer.write(r.tobytes())" % (REPO, os.path.join(REPO, "tests"), d))
    for env in ({"DTS_HASH_SLOTS": "1.2"}, {"DTS_FUSED_KEYS": "0"}, {"DTS_QSORT_MIN": "0"}):
        out = subprocess.run([sys.executable, "-c", code], env={**os.environ, **env},
                             capture_output=True, timeout=600)
        assert out.returncode == 0, out.stderr.decode()[-2000:]
        assert out.stdout == got.tobytes(), env


def _sampled_positions(n):
    """The rows the build's 2^16-entry sample reads: j n / S (k_bounds_sample)."""
    S = min(n, 1 << 16)
    return [j * n // S for j in range(S)]


def _unsampled_positions(n, k):
    """k positions that the build's 2^16-entry stride sample does not read."""
    sampled = set(_sampled_positions(n))
    out = [i for i in range(1, n) if i not in sampled][:k]
    assert len(out) == k
    return out


@pytest.mark.parametrize("kind", ["long_segments", "far_outliers"])
def test_sampled_grid_misses_outliers(dts, oracle_mod, kind):
    """The build derives its grid from a strided sample of D; entries the
    sample misses -- segments far longer than any sampled one (the grid is
    then rebuilt from the exact bounds) or short segments far outside the
    sampled domain (they clamp into the boundary cells) -- must still be
    found, with the stencils taken from the exact extents (the grid is
    rebuilt from the exact bounds when the sample missed part of the
    domain)."""
    c = synth.make_config("C1", scale=0.2)
    D = c.D.reshape(-1, 8).copy()
    n = D.shape[0]
    assert n > (1 << 16)
    pos = _unsampled_positions(n, 6)
    g = synth.rng(77)
    for k, i in enumerate(pos):
        t0 = float(g.uniform(0, 150))
        if kind == "long_segments":      # 40 time units, 30 units of x travel
            D[i] = [t0, -15.0 + k, 0.5, 0.0, t0 + 40.0, 15.0 + k, 0.5, 0.0]
        else:                            # short segments 1e3 away
            D[i] = [t0, 1000.0 + k, -800.0, 5.0, t0 + 1.0, 1000.01 + k, -800.0, 5.0]
    # queries: the headline ones plus segments that cross each outlier
    extra = []
    for i in pos:
        t0, x0, y0, z0, t1, x1, y1, z1 = D[i]
        tm = 0.5 * (t0 + t1)
        xm, ym, zm = 0.5 * (x0 + x1), 0.5 * (y0 + y1), 0.5 * (z0 + z1)
        extra.append([tm - 0.5, xm, ym - 0.002, zm, tm + 0.5, xm, ym + 0.002, zm])
    Q = np.concatenate([c.Q.reshape(-1, 8)[:400], np.array(extra)]).astype(np.float64)
    idx = dts.build_index(D)
    inf = idx.info()
    got = dts.search(idx, Q, c.d)
    ora = oracle_mod.search(D, Q, c.d, threads=THREADS)
    info = parity.compare(got, ora, D, Q, c.d, oracle_mod)
    hit = set(zip(got["query_id"].tolist(), got["entry_id"].tolist()))
    for k, i in enumerate(pos):
        assert (400 + k, i) in hit, (kind, k)
    assert info["common"] >= len(pos)
    if kind == "long_segments":
        # filed as copies along their path (outliers: extent far above the
        # sample's mean), so the grid keeps the short segments' extent;
        # without outlier filing the exact extent sizes the grid instead
        assert inf["outlier_rows"] >= 6 or inf["max_extent"][0] >= 30.0, inf
    idx.free()


def test_periodic_input_sample_not_aliased(dts, oracle_mod):
    """Trajectory-major D whose sample stride is a multiple of the segments
    per trajectory (4 here, as 192 is for the paper's S2 shape): the strided
    sample sees one time step and would build two bins; the exact time range
    (from the fused keys pass) lies well outside the sampled one, so the
    build redoes the keys with the exact grid, one bin per time step.  Results match the
    oracle either way."""
    g = synth.rng(11)
    ntraj, nseg = 1 << 16, 4
    t = np.arange(nseg + 1, dtype=np.float64)
    pos = np.cumsum(g.normal(0, 0.01, (ntraj, nseg + 1, 3)), axis=1) + g.uniform(0, 1, (ntraj, 1, 3))
    D = np.empty((ntraj, nseg, 8))
    D[:, :, 0] = t[:-1]
    D[:, :, 4] = t[1:]
    D[:, :, 1:4] = pos[:, :-1]
    D[:, :, 5:8] = pos[:, 1:]
    D = np.ascontiguousarray(D.reshape(-1, 8))
    Q = np.ascontiguousarray(D[::2621][:100].copy())
    idx = dts.build_index(D)
    inf = idx.info()
    assert inf["bins"] >= nseg, inf
    got = dts.search(idx, Q, 0.003)
    idx.free()
    ora = oracle_mod.search(D, Q, 0.003, threads=THREADS)
    info = parity.compare(got, ora, D, Q, 0.003, oracle_mod)
    assert info["common"] >= Q.shape[0]


def test_build_phase_timings(dts):
    c = synth.make_config("C1", scale=0.1)
    idx = dts.build_index(c.D)
    inf = idx.info()
    ph = list(inf["ms_phase"])
    assert len(ph) == 5 and all(x >= 0.0 for x in ph)
    assert inf["ms_build"] > 0.0
    assert sum(ph) <= inf["ms_build"] * 1.001 + 1e-3
    idx.free()


def test_device_api_matches_host_api(dts):
    import torch
    c = synth.make_config("C0")
    idx_h = dts.build_index(c.D)
    host = dts.search(idx_h, c.Q, c.d, query_id_base=7)
    Dd = torch.from_numpy(c.D).cuda()
    Qd = torch.from_numpy(c.Q).cuda()
    idx_d = dts.build_index_device(Dd)
    res, stats = dts.search_device(idx_d, Qd, c.d, query_id_base=7, time_kernels=True)
    dev = res.numpy()
    assert dev.tobytes() == host.tobytes()
    assert stats["results"] == host.shape[0]
    assert stats["candidates"] >= host.shape[0]
    assert np.all(host["query_id"] >= 7)


# ------------------------------------------------ configs at reduced / full size
@pytest.mark.parametrize("name,scale,dlist", [
    ("C1", 1.0, (0.001, 0.005, 0.02)),
    ("C2", 0.05, (0.03, 0.09, 0.5, 2.0)),
    ("C3", 0.05, (1.0, 5.0, 20.0, 50.0)),
])
def test_configs_sampled(dts, oracle_mod, name, scale, dlist):
    c = synth.make_config(name, scale=scale)
    idx = dts.build_index(c.D)
    g = synth.rng(99)
    qs = np.sort(g.choice(c.Q.shape[0], size=min(96, c.Q.shape[0]), replace=False))
    for d in dlist:
        got = dts.search(idx, c.Q, d)
        ora = oracle_mod.search_queries(c.D, c.Q, qs, d, threads=THREADS)
        parity.compare(parity.restrict(got, qs), ora, c.D, c.Q, d, oracle_mod)
    idx.free()


def test_c2_small_exhaustive_large_d(dts, oracle_mod):
    """Many candidates per query, > 32 stencil cells (chunked lookups) and
    > 32 results per query (CTA sort path)."""
    c = synth.make_config("C2", scale=0.004)
    for d in (2.0, 8.0):
        got, info = run_and_compare(dts, oracle_mod, c.D, c.Q, d)
        assert info["common"] > 0


def test_c4_full_size_sampled(dts, oracle_mod):
    """BASELINE.json configs[4] at full size, in the bench's launch
    configuration (device-resident build + search): sampled queries against
    the oracle, plus size-independent properties."""
    import torch
    c = synth.make_config("C4")
    Dd = torch.from_numpy(c.D).cuda()
    Qd = torch.from_numpy(c.Q).cuda()
    idx = dts.build_index_device(Dd)
    res, stats = dts.search_device(idx, Qd, c.d)
    got = res.numpy()
    parity.assert_canonical(got)
    # every query is a copy of an entry (Q sampled from D): its self pair is a
    # result over the whole segment
    nq = c.Q.shape[0]
    assert np.unique(got["query_id"]).size == nq
    g = synth.rng(123)
    qs = np.sort(g.choice(nq, size=48, replace=False))
    ora = oracle_mod.search_queries(c.D, c.Q, qs, c.d, threads=THREADS)
    parity.compare(parity.restrict(got, qs), ora, c.D, c.Q, c.d, oracle_mod)


# ------------------------------------------------ edge cases and errors
def test_empty_inputs(dts):
    D, Q = synth.random_small(5, 10, 10)
    idx = dts.build_index(D)
    assert dts.search(idx, np.empty((0, 8)), 0.1).shape[0] == 0
    empty = dts.build_index(np.empty((0, 8)))
    assert dts.search(empty, Q, 0.1).shape[0] == 0
    far = Q.copy()
    far[:, [0, 4]] += 1e6
    assert dts.search(idx, far, 0.1).shape[0] == 0


def test_huge_result_segment(dts, oracle_mod):
    """Spilled queries of every segment-sort size class in one tile: 300
    results (a warp), 2,000 (a 256-thread CTA), 6,000 (a 1024-thread CTA)
    and 17,000 (device-wide radix sort of long segments), with the entries
    of each cluster in shuffled order."""
    g = synth.rng(77)
    parts = []
    for k, m in enumerate((17000, 6000, 2000, 300)):
        P = np.zeros((m, 8))
        P[:, 4] = 1.0
        P[:, 1:4] = k + g.uniform(0, 0.01, size=(m, 3))
        P[:, 5:8] = P[:, 1:4]
        parts.append(P)
    D = np.concatenate(parts)
    D = D[g.permutation(D.shape[0])]
    Q = np.array([[0.0, k + 0.005, k + 0.005, k + 0.005, 1.0, k + 0.005, k + 0.005, k + 0.005]
                  for k in range(4)] + [[0.0, 0.5, 0.5, 0.5, 1.0, 0.6, 0.6, 0.6]])
    got, info = run_and_compare(dts, oracle_mod, D, Q, 0.05)
    assert np.array_equal(np.bincount(got["query_id"], minlength=5), [17000, 6000, 2000, 300, 0])
    # caller entry ids over all 32 bits (four radix passes in the warp sort)
    ids = ((g.permutation(D.shape[0]).astype(np.uint64) * 2654435761 + 12345) % (1 << 32)).astype(np.uint32)
    idx = dts.build_index(D, entry_ids=ids)
    got2 = dts.search(idx, Q, 0.05)
    idx.free()
    assert np.array_equal(got2["query_id"], got["query_id"])
    for qi in range(4):
        e = got2["entry_id"][got2["query_id"] == qi]
        assert np.all(np.diff(e.astype(np.int64)) > 0)                 # canonical order
        assert np.array_equal(np.sort(e), np.sort(ids[got["entry_id"][got["query_id"] == qi]]))
    # clustered ids (one far id per query widens the id range): the bucket
    # sort's buckets overflow and those segments go to the radix sort
    ids3 = np.arange(D.shape[0], dtype=np.uint32)
    for qi in (1, 2):
        ids3[got["entry_id"][got["query_id"] == qi][7]] = 4_000_000_000 + qi
    idx = dts.build_index(D, entry_ids=ids3)
    got3 = dts.search(idx, Q, 0.05)
    idx.free()
    assert np.array_equal(got3["query_id"], got["query_id"])
    for qi in range(4):
        e = got3["entry_id"][got3["query_id"] == qi]
        assert np.all(np.diff(e.astype(np.int64)) > 0)
        assert np.array_equal(np.sort(e), np.sort(ids3[got["entry_id"][got["query_id"] == qi]]))


def test_invalid_inputs_raise(dts):
    D, Q = synth.random_small(6, 10, 10)
    bad = D.copy()
    bad[3, 2] = np.nan
    with pytest.raises(dts.DTSError) as e:
        dts.build_index(bad)
    assert e.value.status == -1
    bad = D.copy()
    bad[4, 4] = bad[4, 0] - 1.0
    with pytest.raises(dts.DTSError):
        dts.build_index(bad)
    idx = dts.build_index(D)
    with pytest.raises(dts.DTSError):
        dts.search(idx, Q, -1.0)
    with pytest.raises(dts.DTSError):
        dts.search(idx, Q, float("inf"))
    badq = Q.copy()
    badq[0, 0] = np.inf
    with pytest.raises(dts.DTSError):
        dts.search(idx, badq, 0.1)
    # the index stays usable after an error
    assert dts.search(idx, Q, 0.1).dtype == dts.RESULT_DTYPE


# ------------------------------------------------ candidate generators (§8 f1)
@pytest.mark.parametrize("method,subbins", [("temporal", 0), ("subbin", 2), ("subbin", 4),
                                            ("subbin", 16)])
def test_methods_match_oracle_and_grid(dts, oracle_mod, method, subbins):
    """GPUTemporal / GPUSpatioTemporal candidate generators return the same
    bytes as the grid and match the oracle."""
    cases = [(synth.make_config("C0"), (0.0, 0.05, 0.2)),
             (synth.make_config("C2", scale=0.004), (0.09, 2.0)),
             (synth.make_config("C3", scale=0.01), (5.0, 50.0))]
    for c, dl in cases:
        grid = dts.build_index(c.D)
        alt = dts.build_index(c.D, method=method, subbins=subbins)
        info = alt.info()
        assert info["method"] == {"temporal": 1, "subbin": 2}[method]
        if method == "subbin":
            assert all(v >= 1 for v in info["subbins"])
            assert all(info["subbin_ids"][a] >= c.D.shape[0] for a in range(3))
        for d in dl:
            ref = dts.search(grid, c.Q, d)
            got = dts.search(alt, c.Q, d)
            assert got.tobytes() == ref.tobytes(), (method, subbins, d)
            parity.compare(got, oracle_mod.search(c.D, c.Q, d, threads=THREADS), c.D, c.Q, d,
                           oracle_mod)


def test_subbin_adversarial(dts, oracle_mod):
    for seed in range(60):
        D, Q = synth.adversarial(5000 + seed, 50, 50)
        d = [0.0, 0.03, 0.1, 0.3][seed % 4]
        idx = dts.build_index(D, method="subbin", subbins=[2, 4, 8][seed % 3])
        got = dts.search(idx, Q, d)
        parity.compare(got, oracle_mod.search(D, Q, d), D, Q, d, oracle_mod)


def test_subbin_c1_sampled(dts, oracle_mod):
    c = synth.make_config("C1")
    idx = dts.build_index(c.D, method="subbin")
    g = synth.rng(7)
    qs = np.sort(g.choice(c.Q.shape[0], size=64, replace=False))
    for d in (0.005, 0.02):
        got = dts.search(idx, c.Q, d)
        ora = oracle_mod.search_queries(c.D, c.Q, qs, d, threads=THREADS)
        parity.compare(parity.restrict(got, qs), ora, c.D, c.Q, d, oracle_mod)


def test_streamed_host_search_matches(dts, oracle_mod, monkeypatch):
    """Results larger than the device budget are streamed in query chunks by
    dts_search (host); forced here with DTS_MAX_DEVICE_RESULTS."""
    c = synth.make_config("C2", scale=0.004)
    idx = dts.build_index(c.D)
    ref = dts.search(idx, c.Q, 2.0)
    assert ref.shape[0] > 500
    monkeypatch.setenv("DTS_MAX_DEVICE_RESULTS", str(ref.shape[0] // 7))
    got, st = dts.search_ex(idx, c.Q, 2.0)
    assert got.tobytes() == ref.tobytes()
    assert st["results"] == ref.shape[0]
    # the cap applies to the host API only; the device API returns everything
    import torch
    monkeypatch.setenv("DTS_MAX_DEVICE_RESULTS", "0")
    res, _ = dts.search_device(idx, torch.from_numpy(c.Q).cuda(), 2.0)
    assert res.count == ref.shape[0]


def test_heavy_output_recompute_path(dts, oracle_mod):
    """Tiles whose hits overflow the staging (many results per query) take the
    count-then-scatter recompute + radix canonicalisation path."""
    g = synth.rng(91)
    n = 3000
    D = np.zeros((n, 8))
    D[:, 0], D[:, 4] = 0.0, 1.0
    D[:, 1:4] = g.uniform(0, 0.02, size=(n, 3))
    D[:, 5:8] = D[:, 1:4] + g.uniform(-0.01, 0.01, size=(n, 3))
    Q = D[g.choice(n, size=40, replace=False)].copy()
    for d in (0.01, 0.05):
        got, info = run_and_compare(dts, oracle_mod, D, Q, d)
        assert info["common"] > 1000


def test_spill_paths_same_bytes(dts, oracle_mod):
    """Output-heavy tiles spill their hits (no re-stream); with the spill
    buffer forced small (DTS_SPILL_CAP) tiles find it full and are re-run
    into an exactly sized buffer, and with it forced to 0 every spilling
    tile is re-run.  Same bytes every way, oracle parity, including queries
    with more results than one CTA sorts (device-wide sort of long
    segments)."""
    import subprocess
    import sys
    code = ("import sys; sys.path[:0] = [%r, %r]; import numpy as np, synth, "
            "paper_conf_ipps_gowanlockc15_b200 as m\n"
            "c = synth.make_config('C2', scale=0.004)\n"
            "g = np.random.default_rng(5); n = 4000\n"
            "D = np.zeros((n, 8)); D[:, 4] = 1.0\n"
            "D[:, 1:4] = g.uniform(0, 0.01, (n, 3)); D[:, 5:8] = D[:, 1:4]\n"
            "Q = np.array([[0.0, 0, 0, 0, 1.0, 0.005, 0.005, 0.005]] * 3)\n"
            "out = [m.search(m.build_index(c.D), c.Q, d).tobytes() for d in (2.0, 8.0)]\n"
            "out.append(m.search(m.build_index(D), Q, 0.05).tobytes())\n"
            "sys.stdout.buffer.write(b''.join(len(o).to_bytes(8, 'little') + o for o in out))"
            % (REPO, os.path.join(REPO, "tests")))

    def split(buf):
        parts, k = [], 0
        while k < len(buf):
            n = int.from_bytes(buf[k:k + 8], "little")
            parts.append(buf[k + 8:k + 8 + n])
            k += 8 + n
        return parts
    runs = []
    # (and with 16- and 2-query warp tiles: the tile size sets which hits
    #  share a stage, so which tiles spill)
    for env in ({}, {"DTS_SPILL_CAP": "1000"}, {"DTS_SPILL_CAP": "0"},
                {"DTS_TILE_FILL": "0", "DTS_SPILL_CAP": "1000"},
                {"DTS_TILE_Q": "2", "DTS_SPILL_CAP": "0"}):
        out = subprocess.run([sys.executable, "-c", code], env={**os.environ, **env},
                             capture_output=True, timeout=900)
        assert out.returncode == 0, out.stderr.decode()[-3000:]
        runs.append(split(out.stdout))
    assert all(r == runs[0] for r in runs[1:])
    c = synth.make_config("C2", scale=0.004)
    for k, d in enumerate((2.0, 8.0)):
        got = np.frombuffer(runs[0][k], dtype=dts.RESULT_DTYPE)
        info = parity.compare(got, oracle_mod.search(c.D, c.Q, d, threads=THREADS), c.D, c.Q, d,
                              oracle_mod)
        if d == 8.0:                            # hundreds of results per query: spills
            assert info["common"] > 20 * c.Q.shape[0]
    g = np.random.default_rng(5)
    n = 4000
    D = np.zeros((n, 8))
    D[:, 4] = 1.0
    D[:, 1:4] = g.uniform(0, 0.01, (n, 3))
    D[:, 5:8] = D[:, 1:4]
    Q = np.array([[0.0, 0, 0, 0, 1.0, 0.005, 0.005, 0.005]] * 3)
    got = np.frombuffer(runs[0][2], dtype=dts.RESULT_DTYPE)
    info = parity.compare(got, oracle_mod.search(D, Q, 0.05), D, Q, 0.05, oracle_mod)
    assert info["common"] == 3 * n              # three queries with 4,000 results each


@pytest.mark.parametrize("world", [2, 3])
def test_temporal_shards_on_one_gpu_match_unsharded(dts, world):
    """SURVEY §4 'multi-GPU without a cluster': the temporal-range shards of D
    searched one after another on one GPU (global ids via entry_ids /
    query_ids), concatenated and canonicalised on the device, give the
    unsharded result byte for byte."""
    import torch

    from paper_conf_ipps_gowanlockc15_b200 import dist as dts_dist
    c = synth.make_config("C2", scale=0.004)
    d = 0.5
    ref = dts.search(dts.build_index(c.D), c.Q, d)
    T, rows, maxdur = dts_dist.temporal_partition(c.D, world)
    parts = []
    for r in range(world):
        Dd = torch.from_numpy(np.ascontiguousarray(c.D[rows[r]])).cuda()
        ids = torch.from_numpy(rows[r].astype(np.int32)).cuda()
        qrows = dts_dist.route_queries(c.Q, T, maxdur, r)
        Qd = torch.from_numpy(np.ascontiguousarray(c.Q[qrows])).cuda()
        qids = torch.from_numpy(qrows.astype(np.int32)).cuda()
        idx = dts.build_index_device(Dd, entry_ids=ids)
        res, _ = dts.search_device(idx, Qd, d, query_ids=qids)
        parts.append(res.tensor().clone())
        res.free()
        idx.free()
    allres = torch.cat(parts)
    dts.canonicalize_device(allres)
    got = allres.cpu().numpy().view(dts.RESULT_DTYPE)
    assert got.tobytes() == ref.tobytes()


def test_entry_ids_host_build(dts):
    c = synth.make_config("C0")
    ref = dts.search(dts.build_index(c.D), c.Q, c.d)
    perm = np.random.default_rng(3).permutation(c.D.shape[0])
    idx = dts.build_index(c.D[perm], entry_ids=perm.astype(np.uint32))
    got = dts.search(idx, c.Q, c.d)
    assert got.tobytes() == ref.tobytes()


# ------------------------------------------------ trajectory level (§8 f3)
def test_exclude_same_trajectory(dts, oracle_mod):
    """'any OTHER stellar trajectory': pairs of the same trajectory
    are dropped; everything else is the oracle's result."""
    import torch
    c = synth.make_config("C2", scale=0.004)
    d = 2.0
    ora = oracle_mod.search(c.D, c.Q, d, threads=THREADS)
    keep = c.qtraj[ora["query_id"]] != c.etraj[ora["entry_id"]]
    assert (~keep).sum() >= c.Q.shape[0]            # the self pairs existed
    ora = ora[keep]
    for method in ("grid", "subbin"):
        idx = dts.build_index(c.D, entry_traj=c.etraj, method=method)
        got, _ = dts.search_ex(idx, c.Q, d, query_traj=c.qtraj, exclude_same_trajectory=True)
        parity.compare(got, ora, c.D, c.Q, d, oracle_mod)
        idxd = dts.build_index_device(torch.from_numpy(c.D).cuda(),
                                      entry_traj=torch.from_numpy(c.etraj).cuda())
        res, _ = dts.search_device(idxd, torch.from_numpy(c.Q).cuda(), d,
                                   query_traj=torch.from_numpy(c.qtraj).cuda(),
                                   exclude_same_trajectory=True)
        assert res.numpy().tobytes() == got.tobytes()
    with pytest.raises(dts.DTSError):
        dts.search_ex(dts.build_index(c.D), c.Q, d, query_traj=c.qtraj,
                      exclude_same_trajectory=True)


def test_merge_trajectories_matches_oracle(dts, oracle_mod):
    import torch
    for name, scale, d in (("C0", 1.0, 0.2), ("C2", 0.004, 2.0)):
        c = synth.make_config(name, scale=scale)
        idx = dts.build_index_device(torch.from_numpy(c.D).cuda())
        res, _ = dts.search_device(idx, torch.from_numpy(c.Q).cuda(), d)
        seg = res.numpy()
        m = dts.merge_trajectories_device(res, torch.from_numpy(c.qtraj).cuda(),
                                          torch.from_numpy(c.etraj).cuda())
        got = m.numpy()
        ref = oracle_mod.merge_trajectory_pairs(seg, c.qtraj, c.etraj)
        assert got.shape == ref.shape and got.shape[0] > 0
        assert np.array_equal(got["query_traj"], ref["query_traj"])
        assert np.array_equal(got["entry_traj"], ref["entry_traj"])
        assert np.array_equal(got["t_start"], ref["t_start"])
        assert np.array_equal(got["t_end"], ref["t_end"])
        # and against the merge of the ORACLE's segment results
        ora = oracle_mod.merge_trajectory_pairs(oracle_mod.search(c.D, c.Q, d, threads=THREADS),
                                                c.qtraj, c.etraj)
        assert got.shape == ora.shape
        span = float(c.D[:, 4].max() - c.D[:, 0].min())
        assert np.max(np.abs(got["t_start"] - ora["t_start"])) / span < 1e-9
        assert np.max(np.abs(got["t_end"] - ora["t_end"])) / span < 1e-9


def test_stationary_supernova_queries(dts, oracle_mod):
    """Application (i) of P:L15: stars within d of a supernova -- a stationary
    query point over a time window."""
    c = synth.make_config("C2", scale=0.004)
    g = synth.rng(21)
    k = 40
    P = c.D[g.choice(c.D.shape[0], size=k, replace=False)]
    Q = np.zeros((k, 8))
    Q[:, 0] = P[:, 0] - 0.3
    Q[:, 4] = P[:, 0] + 2.7
    Q[:, 1:4] = P[:, 1:4] + g.normal(0, 0.5, size=(k, 3))
    Q[:, 5:8] = Q[:, 1:4]
    for d in (0.5, 3.0):
        got, info = run_and_compare(dts, oracle_mod, c.D, Q, d)
        if d == 3.0:
            assert info["common"] > 0


# ------------------------------------------------ out-of-core Q (§8 f4)
def test_pipelined_query_chunks_match(dts, oracle_mod, monkeypatch):
    """Host query sets streamed through the device in chunks (H2D of the next
    chunk and D2H of the previous results overlap the search) give the same
    bytes as the one-shot search."""
    c = synth.make_config("C2", scale=0.01)
    idx = dts.build_index(c.D, entry_traj=c.etraj)
    monkeypatch.setenv("DTS_Q_CHUNK", "0")
    ref = dts.search(idx, c.Q, 2.0)
    ref_x, _ = dts.search_ex(idx, c.Q, 2.0, query_traj=c.qtraj, exclude_same_trajectory=True,
                             query_id_base=5)
    for chunk in (97, 400, 1500):
        monkeypatch.setenv("DTS_Q_CHUNK", str(chunk))
        got = dts.search(idx, c.Q, 2.0)
        assert got.tobytes() == ref.tobytes(), chunk
        got_x, st = dts.search_ex(idx, c.Q, 2.0, query_traj=c.qtraj,
                                  exclude_same_trajectory=True, query_id_base=5)
        assert got_x.tobytes() == ref_x.tobytes(), chunk
        assert st["results"] == ref_x.shape[0]
    qs = np.arange(0, c.Q.shape[0], 37)
    parity.compare(parity.restrict(ref, qs), oracle_mod.search_queries(c.D, c.Q, qs, 2.0),
                   c.D, c.Q, 2.0, oracle_mod)


def test_host_results_zero_copy_lifetime(dts, oracle_mod):
    """dts_search's host results are a numpy view of the library's pinned
    array: a view taken from them stays valid after the array itself is gone
    and other searches reuse the library's pinned-buffer cache."""
    import gc
    c = synth.make_config("C0")
    idx = dts.build_index(c.D)
    res = dts.search(idx, c.Q, c.d)
    want = res.copy()
    view = res[["query_id", "entry_id"]][::2]
    tail = res["t_end"][1:]
    del res
    gc.collect()
    for _ in range(5):                       # churn the pinned cache
        r = dts.search(idx, c.Q[::-1].copy(), 0.2)
        del r
        gc.collect()
    assert np.array_equal(view["query_id"], want["query_id"][::2])
    assert np.array_equal(view["entry_id"], want["entry_id"][::2])
    assert np.array_equal(tail, want["t_end"][1:])
    idx.free()


def test_density_cap_invariant(dts, oracle_mod):
    """Sparse data (C3-shaped: a few hundred entries per bin in a 1000^3
    cube) gets coarser cells from the density cap; the result bytes are the
    same as with the plain E + d grid (DTS_DENSITY_CAP=0) and match the
    oracle."""
    import subprocess
    import sys
    c = synth.make_config("C3", scale=0.05)
    code = ("import sys; sys.path[:0] = [%r, %r]; import synth, "
            "paper_conf_ipps_gowanlockc15_b200 as m; c = synth.make_config('C3', scale=0.05); "
            "i = m.build_index(c.D); sys.stderr.write(repr(i.info()['grid'])); "
            "r = m.search(i, c.Q, c.d); sys.stdout.buffer.write(r.tobytes())"
            % (REPO, os.path.join(REPO, "tests")))
    outs, grids = [], []
    for env in ({}, {"DTS_DENSITY_CAP": "0"}):
        out = subprocess.run([sys.executable, "-c", code], env={**os.environ, **env},
                             capture_output=True, timeout=600)
        assert out.returncode == 0, out.stderr.decode()[-2000:]
        outs.append(out.stdout)
        grids.append(out.stderr.decode()[-60:])
    assert outs[0] == outs[1], grids
    assert grids[0] != grids[1], grids          # the cap did change the grid
    got = np.frombuffer(outs[0], dtype=dts.RESULT_DTYPE)
    parity.compare(got, oracle_mod.search(c.D, c.Q, c.d, threads=THREADS), c.D, c.Q, c.d,
                   oracle_mod)


def test_segment_sort_class_boundaries(dts, oracle_mod):
    """Spilled queries with exactly 512 / 513 / 4096 / 4097 / 8192 / 8193 /
    16384 / 16385 results: each side of every segment-sort size boundary
    (warp radix, three bucket-sort CTA sizes, device-wide radix)."""
    g = synth.rng(91)
    sizes = (512, 513, 4096, 4097, 8192, 8193, 16384, 16385)
    parts = []
    for k, m in enumerate(sizes):
        P = np.zeros((m, 8))
        P[:, 4] = 1.0
        P[:, 1:4] = 2.0 * k + g.uniform(0, 0.01, size=(m, 3))
        P[:, 5:8] = P[:, 1:4] + g.uniform(-0.001, 0.001, size=(m, 3))
        parts.append(P)
    D = np.concatenate(parts)
    D = D[g.permutation(D.shape[0])]
    Q = np.array([[0.0, 2.0 * k + 0.005, 2.0 * k + 0.005, 2.0 * k + 0.005, 1.0,
                   2.0 * k + 0.005, 2.0 * k + 0.005, 2.0 * k + 0.005] for k in range(len(sizes))])
    got, info = run_and_compare(dts, oracle_mod, D, Q, 0.05)
    assert np.array_equal(np.bincount(got["query_id"], minlength=len(sizes)), sizes)


@pytest.mark.parametrize("nq", [4096, 8192, 8193, 12287])
def test_query_counts_at_scan_tile_edges(dts, oracle_mod, nq):
    """Query sets of whole and partial single-pass scan tiles (4,096 counts):
    exact offsets and the total at the tile edges (C0, queries repeated)."""
    c = synth.make_config("C0")
    Q = np.ascontiguousarray(np.resize(c.Q, (nq, 8)))
    got, info = run_and_compare(dts, oracle_mod, c.D, Q, 0.2)
    assert info["common"] > 0


def test_repeated_searches_speculative_pass2(dts, oracle_mod):
    """Pass 2 of a repeated search of one index is launched before the total
    is known, into a buffer sized by the previous result count; a larger
    output falls back to an exact buffer.  Growing and shrinking outputs on
    one index give the bytes of a fresh index's search."""
    c = synth.make_config("C1", scale=0.1)
    idx = dts.build_index(c.D)
    seq = (0.005, 0.02, 0.02, 0.05, 0.005, 0.05, 0.001)
    got = [dts.search(idx, c.Q, d).tobytes() for d in seq]
    idx.free()
    for d, g in zip(seq, got):
        fresh = dts.build_index(c.D)
        assert g == dts.search(fresh, c.Q, d).tobytes(), d
        fresh.free()
    r = np.frombuffer(got[3], dtype=dts.RESULT_DTYPE)
    qs = np.arange(0, c.Q.shape[0], 7)
    parity.compare(parity.restrict(r, qs), oracle_mod.search_queries(c.D, c.Q, qs, 0.05),
                   c.D, c.Q, 0.05, oracle_mod)


def test_long_segment_split_and_fallback(dts, oracle_mod):
    """Result segments over one CTA sort are split into ordered id ranges
    sorted separately (k_big_split); a segment whose ids cluster so that one
    range exceeds a CTA sort goes to the device-wide sort instead.  Both
    give the canonical order and match the oracle."""
    g = synth.rng(91)
    m = 20000
    P = np.zeros((m, 8))
    P[:, 4] = 1.0
    P[:, 1:4] = g.uniform(0, 0.01, size=(m, 3))
    P[:, 5:8] = P[:, 1:4]
    D = P[g.permutation(m)]
    Q = np.array([[0.0, 0.005, 0.005, 0.005, 1.0, 0.005, 0.005, 0.005]] * 2)
    got, info = run_and_compare(dts, oracle_mod, D, Q, 0.05)     # uniform ids: split
    assert np.array_equal(np.bincount(got["query_id"], minlength=2), [m, m])
    # clustered caller ids: 19,990 consecutive ids and 10 far away
    ids = np.arange(m, dtype=np.uint32)
    ids[-10:] = (1 << 31) + np.arange(10, dtype=np.uint32)
    ids = ids[g.permutation(m)]
    idx = dts.build_index(D, entry_ids=ids)
    got2 = dts.search(idx, Q, 0.05)
    idx.free()
    for qi in range(2):
        e = got2["entry_id"][got2["query_id"] == qi]
        assert e.shape[0] == m and np.all(np.diff(e.astype(np.int64)) > 0)
        assert np.array_equal(np.sort(e), np.sort(ids))
