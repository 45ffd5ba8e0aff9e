"""Long-segment outliers (internal.cuh "outliers"): a few
entries far longer in space or time than the rest are filed as copies along
their path instead of widening every stencil.  The results must be the
oracle's, with no duplicate from the copies, and byte-identical to plain
filing (DTS_OUTLIERS=0)."""
import os
import subprocess
import sys

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


def with_long_segments(D, k, seed, t_span, length, dur, lo, hi):
    """D plus k long segments: random start in [lo, hi]^3 and time, a random
    direction of the given spatial length, the given duration (some of them
    stationary, some axis-aligned, some diagonal)."""
    g = synth.rng(seed)
    L = np.zeros((k, 8))
    t0 = g.uniform(t_span[0], t_span[1] - dur, k)
    p0 = g.uniform(lo, hi, (k, 3))
    dirs = g.normal(0, 1, (k, 3))
    dirs[::4] = [1.0, 0.0, 0.0]                   # axis-aligned
    dirs /= np.linalg.norm(dirs, axis=1)[:, None]
    length = np.full(k, length)
    length[1::5] = 0.0                              # slow: long in time, still in space
    L[:, 0], L[:, 4] = t0, t0 + dur
    L[:, 1:4] = p0
    L[:, 5:8] = p0 + dirs * length[:, None]
    return np.ascontiguousarray(np.concatenate([D, L])), L


def crossing_queries(L, g, n):
    """Short queries placed on random points of the long segments."""
    i = g.integers(0, L.shape[0], n)
    f = g.uniform(0.05, 0.95, n)
    t = L[i, 0] + f * (L[i, 4] - L[i, 0])
    p = L[i, 1:4] + f[:, None] * (L[i, 5:8] - L[i, 1:4])
    Q = np.zeros((n, 8))
    Q[:, 0], Q[:, 4] = t - 0.4, t + 0.4
    Q[:, 1:4] = p + g.normal(0, 0.002, (n, 3))
    Q[:, 5:8] = Q[:, 1:4] + g.normal(0, 0.01, (n, 3))
    return Q


def _plain_bytes(D, Q, d):
    code = ("import sys, numpy as np; sys.path[:0] = [%r, %r]; "
            "import paper_conf_ipps_gowanlockc15_b200 as m\n"
            "D = np.load(sys.argv[1]); Q = np.load(sys.argv[2])\n"
            "i = m.build_index(D); assert i.info()['outlier_rows'] == 0\n"
            "sys.stdout.buffer.write(m.search(i, Q, float(sys.argv[3])).tobytes())"
            % (REPO, os.path.join(REPO, "tests")))
    import tempfile
    with tempfile.TemporaryDirectory() as td:
        np.save(os.path.join(td, "D.npy"), D)
        np.save(os.path.join(td, "Q.npy"), Q)
        out = subprocess.run([sys.executable, "-c", code, os.path.join(td, "D.npy"),
                              os.path.join(td, "Q.npy"), repr(d)],
                             env={**os.environ, "DTS_OUTLIERS": "0"}, capture_output=True,
                             timeout=900)
    assert out.returncode == 0, out.stderr.decode()[-3000:]
    return out.stdout


@pytest.mark.parametrize("d", [0.0, 0.005, 0.05])
def test_galaxy_with_long_segments(dts, oracle_mod, d):
    """C1-shaped galaxy (scale 0.2) plus 0.1% long segments (30 units of
    travel over 40 time steps, a fifth of them stationary): copies filed,
    the grid keeps the galaxy's cell size, results = oracle = plain filing."""
    c = synth.make_config("C1", scale=0.2)
    D, L = with_long_segments(c.D, max(8, c.D.shape[0] // 1000), 3, (0.0, 192.0), 30.0, 40.0,
                              -12.0, 12.0)
    g = synth.rng(5)
    Q = np.ascontiguousarray(np.concatenate([c.Q[:600], crossing_queries(L, g, 300)]))
    idx = dts.build_index(D)
    inf = idx.info()
    assert inf["outlier_rows"] >= L.shape[0], inf
    assert inf["outlier_copies"] > inf["outlier_rows"]
    assert max(inf["max_extent"]) < 1.0, inf          # the galaxy's, not the long segments'
    got = dts.search(idx, Q, d)
    parity.assert_canonical(got)                        # no duplicate from the copies
    ora = oracle_mod.search(D, Q, d, threads=THREADS)
    info = parity.compare(got, ora, D, Q, d, oracle_mod)
    hit_long = np.isin(got["entry_id"], np.arange(c.D.shape[0], D.shape[0])).sum()
    if d > 0:
        assert hit_long > 50
    assert got.tobytes() == _plain_bytes(D, Q, d)
    # device API, count-only and the spill path agree
    total, counts, _ = dts.search_count(idx, Q, d)
    assert total == got.shape[0]
    idx.free()


def test_random_sets_with_long_segments(dts, oracle_mod):
    """Small random sets where a few entries are 20-50x longer than the rest
    (in space, in time, or both): exhaustive parity with the oracle over many
    seeds and distances."""
    total_long = 0
    for seed in range(60):
        g = synth.rng(900 + seed)
        D, Q = synth.random_small(900 + seed, 400, 60, side=1.0, tspan=6.0, maxdur=0.5,
                                  maxlen=0.03)
        k = 4 + seed % 5
        D, L = with_long_segments(D, k, 2000 + seed, (0.0, 6.0), [1.0, 0.0, 1.5][seed % 3],
                                  [0.5, 4.0, 5.5][seed % 3], 0.0, 1.0)
        Q = np.ascontiguousarray(np.concatenate([Q, crossing_queries(L, g, 20)]))
        d = [0.0, 0.01, 0.05, 0.2][seed % 4]
        idx = dts.build_index(D)
        inf = idx.info()
        got = dts.search(idx, Q, d)
        idx.free()
        parity.assert_canonical(got)
        ora = oracle_mod.search(D, Q, d)
        parity.compare(got, ora, D, Q, d, oracle_mod)
        total_long += int(inf["outlier_rows"])
    assert total_long > 100                              # the copies path was exercised


def test_output_heavy_with_long_segments_all_buffer_paths(dts, oracle_mod):
    """Output-heavy tiles on an index with copies: spilled records carry
    sorted positions and are resolved and filtered after pass 1
    (k_spill_filter); with the spill or the staging buffer forced small
    (DTS_SPILL_CAP, DTS_STAGE_CAP) pass 1 goes round again with buffers sized
    by its counts.  Same bytes every way, = plain filing, = the oracle."""
    code = ("import sys; sys.path[:0] = [%r, %r]; import numpy as np, "
            "paper_conf_ipps_gowanlockc15_b200 as m\n"
            "D = np.load(sys.argv[1]); Q = np.load(sys.argv[2])\n"
            "i = m.build_index(D); inf = i.info()\n"
            "import os\n"
            "if os.environ.get('DTS_OUTLIERS') != '0': assert inf['outlier_rows'] >= 20, inf\n"
            "r = m.search(i, Q, 0.01); assert m.search_count(i, Q, 0.01)[0] == r.shape[0]\n"
            "sys.stdout.buffer.write(r.tobytes())" % (REPO, os.path.join(REPO, "tests")))
    g = np.random.default_rng(17)
    n = 3000
    D = np.zeros((n, 8))
    D[:, 4] = 1.0
    D[:, 1:4] = g.uniform(0, 0.05, (n, 3))
    D[:, 5:8] = D[:, 1:4] + g.uniform(-0.002, 0.002, (n, 3))
    L = np.zeros((24, 8))                     # 30 units of travel across the cube
    L[:, 4] = 1.0
    L[:, 1], L[:, 5] = -15.0, 15.0
    L[:, [2, 3]] = g.uniform(0, 0.05, (24, 2))
    L[:, [6, 7]] = L[:, [2, 3]]
    L[::3, 5:8] = L[::3, 1:4] + [30.0, 0.02, -0.01]
    D = np.ascontiguousarray(np.concatenate([D, L]))
    Q = np.ascontiguousarray(D[g.choice(n, 300, replace=False)])
    import tempfile
    outs = []
    with tempfile.TemporaryDirectory() as td:
        np.save(os.path.join(td, "D.npy"), D)
        np.save(os.path.join(td, "Q.npy"), Q)
        for env in ({}, {"DTS_SPILL_CAP": "1000"}, {"DTS_SPILL_CAP": "0"},
                    {"DTS_STAGE_CAP": "0"}, {"DTS_OUTLIERS": "0"}):
            out = subprocess.run([sys.executable, "-c", code, os.path.join(td, "D.npy"),
                                  os.path.join(td, "Q.npy")], env={**os.environ, **env},
                                 capture_output=True, timeout=900)
            assert out.returncode == 0, (env, out.stderr.decode()[-3000:])
            outs.append(out.stdout)
    assert all(o == outs[0] for o in outs[1:])
    got = np.frombuffer(outs[0], dtype=dts.RESULT_DTYPE)
    parity.assert_canonical(got)
    info = parity.compare(got, oracle_mod.search(D, Q, 0.01, threads=THREADS), D, Q, 0.01,
                          oracle_mod)
    assert info["common"] > 30 * Q.shape[0]                   # output-heavy: tiles spill
    assert np.isin(got["entry_id"], np.arange(n, D.shape[0])).sum() > 100   # copies hit
