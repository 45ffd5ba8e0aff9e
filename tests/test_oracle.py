"""Pins for the oracle (oracle/oracle.c) against things other than itself.

Each test names what fixes the expected value: the paper's printed example
(P:L32), hand-worked pairs (tests/golden/pairs.json), a closed form written
differently from the oracle's root formula, dense sampling of the distance
function, an independent golden-section minimisation, and invariants of the
mathematics (symmetry, monotonicity in d, exact power-of-two scaling,
translation, axis permutation, segment splitting, self pairs).
"""
import json
import math
import os

import numpy as np
import pytest

import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ---- independent helpers (not the oracle's formulas) -----------------------

def pos(seg, t):
    """Point of a segment at time t, written as start + direction * fraction."""
    seg = np.asarray(seg, dtype=np.float64)
    frac = (t - seg[0]) / (seg[4] - seg[0])
    return seg[1:4] + (seg[5:8] - seg[1:4]) * frac


def dist(q, l, t):
    return float(np.linalg.norm(pos(l, t) - pos(q, t)))


def overlap(q, l):
    ts, te = max(q[0], l[0]), min(q[4], l[4])
    return (ts, te) if ts < te else None


def golden_min(q, l, ts, te, iters=200):
    """Minimum of the convex |Delta(t)| on [ts, te] by golden-section search."""
    g = (math.sqrt(5) - 1) / 2
    a, b = ts, te
    c, e = b - g * (b - a), a + g * (b - a)
    fc, fe = dist(q, l, c), dist(q, l, e)
    for _ in range(iters):
        if fc < fe:
            b, e, fe = e, c, fc
            c = b - g * (b - a)
            fc = dist(q, l, c)
        else:
            a, c, fc = c, e, fe
            e = a + g * (b - a)
            fe = dist(q, l, e)
    cands = [(dist(q, l, ts), ts), (dist(q, l, te), te), (fc, c), (fe, e)]
    return min(cands)


# ---- paper / hand-worked values -------------------------------------------

def test_golden_pairs(oracle_mod):
    spec = json.load(open(os.path.join(GOLDEN, "pairs.json")))
    assert len(spec["pairs"]) == 13
    for p in spec["pairs"]:
        got = oracle_mod.compare(p["q"], p["l"], p["d"])
        exp = p["expected"]
        if exp is None:
            assert got is None, p["id"]
        else:
            assert got is not None, p["id"]
            assert got[0] == pytest.approx(exp[0], abs=4e-16), p["id"]
            assert got[1] == pytest.approx(exp[1], abs=4e-16), p["id"]
        # swapping the roles of query and entry gives the same interval
        got2 = oracle_mod.compare(p["l"], p["q"], p["d"])
        assert got2 == got, p["id"]


def test_paper_example(oracle_mod):
    ex = json.load(open(os.path.join(GOLDEN, "paper_example.json")))
    res = oracle_mod.search(np.array(ex["D"]), np.array(ex["Q"]), ex["d"])
    got = [[int(r["query_id"]), int(r["entry_id"]), r["t_start"], r["t_end"]] for r in res]
    assert len(got) == len(ex["expected"])
    for g, e in zip(got, ex["expected"]):
        assert g[:2] == e[:2]
        assert g[2] == pytest.approx(e[2], abs=1e-15)
        assert g[3] == pytest.approx(e[3], abs=1e-15)


# ---- closed form and sampling ---------------------------------------------

def _random_pairs(seed, m, d_scale=0.2):
    g = synth.rng(seed)
    D, Q = synth.random_small(seed, m, m, side=0.5, tspan=1.0, maxdur=1.0, maxlen=0.4)
    return D, Q, g


def test_closed_form_roots(oracle_mod):
    """Interval = tau* +- sqrt(d^2 - dmin^2)/|V| (projection form), clipped."""
    D, Q, g = _random_pairs(11, 400)
    checked = 0
    for i in range(400):
        q, l = Q[i], D[i]
        ov = overlap(q, l)
        if ov is None:
            continue
        ts, te = ov
        A = pos(l, ts) - pos(q, ts)
        V = (pos(l, te) - pos(q, te)) - A
        nv = float(np.linalg.norm(V))
        if nv < 1e-6:
            continue
        tau_star = -float(A @ V) / nv ** 2
        closest = A + tau_star * V
        dperp = float(np.linalg.norm(closest))
        d = dperp + float(g.uniform(0.001, 0.3))
        half = math.sqrt(d * d - dperp * dperp) / nv
        lo, hi = max(tau_star - half, 0.0), min(tau_star + half, 1.0)
        got = oracle_mod.compare(q, l, d)
        if lo > hi:
            # the closest approach lies outside the overlap: no result unless an end is inside
            if got is not None:
                assert min(dist(q, l, ts), dist(q, l, te)) <= d * (1 + 1e-9)
            continue
        assert got is not None
        assert got[0] == pytest.approx(ts + lo * (te - ts), abs=1e-11)
        assert got[1] == pytest.approx(ts + hi * (te - ts), abs=1e-11)
        checked += 1
    assert checked > 50


def test_dense_sampling(oracle_mod):
    """Inside the returned interval |Delta| <= d, outside it |Delta| >= d."""
    D, Q, g = _random_pairs(12, 300)
    hits = 0
    for i in range(300):
        q, l = Q[i], D[i]
        ov = overlap(q, l)
        if ov is None:
            assert oracle_mod.compare(q, l, 0.3) is None
            continue
        ts, te = ov
        d = float(g.uniform(0.05, 0.5))
        got = oracle_mod.compare(q, l, d)
        tt = np.linspace(ts, te, 2001)
        dd = np.array([dist(q, l, t) for t in tt])
        if got is None:
            assert np.all(dd > d * (1 - 1e-9)), i
            continue
        hits += 1
        inside = (tt >= got[0]) & (tt <= got[1])
        assert np.all(dd[inside] <= d * (1 + 1e-9) + 1e-12), i
        assert np.all(dd[~inside] >= d * (1 - 1e-9) - 1e-12), i
    assert hits > 30


def test_bruteforce_independent_minimum(oracle_mod):
    """Whole search on tiny inputs vs an independent golden-section minimum of
    the distance per pair: membership outside a 1e-6 band, endpoints on |Delta|=d."""
    D, Q = synth.random_small(13, 40, 30, side=0.6, tspan=2.0, maxdur=1.0, maxlen=0.3)
    d = 0.12
    res = oracle_mod.search(D, Q, d)
    got = {(int(r["query_id"]), int(r["entry_id"])): (r["t_start"], r["t_end"]) for r in res}
    assert len(got) == len(res)
    n_in = 0
    for qi in range(Q.shape[0]):
        for li in range(D.shape[0]):
            q, l = Q[qi], D[li]
            ov = overlap(q, l)
            if ov is None:
                assert (qi, li) not in got
                continue
            dm, tm = golden_min(q, l, *ov)
            if dm < d * (1 - 1e-6):
                assert (qi, li) in got
                n_in += 1
                a, b = got[(qi, li)]
                assert a <= tm + 1e-9 and tm - 1e-9 <= b
                if a > ov[0]:
                    assert abs(dist(q, l, a) - d) <= 1e-8
                if b < ov[1]:
                    assert abs(dist(q, l, b) - d) <= 1e-8
            elif dm > d * (1 + 1e-6):
                assert (qi, li) not in got
    assert n_in > 20
    # canonical order, no duplicates (reading c7)
    keys = res["query_id"].astype(np.int64) * 2**32 + res["entry_id"]
    assert np.all(np.diff(keys) > 0)


def test_dmin_independent_minimum(oracle_mod):
    """The tie-band distance (oracle_dmin, reading c11) against an independent
    golden-section minimum of |Delta(t)| over the strict overlap, on >= 300
    random pairs (with overlap), plus NaN for pairs without overlap."""
    D, Q = synth.random_small(21, 700, 700, side=0.6, tspan=1.5, maxdur=1.0, maxlen=0.4)
    qids = np.arange(700)
    eids = (np.arange(700) * 7) % 700
    dm = oracle_mod.dmin_pairs(D, Q, qids, eids)
    checked = interior = 0
    for i in range(700):
        q, l = Q[qids[i]], D[eids[i]]
        ov = overlap(q, l)
        if ov is None:
            assert np.isnan(dm[i]), i
            continue
        ref, tm = golden_min(q, l, *ov)
        assert abs(dm[i] - ref) <= 1e-9 * max(1.0, ref), (i, dm[i], ref)
        checked += 1
        interior += ov[0] + 1e-6 < tm < ov[1] - 1e-6
    assert checked >= 300 and interior >= 50


def test_dmin_hand_worked(oracle_mod):
    """d_min of the hand-worked pairs (tests/golden/pairs.json): the closest
    approach over the common time span, worked out from the geometry."""
    spec = {p["id"]: p for p in json.load(open(os.path.join(GOLDEN, "pairs.json")))["pairs"]}
    want = {
        "P1": 0.05,        # parallel, 0.05 apart the whole time
        "P2": 0.2,         # parallel, 0.2 apart
        "P3": 0.0,         # crossing paths meet at t = 0.5
        "P4": 0.25,        # tangent: closest at t = 0.5, distance 0.25
        "P7": 0.0,         # head-on, meet at t = 0.5
        "P8": 0.0,         # q passes the stationary l at t = 0.2
        "P10": 0.0,        # same line, same place over [0.5, 1]
        "P12": 0.0,        # q reaches x = 0.95 at t = 0.95
        "P13": 0.0,        # 3-D: diff = (2 - 2t, 0, 0), zero at t = 1
    }
    for pid, exp in want.items():
        p = spec[pid]
        got = oracle_mod.dmin_pairs(np.array([p["l"]]), np.array([p["q"]]), [0], [0])[0]
        assert got == pytest.approx(exp, abs=1e-15), pid
    for pid in ("P5", "P6"):                       # no strict overlap
        p = spec[pid]
        assert np.isnan(oracle_mod.dmin_pairs(np.array([p["l"]]), np.array([p["q"]]), [0], [0])[0])
    # closest approach after the overlap ends (upper clamp) and before it starts
    q = [0.0, 0.0, 0.0, 0.0, 1.0, 1.0, 0.0, 0.0]
    l_after = [0.0, 3.0, 0.5, 0.0, 1.0, 2.5, 0.5, 0.0]     # gap 3 -> 1.5 in x, 0.5 in y
    assert oracle_mod.dmin_pairs(np.array([l_after]), np.array([q]), [0], [0])[0] == \
        pytest.approx(math.hypot(1.5, 0.5), abs=1e-15)
    l_before = [0.0, -1.0, 0.0, 0.25, 1.0, -1.5, 0.0, 0.25]  # moving away from the start
    assert oracle_mod.dmin_pairs(np.array([l_before]), np.array([q]), [0], [0])[0] == \
        pytest.approx(math.hypot(1.0, 0.25), abs=1e-15)


# ---- invariants ------------------------------------------------------------

def _as_dict(res):
    return {(int(r["query_id"]), int(r["entry_id"])): (float(r["t_start"]), float(r["t_end"]))
            for r in res}


def test_symmetry(oracle_mod):
    D, Q = synth.random_small(14, 60, 50)
    a = _as_dict(oracle_mod.search(D, Q, 0.15))
    b = _as_dict(oracle_mod.search(Q, D, 0.15))
    assert {(e, q) for (q, e) in b} == set(a)
    for (q, e), iv in a.items():
        assert b[(e, q)] == pytest.approx(iv, abs=1e-12)


def test_monotone_in_d(oracle_mod):
    D, Q = synth.random_small(15, 60, 50)
    prev = None
    for d in (0.0, 0.02, 0.05, 0.1, 0.2, 0.4):
        cur = _as_dict(oracle_mod.search(D, Q, d))
        if prev is not None:
            assert set(prev) <= set(cur)
            for k, (a, b) in prev.items():
                assert cur[k][0] <= a + 1e-12 and b - 1e-12 <= cur[k][1]
        prev = cur
    assert len(prev) > 50


def test_power_of_two_scaling_is_exact(oracle_mod):
    D, Q = synth.random_small(16, 60, 50)
    base = oracle_mod.search(D, Q, 0.15)
    D2, Q2 = D.copy(), Q.copy()
    for A in (D2, Q2):
        A[:, [1, 2, 3, 5, 6, 7]] *= 4.0
        A[:, [0, 4]] *= 2.0
    sc = oracle_mod.search(D2, Q2, 0.6)
    assert np.array_equal(base[["query_id", "entry_id"]], sc[["query_id", "entry_id"]])
    assert np.array_equal(base["t_start"] * 2.0, sc["t_start"])
    assert np.array_equal(base["t_end"] * 2.0, sc["t_end"])


def _compare_sets(oracle_mod, D, Q, d, a, b, tol=1e-9):
    """pair sets equal outside the tie band, intervals within tol."""
    da, db = _as_dict(a), _as_dict(b)
    for k in set(da) ^ set(db):
        dm = oracle_mod.dmin_pairs(D, Q, [k[0]], [k[1]])[0]
        assert abs(dm - d) <= 1e-9 * d, k
    for k in set(da) & set(db):
        assert da[k] == pytest.approx(db[k], abs=tol)


def test_translation_rotation_timeshift(oracle_mod):
    D, Q = synth.random_small(17, 60, 50)
    d = 0.15
    base = oracle_mod.search(D, Q, d)
    # translation
    D2, Q2 = D.copy(), Q.copy()
    for A in (D2, Q2):
        A[:, [1, 5]] += 0.375
        A[:, [2, 6]] -= 1.25
        A[:, [3, 7]] += 3.5
    _compare_sets(oracle_mod, D, Q, d, base, oracle_mod.search(D2, Q2, d))
    # rotation by 90 degrees about z: (x, y) -> (-y, x)
    D3, Q3 = D.copy(), Q.copy()
    for A, S in ((D3, D), (Q3, Q)):
        A[:, [1, 5]] = -S[:, [2, 6]]
        A[:, [2, 6]] = S[:, [1, 5]]
    _compare_sets(oracle_mod, D, Q, d, base, oracle_mod.search(D3, Q3, d))
    # common time shift
    D4, Q4 = D.copy(), Q.copy()
    for A in (D4, Q4):
        A[:, [0, 4]] += 10.0
    sh = oracle_mod.search(D4, Q4, d)
    sh["t_start"] -= 10.0
    sh["t_end"] -= 10.0
    _compare_sets(oracle_mod, D, Q, d, base, sh, tol=1e-12 * 100)


def test_segment_splitting(oracle_mod):
    """Splitting an entry at an interior time along its own line: the union of
    the two pieces' intervals equals the original interval."""
    D, Q = synth.random_small(18, 80, 1, side=0.4, tspan=1.0, maxdur=1.5, maxlen=0.3)
    q = Q[0]
    d = 0.2
    n_checked = 0
    for l in D:
        if l[4] - l[0] < 1e-3:
            continue
        tm = l[0] + 0.37 * (l[4] - l[0])
        pm = pos(l, tm)
        l1 = np.concatenate([[l[0]], l[1:4], [tm], pm])
        l2 = np.concatenate([[tm], pm, [l[4]], l[5:8]])
        whole = oracle_mod.compare(q, l, d)
        p1 = oracle_mod.compare(q, l1, d)
        p2 = oracle_mod.compare(q, l2, d)
        parts = [p for p in (p1, p2) if p is not None]
        if whole is None:
            assert not parts or all(min(dist(q, l, p[0]), dist(q, l, p[1])) >= d * (1 - 1e-9)
                                    for p in parts)
            continue
        assert parts
        lo = min(p[0] for p in parts)
        hi = max(p[1] for p in parts)
        assert lo == pytest.approx(whole[0], abs=1e-9)
        assert hi == pytest.approx(whole[1], abs=1e-9)
        if p1 is not None and p2 is not None:
            assert p1[1] == pytest.approx(p2[0], abs=1e-9)   # meet at the split
        n_checked += 1
    assert n_checked > 10


def test_self_pairs(oracle_mod):
    D, _ = synth.random_small(19, 40, 1)
    D = D[D[:, 4] > D[:, 0]]
    for d in (0.0, 0.1, 1.0):
        hit, ts, te = oracle_mod.compare_pairs(D, D, np.arange(len(D)), np.arange(len(D)), d)
        assert hit.all()
        assert np.array_equal(ts, D[:, 0]) and np.array_equal(te, D[:, 4])


def test_zero_duration_never_matches(oracle_mod):
    q = [0, 0, 0, 0, 1, 1, 0, 0]
    for t in (0.0, 0.5, 1.0):
        l = [t, t, 0, 0, t, t, 0, 0]
        assert oracle_mod.compare(q, l, 1.0) is None
        assert oracle_mod.compare(l, q, 1.0) is None


# ---- generator arithmetic (paper dataset sizes, P:L127-P:L141) -------------

def test_paper_dataset_sizes():
    assert synth.segment_count(2500, 400) == 997_500          # Random
    assert synth.segment_count(131_072, 193) == 25_165_824    # Merger
    assert synth.segment_count(65_536, 193) == 12_582_912     # Random-dense
    assert synth.segment_count(100, 400) == 39_900            # S1
    assert synth.segment_count(265, 193) == 50_880            # S2/S3
    assert round(65536 / 0.112) == 585_143                    # P:L131 cube volume 585142.86 pc^3


def test_config_shapes_small():
    c0 = synth.make_config("C0")
    assert c0.D.shape == (2000, 8) and c0.Q.shape == (200, 8)
    assert np.all(c0.D[:, 4] >= c0.D[:, 0])
    c1 = synth.make_config("C1", scale=0.02)
    n = c1.D.shape[0]
    assert n % 192 == 0 and c1.Q.shape[0] % 192 == 0
    c2 = synth.make_config("C2", scale=0.01)
    ntraj = c2.D.shape[0] // 192
    side = c2.D[:, [1, 2, 3]].max() - c2.D[:, [1, 2, 3]].min()
    assert ntraj / side ** 3 == pytest.approx(0.112, rel=0.1)   # P:L131 density


def test_paper_replica_shapes():
    """S1-S3 reproduce the paper's dataset and query sizes (P:L127-P:L141)."""
    s1 = synth.make_config("S1", scale=0.02)
    assert s1.D.shape[0] == synth.segment_count(50, 400)
    assert s1.Q.shape[0] == synth.segment_count(2, 400)
    s3 = synth.make_config("S3", scale=0.002)
    ntraj = s3.D.shape[0] // 192
    side = s3.D[:, [1, 2, 3, 5, 6, 7]].max() - s3.D[:, [1, 2, 3, 5, 6, 7]].min()
    assert ntraj / side ** 3 == pytest.approx(0.112, rel=0.15)      # P:L131 density
    # full sizes follow from the same formulas
    assert synth.segment_count(2500, 400) == 997_500
    assert synth.segment_count(2 * 65536, 193) == 25_165_824
    assert synth.segment_count(65536, 193) == 12_582_912


def test_merge_trajectory_pairs_hand_example(oracle_mod):
    """Union of closed intervals per trajectory pair (P:L15 application):
    touching pieces merge, gaps split, pairs stay separate."""
    dt = oracle_mod.RESULT_DTYPE
    res = np.array([(0, 0, 0.0, 1.0), (0, 1, 1.0, 2.0), (0, 2, 3.0, 4.0),
                    (1, 0, 0.5, 0.7), (0, 3, 1.5, 1.8), (2, 1, 5.0, 5.0)], dtype=dt)
    qtraj = [7, 7, 9]
    etraj = [1, 1, 1, 2]
    m = oracle_mod.merge_trajectory_pairs(res, qtraj, etraj)
    got = [(int(r["query_traj"]), int(r["entry_traj"]), r["t_start"], r["t_end"]) for r in m]
    assert got == [(7, 1, 0.0, 2.0), (7, 1, 3.0, 4.0), (7, 2, 1.5, 1.8), (9, 1, 5.0, 5.0)]
