"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module generates *inputs only*: trajectories sampled as in the paper's
datasets (Gowanlock & Casanova, §V-A) and turned into
4-D line segments (§III: a segment joins two consecutive spatiotemporal
samples of one trajectory).  It holds none of the search method's arithmetic
(no overlap test, no distance, no index), so the oracle (`oracle/`) and the
CUDA path (`paper_conf_ipps_gowanlockc15_b200/`) can both consume it without
sharing any code of the method.

Segment layout (float64, one row per segment, the order of `dts_segment` in
include/dts.h):  t_start, x_start, y_start, z_start, t_end, x_end, y_end, z_end.
Ids are row positions; trajectory-major, time-minor order, so the id of the
k-th segment of trajectory j is j * (samples - 1) + k.

The recipes (sizes, distributions, seeds) are stated in DESIGN.md §"Input
recipe" and SURVEY.md §8(d).
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

__all__ = [
    "SEG_COLS", "segment_count", "rng", "random_walks", "galaxy",
    "segments_from_trajectories", "Config", "make_config", "CONFIG_NAMES",
    "adversarial", "random_small",
]

SEG_COLS = ("t_start", "x_start", "y_start", "z_start",
            "t_end", "x_end", "y_end", "z_end")


def segment_count(trajectories: int, samples: int) -> int:
    """Segments produced by `trajectories` trajectories of `samples` samples.

    The paper counts e.g. 2,500 trajectories x 400 timesteps = 997,500 entry
    segments, i.e. one segment between consecutive timesteps."""
    return trajectories * (samples - 1)


def rng(seed: int) -> np.random.Generator:
    """Counter-based generator (Philox4x32-10) so streams are reproducible."""
    return np.random.Generator(np.random.Philox(key=seed))


def segments_from_trajectories(t: np.ndarray, pos: np.ndarray) -> np.ndarray:
    """t: (ntraj, nsamp) sample times; pos: (ntraj, nsamp, 3) positions.
    Returns (ntraj*(nsamp-1), 8) float64 segments, trajectory-major."""
    ntraj, nsamp = t.shape
    seg = np.empty((ntraj, nsamp - 1, 8), dtype=np.float64)
    seg[:, :, 0] = t[:, :-1]
    seg[:, :, 1:4] = pos[:, :-1, :]
    seg[:, :, 4] = t[:, 1:]
    seg[:, :, 5:8] = pos[:, 1:, :]
    return seg.reshape(-1, 8)


def _reflect(x: np.ndarray, lo: float, hi: float) -> np.ndarray:
    x = np.where(x < lo, 2 * lo - x, x)
    x = np.where(x > hi, 2 * hi - x, x)
    return np.clip(x, lo, hi)


def random_walks(g: np.random.Generator, ntraj: int, nsamp: int, side: float,
                 sigma: float, t0_max: float, dt: float = 1.0):
    """Random-walk trajectories as for the paper's Random / Random-dense sets
    (P:L127): start position U[0,side]^3, i.i.d. N(0, sigma^2) steps
    per axis reflected at the walls, start time U[0, t0_max], dt per sample."""
    pos = np.empty((ntraj, nsamp, 3), dtype=np.float64)
    pos[:, 0, :] = g.uniform(0.0, side, size=(ntraj, 3))
    steps = g.normal(0.0, sigma, size=(ntraj, nsamp - 1, 3))
    for k in range(1, nsamp):
        pos[:, k, :] = _reflect(pos[:, k - 1, :] + steps[:, k - 1, :], 0.0, side)
    t0 = g.uniform(0.0, t0_max, size=ntraj)
    t = t0[:, None] + dt * np.arange(nsamp, dtype=np.float64)[None, :]
    return t, pos


def galaxy(g: np.random.Generator, n1: int, n2: int, nsamp: int):
    """Two-disk galaxy-merger-shaped trajectories (the Merger dataset's shape,
    P:L129: particles of two galactic disks sampled at synchronised timesteps).

    Per particle: R0 ~ Gamma(2, 1) (exponential disk), floored at 0.05;
    z0 = 0.1 atanh(2u-1) (sech^2 profile); flat rotation with 0.05 rad/step at
    R = 1 (angular rate 0.05/R0); epicyclic radial and vertical oscillations of
    amplitude U(0, 0.05 R0) at rates sqrt(2) w and 2 w.  Disk 1 is centred at the
    origin; disk 2 starts at (12, 4, 0), is tilted 60 degrees about x, and its
    centre drifts by (-0.06, -0.02, 0) per step.  Samples at t = 0, 1, ...
    """
    P = n1 + n2
    R0 = np.maximum(g.gamma(2.0, 1.0, size=P), 0.05)
    phi0 = g.uniform(0.0, 2 * math.pi, size=P)
    u = g.uniform(1e-6, 1 - 1e-6, size=P)
    z0 = 0.1 * np.arctanh(2 * u - 1)
    aR = g.uniform(0.0, 0.05, size=P) * R0
    az = g.uniform(0.0, 0.05, size=P) * R0
    psiR = g.uniform(0.0, 2 * math.pi, size=P)
    psiz = g.uniform(0.0, 2 * math.pi, size=P)
    omega = 0.05 / R0
    tilt = math.radians(60.0)
    ct, st = math.cos(tilt), math.sin(tilt)
    pos = np.empty((P, nsamp, 3), dtype=np.float64)
    for k in range(nsamp):
        R = R0 + aR * np.sin(math.sqrt(2.0) * omega * k + psiR)
        th = phi0 + omega * k
        x = R * np.cos(th)
        y = R * np.sin(th)
        z = z0 + az * np.sin(2.0 * omega * k + psiz)
        # disk 1: static, untilted
        pos[:n1, k, 0] = x[:n1]
        pos[:n1, k, 1] = y[:n1]
        pos[:n1, k, 2] = z[:n1]
        # disk 2: tilted about x, drifting centre
        cx, cy = 12.0 - 0.06 * k, 4.0 - 0.02 * k
        pos[n1:, k, 0] = cx + x[n1:]
        pos[n1:, k, 1] = cy + ct * y[n1:] - st * z[n1:]
        pos[n1:, k, 2] = st * y[n1:] + ct * z[n1:]
    t = np.broadcast_to(np.arange(nsamp, dtype=np.float64), (P, nsamp)).copy()
    return t, pos


@dataclasses.dataclass
class Config:
    name: str
    D: np.ndarray          # (n, 8) float64 entry segments
    Q: np.ndarray          # (nq, 8) float64 query segments
    d: float               # headline distance
    d_sweep: tuple         # other distances used by tests / sweeps
    note: str
    etraj: np.ndarray = None   # trajectory id of each entry segment
    qtraj: np.ndarray = None   # trajectory id of each query segment


CONFIG_NAMES = ("C0", "C1", "C2", "C3", "C4")


def _sample_query_trajectories(D: np.ndarray, ntraj: int, nseg: int,
                               nq_traj: int, seed: int) -> np.ndarray:
    return _sample_with_ids(D, ntraj, nseg, nq_traj, seed)[0]


def _sample_with_ids(D: np.ndarray, ntraj: int, nseg: int, nq_traj: int, seed: int):
    g = rng(seed)
    chosen = np.sort(g.choice(ntraj, size=nq_traj, replace=False))
    Q = np.ascontiguousarray(D.reshape(ntraj, nseg, 8)[chosen].reshape(-1, 8))
    return Q, np.repeat(chosen, nseg).astype(np.uint32)


def _traj_ids(ntraj: int, nseg: int) -> np.ndarray:
    return np.repeat(np.arange(ntraj, dtype=np.uint32), nseg)


def make_config(name: str, rank: int = 0, scale: float = 1.0) -> Config:
    """Build one of the five BASELINE.json configs.

    rank: for weak scaling each rank draws its own query set (query seed
    data_seed + 1000 + rank) against the same entry set D.
    scale: < 1 shrinks the particle/trajectory counts (tests only)."""
    if name == "C0":
        g = rng(1)
        t, pos = random_walks(g, 20, 101, 1.0, 0.02, 100.0)
        D = segments_from_trajectories(t, pos)
        gq = rng(1001 + rank)
        off = np.full(3, 0.03 / math.sqrt(3.0))
        t1 = t[0:1] + 0.37
        p1 = pos[0:1] + off
        t2, p2 = random_walks(gq, 1, 101, 1.0, 0.02, 100.0)
        Q = np.concatenate([segments_from_trajectories(t1, p1),
                            segments_from_trajectories(t2, p2)])
        return Config(name, D, Q, 0.05, (0.0, 0.01, 0.05, 0.2),
                      "tiny random walks (P:L127 shape), unit cube", _traj_ids(20, 100),
                      np.repeat(np.array([1000, 1001], dtype=np.uint32), 100))
    if name in ("C1", "C4"):
        if name == "C1":
            n1, n2, nq_traj, seed = 2731, 2730, 52, 2
        else:
            n1, n2, nq_traj, seed = 52429, 52429, 5209, 5
        n1 = max(1, int(n1 * scale)); n2 = max(1, int(n2 * scale))
        nq_traj = max(1, int(nq_traj * scale))
        t, pos = galaxy(rng(seed), n1, n2, 193)
        D = segments_from_trajectories(t, pos)
        del t, pos
        Q, qt = _sample_with_ids(D, n1 + n2, 192, nq_traj, seed + 1000 + rank)
        return Config(name, D, Q, 0.005, (0.001, 0.005, 0.02),
                      "two-disk galaxy merger shape (P:L129), 193 synchronised samples",
                      _traj_ids(n1 + n2, 192), qt)
    if name == "C2":
        ntraj, nq_traj = max(2, int(21846 * scale)), max(1, int(521 * scale))
        side = (ntraj / 0.112) ** (1.0 / 3.0)   # density 0.112 pc^-3
        t, pos = random_walks(rng(3), ntraj, 193, side, 0.05, 100.0)
        D = segments_from_trajectories(t, pos)
        del t, pos
        Q, qt = _sample_with_ids(D, ntraj, 192, nq_traj, 3 + 1000 + rank)
        return Config(name, D, Q, 0.09, (0.03, 0.09, 0.5, 2.0, 8.0),
                      "uniform dense random walks at 0.112 pc^-3 (P:L131)",
                      _traj_ids(ntraj, 192), qt)
    if name == "C3":
        ntraj, nq_traj = max(2, int(10000 * scale)), max(1, int(250 * scale))
        t, pos = random_walks(rng(4), ntraj, 400, 1000.0, 1.0, 10000.0)
        D = segments_from_trajectories(t, pos)
        tq, pq = random_walks(rng(4 + 1000 + rank), nq_traj, 400, 1000.0, 1.0, 10000.0)
        Q = segments_from_trajectories(tq, pq)
        return Config(name, D, Q, 5.0, (1.0, 5.0, 20.0, 50.0),
                      "sparse long-span random walks (P:L127 shape stretched)",
                      _traj_ids(ntraj, 399), _traj_ids(nq_traj, 399) + np.uint32(ntraj))
    # ---- paper-replica scenarios; sizes exactly as P:L127-P:L141
    if name == "S1":
        # Random: 2,500 random-walk trajectories x 400 timesteps = 997,500
        # segments, start times U[0,100]; query: 100 trajectories x
        # 400 timesteps = 39,900 segments.  The paper gives no spatial
        # scale; the walk is C3's ([0,1000]^3, N(0,1) steps).
        ntraj, nq_traj = max(2, int(2500 * scale)), max(1, int(100 * scale))
        t, pos = random_walks(rng(11), ntraj, 400, 1000.0, 1.0, 100.0)
        D = segments_from_trajectories(t, pos)
        tq, pq = random_walks(rng(11 + 1000 + rank), nq_traj, 400, 1000.0, 1.0, 100.0)
        Q = segments_from_trajectories(tq, pq)
        return Config(name, D, Q, 50.0, (1.0, 5.0, 20.0, 50.0, 100.0),
                      "paper S1: Random (P:L127, P:L139)")
    if name == "S2":
        # Merger shape: 131,072 particles x 193 timesteps = 25,165,824
        # segments; query: 265 trajectories x 193 timesteps = 50,880
        # segments, drawn from D.
        n1 = max(1, int(65536 * scale))
        nq_traj = max(1, int(265 * scale))
        t, pos = galaxy(rng(12), n1, n1, 193)
        D = segments_from_trajectories(t, pos)
        del t, pos
        Q = _sample_query_trajectories(D, 2 * n1, 192, nq_traj, 12 + 1000 + rank)
        return Config(name, D, Q, 0.001, (0.001, 0.01, 0.1, 1.0, 5.0),
                      "paper S2: Merger-shaped (P:L129, P:L140)")
    if name == "S3":
        # Random-dense: 65,536 particles x 193 timesteps = 12,582,912 segments
        # at 0.112 stars/pc^3, i.e. a 585,142 pc^3 cube; query: 265
        # trajectories x 193 timesteps = 50,880 segments, from D.
        ntraj, nq_traj = max(2, int(65536 * scale)), max(1, int(265 * scale))
        side = (ntraj / 0.112) ** (1.0 / 3.0)
        t, pos = random_walks(rng(13), ntraj, 193, side, 0.05, 100.0)
        D = segments_from_trajectories(t, pos)
        del t, pos
        Q = _sample_query_trajectories(D, ntraj, 192, nq_traj, 13 + 1000 + rank)
        return Config(name, D, Q, 0.05, (0.01, 0.02, 0.03, 0.05, 0.09),
                      "paper S3: Random-dense (P:L131, P:L141)")
    raise ValueError(f"unknown config {name!r}")


def random_small(seed: int, n: int, nq: int, side: float = 1.0,
                 tspan: float = 4.0, maxdur: float = 1.0, maxlen: float = 0.3):
    """Independent random segments (tiny parity / pin cases)."""
    g = rng(seed)

    def seg(k):
        t0 = g.uniform(0.0, tspan, size=k)
        t1 = t0 + g.uniform(0.0, maxdur, size=k)
        p0 = g.uniform(0.0, side, size=(k, 3))
        p1 = p0 + g.uniform(-maxlen, maxlen, size=(k, 3))
        return np.column_stack([t0, p0, t1, p1])

    return seg(n), seg(nq)


def adversarial(seed: int, n: int = 50, nq: int = 50):
    """Degenerate geometry mixed into random segments: parallel, coincident,
    stationary, zero-duration, shared timesteps (integer times), coordinates on
    round cell-boundary values, and touching-in-time neighbours."""
    g = rng(seed)
    D, Q = random_small(seed + 77, n, nq)
    kinds = g.integers(0, 7, size=n)
    for i in range(n):
        k = kinds[i]
        j = int(g.integers(0, nq))
        if k == 0:      # coincident with a query
            D[i] = Q[j]
        elif k == 1:    # parallel copy offset in space
            D[i] = Q[j]
            D[i, [1, 2, 3, 5, 6, 7]] += np.repeat(g.uniform(-0.1, 0.1, size=(1, 3)), 2, axis=0).ravel()
        elif k == 2:    # stationary
            D[i, 5:8] = D[i, 1:4]
        elif k == 3:    # zero duration
            D[i, 4] = D[i, 0]
        elif k == 4:    # shared integer timesteps
            t0 = float(g.integers(0, 4))
            D[i, 0], D[i, 4] = t0, t0 + 1.0
            Q[j, 0], Q[j, 4] = t0, t0 + 1.0
        elif k == 5:    # round coordinates (cell-boundary-like values)
            D[i, 1:4] = np.round(D[i, 1:4] * 8) / 8
            D[i, 5:8] = np.round(D[i, 5:8] * 8) / 8
        else:           # touching a query in time only
            D[i, 0] = Q[j, 4]
            D[i, 4] = D[i, 0] + 0.5
    return np.ascontiguousarray(D), np.ascontiguousarray(Q)


def crowded(seed: int, big: int = 70000, clusters: int = 120, per_cluster: int = 50,
            background: int = 3000, nq: int = 12):
    """Crowded grid cells: `big` short segments inside one tiny box (one
    8-cell hash block holding more than 65,535 entries), `clusters` boxes of
    `per_cluster` segments (blocks longer than a warp), and `background`
    short random segments in [0,1]^3, all over times in [0, 1]; queries cross
    the big box, the clusters and empty space."""
    g = rng(seed)

    def box(n, c, r):
        s = np.empty((n, 8))
        s[:, 0] = g.uniform(0.0, 0.4, n)
        s[:, 4] = s[:, 0] + g.uniform(0.2, 0.6, n)
        s[:, 1:4] = c + g.uniform(-r, r, (n, 3))
        s[:, 5:8] = c + g.uniform(-r, r, (n, 3))
        return s

    parts = [box(big, np.array([0.5, 0.5, 0.5]), 1e-4)]
    for c in g.uniform(0.05, 0.95, (clusters, 3)):
        parts.append(box(per_cluster, c, 2e-4))
    bg = box(background, np.zeros(3), 0.0)
    bg[:, 1:4] = g.uniform(0.0, 1.0, (background, 3))
    bg[:, 5:8] = bg[:, 1:4] + g.uniform(-0.01, 0.01, (background, 3))
    parts.append(bg)
    D = np.concatenate(parts)
    D = D[g.permutation(D.shape[0])]
    Q = np.empty((nq, 8))
    Q[:, 0] = g.uniform(0.0, 0.3, nq)
    Q[:, 4] = Q[:, 0] + 0.5
    a = np.concatenate([np.full((nq // 3, 3), 0.5), g.uniform(0.05, 0.95, (nq - nq // 3, 3))])
    Q[:, 1:4] = a - 0.003
    Q[:, 5:8] = a + 0.003
    return np.ascontiguousarray(D), np.ascontiguousarray(Q)
