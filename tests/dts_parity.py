"""Parity rule (BASELINE.json north_star; readings c11, c10):

* the result pair set must equal the oracle's, except pairs whose minimum
  distance (computed by the oracle's routine, pinned in tests/test_oracle.py)
  lies within 1e-9*d of d -- exactly the north star's band for every d > 0.
  At d = 0 that band is empty; there, and only there, the band is the fp64
  rounding floor 1e-12*L of a distance computed from coordinates of magnitude
  L = max |coordinate| (reading c11: a pair that touches at one instant is a
  rounding decision of either implementation);
* interval endpoints of common pairs agree within 1e-9 in normalised time
  t^ = (t - t_min(D)) / (t_max(D) - t_min(D));
* results are in canonical (query_id, entry_id) order with no duplicates.
"""
import numpy as np

BAND = 1e-9
FLOOR = 1e-12
TOL_T = 1e-9


SUMMARY = []          # one dict per compare() call (written by conftest at session end)


def band(D, Q, d):
    if d > 0:
        return BAND * d
    Dv = np.asarray(D).reshape(-1, 8)[:, [1, 2, 3, 5, 6, 7]]
    Qv = np.asarray(Q).reshape(-1, 8)[:, [1, 2, 3, 5, 6, 7]]
    L = max(float(np.abs(Dv).max()) if Dv.size else 0.0,
            float(np.abs(Qv).max()) if Qv.size else 0.0)
    return FLOOR * L


def keys(res) -> np.ndarray:
    return res["query_id"].astype(np.uint64) << np.uint64(32) | res["entry_id"].astype(np.uint64)


def assert_canonical(res):
    k = keys(res)
    if k.size > 1:
        assert np.all(k[1:] > k[:-1]), "results not strictly sorted by (query_id, entry_id)"
    assert np.all(res["t_start"] <= res["t_end"]), "t_start > t_end"


def compare(gpu, ora, D, Q, d, oracle_mod, qid_base=0, tol_t=TOL_T):
    """Returns a dict of counts; raises AssertionError on a parity violation."""
    assert_canonical(gpu)
    assert_canonical(ora)
    kg, ko = keys(gpu), keys(ora)
    only_g = np.setdiff1d(kg, ko, assume_unique=True)
    only_o = np.setdiff1d(ko, kg, assume_unique=True)
    diff = np.concatenate([only_g, only_o])
    if diff.size:
        qids = (diff >> np.uint64(32)).astype(np.int64) - qid_base
        eids = (diff & np.uint64(0xffffffff)).astype(np.int64)
        dm = oracle_mod.dmin_pairs(D, Q, qids, eids)
        bad = ~(np.abs(dm - d) <= band(D, Q, d))
        if np.any(bad):
            i = int(np.flatnonzero(bad)[0])
            raise AssertionError(
                f"pair (q={qids[i]}, e={eids[i]}) differs outside the tie band: dmin={dm[i]!r}, "
                f"d={d!r}; only_gpu={only_g.size} only_oracle={only_o.size}")
    common, ig, io = np.intersect1d(kg, ko, assume_unique=True, return_indices=True)
    if common.size:
        Dv = np.asarray(D).reshape(-1, 8)
        span = float(Dv[:, 4].max() - Dv[:, 0].min()) or 1.0
        e0 = np.abs(gpu["t_start"][ig] - ora["t_start"][io]) / span
        e1 = np.abs(gpu["t_end"][ig] - ora["t_end"][io]) / span
        worst = float(max(e0.max(), e1.max()))
        assert worst <= tol_t, f"endpoint error {worst} in normalised time > {tol_t}"
    else:
        worst = 0.0
    info = {"gpu": int(kg.size), "oracle": int(ko.size), "common": int(common.size),
            "band_only_gpu": int(only_g.size), "band_only_oracle": int(only_o.size),
            "worst_endpoint": worst, "d": float(d), "band": float(band(D, Q, d))}
    SUMMARY.append(info)
    return info


def restrict(res, qids):
    return res[np.isin(res["query_id"], np.asarray(qids, dtype=np.uint32))]
