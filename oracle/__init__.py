"""ctypes front of oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` legs may import this package.  The product path
(paper_conf_ipps_gowanlockc15_b200) never imports it.

The C code is the plain brute-force definition of the distance threshold
search (§III, compare() of Alg. 1 l.14 P:L64); see the header
of oracle.c for the step-by-step reading and tests/test_oracle.py for the pins.
The thread pool below is only a harness: each thread runs the single-threaded
C search on a disjoint, contiguous query range, and the outputs are
concatenated in range order, which is the (query, entry) canonical order.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from concurrent.futures import ThreadPoolExecutor

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

RESULT_DTYPE = np.dtype([("query_id", "<u4"), ("entry_id", "<u4"),
                         ("t_start", "<f8"), ("t_end", "<f8")], align=True)
assert RESULT_DTYPE.itemsize == 24


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc -O2 -ffp-contract=off, single-threaded C)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math",
                               "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        lib.oracle_search.argtypes = [P, ctypes.c_uint64, P, ctypes.c_uint64, ctypes.c_uint64,
                                      ctypes.c_double, ctypes.POINTER(P),
                                      ctypes.POINTER(ctypes.c_uint64)]
        lib.oracle_search.restype = ctypes.c_int
        lib.oracle_dmin_pairs.argtypes = [P, P, P, P, ctypes.c_uint64, P]
        lib.oracle_dmin_pairs.restype = None
        lib.oracle_compare_pairs.argtypes = [P, P, P, P, ctypes.c_uint64, ctypes.c_double,
                                             P, P, P]
        lib.oracle_compare_pairs.restype = None
        lib.oracle_free.argtypes = [P]
        lib.oracle_free.restype = None
        _lib = lib
    return _lib


def _seg(a) -> np.ndarray:
    a = np.ascontiguousarray(np.asarray(a, dtype=np.float64))
    if a.ndim != 2 or a.shape[1] != 8:
        a = a.reshape(-1, 8)
    return a


def _search_range(D, Q, q0, q1, d) -> np.ndarray:
    lib = _load()
    out = ctypes.c_void_p()
    cnt = ctypes.c_uint64()
    rc = lib.oracle_search(D.ctypes.data, D.shape[0], Q.ctypes.data, q0, q1, float(d),
                           ctypes.byref(out), ctypes.byref(cnt))
    if rc != 0:
        raise MemoryError("oracle_search: allocation failed")
    try:
        n = cnt.value
        res = np.empty(n, dtype=RESULT_DTYPE)
        if n:
            ctypes.memmove(res.ctypes.data, out.value, n * RESULT_DTYPE.itemsize)
    finally:
        lib.oracle_free(out)
    return res


def search(D, Q, d: float, q_range=None, threads: int = 1) -> np.ndarray:
    """All (query_id, entry_id, t_start, t_end) with the pair within d
    (P:L32), sorted by (query_id, entry_id).  q_range = (q0, q1) restricts the
    queries (ids stay global)."""
    D = _seg(D)
    Q = _seg(Q)
    q0, q1 = (0, Q.shape[0]) if q_range is None else (int(q_range[0]), int(q_range[1]))
    if threads <= 1 or q1 - q0 < 2:
        return _search_range(D, Q, q0, q1, d)
    bounds = np.linspace(q0, q1, threads + 1).astype(np.int64)
    with ThreadPoolExecutor(threads) as ex:
        parts = list(ex.map(lambda i: _search_range(D, Q, int(bounds[i]), int(bounds[i + 1]), d),
                            range(threads)))
    return np.concatenate(parts)


def search_queries(D, Q, qids, d: float, threads: int = 1) -> np.ndarray:
    """Brute force for an arbitrary subset of query ids (sampled parity at full
    size): each query is searched against all of D."""
    D = _seg(D)
    Q = _seg(Q)
    qids = np.asarray(qids, dtype=np.int64)

    def one(q):
        return _search_range(D, Q, int(q), int(q) + 1, d)

    if threads <= 1:
        parts = [one(q) for q in qids]
    else:
        with ThreadPoolExecutor(threads) as ex:
            parts = list(ex.map(one, qids))
    return np.concatenate(parts) if parts else np.empty(0, dtype=RESULT_DTYPE)


def dmin_pairs(D, Q, qids, eids) -> np.ndarray:
    """Minimum distance over the strict temporal overlap of each pair (NaN if
    none) -- the tie-band quantity of reading c11."""
    lib = _load()
    D = _seg(D)
    Q = _seg(Q)
    qids = np.ascontiguousarray(qids, dtype=np.uint32)
    eids = np.ascontiguousarray(eids, dtype=np.uint32)
    out = np.empty(qids.shape[0], dtype=np.float64)
    lib.oracle_dmin_pairs(D.ctypes.data, Q.ctypes.data, qids.ctypes.data, eids.ctypes.data,
                          qids.shape[0], out.ctypes.data)
    return out


def compare_pairs(D, Q, qids, eids, d: float):
    """compare() on explicit pairs: (hit bool array, t_start, t_end)."""
    lib = _load()
    D = _seg(D)
    Q = _seg(Q)
    qids = np.ascontiguousarray(qids, dtype=np.uint32)
    eids = np.ascontiguousarray(eids, dtype=np.uint32)
    m = qids.shape[0]
    hit = np.empty(m, dtype=np.int32)
    ts = np.empty(m, dtype=np.float64)
    te = np.empty(m, dtype=np.float64)
    lib.oracle_compare_pairs(D.ctypes.data, Q.ctypes.data, qids.ctypes.data, eids.ctypes.data,
                             m, float(d), hit.ctypes.data, ts.ctypes.data, te.ctypes.data)
    return hit.astype(bool), ts, te


def compare(q, l, d: float):
    """compare() of one query segment q and one entry segment l (8-vectors)."""
    hit, ts, te = compare_pairs(np.asarray(l, dtype=np.float64).reshape(1, 8),
                                np.asarray(q, dtype=np.float64).reshape(1, 8),
                                [0], [0], d)
    return (float(ts[0]), float(te[0])) if hit[0] else None


def merge_trajectory_pairs(res, query_traj, entry_traj) -> np.ndarray:
    """Trajectory-level results (the application of P:L15): map each
    segment-level result (q, l, [ts, te]) to (query_traj[q], entry_traj[l])
    and replace the intervals of each pair by the maximal connected pieces of
    their union (closed intervals: touching ones merge).  Plain loops; sorted
    by (query_traj, entry_traj, t_start)."""
    qt = np.asarray(query_traj, dtype=np.int64)[res["query_id"].astype(np.int64)]
    et = np.asarray(entry_traj, dtype=np.int64)[res["entry_id"].astype(np.int64)]
    groups = {}
    for a, b, s, e in zip(qt.tolist(), et.tolist(), res["t_start"].tolist(),
                          res["t_end"].tolist()):
        groups.setdefault((a, b), []).append((s, e))
    out = []
    for (a, b) in sorted(groups):
        iv = sorted(groups[(a, b)])
        lo, hi = iv[0]
        for s, e in iv[1:]:
            if s <= hi:
                hi = max(hi, e)
            else:
                out.append((a, b, lo, hi))
                lo, hi = s, e
        out.append((a, b, lo, hi))
    dt = np.dtype([("query_traj", "<u4"), ("entry_traj", "<u4"), ("t_start", "<f8"),
                   ("t_end", "<f8")], align=True)
    return np.array(out, dtype=dt)
