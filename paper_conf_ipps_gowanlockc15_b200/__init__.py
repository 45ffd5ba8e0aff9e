"""Thin Python binding of libdts.so (include/dts.h): argument marshalling only.

Every step of the distance threshold search (§III) runs in the
library's sm_100a kernels; this module converts numpy arrays / torch tensors
to pointers and back.  There is no CPU fallback: if libdts.so is missing or
the device is not an sm_100 part, the calls raise.

Names follow the C ABI: build_index, build_index_device, search, search_ex,
search_device, free_results (implicit, by garbage collection), index info.
"""
from __future__ import annotations

import ctypes
import os
import weakref

import numpy as np

__all__ = ["RESULT_DTYPE", "IndexParams", "Index", "DeviceResults", "DTSError",
           "build_index", "build_index_device", "search", "search_ex", "search_device",
           "lib_path", "load", "EXPORTED_SYMBOLS"]

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.environ.get("DTS_LIB") or os.path.join(_HERE, "libdts.so")   # DTS_LIB: A/B builds

RESULT_DTYPE = np.dtype([("query_id", "<u4"), ("entry_id", "<u4"),
                         ("t_start", "<f8"), ("t_end", "<f8")], align=True)
assert RESULT_DTYPE.itemsize == 24

EXPORTED_SYMBOLS = (
    "dts_build_index", "dts_build_index_device", "dts_search", "dts_search_ex",
    "dts_search_device", "dts_free_results", "dts_free_results_device", "dts_free_index",
    "dts_index_get_info", "dts_last_error", "dts_version", "dts_kernel_launches",
    "dts_search_device_ex", "dts_canonicalize_device", "dts_merge_trajectories_device",
    "dts_query_costs_device", "dts_search_count", "dts_search_count_device",
    "dts_search_stream", "dts_search_read_times", "dts_query_costs_sampled_device",
)

_STATUS = {0: "DTS_OK", -1: "DTS_EINVAL", -2: "DTS_ENOMEM", -3: "DTS_ECUDA",
           -4: "DTS_ENOTSUP", -5: "DTS_EINTERNAL"}


class DTSError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


class IndexParams(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("temporal_bins", ctypes.c_uint32),
                ("cells_per_dim", ctypes.c_uint32), ("d_hint", ctypes.c_double),
                ("mem_budget_bytes", ctypes.c_uint64), ("method", ctypes.c_uint32),
                ("subbins", ctypes.c_uint32), ("entry_ids", ctypes.c_void_p),
                ("entry_traj", ctypes.c_void_p)]


class SearchOptions(ctypes.Structure):
    _fields_ = [("query_id_base", ctypes.c_uint32), ("query_ids", ctypes.c_void_p),
                ("query_traj", ctypes.c_void_p), ("exclude_same_trajectory", ctypes.c_uint32)]


METHODS = {"grid": 0, "temporal": 1, "subbin": 2}

# int callback(const dts_result* results, size_t count, void* user)
RESULT_CALLBACK = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t,
                                   ctypes.c_void_p)

TRAJ_DTYPE = np.dtype([("query_traj", "<u4"), ("entry_traj", "<u4"),
                       ("t_start", "<f8"), ("t_end", "<f8")], align=True)


class SearchStats(ctypes.Structure):
    _fields_ = [("candidates", ctypes.c_uint64), ("cell_lookups", ctypes.c_uint64),
                ("results", ctypes.c_uint64), ("max_results_per_query", ctypes.c_uint32),
                ("time_kernels", ctypes.c_uint32), ("ms_prep", ctypes.c_float),
                ("ms_count", ctypes.c_float), ("ms_scan", ctypes.c_float),
                ("ms_scatter", ctypes.c_float), ("ms_canon", ctypes.c_float),
                ("timer_slot", ctypes.c_uint32), ("tile_queries", ctypes.c_uint32),
                ("work_estimate", ctypes.c_float)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class IndexInfo(ctypes.Structure):
    _fields_ = [("n", ctypes.c_uint64), ("cells", ctypes.c_uint64), ("bins", ctypes.c_uint32),
                ("grid", ctypes.c_uint32 * 3), ("bin_width", ctypes.c_double),
                ("cell_width", ctypes.c_double * 3), ("max_extent", ctypes.c_double * 3),
                ("max_duration", ctypes.c_double), ("ms_build", ctypes.c_float),
                ("method", ctypes.c_uint32), ("subbins", ctypes.c_uint32 * 3),
                ("subbin_ids", ctypes.c_uint64 * 3), ("ms_phase", ctypes.c_float * 5),
                ("build_flags", ctypes.c_uint32), ("hash_kind", ctypes.c_uint32),
                ("hash_items", ctypes.c_uint64), ("hash_bytes", ctypes.c_uint64),
                ("shards", ctypes.c_uint32), ("outlier_rows", ctypes.c_uint64),
                ("outlier_copies", ctypes.c_uint64)]

    def as_dict(self):
        out = {}
        for k, _ in self._fields_:
            v = getattr(self, k)
            out[k] = list(v) if isinstance(v, ctypes.Array) else v
        return out


_lib = None


def lib_path() -> str:
    return _LIB_PATH


def load():
    """Load libdts.so (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise ImportError(f"{_LIB_PATH} not built; run __graft_entry__.build() "
                          "or python paper_conf_ipps_gowanlockc15_b200/build.py")
    lib = ctypes.CDLL(_LIB_PATH)
    P = ctypes.c_void_p
    S = ctypes.c_size_t
    pp = ctypes.POINTER(ctypes.c_void_p)
    ps = ctypes.POINTER(ctypes.c_size_t)
    lib.dts_build_index.argtypes = [P, S, ctypes.POINTER(IndexParams), pp]
    lib.dts_build_index_device.argtypes = [P, S, ctypes.POINTER(IndexParams), P, pp]
    lib.dts_search.argtypes = [P, P, S, ctypes.c_double, ctypes.c_uint32, P, pp, ps]
    lib.dts_search_ex.argtypes = [P, P, S, ctypes.c_double, ctypes.POINTER(SearchOptions), P,
                                  pp, ps, ctypes.POINTER(SearchStats)]
    lib.dts_search_device_ex.argtypes = [P, P, S, ctypes.c_double,
                                         ctypes.POINTER(SearchOptions), P, pp, ps,
                                         ctypes.POINTER(SearchStats)]
    lib.dts_merge_trajectories_device.argtypes = [P, S, P, S, P, S, P, pp, ps]
    lib.dts_merge_trajectories_device.restype = ctypes.c_int
    lib.dts_search_device_ex.restype = ctypes.c_int
    lib.dts_search_count.argtypes = [P, P, S, ctypes.c_double, ctypes.POINTER(SearchOptions), P,
                                     P, ctypes.POINTER(ctypes.c_uint64),
                                     ctypes.POINTER(SearchStats)]
    lib.dts_search_count.restype = ctypes.c_int
    lib.dts_search_count_device.argtypes = [P, P, S, ctypes.c_double,
                                            ctypes.POINTER(SearchOptions), P, P,
                                            ctypes.POINTER(ctypes.c_uint64),
                                            ctypes.POINTER(SearchStats)]
    lib.dts_search_count_device.restype = ctypes.c_int
    lib.dts_search_stream.argtypes = [P, P, S, ctypes.c_double, ctypes.POINTER(SearchOptions),
                                      ctypes.c_uint64, RESULT_CALLBACK, P, P,
                                      ctypes.POINTER(SearchStats)]
    lib.dts_search_stream.restype = ctypes.c_int
    lib.dts_query_costs_device.argtypes = [P, P, S, ctypes.c_double, ctypes.c_uint32, P, P]
    lib.dts_query_costs_sampled_device.argtypes = [P, P, S, ctypes.c_double, ctypes.c_uint32,
                                                   ctypes.c_uint32, P, P]
    lib.dts_query_costs_sampled_device.restype = ctypes.c_int
    lib.dts_query_costs_device.restype = ctypes.c_int
    lib.dts_search_read_times.argtypes = [ctypes.POINTER(SearchStats)]
    lib.dts_search_read_times.restype = ctypes.c_int
    lib.dts_canonicalize_device.argtypes = [P, S, P]
    lib.dts_canonicalize_device.restype = ctypes.c_int
    lib.dts_search_device.argtypes = [P, P, S, ctypes.c_double, ctypes.c_uint32, P, pp, ps,
                                      ctypes.POINTER(SearchStats)]
    for f in ("dts_build_index", "dts_build_index_device", "dts_search", "dts_search_ex",
              "dts_search_device", "dts_index_get_info"):
        getattr(lib, f).restype = ctypes.c_int
    lib.dts_index_get_info.argtypes = [P, ctypes.POINTER(IndexInfo)]
    lib.dts_free_results.argtypes = [P]
    lib.dts_free_results.restype = None
    lib.dts_free_results_device.argtypes = [P]
    lib.dts_free_results_device.restype = None
    lib.dts_free_index.argtypes = [P]
    lib.dts_free_index.restype = None
    lib.dts_last_error.restype = ctypes.c_char_p
    lib.dts_version.restype = ctypes.c_char_p
    lib.dts_kernel_launches.restype = ctypes.c_uint64
    lib.dts_kernel_launches.argtypes = []
    _lib = lib
    return lib


def _check(rc: int):
    if rc != 0:
        raise DTSError(rc, _lib.dts_last_error().decode())


def _segments(a) -> np.ndarray:
    a = np.ascontiguousarray(np.asarray(a, dtype=np.float64))
    if a.size == 0:
        return a.reshape(0, 8)
    if a.ndim != 2 or a.shape[1] != 8:
        raise ValueError("segments must have shape (n, 8)")
    return a


def _params(device=0, temporal_bins=0, cells_per_dim=0, d_hint=0.0, method="grid",
            subbins=0, entry_ids_ptr=None, entry_traj_ptr=None,
            mem_budget_bytes=0) -> IndexParams:
    m = METHODS[method] if isinstance(method, str) else int(method)
    return IndexParams(int(device), int(temporal_bins), int(cells_per_dim), float(d_hint),
                       int(mem_budget_bytes), m, int(subbins), entry_ids_ptr, entry_traj_ptr)


def _u32_host(a, n, what):
    if a is None:
        return None
    a = np.ascontiguousarray(a, dtype=np.uint32)
    if a.shape[0] != n:
        raise ValueError(f"{what} must have {n} entries")
    return a


def _dev_ptr(t):
    if t is None:
        return None
    return t.data_ptr() if hasattr(t, "data_ptr") else int(t)


def _stream_ptr(stream) -> int:
    if stream is None:
        return 0
    if hasattr(stream, "cuda_stream"):
        return int(stream.cuda_stream)
    return int(stream)


class Index:
    """Owns a dts_index*; freed with dts_free_index."""

    def __init__(self, handle: int, device: int):
        self._h = ctypes.c_void_p(handle)
        self.device = device

    @property
    def handle(self):
        return self._h

    def info(self) -> dict:
        inf = IndexInfo()
        _check(load().dts_index_get_info(self._h, ctypes.byref(inf)))
        return inf.as_dict()

    def free(self):
        if self._h and self._h.value:
            load().dts_free_index(self._h)
            self._h = ctypes.c_void_p(0)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class DeviceResults:
    """Results in library-owned device memory (dts_free_results_device on
    release).  Exposes __cuda_array_interface__ as a flat uint8 buffer."""

    def __init__(self, ptr: int, count: int, device: int, dtype=RESULT_DTYPE):
        self.ptr = ptr
        self.count = count
        self.device = device
        self.dtype = dtype

    @property
    def __cuda_array_interface__(self):
        return {"shape": (self.count * self.dtype.itemsize,), "typestr": "|u1",
                "data": (self.ptr or 0, False), "version": 3}

    def tensor(self):
        import torch
        if self.count == 0:
            return torch.empty(0, dtype=torch.uint8, device=f"cuda:{self.device}")
        return torch.as_tensor(self, device=f"cuda:{self.device}")

    def numpy(self) -> np.ndarray:
        if self.count == 0:
            return np.empty(0, dtype=self.dtype)
        return self.tensor().cpu().numpy().view(self.dtype)

    def free(self):
        if self.ptr:
            load().dts_free_results_device(ctypes.c_void_p(self.ptr))
            self.ptr = 0
            self.count = 0

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def build_index(D, device: int = 0, temporal_bins: int = 0, cells_per_dim: int = 0,
                d_hint: float = 0.0, method="grid", subbins: int = 0,
                entry_ids=None, entry_traj=None, mem_budget_bytes: int = 0) -> Index:
    """dts_build_index: D is host (n, 8) float64 (copied); entry_ids /
    entry_traj: optional host uint32 reported ids / trajectory ids per row;
    mem_budget_bytes: device budget (over it: temporal shards on the host)."""
    lib = load()
    D = _segments(D)
    ids = _u32_host(entry_ids, D.shape[0], "entry_ids")
    traj = _u32_host(entry_traj, D.shape[0], "entry_traj")
    p = _params(device, temporal_bins, cells_per_dim, d_hint, method, subbins,
                ids.ctypes.data if ids is not None else None,
                traj.ctypes.data if traj is not None else None, mem_budget_bytes)
    h = ctypes.c_void_p()
    _check(lib.dts_build_index(D.ctypes.data if D.size else None, D.shape[0], ctypes.byref(p),
                               ctypes.byref(h)))
    return Index(h.value, device)


def build_index_device(D_dev, n: int = None, device: int = 0, temporal_bins: int = 0,
                       cells_per_dim: int = 0, d_hint: float = 0.0, stream=None,
                       method="grid", subbins: int = 0, entry_ids=None,
                       entry_traj=None) -> Index:
    """dts_build_index_device: D_dev is a CUDA tensor (n, 8) float64;
    entry_ids / entry_traj: optional CUDA int32/uint32 tensors."""
    lib = load()
    ptr = D_dev.data_ptr() if hasattr(D_dev, "data_ptr") else int(D_dev)
    if n is None:
        n = D_dev.shape[0]
    p = _params(device, temporal_bins, cells_per_dim, d_hint, method, subbins,
                _dev_ptr(entry_ids), _dev_ptr(entry_traj))
    h = ctypes.c_void_p()
    _check(lib.dts_build_index_device(ctypes.c_void_p(ptr), n, ctypes.byref(p),
                                      ctypes.c_void_p(_stream_ptr(stream)), ctypes.byref(h)))
    return Index(h.value, device)


def _free_results(ptr: int) -> None:
    load().dts_free_results(ctypes.c_void_p(ptr))


def _host_results(ptr, count) -> np.ndarray:
    """The library's pinned result array as a numpy array, without a copy
    (copying 0.8 GB of results into fresh pageable memory took longer than
    the search): dts_free_results runs when the array and every view of it
    are gone."""
    if count == 0:
        if ptr:
            _free_results(ptr)
        return np.empty(0, dtype=RESULT_DTYPE)
    buf = (ctypes.c_char * (count * RESULT_DTYPE.itemsize)).from_address(ptr)
    weakref.finalize(buf, _free_results, ptr)
    return np.frombuffer(buf, dtype=RESULT_DTYPE, count=count)


def search_ex(index: Index, Q, d: float, query_id_base: int = 0, stream=None,
              time_kernels: bool = False, query_ids=None, query_traj=None,
              exclude_same_trajectory: bool = False):
    """dts_search_ex: host Q (+ optional host uint32 query_ids / query_traj)
    -> (results structured array, stats dict)."""
    lib = load()
    Q = _segments(Q)
    qids = _u32_host(query_ids, Q.shape[0], "query_ids")
    qtraj = _u32_host(query_traj, Q.shape[0], "query_traj")
    opts = SearchOptions(int(query_id_base), qids.ctypes.data if qids is not None else None,
                         qtraj.ctypes.data if qtraj is not None else None,
                         1 if exclude_same_trajectory else 0)
    out = ctypes.c_void_p()
    cnt = ctypes.c_size_t()
    st = SearchStats()
    st.time_kernels = _timing_mode(time_kernels)
    _check(lib.dts_search_ex(index.handle, Q.ctypes.data if Q.size else None, Q.shape[0],
                             float(d), ctypes.byref(opts), ctypes.c_void_p(_stream_ptr(stream)),
                             ctypes.byref(out), ctypes.byref(cnt), ctypes.byref(st)))
    return _host_results(out.value, cnt.value), st.as_dict()


def search(index: Index, Q, d: float, query_id_base: int = 0, stream=None) -> np.ndarray:
    """dts_search: host Q -> results sorted by (query_id, entry_id)."""
    lib = load()
    Q = _segments(Q)
    out = ctypes.c_void_p()
    cnt = ctypes.c_size_t()
    _check(lib.dts_search(index.handle, Q.ctypes.data if Q.size else None, Q.shape[0], float(d),
                          int(query_id_base), ctypes.c_void_p(_stream_ptr(stream)),
                          ctypes.byref(out), ctypes.byref(cnt)))
    return _host_results(out.value, cnt.value)


def _timing_mode(time_kernels) -> int:
    """time_kernels: False/0 off, True/1 phase times read before the call
    returns, "defer"/2 recorded only (read later by read_times), "pass1"/3
    as "defer" for pass 1's two events only."""
    if time_kernels == "defer":
        return 2
    if time_kernels == "pass1":
        return 3
    return int(time_kernels) if time_kernels in (0, 1, 2, 3) else (1 if time_kernels else 0)


def read_times(stats: dict) -> dict:
    """dts_search_read_times: the phase times of a search made with
    time_kernels="defer" (same thread), as a new stats dict."""
    st = SearchStats(**{k: stats[k] for k, _ in SearchStats._fields_})
    _check(load().dts_search_read_times(ctypes.byref(st)))
    return st.as_dict()


def search_device(index: Index, Q_dev, d: float, query_id_base: int = 0, stream=None,
                  n: int = None, time_kernels: bool = False, query_ids=None, query_traj=None,
                  exclude_same_trajectory: bool = False):
    """dts_search_device (dts_search_device_ex when query_ids, a CUDA int32 /
    uint32 tensor of increasing reported ids, is given): Q_dev CUDA tensor
    (nq, 8) float64 -> (DeviceResults, stats)."""
    lib = load()
    ptr = Q_dev.data_ptr() if hasattr(Q_dev, "data_ptr") else int(Q_dev)
    if n is None:
        n = Q_dev.shape[0]
    out = ctypes.c_void_p()
    cnt = ctypes.c_size_t()
    st = SearchStats()
    st.time_kernels = _timing_mode(time_kernels)
    if query_ids is None and query_traj is None and not exclude_same_trajectory:
        _check(lib.dts_search_device(index.handle, ctypes.c_void_p(ptr), n, float(d),
                                     int(query_id_base), ctypes.c_void_p(_stream_ptr(stream)),
                                     ctypes.byref(out), ctypes.byref(cnt), ctypes.byref(st)))
    else:
        opts = SearchOptions(int(query_id_base), _dev_ptr(query_ids), _dev_ptr(query_traj),
                             1 if exclude_same_trajectory else 0)
        _check(lib.dts_search_device_ex(index.handle, ctypes.c_void_p(ptr), n, float(d),
                                        ctypes.byref(opts),
                                        ctypes.c_void_p(_stream_ptr(stream)),
                                        ctypes.byref(out), ctypes.byref(cnt), ctypes.byref(st)))
    return DeviceResults(out.value or 0, cnt.value, index.device), st.as_dict()


def _options(query_id_base=0, query_ids=None, query_traj=None, exclude_same_trajectory=False):
    return SearchOptions(int(query_id_base), query_ids, query_traj,
                         1 if exclude_same_trajectory else 0)


def search_count(index: Index, Q, d: float, query_traj=None,
                 exclude_same_trajectory: bool = False, stream=None, time_kernels=False):
    """dts_search_count: host Q -> (total, per-query counts uint32 array, stats)."""
    lib = load()
    Q = _segments(Q)
    qtraj = _u32_host(query_traj, Q.shape[0], "query_traj")
    opts = _options(0, None, qtraj.ctypes.data if qtraj is not None else None,
                    exclude_same_trajectory)
    counts = np.empty(Q.shape[0], dtype=np.uint32)
    total = ctypes.c_uint64()
    st = SearchStats()
    st.time_kernels = _timing_mode(time_kernels)
    _check(lib.dts_search_count(index.handle, Q.ctypes.data if Q.size else None, Q.shape[0],
                                float(d), ctypes.byref(opts),
                                ctypes.c_void_p(_stream_ptr(stream)),
                                counts.ctypes.data if Q.size else None, ctypes.byref(total),
                                ctypes.byref(st)))
    return int(total.value), counts, st.as_dict()


def search_count_device(index: Index, Q_dev, d: float, counts_out=None, stream=None,
                        time_kernels=False):
    """dts_search_count_device: CUDA Q -> (total, CUDA int32 counts tensor, stats)."""
    import torch
    lib = load()
    nq = int(Q_dev.shape[0])
    if counts_out is None:
        counts_out = torch.empty(nq, dtype=torch.int32, device=Q_dev.device)
    total = ctypes.c_uint64()
    st = SearchStats()
    st.time_kernels = _timing_mode(time_kernels)
    opts = _options()
    _check(lib.dts_search_count_device(index.handle, ctypes.c_void_p(Q_dev.data_ptr() if nq else 0),
                                       nq, float(d), ctypes.byref(opts),
                                       ctypes.c_void_p(_stream_ptr(stream)),
                                       ctypes.c_void_p(counts_out.data_ptr() if nq else 0),
                                       ctypes.byref(total), ctypes.byref(st)))
    return int(total.value), counts_out, st.as_dict()


def search_stream(index: Index, Q, d: float, callback, chunk_results: int = 0,
                  query_id_base: int = 0, query_ids=None, query_traj=None,
                  exclude_same_trajectory: bool = False, stream=None):
    """dts_search_stream: host Q; `callback(chunk)` receives each chunk of
    results in canonical order as a numpy structured view of library memory,
    valid only during the call (copy what must outlive it); returning True
    stops the search.  Returns the stats dict."""
    lib = load()
    Q = _segments(Q)
    qids = _u32_host(query_ids, Q.shape[0], "query_ids")
    qtraj = _u32_host(query_traj, Q.shape[0], "query_traj")
    opts = _options(query_id_base, qids.ctypes.data if qids is not None else None,
                    qtraj.ctypes.data if qtraj is not None else None, exclude_same_trajectory)
    errors = []

    def trampoline(ptr, count, _user):
        try:
            buf = (ctypes.c_char * (count * RESULT_DTYPE.itemsize)).from_address(ptr)
            stop = callback(np.frombuffer(buf, dtype=RESULT_DTYPE, count=count))
            return 1 if stop else 0
        except BaseException as e:          # surfaced after the call
            errors.append(e)
            return 1

    cb = RESULT_CALLBACK(trampoline)
    st = SearchStats()
    rc = lib.dts_search_stream(index.handle, Q.ctypes.data if Q.size else None, Q.shape[0],
                               float(d), ctypes.byref(opts), int(chunk_results), cb, None,
                               ctypes.c_void_p(_stream_ptr(stream)), ctypes.byref(st))
    if errors:
        raise errors[0]
    _check(rc)
    return st.as_dict()


def query_costs_device(index: Index, Q_dev, d: float, block: int = 1, stream=None, out=None,
                       stride: int = 1):
    """dts_query_costs_device (dts_query_costs_sampled_device when stride >
    1): Q_dev CUDA tensor (nq, 8) float64 -> CUDA int64 tensor of
    ceil(nq / block) candidate counts (sum over each block of `block`
    consecutive queries of the pairs the search would refine; estimated from
    every stride-th query)."""
    import torch
    lib = load()
    nq = int(Q_dev.shape[0])
    nb = (nq + int(block) - 1) // int(block)
    if out is None:
        out = torch.empty(nb, dtype=torch.int64, device=Q_dev.device)
    qp = ctypes.c_void_p(Q_dev.data_ptr() if nq else 0)
    op = ctypes.c_void_p(out.data_ptr() if nb else 0)
    sp = ctypes.c_void_p(_stream_ptr(stream))
    if int(stride) == 1:
        _check(lib.dts_query_costs_device(index.handle, qp, nq, float(d), int(block), sp, op))
    else:
        _check(lib.dts_query_costs_sampled_device(index.handle, qp, nq, float(d), int(block),
                                                  int(stride), sp, op))
    return out


def merge_trajectories_device(results, query_traj, entry_traj, stream=None):
    """dts_merge_trajectories_device: DeviceResults (or a CUDA uint8 tensor of
    24-byte records) + CUDA uint32/int32 tensors of trajectory ids indexed by
    reported query id / entry id -> DeviceResults-like buffer of 24-byte
    dts_traj_result records (numpy(TRAJ_DTYPE))."""
    lib = load()
    if isinstance(results, DeviceResults):
        rptr, n, dev = results.ptr, results.count, results.device
    else:
        rptr, n, dev = results.data_ptr(), results.numel() // RESULT_DTYPE.itemsize, \
            results.device.index or 0
    out = ctypes.c_void_p()
    cnt = ctypes.c_size_t()
    _check(lib.dts_merge_trajectories_device(ctypes.c_void_p(rptr or 0), int(n),
                                             ctypes.c_void_p(_dev_ptr(query_traj)),
                                             int(query_traj.numel()),
                                             ctypes.c_void_p(_dev_ptr(entry_traj)),
                                             int(entry_traj.numel()),
                                             ctypes.c_void_p(_stream_ptr(stream)),
                                             ctypes.byref(out), ctypes.byref(cnt)))
    return DeviceResults(out.value or 0, cnt.value, dev, dtype=TRAJ_DTYPE)


def canonicalize_device(results_dev, n: int = None, stream=None) -> None:
    """dts_canonicalize_device: sort results in device memory (a CUDA uint8
    tensor of n * 24 bytes, or a DeviceResults) by (query_id, entry_id)."""
    lib = load()
    if isinstance(results_dev, DeviceResults):
        ptr, n = results_dev.ptr, results_dev.count
    else:
        ptr = results_dev.data_ptr()
        if n is None:
            n = results_dev.numel() // RESULT_DTYPE.itemsize
    _check(lib.dts_canonicalize_device(ctypes.c_void_p(ptr or 0), int(n),
                                       ctypes.c_void_p(_stream_ptr(stream))))


def kernel_launches() -> int:
    return int(load().dts_kernel_launches())


def version() -> str:
    return load().dts_version().decode()
