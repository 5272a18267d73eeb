"""B200-native ALGAS: small-batch graph ANN search on sm_100a.

Thin Python binding over the C-ABI in ``include/algas.h`` (``libalgas.so``,
built in-tree by ``build.py``).  This module only marshals arguments: every
step of the search runs in the library's CUDA kernels.  There is no CPU
fallback -- if the extension is missing or CUDA is unavailable, calls raise.

Arrays may be numpy arrays (host) or torch tensors (host or CUDA); the
library detects device pointers itself.
"""
from __future__ import annotations

import ctypes
import os
import threading

import numpy as np

from .build import LIB as _LIB_PATH, build as _build, built_hash as _built_hash, source_hash as _source_hash

SENTINEL = 0xFFFFFFFF
L2 = 0
IP = 1
COSINE = 2  # -(q.x)/(|q||x|): IP on unit rows (include/algas.h, R29)
VISITED_PRIVATE = 0
VISITED_SHARED = 1

OK, EINVAL, ENOMEM, ECUDA, EAGAIN, ESTATE, ENCCL, EOVERFLOW = 0, -1, -2, -3, -4, -5, -6, -7

__all__ = ["Index", "Server", "Params", "QueryStats", "RunInfo", "lib", "knn", "prune", "build_graph",
           "merge_topk", "merge_topk_parts", "knn_partitioned", "build_graph_partitioned", "knn_refine", "tune", "device_props", "AlgasError", "SENTINEL", "L2", "IP", "COSINE"]


class AlgasError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"algas error {code}: {msg}")
        self.code = code


class Params(ctypes.Structure):
    _fields_ = [("k", ctypes.c_int32), ("itopk", ctypes.c_int32), ("width", ctypes.c_int32),
                ("offset_beam", ctypes.c_int32), ("ctas_per_query", ctypes.c_int32),
                ("threads_per_cta", ctypes.c_int32), ("n_seeds", ctypes.c_int32),
                ("max_iter", ctypes.c_int32), ("visited_mode", ctypes.c_int32), ("slots", ctypes.c_int32),
                ("hash_bits", ctypes.c_int32), ("stage_rows", ctypes.c_int32),
                ("cluster_size", ctypes.c_int32), ("host_threads", ctypes.c_int32),
                ("state_mirror", ctypes.c_int32), ("watchdog_ms", ctypes.c_int32), ("seed", ctypes.c_uint64)]


class QueryStats(ctypes.Structure):
    _fields_ = [("iters", ctypes.c_uint32), ("max_iters", ctypes.c_uint32), ("parents", ctypes.c_uint32),
                ("dist_evals", ctypes.c_uint32), ("cap_hits", ctypes.c_uint32), ("spills", ctypes.c_uint32),
                ("overflows", ctypes.c_uint32), ("ctas", ctypes.c_uint32), ("t_start_ns", ctypes.c_uint64),
                ("t_end_ns", ctypes.c_uint64), ("latency_ns", ctypes.c_uint64), ("cyc_select", ctypes.c_uint64),
                ("cyc_gather", ctypes.c_uint64), ("cyc_dist", ctypes.c_uint64), ("cyc_sort", ctypes.c_uint64),
                ("t_loop_first_ns", ctypes.c_uint64), ("t_loop_last_ns", ctypes.c_uint64),
                ("t_loop_end_ns", ctypes.c_uint64), ("t_entry_last_ns", ctypes.c_uint64),
                ("queue_ns", ctypes.c_uint64), ("merges_bitonic", ctypes.c_uint32),
                ("merges_rank", ctypes.c_uint32)]


STATS_DTYPE = np.dtype([("iters", np.uint32), ("max_iters", np.uint32), ("parents", np.uint32),
                        ("dist_evals", np.uint32), ("cap_hits", np.uint32), ("spills", np.uint32),
                        ("overflows", np.uint32), ("ctas", np.uint32), ("t_start_ns", np.uint64),
                        ("t_end_ns", np.uint64), ("latency_ns", np.uint64), ("cyc_select", np.uint64),
                        ("cyc_gather", np.uint64), ("cyc_dist", np.uint64), ("cyc_sort", np.uint64),
                        ("t_loop_first_ns", np.uint64), ("t_loop_last_ns", np.uint64), ("t_loop_end_ns", np.uint64),
                        ("t_entry_last_ns", np.uint64), ("queue_ns", np.uint64), ("merges_bitonic", np.uint32),
                        ("merges_rank", np.uint32)])
assert STATS_DTYPE.itemsize == ctypes.sizeof(QueryStats)


class RunInfo(ctypes.Structure):
    _fields_ = [("kernel_ms", ctypes.c_float), ("grid", ctypes.c_int32), ("threads_per_cta", ctypes.c_int32),
                ("ctas_per_query", ctypes.c_int32), ("smem_per_cta", ctypes.c_int32),
                ("blocks_per_sm", ctypes.c_int32), ("hash_bits", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("call_ms", ctypes.c_float), ("merge_ms", ctypes.c_float)]


class DeviceProps(ctypes.Structure):
    _fields_ = [("n_sm", ctypes.c_int32), ("max_blocks_per_sm", ctypes.c_int32), ("smem_per_sm", ctypes.c_int64),
                ("smem_reserved_per_block", ctypes.c_int64), ("smem_per_block_optin", ctypes.c_int64),
                ("max_threads_per_sm", ctypes.c_int32), ("regs_per_sm", ctypes.c_int32)]


class Tuning(ctypes.Structure):
    _fields_ = [("ctas_per_query", ctypes.c_int32), ("blocks_per_sm", ctypes.c_int32),
                ("smem_avail_per_block", ctypes.c_int64), ("smem_per_block", ctypes.c_int64),
                ("threads_per_cta", ctypes.c_int32), ("width", ctypes.c_int32), ("offset_beam", ctypes.c_int32),
                ("hash_bits", ctypes.c_int32), ("stage_rows", ctypes.c_int32), ("visited_mode", ctypes.c_int32)]


# every symbol include/algas.h declares (checked by tests/test_abi.py)
EXPORTS = ["algas_params_default", "algas_last_error", "algas_version", "algas_index_create",
           "algas_index_destroy", "algas_index_info", "algas_search", "algas_search_ex", "algas_search_dynamic",
           "algas_server_create", "algas_server_create_deferred", "algas_server_create_emulated",
           "algas_server_emulated_stall", "algas_server_start", "algas_submit", "algas_submit_many", "algas_enqueue", "algas_poll", "algas_server_inflight", "algas_server_destroy",
           "algas_merge_topk", "algas_merge_topk_parts", "algas_device_query", "algas_tuner_max_parallel", "algas_tuner_blocks_per_sm",
           "algas_tuner_smem_per_block", "algas_tune", "algas_knn", "algas_knn_last_stats", "algas_prune",
           "algas_build_graph", "algas_knn_partitioned", "algas_build_graph_partitioned", "algas_knn_refine"]

_lock = threading.Lock()
_lib = None


def lib(build_if_missing: bool = True):
    """Load libalgas.so, (re)building it first if it is missing or stale --
    stale = its recorded source hash differs from the current sources' (a
    stale library never loads silently: without build_if_missing it raises)."""
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        stale = not os.path.exists(_LIB_PATH) or _built_hash() != _source_hash()
        if stale and build_if_missing:
            _build()
            stale = not os.path.exists(_LIB_PATH) or _built_hash() != _source_hash()
        if not os.path.exists(_LIB_PATH):
            raise AlgasError(ECUDA, f"CUDA extension {_LIB_PATH} is missing (run build.py)")
        if stale:
            raise AlgasError(ECUDA, f"CUDA extension {_LIB_PATH} is stale (sources changed; run build.py)")
        L = ctypes.CDLL(_LIB_PATH)
        P, i32, i64, u32, u64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32, ctypes.c_uint64
        L.algas_params_default.argtypes = [ctypes.POINTER(Params)]
        L.algas_params_default.restype = None
        L.algas_last_error.restype = ctypes.c_char_p
        L.algas_version.restype = ctypes.c_char_p
        L.algas_index_create.argtypes = [P, i64, i32, i32, P, i32]
        L.algas_index_create.restype = P
        L.algas_index_destroy.argtypes = [P]
        L.algas_index_info.argtypes = [P, P, P, P, P, P, P, P]
        L.algas_search.argtypes = [P, P, i64, i32, i32, i32, P, P]
        L.algas_search_ex.argtypes = [P, P, i64, ctypes.POINTER(Params), u64, P, P, P, P, P, P,
                                      ctypes.POINTER(RunInfo)]
        L.algas_search_dynamic.argtypes = [P, P, i64, ctypes.POINTER(Params), u64, P, P, P, P,
                                           ctypes.POINTER(RunInfo)]
        L.algas_server_create.argtypes = [P, ctypes.POINTER(Params), ctypes.POINTER(P)]
        L.algas_server_create_deferred.argtypes = [P, ctypes.POINTER(Params), ctypes.POINTER(P)]
        L.algas_server_create_emulated.argtypes = [ctypes.POINTER(Params), i32, i32, ctypes.POINTER(P)]
        L.algas_server_emulated_stall.argtypes = [P, u64]
        L.algas_server_start.argtypes = [P, i32]
        L.algas_submit.argtypes = [P, P, u64, i32, i32, i32]
        L.algas_submit_many.argtypes = [P, P, i64, u64, i32, i32, i32, ctypes.POINTER(i64)]
        L.algas_enqueue.argtypes = [P, P, i64, u64, i32, i32, i32]
        L.algas_poll.argtypes = [P, P, P, P, P, i32, ctypes.POINTER(i32)]
        L.algas_server_inflight.argtypes = [P, ctypes.POINTER(i64)]
        L.algas_server_destroy.argtypes = [P]
        L.algas_merge_topk.argtypes = [P, P, i32, i32, P, P]
        L.algas_merge_topk.restype = i32
        L.algas_merge_topk_parts.argtypes = [P, P, i32, i64, i32, i32, P, P]
        L.algas_device_query.argtypes = [ctypes.POINTER(DeviceProps)]
        L.algas_tuner_max_parallel.argtypes = [i32, i32, i32]
        L.algas_tuner_max_parallel.restype = i32
        L.algas_tuner_blocks_per_sm.argtypes = [i32, i32, i32]
        L.algas_tuner_blocks_per_sm.restype = i32
        L.algas_tuner_smem_per_block.argtypes = [i64, i32, i64]
        L.algas_tuner_smem_per_block.restype = i64
        L.algas_tune.argtypes = [ctypes.POINTER(DeviceProps), i32, i32, i32, i32, i32, ctypes.POINTER(Tuning)]
        L.algas_knn.argtypes = [P, i64, P, i64, i32, i32, i32, i64, P, P]
        L.algas_knn_last_stats.argtypes = [ctypes.POINTER(i64)]
        L.algas_knn_last_stats.restype = i64
        L.algas_prune.argtypes = [P, i64, i32, i32, P]
        L.algas_build_graph.argtypes = [P, i64, i32, i32, i32, i32, i32, P]
        L.algas_knn_partitioned.argtypes = [P, i64, i32, i32, i32, i32, i32, P, P]
        L.algas_build_graph_partitioned.argtypes = [P, i64, i32, i32, i32, i32, i32, i32, i32, i32, i32, P]
        L.algas_knn_refine.argtypes = [P, i64, i32, i32, i32, i32, i32, P, P]
        _lib = L
        return L


def _check(rc: int, allow=()):
    if rc != OK and rc not in allow:
        raise AlgasError(rc, lib().algas_last_error().decode())
    return rc


def _ptr(a):
    """(pointer, keepalive) for a numpy array or torch tensor (host or CUDA)."""
    if a is None:
        return None, None
    if isinstance(a, np.ndarray):
        if not a.flags["C_CONTIGUOUS"]:
            raise ValueError("array must be C-contiguous")
        return ctypes.c_void_p(a.ctypes.data), a
    # torch tensor (imported lazily: torch is plumbing only)
    if not a.is_contiguous():
        raise ValueError("tensor must be contiguous")
    return ctypes.c_void_p(a.data_ptr()), a


def _is_torch(a):
    return type(a).__module__.startswith("torch")


def _alloc_like(ref, shape, np_dtype, torch_dtype_name):
    if ref is not None and _is_torch(ref):
        import torch
        return torch.empty(shape, dtype=getattr(torch, torch_dtype_name), device=ref.device)
    return np.empty(shape, np_dtype)


def _stream_ptr(stream):
    if stream is None:
        return None
    if isinstance(stream, int):
        return ctypes.c_void_p(stream)
    return ctypes.c_void_p(stream.cuda_stream)


def default_params(**kw) -> Params:
    p = Params()
    lib().algas_params_default(ctypes.byref(p))
    for k, v in kw.items():
        if not hasattr(p, k):
            raise KeyError(k)
        setattr(p, k, int(v))
    return p


class Index:
    """Graph index in HBM.  data: n x dim float32; graph: n x degree uint32 or None (build)."""

    def __init__(self, data, graph=None, metric: int = L2, degree: int | None = None):
        L = lib()
        n, dim = int(data.shape[0]), int(data.shape[1])
        if graph is not None:
            degree = int(graph.shape[1])
        if degree is None:
            raise ValueError("degree is required when graph is None")
        dp, _k1 = _ptr(data)
        gp, _k2 = _ptr(graph)
        h = L.algas_index_create(dp, n, dim, metric, gp, degree)
        if not h:
            raise AlgasError(EINVAL, L.algas_last_error().decode())
        self._h = ctypes.c_void_p(h)
        self.n, self.dim, self.metric, self.degree = n, dim, metric, degree

    def close(self):
        if getattr(self, "_h", None):
            lib().algas_index_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def handle(self):
        return self._h

    def search(self, queries, k=10, itopk=64, width=1, params: Params | None = None, tag0: int = 0,
               want_cta: bool = False, want_stats: bool = True, stream=None, out=None):
        """Static batch search (algas_search_ex).  Returns dict(ids, dists, stats, info[, cta_ids, cta_dists])."""
        p = params if params is not None else default_params(k=k, itopk=itopk, width=width)
        nq = int(queries.shape[0])
        kk = p.k
        if out is None:
            ids = _alloc_like(queries, (nq, kk), np.uint32, "int32")
            ds = _alloc_like(queries, (nq, kk), np.float32, "float32")
        else:
            ids, ds = out
        T = p.ctas_per_query if p.ctas_per_query > 0 else None
        cti = ctd = None
        if want_cta:
            if T is None:
                raise ValueError("want_cta needs an explicit ctas_per_query")
            cti = np.empty((nq, T, kk), np.uint32)
            ctd = np.empty((nq, T, kk), np.float32)
        st = np.zeros(nq, STATS_DTYPE) if want_stats else None
        info = RunInfo()
        qp, _a = _ptr(queries)
        ip, _b = _ptr(ids)
        dp, _c = _ptr(ds)
        cip, _d = _ptr(cti)
        cdp, _e = _ptr(ctd)
        sp, _f = _ptr(st)
        rc = lib().algas_search_ex(self._h, qp, nq, ctypes.byref(p), tag0, ip, dp, cip, cdp, sp,
                                   _stream_ptr(stream), ctypes.byref(info))
        _check(rc, allow=(EOVERFLOW,))
        r = dict(ids=ids, dists=ds, stats=st, info=info, overflow=(rc == EOVERFLOW))
        if want_cta:
            r["cta_ids"], r["cta_dists"] = cti, ctd
        return r

    def search_dynamic(self, queries_dev, params: Params, tag0: int = 0, stream=None, out=None):
        """Dynamic batching from an HBM query queue (algas_search_dynamic)."""
        nq = int(queries_dev.shape[0])
        kk = params.k
        if out is None:
            ids = np.empty((nq, kk), np.uint32)
            ds = np.empty((nq, kk), np.float32)
        else:
            ids, ds = out
        st = np.zeros(nq, STATS_DTYPE)
        info = RunInfo()
        qp, _a = _ptr(queries_dev)
        ip, _b = _ptr(ids)
        dp, _c = _ptr(ds)
        sp, _d = _ptr(st)
        rc = lib().algas_search_dynamic(self._h, qp, nq, ctypes.byref(params), tag0, ip, dp, sp,
                                        _stream_ptr(stream), ctypes.byref(info))
        _check(rc, allow=(EOVERFLOW,))
        return dict(ids=ids, dists=ds, stats=st, info=info, overflow=(rc == EOVERFLOW))


class Server:
    """Persistent kernel + host-mapped slot ring (algas_server_*)."""

    def __init__(self, index: Index, params: Params, deferred: bool = False, emulated_dim: int = 0):
        """deferred=True: algas_server_create_deferred -- stage queries with
        submit(), then start() launches the kernel.  emulated_dim > 0:
        algas_server_create_emulated -- a TEST HARNESS whose device side is a
        host thread following the ring protocol (no GPU; results are a fixed
        function of the query, not a search); index must be None."""
        self.index = index
        self.params = params
        h = ctypes.c_void_p()
        if emulated_dim > 0:
            assert index is None, "an emulated server has no index"
            _check(lib().algas_server_create_emulated(ctypes.byref(params), int(emulated_dim), 1 if deferred else 0,
                                                      ctypes.byref(h)))
        else:
            create = lib().algas_server_create_deferred if deferred else lib().algas_server_create
            _check(create(index.handle, ctypes.byref(params), ctypes.byref(h)))
        self._h = h
        self.kmax = params.k

    def emulated_stall(self, tag: int) -> None:
        """Emulated server: never finish the query with this tag."""
        _check(lib().algas_server_emulated_stall(self._h, ctypes.c_uint64(tag)))

    def start(self, quit_when_idle: bool = False) -> None:
        """Launch a deferred server's kernel (algas_server_start); with
        quit_when_idle the kernel exits after the staged queries."""
        _check(lib().algas_server_start(self._h, 1 if quit_when_idle else 0))

    def submit(self, query: np.ndarray, tag: int, k: int = 0, itopk: int = 0, width: int = 0) -> bool:
        """True if accepted, False if every slot is busy (EAGAIN)."""
        qp, _a = _ptr(query)
        rc = lib().algas_submit(self._h, qp, tag, k, itopk, width)
        _check(rc, allow=(EAGAIN,))
        return rc == OK

    def submit_many(self, queries: np.ndarray, tag0: int, k: int = 0, itopk: int = 0, width: int = 0) -> int:
        """Submit rows of a contiguous HOST fp32 array with tags tag0 + i until
        the ring is full; returns how many were accepted."""
        n = ctypes.c_int64(0)
        qp, _a = _ptr(queries)
        _check(lib().algas_submit_many(self._h, qp, int(queries.shape[0]), tag0, k, itopk, width, ctypes.byref(n)))
        return n.value

    def enqueue(self, queries: np.ndarray, tag0: int, k: int = 0, itopk: int = 0, width: int = 0) -> None:
        """Append rows of a contiguous HOST fp32 array (tags tag0 + i) to the
        server's host FIFO; the poller thread feeds them into slots as they
        free up (never refuses)."""
        qp, _a = _ptr(queries)
        _check(lib().algas_enqueue(self._h, qp, int(queries.shape[0]), tag0, k, itopk, width))

    def poll(self, max_results: int = 64):
        tags = np.empty(max_results, np.uint64)
        ids = np.empty((max_results, self.kmax), np.uint32)
        ds = np.empty((max_results, self.kmax), np.float32)
        st = np.zeros(max_results, STATS_DTYPE)
        n = ctypes.c_int32(0)
        _check(lib().algas_poll(self._h, _ptr(tags)[0], _ptr(ids)[0], _ptr(ds)[0], _ptr(st)[0], max_results,
                                ctypes.byref(n)))
        m = n.value
        return tags[:m], ids[:m], ds[:m], st[:m]

    def inflight(self) -> int:
        n = ctypes.c_int64(0)
        _check(lib().algas_server_inflight(self._h, ctypes.byref(n)))
        return n.value

    def close(self):
        if getattr(self, "_h", None):
            _check(lib().algas_server_destroy(self._h))
            self._h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def knn(base, queries, k: int, metric: int = L2, self_base: int = -1):
    """Exact kNN on the GPU (algas_knn)."""
    nq, dim = int(queries.shape[0]), int(queries.shape[1])
    ids = _alloc_like(queries, (nq, k), np.uint32, "int32")
    ds = _alloc_like(queries, (nq, k), np.float32, "float32")
    bp, _a = _ptr(base)
    qp, _b = _ptr(queries)
    ip, _c = _ptr(ids)
    dp, _d = _ptr(ds)
    _check(lib().algas_knn(bp, int(base.shape[0]), qp, nq, dim, metric, k, self_base, ip, dp))
    return ids, ds


def knn_partitioned(data, k: int, n_clusters: int, overlap: int = 2, metric: int = L2):
    """Partitioned approximate kNN of the base set (algas_knn_partitioned, R30)."""
    n, dim = int(data.shape[0]), int(data.shape[1])
    ids = _alloc_like(data, (n, k), np.uint32, "int32")
    ds = _alloc_like(data, (n, k), np.float32, "float32")
    dp, _a = _ptr(data)
    ip, _c = _ptr(ids)
    sp, _d = _ptr(ds)
    _check(lib().algas_knn_partitioned(dp, n, dim, metric, k, n_clusters, overlap, ip, sp))
    return ids, ds


def build_graph_partitioned(data, degree: int, n_clusters: int, overlap: int = 2, knn_degree: int | None = None,
                            metric: int = L2, prune: bool = True, refine_fan: int = 16, refine_rounds: int = 0):
    """algas_build_graph_partitioned: partitioned kNN (+ refinement rounds) + the same prune as build_graph."""
    n, dim = int(data.shape[0]), int(data.shape[1])
    kd = knn_degree if knn_degree is not None else 2 * degree
    out = np.empty((n, degree), np.uint32)
    dp, _a = _ptr(data)
    _check(lib().algas_build_graph_partitioned(dp, n, dim, metric, kd, degree, 1 if prune else 0, n_clusters,
                                               overlap, refine_fan, refine_rounds, _ptr(out)[0]))
    return out


def knn_refine(data, ids, dists, fan: int, rounds: int = 1, metric: int = L2, reverse: bool = False):
    """algas_knn_refine: neighbour-of-neighbour refinement rounds (R33; reverse=True: R35 with
    reverse neighbours, passed as a negative fan); returns new (ids, dists)."""
    if reverse:
        fan = -abs(int(fan))
    n, dim = int(data.shape[0]), int(data.shape[1])
    ids = ids.clone() if _is_torch(ids) else np.array(ids, np.uint32, copy=True)
    dists = dists.clone() if _is_torch(dists) else np.array(dists, np.float32, copy=True)
    k = int(ids.shape[1])
    dp, _a = _ptr(data)
    _check(lib().algas_knn_refine(dp, n, dim, metric, k, fan, rounds, _ptr(ids)[0], _ptr(dists)[0]))
    return ids, dists


def knn_last_stats():
    """(rows screened on tensor cores, rows re-done on the direct path) since
    the last call (algas_knn_last_stats); resets the counters."""
    fb = ctypes.c_int64(0)
    n = lib().algas_knn_last_stats(ctypes.byref(fb))
    return int(n), int(fb.value)


def prune(knn_graph, degree: int):
    n, K = int(knn_graph.shape[0]), int(knn_graph.shape[1])
    out = _alloc_like(knn_graph, (n, degree), np.uint32, "int32")
    kp, _a = _ptr(knn_graph)
    op, _b = _ptr(out)
    _check(lib().algas_prune(kp, n, K, degree, op))
    return out


def build_graph(data, degree: int, knn_degree: int | None = None, metric: int = L2, prune: bool = True):
    n, dim = int(data.shape[0]), int(data.shape[1])
    kd = knn_degree if knn_degree is not None else 2 * degree
    out = np.empty((n, degree), np.uint32)
    dp, _a = _ptr(data)
    _check(lib().algas_build_graph(dp, n, dim, metric, kd, degree, 1 if prune else 0, _ptr(out)[0]))
    return out


def merge_topk(ids, dists, k: int):
    ids = np.ascontiguousarray(ids, np.uint32).ravel()
    dists = np.ascontiguousarray(dists, np.float32).ravel()
    oi = np.empty(k, np.uint32)
    od = np.empty(k, np.float32)
    n = lib().algas_merge_topk(_ptr(ids)[0], _ptr(dists)[0], ids.shape[0], k, _ptr(oi)[0], _ptr(od)[0])
    if n < 0:
        _check(n)
    return oi, od, n


def merge_topk_parts(ids, dists, k: int):
    """Host merge of per-part sorted rows: ids/dists [nparts, nq, m] -> [nq, k]."""
    ids = np.ascontiguousarray(ids, np.uint32)
    dists = np.ascontiguousarray(dists, np.float32)
    P_, nq, m = ids.shape
    oi = np.empty((nq, k), np.uint32)
    od = np.empty((nq, k), np.float32)
    _check(lib().algas_merge_topk_parts(_ptr(ids)[0], _ptr(dists)[0], P_, nq, m, k, _ptr(oi)[0], _ptr(od)[0]))
    return oi, od


def device_props() -> DeviceProps:
    d = DeviceProps()
    _check(lib().algas_device_query(ctypes.byref(d)))
    return d


def tune(slots: int, dim: int, degree: int, itopk: int, k: int, props: DeviceProps | None = None) -> Tuning:
    t = Tuning()
    _check(lib().algas_tune(ctypes.byref(props) if props is not None else None, slots, dim, degree, itopk, k,
                            ctypes.byref(t)))
    return t
