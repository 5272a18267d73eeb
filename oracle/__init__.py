"""CPU oracle for the ALGAS hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` leg may import this package.  The
product path (``paper_conf_ipps_chencyzw025_b200``) never imports it and shares
no code with it; see ``oracle/oracle.c`` for the function-by-function citation
of /root/reference/PAPER.md (P:L<line>).

This module is argument marshalling (numpy <-> ``liboracle.so``) for every
function whose arithmetic lives in ``oracle.c`` -- with ONE documented
exception: ``knn_partitioned`` (f4, R30) writes its clustering
steps (Lloyd means in float64, the capacity-constrained assignment) in plain
numpy/Python here, calling O1 (``orc_brute_force``) and the merge
(``orc_merge_topk``) for its distance and top-k steps.

Parity status per function:
  * orc_distance / orc_brute_force (O1)   pinned: numpy float64 argsort,
    integer-lattice exactness, hand-computed values.
  * orc_search (O2)                        pinned: exhaustive special cases
    (== O1), hand-worked path / star / disconnected graphs, w=1 == off>=L.
  * orc_merge_topk (A9)                    pinned: brute-force sort + dedupe.
  * orc_tuner_*                            pinned: Table II closed form.
  * COSINE metric (R29)                     pinned: hand values, angle closed
    form, unit-circle ordering with random radii.
  * knn_partitioned (f4, R30)              parity unpinned by the paper (no
    build algorithm in it); pinned by m = 1 / overlap = m == O1 and two
    hand-worked 1-d examples, one where a Lloyd move and the capacity bound
    (4c < m) each change a cluster.
  * orc_knn_refine (f4, R33)               parity unpinned by the paper; pinned
    by its fixed point (an exact kNN list is unchanged), a hand-worked 1-d
    example and monotonicity (no row's k-th distance grows).
  * orc_knn_refine_rev (f4, R35)           parity unpinned by the paper; pinned
    by a hand-worked example (p-1 reached only through the reverse list), the
    exact-list fixed point and the superset property over R33.
  * orc_prune (K10)                        parity unpinned by the paper (the
    CAGRA algorithm is only cited); pinned by a hand-worked
    example and invariants.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

SENTINEL = 0xFFFFFFFF
L2 = 0
IP = 1
COSINE = 2  # -(q.x)/(|q||x|), R29


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (-O2, no fast-math, no FP contraction)."""
    if (not force and os.path.exists(_LIB_PATH)
            and os.path.getmtime(_LIB_PATH) >= os.path.getmtime(_SRC)):
        return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", "-O2", "-std=c99", "-ffp-contract=off", "-fno-fast-math",
                           "-fPIC", "-shared", "-Wall", "-o", tmp, _SRC, "-lm"])
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


class Params(ctypes.Structure):
    _fields_ = [("k", ctypes.c_int32), ("L", ctypes.c_int32), ("w", ctypes.c_int32),
                ("off", ctypes.c_int32), ("T", ctypes.c_int32), ("S", ctypes.c_int32),
                ("max_iter", ctypes.c_int32), ("shared_visited", ctypes.c_int32),
                ("seed", ctypes.c_uint64)]


class Stats(ctypes.Structure):
    _fields_ = [("iters", ctypes.c_int64), ("parents", ctypes.c_int64),
                ("dist_evals", ctypes.c_int64), ("cap_hits", ctypes.c_int64),
                ("max_iters", ctypes.c_int64)]


STATS_DTYPE = np.dtype([("iters", np.int64), ("parents", np.int64), ("dist_evals", np.int64),
                        ("cap_hits", np.int64), ("max_iters", np.int64)])


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB_PATH)
            P = ctypes.c_void_p
            i32, i64, u32, u64 = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32, ctypes.c_uint64
            L.orc_splitmix64.argtypes = [u64]
            L.orc_splitmix64.restype = u64
            L.orc_entry_point.argtypes = [u64, u64, u32, u32, i64]
            L.orc_entry_point.restype = u32
            L.orc_distance.argtypes = [P, P, i32, i32]
            L.orc_distance.restype = ctypes.c_float
            L.orc_brute_force.argtypes = [P, i64, i32, i32, P, i64, i32, i64, P, P]
            L.orc_brute_force.restype = None
            L.orc_merge_topk.argtypes = [P, P, i32, i32, P, P]
            L.orc_merge_topk.restype = i32
            L.orc_search.argtypes = [P, i64, i32, i32, P, i32, P, u64, ctypes.POINTER(Params),
                                     P, P, P, P, P]
            L.orc_search.restype = i32
            L.orc_search_batch.argtypes = [P, i64, i32, i32, P, i32, P, i64, u64,
                                           ctypes.POINTER(Params), P, P, P, P, P]
            L.orc_search_batch.restype = i32
            L.orc_tuner_max_parallel.argtypes = [i32, i32, i32]
            L.orc_tuner_max_parallel.restype = i32
            L.orc_tuner_blocks_per_sm.argtypes = [i32, i32, i32]
            L.orc_tuner_blocks_per_sm.restype = i32
            L.orc_tuner_smem_per_block.argtypes = [i64, i32, i64]
            L.orc_tuner_smem_per_block.restype = i64
            L.orc_prune.argtypes = [P, i64, i32, i32, P, P]
            L.orc_prune.restype = i32
            L.orc_knn_refine.argtypes = [P, i64, i32, i32, i32, i32, P, P, P, P]
            L.orc_knn_refine.restype = i32
            L.orc_knn_refine_rev.argtypes = [P, i64, i32, i32, i32, i32, P, P, P, P]
            L.orc_knn_refine_rev.restype = i32
            _lib = L
    return _lib


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _u32(a):
    return np.ascontiguousarray(a, dtype=np.uint32)


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def splitmix64(z: int) -> int:
    return int(lib().orc_splitmix64(z & 0xFFFFFFFFFFFFFFFF))


def entry_point(seed: int, tag: int, cta: int, j: int, n: int) -> int:
    return int(lib().orc_entry_point(seed, tag, cta, j, n))


def distance(q, x, metric: int = L2) -> float:
    q, x = _f32(q), _f32(x)
    return float(lib().orc_distance(_ptr(q), _ptr(x), q.shape[0], metric))


def brute_force(X, Q, k: int, metric: int = L2, self_base: int = -1):
    """O1: exact kNN of each row of Q in X; returns (ids uint32 [nq,k], dists f32 [nq,k])."""
    X, Q = _f32(X), _f32(Q)
    n, d = X.shape
    nq = Q.shape[0]
    ids = np.empty((nq, k), np.uint32)
    ds = np.empty((nq, k), np.float32)
    lib().orc_brute_force(_ptr(X), n, d, metric, _ptr(Q), nq, k, self_base, _ptr(ids), _ptr(ds))
    return ids, ds


def knn_graph(X, K: int, metric: int = L2):
    """kNN graph excluding self (O1 with self exclusion)."""
    return brute_force(X, X, K, metric, self_base=0)


def knn_partitioned(X, k: int, n_clusters: int, overlap: int, metric: int = L2):
    """Partitioned approximate kNN graph (R30), step by
    step: (1) centres = rows floor(j n / m); (2) each point's `overlap`
    nearest centres with room (capacity ceil(2 c n / m), n if 4c >= m), after
    8 Lloyd iterations on a row sample; (3) cluster members in ascending
    id; (4) O1 inside each cluster, self excluded, k_j = min(k, s_j - 1);
    (5) per point: its cluster lists merged by (dist, id), repeated ids
    dropped, first k (orc_merge_topk).  Parity unpinned by the paper (it
    gives no build algorithm); pinned by m = 1 and overlap = m (== O1) and a
    hand-worked example (tests/test_oracle.py)."""
    X = _f32(X)
    n = X.shape[0]
    m, c = n_clusters, overlap
    centres = X[[(j * n) // m for j in range(m)]].copy()
    # (1b) 8 Lloyd iterations on the sample rows floor(i n / ns), ns = min(n, 32 m):
    # nearest centre (O1), centre = mean of its rows (double, row order), empty stays
    if m > 1:
        ns = min(n, 32 * m)
        S = X[[(i * n) // ns for i in range(ns)]]
        for _ in range(8):
            a1, _d = brute_force(centres, S, 1, metric)
            for j in range(m):
                rows = [i for i in range(ns) if a1[i, 0] == j]
                if rows:
                    acc = np.zeros(X.shape[1], np.float64)
                    for i in rows:
                        acc += S[i].astype(np.float64)
                    centres[j] = (acc / len(rows)).astype(np.float32)
    # (2) capacity-constrained: P nearest centres per point; points in id
    # order take the first c with room, else the lowest-index ones with room
    P = min(m, 4 * c + 4)
    pref, _ = brute_force(centres, X, P, metric)
    cap = n if 4 * c >= m else -(-2 * c * n // m)
    load = [0] * m
    asg = np.zeros((n, c), np.int64)
    for i in range(n):
        got = []
        for j in list(pref[i]) + list(range(m)):
            if len(got) == c:
                break
            if load[j] < cap and j not in got:
                got.append(int(j))
                load[j] += 1
        assert len(got) == c
        asg[i] = got
    cand_i = np.full((n, c, k), SENTINEL, np.uint32)
    cand_d = np.full((n, c, k), np.inf, np.float32)
    for j in range(m):
        mem = np.array([i for i in range(n) if j in asg[i]], np.int64)
        if mem.shape[0] < 2:
            continue
        kj = min(k, mem.shape[0] - 1)
        li, ld = brute_force(X[mem], X[mem], kj, metric, self_base=0)
        for t, i in enumerate(mem):
            r = list(asg[i]).index(j)
            cand_i[i, r, :kj] = mem[li[t]]
            cand_d[i, r, :kj] = ld[t]
    ids = np.empty((n, k), np.uint32)
    ds = np.empty((n, k), np.float32)
    for i in range(n):
        ids[i], ds[i], _ = merge_topk(cand_i[i], cand_d[i], k)
    return ids, ds


def knn_refine(X, ids, ds, fan: int, rounds: int = 1, metric: int = L2, reverse: bool = False):
    """R33: `rounds` neighbour-of-neighbour refinement rounds (orc_knn_refine,
    each a Jacobi round over the previous round's lists); reverse=True: R35,
    the same with reverse neighbours (orc_knn_refine_rev)."""
    X = _f32(X)
    ids, ds = _u32(ids).copy(), _f32(ds).copy()
    n, k = ids.shape
    for _ in range(rounds):
        oi = np.empty_like(ids)
        od = np.empty_like(ds)
        fn = lib().orc_knn_refine_rev if reverse else lib().orc_knn_refine
        rc = fn(_ptr(X), n, X.shape[1], metric, k, fan, _ptr(ids), _ptr(ds), _ptr(oi), _ptr(od))
        if rc != 0:
            raise RuntimeError("orc_knn_refine failed")
        ids, ds = oi, od
    return ids, ds


def merge_topk(ids, dists, k: int):
    ids, dists = _u32(ids).ravel(), _f32(dists).ravel()
    oi = np.empty(k, np.uint32)
    od = np.empty(k, np.float32)
    n = lib().orc_merge_topk(_ptr(ids), _ptr(dists), ids.shape[0], k, _ptr(oi), _ptr(od))
    return oi, od, int(n)


def make_params(k=10, L=64, w=1, off=None, T=1, S=32, max_iter=None, shared_visited=0, seed=0):
    if off is None:
        off = L  # beam extend disabled unless asked for
    if max_iter is None:
        max_iter = 4 * L + 256
    return Params(k, L, w, off, T, S, max_iter, shared_visited, seed & 0xFFFFFFFFFFFFFFFF)


def search(X, G, Q, params: Params, metric: int = L2, tag0: int = 0, want_cta: bool = False):
    """O2 over a batch: query i has tag tag0+i.  Returns ids, dists, stats[, cta_ids, cta_d]."""
    X, Q, G = _f32(X), _f32(np.atleast_2d(Q)), _u32(G)
    n, d = X.shape
    R = G.shape[1]
    nq = Q.shape[0]
    k, T = params.k, params.T
    ids = np.empty((nq, k), np.uint32)
    ds = np.empty((nq, k), np.float32)
    st = np.zeros(nq, STATS_DTYPE)
    ci = np.empty((nq, T, k), np.uint32) if want_cta else None
    cd = np.empty((nq, T, k), np.float32) if want_cta else None
    rc = lib().orc_search_batch(_ptr(X), n, d, metric, _ptr(G), R, _ptr(Q), nq, tag0,
                                ctypes.byref(params), _ptr(ids), _ptr(ds), _ptr(ci), _ptr(cd),
                                _ptr(st))
    if rc != 0:
        raise RuntimeError(f"orc_search_batch failed rc={rc}")
    if want_cta:
        return ids, ds, st, ci, cd
    return ids, ds, st


def tuner_max_parallel(slots, n_sm, max_block_per_sm):
    return int(lib().orc_tuner_max_parallel(slots, n_sm, max_block_per_sm))


def tuner_blocks_per_sm(n_parallel, slots, n_sm):
    return int(lib().orc_tuner_blocks_per_sm(n_parallel, slots, n_sm))


def tuner_smem_per_block(m_per_sm, blocks_per_sm, m_reserved):
    return int(lib().orc_tuner_smem_per_block(m_per_sm, blocks_per_sm, m_reserved))


def prune(knn, R: int, want_pruned: bool = False):
    knn = _u32(knn)
    n, K = knn.shape
    out = np.empty((n, R), np.uint32)
    pr = np.empty((n, R), np.uint32) if want_pruned else None
    rc = lib().orc_prune(_ptr(knn), n, K, R, _ptr(out), _ptr(pr))
    if rc != 0:
        raise RuntimeError("orc_prune failed")
    return (out, pr) if want_pruned else out


def recall(found_ids, truth_ids, k: int) -> float:
    """recall = |K_approx ∩ K_truth| / |K_truth|, averaged over queries."""
    found_ids = np.asarray(found_ids)[:, :k]
    truth_ids = np.asarray(truth_ids)[:, :k]
    hits = 0
    for f, t in zip(found_ids, truth_ids):
        hits += len(set(f.tolist()) & set(t.tolist()) - {SENTINEL})
    return hits / float(truth_ids.shape[0] * k)
