"""Multi-process host logic of the multi-GPU layouts, on CPU with
the gloo backend and world_size 2.  The per-shard / per-replica searches are
stood in for by the oracle (CPU), so these tests check the partitioning,
global-id translation, all-gather exchange and host merge -- the parts that
do not need a GPU."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch.multiprocessing as mp

import oracle
import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, fn, out_dir):
    import sys
    sys.path.insert(0, ROOT)
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        res = fn(rank, world)
        np.save(os.path.join(out_dir, f"r{rank}.npy"), res, allow_pickle=True)
    finally:
        dist.destroy_process_group()


def _run(fn, world=2):
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_worker, args=(world, _free_port(), fn, d), nprocs=world, join=True, start_method="spawn")
        return [np.load(os.path.join(d, f"r{r}.npy"), allow_pickle=True).item() for r in range(world)]


def _shard_exact(rank, world):
    from paper_conf_ipps_chencyzw025_b200 import shard
    X = synth.lattice(3001, 16, seed=71)
    Q = synth.lattice(40, 16, seed=72)
    lo, hi = shard.shard_range(X.shape[0], world, rank)
    li, ld = oracle.brute_force(X[lo:hi], Q, 12)      # exact per-shard top-k (stand-in for the GPU search)
    gi, gd = shard.gather_and_merge(shard.to_global(li, lo), ld, 12)
    return dict(ids=gi, dists=gd, lo=lo, hi=hi)


def test_sharded_exact_topk_equals_global_bruteforce():
    """Exact per-shard top-k + all-gather + merge == global exact top-k (O1)."""
    res = _run(_shard_exact)
    X = synth.lattice(3001, 16, seed=71)
    Q = synth.lattice(40, 16, seed=72)
    ei, ed = oracle.brute_force(X, Q, 12)
    for r in res:
        np.testing.assert_array_equal(r["ids"], ei)
        np.testing.assert_array_equal(r["dists"], ed)
    # shards partition the base set
    assert res[0]["lo"] == 0 and res[0]["hi"] == res[1]["lo"] and res[1]["hi"] == X.shape[0]


def _shard_graph_search(rank, world):
    from paper_conf_ipps_chencyzw025_b200 import shard
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 3000)
    Q = synth.query_vectors(w, 30)
    lo, hi = shard.shard_range(X.shape[0], world, rank)
    G, _ = oracle.knn_graph(X[lo:hi], 16)             # subgraph built inside the shard
    p = oracle.make_params(k=10, L=48, w=2, off=12, T=1, S=16, seed=3)
    li, ld, _ = oracle.search(X[lo:hi], G, Q, p)
    gi, gd = shard.gather_and_merge(shard.to_global(li, lo), ld, 10)
    return dict(ids=gi, dists=gd)


def test_sharded_graph_search_is_consistent_and_accurate():
    res = _run(_shard_graph_search)
    np.testing.assert_array_equal(res[0]["ids"], res[1]["ids"])  # every rank holds the merged answer
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 3000)
    Q = synth.query_vectors(w, 30)
    # expected: the same per-shard searches, merged in-process with the oracle's merge
    from paper_conf_ipps_chencyzw025_b200 import shard
    parts_i, parts_d = [], []
    for r in range(2):
        lo, hi = shard.shard_range(X.shape[0], 2, r)
        G, _ = oracle.knn_graph(X[lo:hi], 16)
        li, ld, _ = oracle.search(X[lo:hi], G, Q, oracle.make_params(k=10, L=48, w=2, off=12, T=1, S=16, seed=3))
        parts_i.append(shard.to_global(li, lo))
        parts_d.append(ld)
    for t in range(Q.shape[0]):
        ei, ed, _ = oracle.merge_topk(np.concatenate([p[t] for p in parts_i]),
                                      np.concatenate([p[t] for p in parts_d]), 10)
        np.testing.assert_array_equal(res[0]["ids"][t], ei)
    bi, _ = oracle.brute_force(X, Q, 10)
    assert oracle.recall(res[0]["ids"], bi, 10) > 0.5
    for t in range(Q.shape[0]):
        row = [int(i) for i in res[0]["ids"][t]]
        assert len(set(row)) == 10 and np.all(np.diff(res[0]["dists"][t]) >= 0)


def _replicas(rank, world):
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_chencyzw025_b200 import shard
    X = synth.lattice(1500, 16, seed=81)
    Q = synth.lattice(37, 16, seed=82)
    G, _ = oracle.knn_graph(X, 12)
    sl = shard.replica_slice(Q.shape[0], world, rank)
    p = oracle.make_params(k=8, L=32, w=2, off=8, T=1, S=8, seed=1)
    ids, ds, _ = oracle.search(X, G, Q[sl], p, tag0=sl.start)  # tags follow the global query index
    # reassemble (test harness only; replicas need no collective on the data path)
    parts = [None] * world
    dist.all_gather_object(parts, ids)
    return dict(ids=np.concatenate(parts).astype(np.uint32))


def test_replicas_equal_single_process():
    """Query-parallel replicas return exactly the single-process answers."""
    res = _run(_replicas)
    X = synth.lattice(1500, 16, seed=81)
    Q = synth.lattice(37, 16, seed=82)
    G, _ = oracle.knn_graph(X, 12)
    ids, _, _ = oracle.search(X, G, Q, oracle.make_params(k=8, L=32, w=2, off=8, T=1, S=8, seed=1))
    np.testing.assert_array_equal(res[0]["ids"], ids)


def test_shard_range_partitions():
    from paper_conf_ipps_chencyzw025_b200 import shard
    for n in (1, 7, 100, 1001):
        for world in (1, 2, 3, 8):
            rs = [shard.shard_range(n, world, r) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(world - 1))
            assert max(b - a for a, b in rs) - min(b - a for a, b in rs) <= 1
    ids = np.array([0, 5, 0xFFFFFFFF], np.uint32)
    np.testing.assert_array_equal(shard.to_global(ids, 100), [100, 105, 0xFFFFFFFF])


def _sharded_server_emulated(rank, world):
    """Each rank serves its 'shard' with an emulated ring device (host logic
    only); rank 0 alone holds the query stream."""
    import paper_conf_ipps_chencyzw025_b200 as algas
    from paper_conf_ipps_chencyzw025_b200 import shard
    Q = synth.uniform(300, 8, seed=90).astype(np.float32)
    Q[:, 0] = np.round(Q[:, 0] * 100)  # exact small-integer q[0] (the emulated dists)
    offset = rank * 10_000_000
    p = algas.default_params(k=6, itopk=16, width=4, ctas_per_query=2, slots=4)
    with algas.Server(None, p, emulated_dim=8, deferred=True) as srv:
        ss = shard.ShardedServer(srv, offset, 6)
        ss.warmup(8, 64)
        srv.start()
        gi, gd = ss.serve(Q if rank == 0 else None, batch=64, tag0=5)
    return dict(ids=gi, dists=gd, Q=Q)


def test_sharded_server_broadcast_enqueue_gather_merge():
    """ShardedServer: rank 0's stream is broadcast, every rank's server
    answers every query, and the merged lists equal the (dist, id)-sorted
    union of the ranks' per-shard lists with global ids -- on every rank."""
    res = _run(_sharded_server_emulated)
    Q = res[0]["Q"]
    for q in range(Q.shape[0]):
        tag = 5 + q
        union = [(Q[q, 0] + j, tag * 1000 + j + r * 10_000_000) for r in range(2) for j in range(6)]
        union.sort()
        exp_i = np.array([u[1] for u in union[:6]], np.uint32)
        exp_d = np.array([u[0] for u in union[:6]], np.float32)
        for r in range(2):
            np.testing.assert_array_equal(res[r]["ids"][q], exp_i)
            np.testing.assert_array_equal(res[r]["dists"][q], exp_d)
