"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself:
published constants, closed forms, the paper's worked table, hand-worked
traces, exhaustive special cases that reduce to the plain definition, and
numpy/float64 or exact-integer recomputation.  CPU only."""
import json
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")
SENT = oracle.SENTINEL


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------- generator
def test_splitmix64_published_sequence():
    g = _gold("splitmix64.json")
    gamma = int(g["gamma_hex"], 16)
    for i, h in enumerate(g["state0_outputs_hex"]):
        # the generator's i-th output from state 0 is one mix step of state (i*gamma)
        assert oracle.splitmix64((i * gamma) & (2**64 - 1)) == int(h, 16)


def test_entry_points_in_range_and_spread():
    n = 1000
    e = [oracle.entry_point(7, t, c, j, n) for t in range(20) for c in range(4) for j in range(8)]
    assert min(e) >= 0 and max(e) < n
    assert len(set(e)) > 0.7 * len(e)  # not degenerate
    assert oracle.entry_point(7, 3, 1, 2, n) == oracle.entry_point(7, 3, 1, 2, n)
    # the seed enters the composition: another seed moves (almost) every entry point
    moved = sum(oracle.entry_point(7, t, c, j, n) != oracle.entry_point(8, t, c, j, n)
                for t in range(20) for c in range(4) for j in range(8))
    assert moved > 0.95 * 640, moved


def test_entry_point_hand_derived_from_published_vectors():
    """R5: e = splitmix64(seed ^ splitmix64(tag ^ splitmix64(cta << 32 | j))) mod n,
    evaluated by hand from the published state-0 outputs o0, o1, o2 of SplitMix64
    (o_i = splitmix64(i * gamma)):  cta = j = 0 gives splitmix64(0) = o0; with
    tag = o0 ^ gamma the middle call is splitmix64(gamma) = o1; with
    seed = o1 ^ (2 gamma mod 2^64) the outer call is splitmix64(2 gamma) = o2.
    So e = o2 mod n -- any other composition (e.g. tag + a) breaks it."""
    g = _gold("splitmix64.json")
    gamma = int(g["gamma_hex"], 16)
    o0, o1, o2 = (int(h, 16) for h in g["state0_outputs_hex"])
    M = 2**64 - 1
    tag = o0 ^ gamma
    seed = o1 ^ ((2 * gamma) & M)
    for n in (7, 1000, 1_000_000, 100_000_000, 2**31 - 1):
        assert oracle.entry_point(seed, tag, 0, 0, n) == o2 % n
    # the cta / j word: (cta << 32) | j = gamma (cta = gamma >> 32, j = low 32
    # bits) makes the inner call o1; tag = o1 ^ 2 gamma -> o2; seed = o2 ^ 0 -> o0
    cta, j = gamma >> 32, gamma & 0xFFFFFFFF
    assert oracle.entry_point(o2, o1 ^ ((2 * gamma) & M), cta, j, 1_000_003) == \
        oracle.splitmix64(0) % 1_000_003 == o0 % 1_000_003


# ---------------------------------------------------------------- distance
def test_distance_hand_values():
    q = np.array([1, 2, 3], np.float32)
    x = np.array([4, 6, 3], np.float32)
    assert oracle.distance(q, x, oracle.L2) == 25.0       # 9 + 16 + 0
    assert oracle.distance(q, x, oracle.IP) == -25.0      # -(4 + 12 + 9)
    assert oracle.distance(q, q, oracle.L2) == 0.0


def test_distance_close_to_float64():
    rng = np.random.default_rng(0)
    for d in (1, 7, 96, 100, 128, 960):
        q = rng.standard_normal(d).astype(np.float32)
        x = rng.standard_normal(d).astype(np.float32)
        l2 = float(((q.astype(np.float64) - x) ** 2).sum())
        ip = -float((q.astype(np.float64) * x).sum())
        assert abs(oracle.distance(q, x, oracle.L2) - l2) <= 1e-5 * l2
        scale = float(np.abs(q.astype(np.float64) * x).sum())
        assert abs(oracle.distance(q, x, oracle.IP) - ip) <= 1e-5 * scale


# ---------------------------------------------------------------- O1 brute force
def _np_exact_int_topk(X, Q, k, metric, self_base=-1):
    """Exact integer distances (int64) + lexsort by (dist, id)."""
    Xi = X.astype(np.int64)
    ids, ds = [], []
    for qi, q in enumerate(Q.astype(np.int64)):
        d = ((Xi - q) ** 2).sum(1) if metric == oracle.L2 else -(Xi * q).sum(1)
        idx = np.arange(X.shape[0])
        if self_base >= 0:
            keep = idx != self_base + qi
            d, idx = d[keep], idx[keep]
        o = np.lexsort((idx, d))[:k]
        ids.append(idx[o])
        ds.append(d[o])
    return np.array(ids), np.array(ds)


@pytest.mark.parametrize("metric", [oracle.L2, oracle.IP])
def test_brute_force_integer_lattice_exact(metric):
    X = synth.lattice(600, 32, seed=11, metric=metric)
    Q = synth.lattice(20, 32, seed=12, metric=metric)
    ids, ds = oracle.brute_force(X, Q, 15, metric)
    ei, ed = _np_exact_int_topk(X, Q, 15, metric)
    np.testing.assert_array_equal(ids, ei)
    np.testing.assert_array_equal(ds, ed.astype(np.float32))


def test_brute_force_self_exclusion_lattice():
    X = synth.lattice(300, 16, seed=13)
    ids, ds = oracle.knn_graph(X, 10)
    ei, ed = _np_exact_int_topk(X, X, 10, oracle.L2, self_base=0)
    np.testing.assert_array_equal(ids, ei)
    assert not np.any(ids == np.arange(300)[:, None])


def test_brute_force_float_vs_float64_argsort():
    X = synth.uniform(800, 24, seed=3)
    Q = synth.uniform(30, 24, seed=4)
    k = 10
    ids, ds = oracle.brute_force(X, Q, k)
    d64 = ((Q[:, None, :].astype(np.float64) - X[None].astype(np.float64)) ** 2).sum(-1)
    for r in range(Q.shape[0]):
        order = np.argsort(d64[r], kind="stable")[:k]
        kth = d64[r, order[-1]]
        # identical except where two float64 distances lie within the tolerance of the k-th
        for a, b in zip(ids[r], order):
            if a != b:
                assert abs(d64[r, a] - d64[r, b]) <= 1e-5 * kth
        np.testing.assert_allclose(ds[r], d64[r, ids[r]], rtol=1e-5)


def test_brute_force_padding_when_k_exceeds_n():
    X = synth.uniform(5, 4, seed=5)
    ids, ds = oracle.brute_force(X, X[:1], 8)
    assert list(ids[0, 5:]) == [SENT] * 3
    assert np.all(np.isinf(ds[0, 5:]))
    ids, ds = oracle.brute_force(X, X[:1], 8, self_base=0)
    assert list(ids[0, 4:]) == [SENT] * 4


# ---------------------------------------------------------------- A9 merge
def test_merge_topk_vs_bruteforce_sort():
    rng = np.random.default_rng(9)
    for trial in range(50):
        m = int(rng.integers(1, 60))
        ids = rng.integers(0, 25, size=m).astype(np.uint32)
        ids[rng.random(m) < 0.1] = SENT
        # a duplicate id always carries the same distance (deterministic F)
        table = rng.integers(0, 6, size=25).astype(np.float32)
        ds = np.where(ids == SENT, np.float32(np.inf), table[np.minimum(ids, 24)])
        k = int(rng.integers(1, 12))
        oi, od, n = oracle.merge_topk(ids, ds, k)
        uniq = sorted({(float(table[i]), int(i)) for i in ids if i != SENT})[:k]
        assert n == len(uniq)
        assert [int(x) for x in oi[:n]] == [i for _, i in uniq]
        assert [float(x) for x in od[:n]] == [d for d, _ in uniq]
        assert all(x == SENT for x in oi[n:])


# ---------------------------------------------------------------- tuner (Table II)
def test_tuner_equations_table2():
    g = _gold("table2_tuner.json")
    a = g["a6000"]
    for w in g["worked"]:
        if "expect_max_parallel" in w:
            assert oracle.tuner_max_parallel(w["slots"], a["n_sm"], a["max_blocks_per_sm"]) == w["expect_max_parallel"]
        if "expect_blocks_per_sm" in w:
            assert oracle.tuner_blocks_per_sm(w["n_parallel"], w["slots"], a["n_sm"]) == w["expect_blocks_per_sm"]
        if "expect_smem_per_block" in w:
            assert oracle.tuner_smem_per_block(a["shared_mem_per_sm_bytes"], w["blocks_per_sm"],
                                               a["reserved_shared_mem_per_block_bytes"]) == w["expect_smem_per_block"]


def test_tuner_equations_b200_numbers():
    # B200: 148 SMs, 32 blocks/SM, 228 KB smem/SM, 1 KB reserved per block
    assert oracle.tuner_max_parallel(32, 148, 32) == 148
    assert oracle.tuner_blocks_per_sm(148, 32, 148) == 32
    assert oracle.tuner_smem_per_block(228 * 1024, 32, 1024) == 6272   # 6.125 KB
    assert oracle.tuner_smem_per_block(228 * 1024, 8, 1024) == 28160    # 27.5 KB


# ---------------------------------------------------------------- O2 search
def _reachable(G, seeds):
    n = G.shape[0]
    seen = np.zeros(n, bool)
    stack = list(seeds)
    for s in stack:
        seen[s] = True
    while stack:
        u = stack.pop()
        for v in G[u]:
            if v != SENT and not seen[v]:
                seen[v] = True
                stack.append(int(v))
    return seen


@pytest.mark.parametrize("metric", [oracle.L2, oracle.IP])
@pytest.mark.parametrize("T,shared", [(1, 0), (3, 0), (3, 1)])
def test_search_exhaustive_equals_bruteforce(metric, T, shared):
    """L >= n and max_iter >= n on a graph reachable from the seeds: the list is
    never truncated, every reachable point is scored, so O2 == O1 exactly."""
    n, d = 150, 8
    X = synth.lattice(n, d, seed=21, metric=metric)
    Q = synth.lattice(6, d, seed=22, metric=metric)
    G = synth.random_graph(n, 6, seed=23)
    p = oracle.make_params(k=12, L=n, w=2, off=4, T=T, S=2, max_iter=10 * n, shared_visited=shared, seed=5)
    seeds = [oracle.entry_point(5, t, c, j, n) for t in range(6) for c in range(T) for j in range(2)]
    assert _reachable(G, seeds).all()
    ids, ds, st = oracle.search(X, G, Q, p, metric=metric)
    ei, ed = oracle.brute_force(X, Q, 12, metric)
    np.testing.assert_array_equal(ids, ei)
    np.testing.assert_array_equal(ds, ed)
    assert (st["cap_hits"] == 0).all()
    if T == 1 or not shared:
        assert (st["dist_evals"] == T * n).all()      # every point scored once per table
    else:
        assert (st["dist_evals"] <= n + T * 2).all()  # shared table: + re-scored foreign seeds


def test_search_complete_graph_one_expansion():
    n = 40
    X = synth.uniform(n, 4, seed=31)
    Q = synth.uniform(5, 4, seed=32)
    G = np.array([[j for j in range(n) if j != i] for i in range(n)], np.uint32)
    p = oracle.make_params(k=5, L=8, w=1, T=1, S=1, seed=1)
    ids, ds, st = oracle.search(X, G, Q, p)
    ei, ed = oracle.brute_force(X, Q, 5)
    np.testing.assert_array_equal(ids, ei)
    assert (st["dist_evals"] == n).all()


def test_search_path_graph_hand_trace():
    """1-D points x_i = i on a path graph (i-1, i+1), query 7.2, one seed e<=5, L=3.
    Hand trace: the walk expands e, e+1, ..., 6, 7, 8 (9-e steps); it scores the
    seed, e-1, e+1 .. 8 and 9 (11-e points); the final list is [7, 8, 6]."""
    n = 20
    X = np.arange(n, dtype=np.float32)[:, None]
    G = np.array([[i - 1 if i > 0 else SENT, i + 1 if i < n - 1 else SENT] for i in range(n)], np.uint32)
    q = np.array([[7.2]], np.float32)
    seed = next(s for s in range(1000) if 1 <= oracle.entry_point(s, 0, 0, 0, n) <= 5)
    e = oracle.entry_point(seed, 0, 0, 0, n)
    p = oracle.make_params(k=3, L=3, w=1, T=1, S=1, seed=seed)
    ids, ds, st = oracle.search(X, G, q, p)
    assert list(ids[0]) == [7, 8, 6]
    np.testing.assert_allclose(ds[0], [0.2 ** 2, 0.8 ** 2, 1.2 ** 2], rtol=1e-5)  # 7.2 is not exact in fp32
    assert st["iters"][0] == 9 - e
    assert st["dist_evals"][0] == 11 - e
    assert st["parents"][0] == 9 - e


# The beam-extend hand trace (R6/R7).  1-d points (d padded
# to 4 with zeros) on a small directed graph, query at 0; squared distances
# A=100 B=144 C=169 D=25 E=400 F=16 G=900.
BEAM_X = [10, 12, 13, 5, 20, 4, 30]           # ids 0..6 = A B C D E F G
BEAM_G = [[1, 2], [3, SENT], [4, SENT], [5, 0], [6, SENT], [3, SENT], [4, SENT]]
BEAM_SEED = 3                                  # entry_point(3, tag 0, cta 0, j 0, n 7) = 0 = A


def beam_case():
    X = np.zeros((7, 4), np.float32)
    X[:, 0] = BEAM_X
    return X, np.array(BEAM_G, np.uint32), np.zeros((1, 4), np.float32)


# (off, iters, parents, dist_evals), worked by hand in test_beam_extend_trigger_hand_trace
BEAM_TRACES = [(1, 4, 6, 7), (2, 5, 5, 6), (5, 5, 5, 6)]


@pytest.mark.parametrize("off,iters,parents,evals", BEAM_TRACES)
def test_beam_extend_trigger_hand_trace(off, iters, parents, evals):
    """L = 5, w = 2, one seed (A), T = 1.  Diffusing latches when the FIRST
    unchecked position U[0] >= off and stays on (R6, sticky).

    off = 1:  s1 list [A] U=[0], 0<1 greedy: expand A -> B, C; list [A* B C].
              s2 U=[1,2], 1>=1 -> diffusing: expand B, C -> D, E; [D A* B* C* E].
              s3 U=[0,4]: sticky, so 2 parents D, E -> F, G; [F D* A* B* C*] (E, G cut).
              s4 U=[0] -> F (D visited).  s5 U=[] Finish.
              iters 4, parents 1+2+2+1 = 6, evals 1+2+2+2 = 7.
              (with '>' instead of '>=': s2 is greedy -> iters 5, parents 5;
               non-sticky: s3 has U[0]=0 < 1 -> one parent -> parents 5, evals 6)
    off = 2:  s2 U[0]=1 <2 greedy: B -> D; [D A* B* C].  s3 U=[0,3] greedy D -> F;
              [F D* A* B* C].  s4 U=[0,4] greedy F.  s5 U=[4], 4>=2 diffusing: C -> E;
              [F D* A* B* C*] (E cut).  s6 U=[] Finish: iters 5, parents 5, evals 6.
    off = 5 (= L, beam extend off, Alg. 1): the same walk as off = 2.
    In every case the result (k = 3) is F, D, A at 16, 25, 100."""
    X, G, q = beam_case()
    assert oracle.entry_point(BEAM_SEED, 0, 0, 0, 7) == 0
    p = oracle.make_params(k=3, L=5, w=2, off=off, T=1, S=1, seed=BEAM_SEED)
    ids, ds, st = oracle.search(X, G, q, p)
    assert ids[0].tolist() == [5, 3, 0] and ds[0].tolist() == [16.0, 25.0, 100.0]
    assert (st["iters"][0], st["parents"][0], st["dist_evals"][0]) == (iters, parents, evals)


def test_search_star_graph():
    """Star: leaves connect only to the centre 0, the centre to every leaf.
    From any leaf the second step expands the centre and scores everything."""
    n = 30
    X = synth.uniform(n, 4, seed=41)
    Q = synth.uniform(4, 4, seed=42)
    G = np.full((n, n - 1), SENT, np.uint32)
    G[0] = np.arange(1, n)
    G[1:, 0] = 0
    p = oracle.make_params(k=4, L=6, w=1, T=1, S=1, seed=3)
    ids, ds, st = oracle.search(X, G, Q, p)
    ei, ed = oracle.brute_force(X, Q, 4)
    np.testing.assert_array_equal(ids, ei)
    assert (st["dist_evals"] == n).all()


def test_search_disconnected_graph_stays_in_component():
    n = 40
    X = synth.uniform(n, 4, seed=51)
    half = n // 2
    G = np.array([[j for j in range((i // half) * half, (i // half + 1) * half) if j != i] for i in range(n)],
                 np.uint32)
    Q = synth.uniform(6, 4, seed=52)
    p = oracle.make_params(k=5, L=n, w=1, T=1, S=1, seed=4)
    ids, ds, st = oracle.search(X, G, Q, p)
    for t in range(6):
        comp = oracle.entry_point(4, t, 0, 0, n) // half
        assert all(int(i) // half == comp for i in ids[t])
        # exact within the reachable component
        sub = np.arange(comp * half, (comp + 1) * half)
        ei, _ = oracle.brute_force(X[sub], Q[t:t + 1], 5)
        assert list(ids[t]) == [int(sub[i]) for i in ei[0]]


def test_beam_extend_disabled_equals_greedy():
    """w>1 with off >= L never enters the diffusing phase: identical to Alg.1."""
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 3000)
    Q = synth.query_vectors(w, 20)
    G, _ = oracle.knn_graph(X, 16)
    a = oracle.search(X, G, Q, oracle.make_params(k=10, L=32, w=1, T=1, S=8, seed=2))
    b = oracle.search(X, G, Q, oracle.make_params(k=10, L=32, w=4, off=32, T=1, S=8, seed=2))
    np.testing.assert_array_equal(a[0], b[0])
    np.testing.assert_array_equal(a[2]["iters"], b[2]["iters"])
    c = oracle.search(X, G, Q, oracle.make_params(k=10, L=32, w=4, off=4, T=1, S=8, seed=2))
    # beam extend: fewer maintenance steps ...
    assert c[2]["iters"].mean() < 0.8 * a[2]["iters"].mean()
    # ... and each diffusing step expands up to w parents
    assert (c[2]["parents"] >= c[2]["iters"]).all()


def test_multi_cta_private_is_union_of_ctas():
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 2000)
    Q = synth.query_vectors(w, 10)
    G, _ = oracle.knn_graph(X, 16)
    p1 = oracle.make_params(k=10, L=24, w=1, T=1, S=4, seed=9)
    p3 = oracle.make_params(k=10, L=24, w=1, T=3, S=4, seed=9)
    i1, d1, s1 = oracle.search(X, G, Q, p1)
    i3, d3, s3, ci, cd = oracle.search(X, G, Q, p3, want_cta=True)
    # CTA 0 of a private-visited T=3 run is the T=1 run (same seeds, same table)
    np.testing.assert_array_equal(ci[:, 0, :], i1)
    # the merged result is the (dist,id)-sorted, deduplicated union of the CTA lists
    for t in range(Q.shape[0]):
        u = sorted({(float(dd), int(ii)) for ii, dd in zip(ci[t].ravel(), cd[t].ravel()) if ii != SENT})[:10]
        assert [i for _, i in u] == [int(x) for x in i3[t]]


def test_search_invariants_float():
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 3000)
    Q = synth.query_vectors(w, 30)
    G, _ = oracle.knn_graph(X, 16)
    for metric in (oracle.L2, oracle.IP):
        ids, ds, st = oracle.search(X, G, Q, oracle.make_params(k=10, L=32, w=2, off=8, T=2, S=8, seed=1),
                                    metric=metric)
        for t in range(Q.shape[0]):
            assert len(set(ids[t].tolist())) == 10
            assert np.all(np.diff(ds[t]) >= 0)
            x = X[ids[t]].astype(np.float64)
            q = Q[t].astype(np.float64)
            ref = ((x - q) ** 2).sum(1) if metric == oracle.L2 else -(x * q).sum(1)
            scale = ref if metric == oracle.L2 else np.abs(x * q).sum(1)
            assert np.all(np.abs(ds[t] - ref) <= 1e-5 * scale + 1e-30)


def test_max_iter_cap_counted():
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 1000)
    Q = synth.query_vectors(w, 5)
    G, _ = oracle.knn_graph(X, 8)
    ids, ds, st = oracle.search(X, G, Q, oracle.make_params(k=5, L=16, T=1, S=4, max_iter=3, seed=1))
    assert (st["iters"] == 3).all() and (st["cap_hits"] == 1).all()


# ---------------------------------------------------------------- K10 prune
def test_prune_hand_examples():
    """Derivation of example 2 (knn rows 0:[1,2,3] 1:[0,2,3] 2:[0,1,3] 3:[0,1,2], R=2):
    detours -- node 2: y=1 (j=1) is reachable as 0->1 with rank 0 < 1 -> count 1;
    node 3: y=1 via 0 (count 1), y=2 via 0 and via 1 (count 2).  Pruned
    rows = first R by (count, j): [1,2] [0,2] [0,3] [0,1].  Reverse lists by
    (rank, src): Rev0=[1,2], Rev1=[0,3], Rev2=[0,1], Rev3=[2].  Output = first
    R/2 pruned + reverse (skip dups) + rest: [1,2] [0,3] [0,1] [0,2]."""
    g = _gold("prune_hand.json")
    for ex in g["examples"]:
        knn = np.array(ex["knn"], np.uint32)
        out, pr = oracle.prune(knn, ex["R"], want_pruned=True)
        np.testing.assert_array_equal(pr, np.array(ex["expect_pruned"]))
        np.testing.assert_array_equal(out, np.array(ex["expect_out"]))


def test_prune_invariants():
    X = synth.base_vectors(synth.WORKLOADS["C1"], 1500)
    knn, _ = oracle.knn_graph(X, 32)
    out, pr = oracle.prune(knn, 16, want_pruned=True)
    n = X.shape[0]
    for x in range(n):
        row = [int(v) for v in out[x] if v != SENT]
        assert len(row) == len(set(row)) == 16
        assert x not in row
        assert set(pr[x].tolist()) <= set(knn[x].tolist())
        # every edge is a kNN edge of x or a reverse of a pruned edge into x
        for y in row:
            assert y in set(knn[x].tolist()) or x in set(pr[y].tolist())


def test_generator_acceptance_C1_small():
    """DESIGN.md §4 acceptance: the C1-family kNN graph is one weak component
    and the iteration spread premise (max/mean >= 1.3) holds."""
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 4000)
    Q = synth.query_vectors(w, 60)
    G, _ = oracle.knn_graph(X, 32)
    n = X.shape[0]
    # weak connectivity by union-find over undirected edges
    parent = np.arange(n)

    def find(a):
        while parent[a] != a:
            parent[a] = parent[parent[a]]
            a = parent[a]
        return a
    for u in range(n):
        for v in G[u]:
            ru, rv = find(u), find(int(v))
            if ru != rv:
                parent[ru] = rv
    assert len({find(u) for u in range(n)}) == 1
    ids, ds, st = oracle.search(X, G, Q, oracle.make_params(k=10, L=16, T=1, S=32, seed=0))
    assert st["iters"].max() / st["iters"].mean() >= 1.3


# ---------------------------------------------------------------- COSINE (f3, R29)
def test_cosine_hand_values():
    """-(q.x)/(|q||x|): parallel -1, orthogonal 0, opposite +1, (3,4).(4,3) = 24/25."""
    q = np.array([1, 0], np.float32)
    assert oracle.distance(q, np.array([2, 0], np.float32), oracle.COSINE) == -1.0
    assert oracle.distance(q, np.array([0, 3], np.float32), oracle.COSINE) == 0.0
    assert oracle.distance(q, np.array([-5, 0], np.float32), oracle.COSINE) == 1.0
    assert oracle.distance(np.array([3, 4], np.float32), np.array([4, 3], np.float32),
                           oracle.COSINE) == np.float32(-0.96)
    assert oracle.distance(q, np.zeros(2, np.float32), oracle.COSINE) == 0.0


def test_cosine_angles_closed_form():
    """q = (cos a, sin a), x = r (cos b, sin b), any r > 0: -cos(a - b)."""
    rng = np.random.default_rng(3)
    for _ in range(200):
        a, b = rng.uniform(-np.pi, np.pi, 2)
        r = rng.uniform(0.01, 100.0)
        q = np.array([np.cos(a), np.sin(a)], np.float32)
        x = (r * np.array([np.cos(b), np.sin(b)])).astype(np.float32)
        assert abs(oracle.distance(q, x, oracle.COSINE) + np.cos(a - b)) <= 1e-6


def test_cosine_bruteforce_circle_order():
    """n points on the unit circle at angles 2 pi i / n, each scaled by its own
    random radius (cosine ignores it); the k nearest of a query at angle
    theta are the k smallest angular gaps, a closed-form order."""
    n, k = 360, 9
    rng = np.random.default_rng(4)
    ang = 2 * np.pi * np.arange(n) / n
    rad = rng.uniform(0.1, 10.0, n)
    X = np.stack([rad * np.cos(ang), rad * np.sin(ang)], 1).astype(np.float32)
    X = np.concatenate([X, np.zeros((n, 2), np.float32)], 1)  # d = 4 (row alignment)
    thetas = 2 * np.pi * (np.arange(20) + 0.3) / 20   # never equidistant from two points
    Q = np.stack([np.cos(thetas), np.sin(thetas), np.zeros(20), np.zeros(20)], 1).astype(np.float32)
    ids, ds = oracle.brute_force(X, Q, k, oracle.COSINE)
    for t, th in enumerate(thetas):
        gap = np.abs((ang - th + np.pi) % (2 * np.pi) - np.pi)
        assert set(ids[t].tolist()) == set(np.argsort(gap)[:k].tolist())
        np.testing.assert_allclose(ds[t], -np.cos(np.sort(gap)[:k]), atol=1e-6)


def test_cosine_search_exhaustive_equals_bruteforce():
    """L >= n on a connected graph: O2 scores every point, O2 == O1 (COSINE)."""
    n, d = 150, 8
    rng = np.random.default_rng(24)
    X = rng.standard_normal((n, d)).astype(np.float32) * rng.uniform(0.5, 3.0, (n, 1)).astype(np.float32)
    Q = rng.standard_normal((6, d)).astype(np.float32)
    G = synth.random_graph(n, 6, seed=23)
    p = oracle.make_params(k=12, L=n, w=2, off=4, T=2, S=2, max_iter=10 * n, shared_visited=1, seed=5)
    seeds = [oracle.entry_point(5, t, c, j, n) for t in range(6) for c in range(2) for j in range(2)]
    assert _reachable(G, seeds).all()
    ids, ds, st = oracle.search(X, G, Q, p, metric=oracle.COSINE)
    ei, ed = oracle.brute_force(X, Q, 12, oracle.COSINE)
    np.testing.assert_array_equal(ids, ei)
    np.testing.assert_array_equal(ds, ed)
    # and O1 COSINE ranks like -q.x on rows normalised in float64 (numpy)
    Xn = X / np.linalg.norm(X.astype(np.float64), axis=1, keepdims=True)
    for t in range(6):
        ref = -(Xn @ Q[t].astype(np.float64)) / np.linalg.norm(Q[t].astype(np.float64))
        np.testing.assert_allclose(ed[t], np.sort(ref)[:12], atol=1e-6)


# ---------------------------------------------------------------- partitioned kNN build (f4, R30)
def test_knn_partitioned_hand_example():
    """1-d points 0,1,2 | 10,11,12 (d padded to 4); m = 2 -> centres rows 0
    and 3 (x = 0, x = 10); overlap 1 -> clusters {0,1,2}, {3,4,5}; k = 3:
    each point sees only its own cluster (2 neighbours), the 3rd slot is
    padding, unlike the exact kNN whose 3rd neighbour crosses the gap."""
    x = np.array([0, 1, 2, 10, 11, 12], np.float32)
    X = np.zeros((6, 4), np.float32)
    X[:, 0] = x
    ids, ds = oracle.knn_partitioned(X, 3, 2, 1)
    assert ids[0].tolist() == [1, 2, oracle.SENTINEL] and ds[0].tolist()[:2] == [1.0, 4.0]
    assert ids[1].tolist()[:2] == [0, 2] and ds[1].tolist()[:2] == [1.0, 1.0]   # tie by id
    assert ids[5].tolist()[:2] == [4, 3] and ds[5].tolist()[:2] == [1.0, 4.0]
    assert np.isinf(ds[:, 2]).all()
    ei, ed = oracle.knn_graph(X, 3)
    assert ei[2].tolist() == [1, 0, 3] and ed[2, 2] == 64.0


def test_knn_partitioned_capacity_and_lloyd_hand_example():
    """m = 5 clusters, overlap c = 1 (4c < m: capacity ceil(2cn/m) = 4), n = 10,
    1-d points by id x = 7 16 3 10 4 11 29 9 22 13 (d padded to 4), k = 3.
    Initial centres = rows 0,2,4,6,8 = 7 3 4 29 22.
    Lloyd 1 (sample = all rows; nearest centre, ties to the lower index):
      7,10,11,9,13 -> c0; 16,22 -> c4; 3 -> c1; 4 -> c2; 29 -> c3
      => centres 10 3 4 29 19.  Lloyd 2: same assignment (7 ties c0/c2 at 9
      -> c0) => converged.
    Capacity pass in id order, P = min(m, 4c+4) = 5 preferences:
      c0 takes ids 0 (7), 3 (10), 5 (11), 7 (9) -> full; id 9 (13) prefers c0
      (36) but it is full -> c4 (19, 36 < c2's 81).  Clusters: c0 {0,3,5,7},
      c1 {2}, c2 {4}, c3 {6}, c4 {1,8,9}.
    Without Lloyd, id 9 would go to c2 (tie 81 with c4 at 22, lower index);
    without the capacity, to c0 -- both change row 9 below."""
    x = np.array([7, 16, 3, 10, 4, 11, 29, 9, 22, 13], np.float32)
    X = np.zeros((10, 4), np.float32)
    X[:, 0] = x
    ids, ds = oracle.knn_partitioned(X, 3, 5, 1)
    S = oracle.SENTINEL
    assert ids[9].tolist() == [1, 8, S] and ds[9].tolist()[:2] == [9.0, 81.0]     # c4: 16, 22
    assert ids[1].tolist() == [9, 8, S] and ds[1].tolist()[:2] == [9.0, 36.0]
    assert ids[0].tolist() == [7, 3, 5] and ds[0].tolist() == [4.0, 9.0, 16.0]    # c0: 9, 10, 11
    assert ids[7].tolist() == [3, 0, 5] and ds[7].tolist() == [1.0, 4.0, 4.0]     # tie 4: id order
    for i in (2, 4, 6):                                                           # singletons
        assert ids[i].tolist() == [S, S, S] and np.isinf(ds[i]).all()


@pytest.mark.parametrize("metric", [oracle.L2, oracle.IP])
def test_knn_partitioned_reduces_to_exact(metric):
    """m = 1 (one cluster = everything) and overlap = m (every point in
    every cluster) both reduce to the exact kNN graph (O1, self excluded)."""
    X = synth.lattice(120, 8, seed=31, metric=metric)
    ei, ed = oracle.knn_graph(X, 7, metric)
    for m, c in ((1, 1), (5, 5)):
        ids, ds = oracle.knn_partitioned(X, 7, m, c, metric)
        np.testing.assert_array_equal(ids, ei)
        np.testing.assert_array_equal(ds, ed)


def test_knn_partitioned_entries_are_true_neighbours():
    """Any m: every entry is a real point != self with its exact distance,
    rows sorted and duplicate-free; recall vs the exact graph rises with overlap."""
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 1500)
    ei, _ = oracle.knn_graph(X, 10)
    rec = []
    for c in (1, 3):
        ids, ds = oracle.knn_partitioned(X, 10, 12, c)
        for i in range(0, 1500, 37):
            real = ids[i][ids[i] != oracle.SENTINEL]
            assert i not in real.tolist() and len(set(real.tolist())) == len(real)
            ref = ((X[real].astype(np.float64) - X[i]) ** 2).sum(1)
            np.testing.assert_allclose(ds[i, :len(real)], ref, rtol=1e-5)
            assert np.all(np.diff(ds[i, :len(real)]) >= 0)
        rec.append(oracle.recall(ids, ei, 10))
    assert rec[1] > rec[0] and rec[1] > 0.8, rec


# ---------------------------------------------------------------- refinement round (f4, R33)
def _line_lists(n, k=2):
    """1-d points x_i = i (d padded to 4); input lists in[p] = [p+1, p+3]
    (distances 1, 9), SENTINEL past the end."""
    X = np.zeros((n, 4), np.float32)
    X[:, 0] = np.arange(n)
    ids = np.full((n, k), SENT, np.uint32)
    ds = np.full((n, k), np.inf, np.float32)
    for p in range(n):
        row = [(float((q - p) ** 2), q) for q in (p + 1, p + 3) if q < n]
        for e, (dd, q) in enumerate(row):
            ids[p, e], ds[p, e] = q, dd
    return X, ids, ds


def test_knn_refine_hand_example():
    """k = 2, fan = 2, in[p] = [p+1, p+3].  For p <= 5: the neighbours' lists
    are in[p+1] = [p+2, p+4] and in[p+3] = [p+4, p+6], so the candidates are
    p+2, p+4, p+6 at 4, 16, 36; merged with (p+1: 1, p+3: 9) the first two are
    p+1, p+2 at 1, 4.  A second round finds nothing closer (the lists only
    point forward: p-1, as close as p+1, is never reached)."""
    X, ids, ds = _line_lists(12)
    o1, d1 = oracle.knn_refine(X, ids, ds, fan=2, rounds=1)
    for p in range(6):
        assert o1[p].tolist() == [p + 1, p + 2] and d1[p].tolist() == [1.0, 4.0]
    o2, d2 = oracle.knn_refine(X, ids, ds, fan=2, rounds=2)
    np.testing.assert_array_equal(o2[:6], o1[:6])


@pytest.mark.parametrize("metric", [oracle.L2, oracle.IP])
def test_knn_refine_exact_list_is_a_fixed_point(metric):
    """An exact kNN list cannot be improved: refinement returns it unchanged."""
    X = synth.lattice(400, 16, seed=61, metric=metric)
    ei, ed = oracle.knn_graph(X, 12, metric)
    for fan in (1, 4, 12):
        ri, rd = oracle.knn_refine(X, ei, ed, fan=fan, rounds=1, metric=metric)
        np.testing.assert_array_equal(ri, ei)
        np.testing.assert_array_equal(rd, ed)


def test_knn_refine_monotone_and_improves_partitioned_lists():
    """From the partitioned lists (overlap 2, so lists cross partition
    borders): every row's k-th distance never grows, all entries are true
    distances, and recall vs the exact graph rises."""
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 1500)
    ei, _ = oracle.knn_graph(X, 10)
    pi, pd = oracle.knn_partitioned(X, 10, 12, 2)   # overlap 2: lists link the partitions
    ri, rd = oracle.knn_refine(X, pi, pd, fan=8, rounds=1)
    assert np.all(rd[:, -1] <= pd[:, -1])
    for i in range(0, 1500, 53):
        real = ri[i][ri[i] != SENT]
        ref = ((X[real].astype(np.float64) - X[i]) ** 2).sum(1)
        np.testing.assert_allclose(rd[i, :len(real)], ref, rtol=1e-5)
        assert i not in real.tolist() and len(set(real.tolist())) == len(real)
    assert oracle.recall(ri, ei, 10) > oracle.recall(pi, ei, 10) + 0.05


def test_knn_refine_reverse_hand_example():
    """R35 on the same lines: in[p] = [p+1, p+3], fan = 2.  p's reverse pairs
    are (0, p-1) (in[p-1] = [p, p+2]) and (1, p-3) (in[p-3] = [p-2, p]), so
    rev(p) = [p-1, p-3]: p-1 (at 1) becomes a candidate, which the forward-
    only round never reaches, and for 3 <= p <= 5 the first two are p-1, p+1
    (dist 1 each, id order).  p = 1: rev(1) = [0], first two 0, 2."""
    X, ids, ds = _line_lists(12)
    o, d = oracle.knn_refine(X, ids, ds, fan=2, rounds=1, reverse=True)
    for p in range(3, 6):
        assert o[p].tolist() == [p - 1, p + 1] and d[p].tolist() == [1.0, 1.0], (p, o[p], d[p])
    assert o[1].tolist() == [0, 2] and d[1].tolist() == [1.0, 1.0]
    f, _ = oracle.knn_refine(X, ids, ds, fan=2, rounds=1, reverse=False)
    assert all(p - 1 not in f[p].tolist() for p in range(1, 6))


@pytest.mark.parametrize("metric", [oracle.L2, oracle.IP])
def test_knn_refine_reverse_fixed_point_and_superset(metric):
    """An exact list is a fixed point of R35 too; and R35's candidate set
    contains R33's, so every row's sorted distances are elementwise <= the
    forward-only round's (first k of a superset)."""
    X = synth.lattice(400, 16, seed=61, metric=metric)
    ei, ed = oracle.knn_graph(X, 12, metric)
    ri, rd = oracle.knn_refine(X, ei, ed, fan=4, rounds=1, metric=metric, reverse=True)
    np.testing.assert_array_equal(ri, ei)
    np.testing.assert_array_equal(rd, ed)
    pi, pd = oracle.knn_partitioned(X, 12, 8, 2, metric)
    fi, fd = oracle.knn_refine(X, pi, pd, fan=6, rounds=1, metric=metric)
    bi, bd = oracle.knn_refine(X, pi, pd, fan=6, rounds=1, metric=metric, reverse=True)
    assert np.all(bd <= fd)
    assert oracle.recall(bi, ei, 12) >= oracle.recall(fi, ei, 12)
