"""GPU parity for the partitioned approximate kNN build (
DESIGN.md R30): algas_knn_partitioned against oracle.knn_partitioned on the
same seeded inputs -- bit-exact on integer-lattice data (fp32 sums exact in
any order), ids exact and distances within 1e-5 (relative) on float data."""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_chencyzw025_b200 as algas
import synth

pytestmark = pytest.mark.gpu


def _bits(a):
    return (np.asarray(a, np.float32) + np.float32(0.0)).view(np.uint32)


@pytest.mark.parametrize("metric", [algas.L2, algas.IP])
@pytest.mark.parametrize("m,c", [(1, 1), (7, 1), (16, 2), (9, 9)])
def test_knn_partitioned_lattice_bit_exact(metric, m, c):
    X = synth.lattice(700, 32, seed=41, metric=metric)
    gi, gd = algas.knn_partitioned(X, 12, m, c, metric)
    oi, od = oracle.knn_partitioned(X, 12, m, c, metric)
    np.testing.assert_array_equal(gi, oi)
    np.testing.assert_array_equal(_bits(gd), _bits(od))


def test_knn_partitioned_float_matches_oracle():
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 3000)
    gi, gd = algas.knn_partitioned(X, 16, 10, 2)
    oi, od = oracle.knn_partitioned(X, 16, 10, 2)
    same = (gi == oi).mean()
    assert same > 0.995, same          # near-ties may swap under fp32 rounding order
    np.testing.assert_allclose(gd, od, rtol=1e-5, atol=1e-6)


def test_build_graph_partitioned_search_recall():
    """The partitioned graph serves the search nearly as well as the exact one."""
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 8000)
    Q = synth.query_vectors(w, 200)
    ti, _ = oracle.brute_force(X, Q, 10)
    p = algas.default_params(k=10, itopk=64, width=4, offset_beam=1, n_seeds=16, ctas_per_query=1,
                             threads_per_cta=256, seed=3)
    ge = algas.build_graph(X, 32)
    gp = algas.build_graph_partitioned(X, 32, n_clusters=16, overlap=2)
    assert gp.shape == ge.shape and (gp < X.shape[0]).mean() > 0.99
    re = oracle.recall(algas.Index(X, ge).search(Q, params=p)["ids"], ti, 10)
    rp = oracle.recall(algas.Index(X, gp).search(Q, params=p)["ids"], ti, 10)
    assert rp >= re - 0.02, (rp, re)


def test_knn_partitioned_rejects():
    X = np.zeros((10, 8), np.float32)
    for m, c in ((0, 1), (11, 1), (4, 5)):
        with pytest.raises(algas.AlgasError):
            algas.knn_partitioned(X, 3, m, c)


def test_build_graph_partitioned_short_clusters_completed():
    """Many clusters with overlap 1: some hold <= knn_degree points, their
    rows come back short from algas_knn_partitioned; the graph builder
    completes them (no sentinel reaches the prune, every row is full)."""
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 3000)
    ki, _ = algas.knn_partitioned(X, 48, 200, 1)
    assert (ki == algas.SENTINEL).any()
    g = algas.build_graph_partitioned(X, 24, n_clusters=200, overlap=1, knn_degree=48)
    assert (g < X.shape[0]).mean() > 0.999
    assert not (g == np.arange(X.shape[0])[:, None]).any()


# ------------------------------------------------------------------ refinement round (R33)
@pytest.mark.parametrize("metric", [algas.L2, algas.IP])
@pytest.mark.parametrize("fan,rounds", [(4, 1), (12, 2)])
def test_knn_refine_lattice_bit_exact(metric, fan, rounds):
    """algas_knn_refine == oracle.knn_refine bit for bit on lattice data,
    from the (oracle's) partitioned lists."""
    X = synth.lattice(900, 32, seed=43, metric=metric)
    pi, pd = oracle.knn_partitioned(X, 16, 9, 2, metric)
    gi, gd = algas.knn_refine(X, pi, pd, fan=fan, rounds=rounds, metric=metric)
    oi, od = oracle.knn_refine(X, pi, pd, fan=fan, rounds=rounds, metric=metric)
    np.testing.assert_array_equal(gi, oi)
    np.testing.assert_array_equal(_bits(gd), _bits(od))


def test_knn_refine_hand_example_gpu():
    """The oracle's hand-worked example (tests/test_oracle.py) on the GPU."""
    from test_oracle import _line_lists
    X, ids, ds = _line_lists(12)
    gi, gd = algas.knn_refine(X, ids, ds, fan=2, rounds=1)
    for p in range(6):
        assert gi[p].tolist() == [p + 1, p + 2] and gd[p].tolist() == [1.0, 4.0]


def test_knn_refine_raises_recall_float():
    """Float data: one round from partitioned lists raises kNN recall; every
    entry is a true distance (1e-5) and rows stay sorted and duplicate-free."""
    w = synth.WORKLOADS["C1"]
    X = synth.base_vectors(w, 6000)
    ei, _ = oracle.knn_graph(X, 16)
    pi, pd = algas.knn_partitioned(X, 16, 24, 2)
    ri, rd = algas.knn_refine(X, pi, pd, fan=16, rounds=1)
    assert oracle.recall(ri, ei, 16) > oracle.recall(pi, ei, 16) + 0.05
    assert np.all(rd[:, -1] <= pd[:, -1])
    for i in range(0, 6000, 97):
        real = ri[i][ri[i] != algas.SENTINEL]
        assert i not in real.tolist() and len(set(real.tolist())) == len(real)
        ref = ((X[real].astype(np.float64) - X[i]) ** 2).sum(1)
        np.testing.assert_allclose(rd[i, :len(real)], ref, rtol=1e-5)
        assert np.all(np.diff(rd[i, :len(real)]) >= 0)


# ------------------------------------------------------------------ reverse-neighbour rounds (R35)
@pytest.mark.parametrize("metric", [algas.L2, algas.IP])
@pytest.mark.parametrize("fan,rounds", [(4, 1), (8, 2)])
def test_knn_refine_reverse_lattice_bit_exact(metric, fan, rounds):
    """algas_knn_refine with reverse neighbours == oracle.knn_refine(reverse)
    bit for bit on lattice data, from the (oracle's) partitioned lists."""
    X = synth.lattice(900, 32, seed=47, metric=metric)
    pi, pd = oracle.knn_partitioned(X, 16, 9, 2, metric)
    gi, gd = algas.knn_refine(X, pi, pd, fan=fan, rounds=rounds, metric=metric, reverse=True)
    oi, od = oracle.knn_refine(X, pi, pd, fan=fan, rounds=rounds, metric=metric, reverse=True)
    np.testing.assert_array_equal(gi, oi)
    np.testing.assert_array_equal(_bits(gd), _bits(od))


def test_knn_refine_reverse_hand_example_gpu():
    """The oracle's R35 hand example: p-1 is reached through the reverse list."""
    from test_oracle import _line_lists
    X, ids, ds = _line_lists(12)
    gi, gd = algas.knn_refine(X, ids, ds, fan=2, rounds=1, reverse=True)
    for p in range(3, 6):
        assert gi[p].tolist() == [p - 1, p + 1] and gd[p].tolist() == [1.0, 1.0]
