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
