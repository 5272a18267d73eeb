"""Bounded runs of the persistent ring path (and the device-queue and batch
paths) for compute-sanitizer (racecheck / synccheck / memcheck).

The server runs as a bounded session (algas_server_create_deferred + staged
queries + algas_server_start(quit_when_idle)): the sanitizer serialises the
launch, so the host cannot submit while the kernel runs.  Lattice data (C1
shape, exact) so every result is also checked against the oracle.

usage: compute-sanitizer --tool racecheck python scripts/sanitize_ring.py [threads]
"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import paper_conf_ipps_chencyzw025_b200 as algas  # noqa: E402
import synth  # noqa: E402


def main():
    import torch
    nt = int(sys.argv[1]) if len(sys.argv) > 1 else 128
    X = synth.lattice(2000, 128, seed=42)
    Q = synth.lattice(12, 128, seed=43)
    G, _ = oracle.knn_graph(X, 32)
    idx = algas.Index(X, G)
    for vis, T, mirror in ((0, 2, 0), (1, 4, 0), (1, 4, 1)):
        p = algas.default_params(k=10, itopk=32, width=4, offset_beam=1, n_seeds=16, ctas_per_query=T,
                                 threads_per_cta=nt, slots=6, seed=1, visited_mode=vis, state_mirror=mirror,
                                 watchdog_ms=-1)  # a sanitized kernel runs orders of magnitude slower
        got = {}
        with algas.Server(idx, p, deferred=True) as srv:
            for t in range(Q.shape[0]):
                assert srv.submit(Q[t], tag=t)
            srv.start(quit_when_idle=True)
            t0 = time.time()
            while len(got) < Q.shape[0] and time.time() - t0 < 600:
                for t, i, _d, _s in zip(*srv.poll(32)):
                    got[int(t)] = i
        assert len(got) == Q.shape[0], len(got)
        d = idx.search_dynamic(torch.from_numpy(Q).cuda(), p)
        if vis == 0:
            oi, od, _ = oracle.search(X, G, Q, oracle.make_params(k=10, L=32, w=4, off=1, T=T, S=16, seed=1))
            assert all(np.array_equal(got[t], oi[t]) for t in got), "server != oracle"
            assert np.array_equal(d["ids"], oi), "dynamic != oracle"
            b = idx.search(Q, params=p)
            assert np.array_equal(b["ids"], oi), "batch != oracle"
        print(f"visited_mode={vis} T={T} mirror={mirror} threads={nt}: {len(got)} queries ok", flush=True)
    print("SANITIZE_RUN_OK")


if __name__ == "__main__":
    main()
