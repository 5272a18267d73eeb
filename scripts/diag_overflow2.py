"""Reproduce the full-size test sequence at C2 and report which queries flag a
visited-table overflow (GPU box)."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_chencyzw025_b200 as algas  # noqa: E402
import synth  # noqa: E402

w = synth.WORKLOADS["C2"]
X = torch.from_numpy(synth.base_vectors(w)).cuda()
Q = torch.from_numpy(synth.query_vectors(w, 2000)).cuda()
knn, _ = algas.knn(X, X, w.knn_degree, w.metric, self_base=0)
G = algas.prune(knn, w.degree)
del knn
idx = algas.Index(X, G, w.metric)
POINTS = [(12, 8, 4, 1024, True), (12, 12, 4, 1024, True), (12, 8, 4, 1024, False), (32, 8, 1, 512, False),
          (64, 16, 2, 512, False), (24, 8, 2, 1024, True), (64, 16, 2, 512, False)]
for mode in (None, "1"):
    if mode:
        os.environ["ALGAS_NO_STREAM_MERGE"] = mode
    else:
        os.environ.pop("ALGAS_NO_STREAM_MERGE", None)
    for L, wd, T, nt, sh in POINTS:
        for seed in ((1, 2, 3) if sh else (1,)):
            p = algas.default_params(k=10, itopk=L, width=wd, offset_beam=1, ctas_per_query=T, threads_per_cta=nt,
                                     slots=32, n_seeds=32, seed=seed, visited_mode=1 if sh else 0)
            r = idx.search_dynamic(Q, p, tag0=0)
            st = r["stats"]
            bad = np.nonzero(st["overflows"])[0]
            print(f"classic={bool(mode)} L={L} w={wd} T={T} nt={nt} sh={sh} seed={seed}: overflow={r['overflow']} "
                  f"n={len(bad)} hb={r['info'].hash_bits} spills={int((st['spills'] > 0).sum())}", flush=True)
            for q in bad[:3]:
                print("   ", q, {f: int(st[f][q]) for f in ("iters", "max_iters", "parents", "dist_evals", "spills",
                                                           "overflows", "cap_hits", "merges_bitonic", "merges_rank")},
                      flush=True)
