"""Which queries report a visited-table overflow at a C2 point (GPU box)?
Compares the streaming-merge and the classic (ALGAS_NO_STREAM_MERGE) paths."""
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
for L, wd, T, nt, vis in ((64, 16, 2, 512, 0), (12, 12, 4, 1024, 1), (64, 16, 1, 512, 0), (64, 16, 2, 1024, 0)):
    p = algas.default_params(k=10, itopk=L, width=wd, offset_beam=1, ctas_per_query=T, threads_per_cta=nt, slots=32,
                             n_seeds=32, seed=1, visited_mode=vis)
    for env in (None, "1"):
        if env:
            os.environ["ALGAS_NO_STREAM_MERGE"] = env
        else:
            os.environ.pop("ALGAS_NO_STREAM_MERGE", None)
        r = idx.search_dynamic(Q, p)
        st = r["stats"]
        bad = np.nonzero(st["overflows"])[0]
        print(f"L={L} w={wd} T={T} nt={nt} vis={vis} classic={bool(env)}: overflow={r['overflow']} "
              f"n_over={len(bad)} spills={int((st['spills'] > 0).sum())} hash_bits={r['info'].hash_bits} "
              f"kernel_ms={r['info'].kernel_ms:.2f} mb={st['merges_bitonic'].mean():.1f} mr={st['merges_rank'].mean():.1f} "
              f"first={bad[:5].tolist()}", flush=True)
