"""Graph-build contraction A/B (GPU box): the screened exact kNN with the
hand-written tcgen05 3xTF32 kernel (default) vs cuBLAS (ALGAS_KNN_GEMM=cublas),
same inputs: wall time of algas_knn and the certificate's fallback rows.

usage: python scripts/knn_gemm_ab.py C2 [nq]
"""
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_chencyzw025_b200 as algas  # noqa: E402
import synth  # noqa: E402

w = synth.WORKLOADS[sys.argv[1]]
nq = int(sys.argv[2]) if len(sys.argv) > 2 else 100_000
X = torch.from_numpy(synth.base_vectors(w)).cuda()
Q = X[:nq].contiguous()
os.environ["ALGAS_KNN_MODE"] = "screened"
res = {}
for name, env in (("tcgen05", None), ("cublas", "cublas"), ("tcgen05_again", None)):
    if env:
        os.environ["ALGAS_KNN_GEMM"] = env
    else:
        os.environ.pop("ALGAS_KNN_GEMM", None)
    algas.knn_last_stats()
    torch.cuda.synchronize()
    t0 = time.time()
    ids, ds = algas.knn(X, Q, w.knn_degree, w.metric, self_base=0)
    torch.cuda.synchronize()
    el = time.time() - t0
    sc, fb = algas.knn_last_stats()
    res[name] = (ids.cpu().numpy(), el, sc, fb)
    print(json.dumps({"gemm": name, "n": w.n, "nq": nq, "k": w.knn_degree, "seconds": round(el, 3),
                      "rows_screened": sc, "fallback_rows": fb}), flush=True)
print(json.dumps({"identical_ids": bool(np.array_equal(res["tcgen05"][0], res["cublas"][0]))}))
