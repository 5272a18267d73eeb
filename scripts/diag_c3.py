"""Locate the C3 (960-d) recall failure: kNN rows vs torch fp64, search recall, at growing n."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_chencyzw025_b200 as algas  # noqa: E402
import synth  # noqa: E402

w = synth.WORKLOADS["C3"]
for n in [int(x) for x in sys.argv[1:]]:
    X = synth.base_vectors(w, n)
    Q = synth.query_vectors(w, 500)
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    for mode in ("screened", "direct"):
        os.environ["ALGAS_KNN_MODE"] = mode
        ti, td = algas.knn(Xd, Qd[:50], 10, 0)
        ti = ti.cpu().numpy().view(np.uint32)
        d64 = torch.cdist(Qd[:50].double(), Xd.double()) ** 2
        ref = torch.topk(d64, 10, largest=False).indices.cpu().numpy()
        ov = np.mean([len(set(a.tolist()) & set(b.tolist())) / 10 for a, b in zip(ti, ref)])
        print(f"n={n} knn[{mode}] overlap with fp64 exact: {ov:.3f}; stats {algas.knn_last_stats()}", flush=True)
    os.environ.pop("ALGAS_KNN_MODE")
    knn, _ = algas.knn(Xd, Xd, w.knn_degree, w.metric, self_base=0)
    rows = np.arange(0, n, n // 7)[:7]
    kr = knn[torch.from_numpy(rows).cuda()].cpu().numpy().view(np.uint32)
    d64 = torch.cdist(Xd[torch.from_numpy(rows).cuda()].double(), Xd.double()) ** 2
    d64[torch.arange(len(rows)), torch.from_numpy(rows).cuda()] = float("inf")
    ref = torch.topk(d64, w.knn_degree, largest=False).indices.cpu().numpy()
    ov = np.mean([len(set(a.tolist()) & set(b.tolist())) / w.knn_degree for a, b in zip(kr, ref)])
    print(f"n={n} graph knn rows overlap: {ov:.3f}", flush=True)
    G = algas.prune(knn, w.degree)
    del knn
    ti, _ = algas.knn(Xd, Qd, 10, 0)
    ti = ti.cpu().numpy().view(np.uint32)
    idx = algas.Index(Xd, G, 0)
    for nt in (256, 512):
        p = algas.default_params(k=10, itopk=64, width=8, offset_beam=1, ctas_per_query=1, threads_per_cta=nt, slots=32,
                                 n_seeds=32, seed=1)
        r = idx.search_dynamic(Qd, p)
        rec = np.mean([len(set(a.tolist()) & set(b.tolist())) / 10 for a, b in zip(r["ids"], ti)])
        rs = idx.search(Q, params=p)
        rec2 = np.mean([len(set(a.tolist()) & set(b.tolist())) / 10 for a, b in zip(rs["ids"], ti)])
        print(f"n={n} threads={nt} search recall dynamic {rec:.3f} batch {rec2:.3f}", flush=True)
    del idx, Xd
    torch.cuda.empty_cache()
