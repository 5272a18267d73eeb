"""Graph-build timing: exact kNN + prune vs the partitioned
build (algas_build_graph_partitioned, R30) on a workload's
synthetic base set; kNN-graph recall of the partitioned lists on a sample of
rows and search recall@k of both graphs at one fixed search point.

    python scripts/build_timing.py C2 --clusters 64 128 --overlap 2
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch

    import paper_conf_ipps_chencyzw025_b200 as algas
    import synth
    ap = argparse.ArgumentParser()
    ap.add_argument("workload", default="C2")
    ap.add_argument("--clusters", type=int, nargs="+", default=[64, 128])
    ap.add_argument("--overlap", type=int, nargs="+", default=[2])
    ap.add_argument("--refine", type=int, nargs="+", default=[0, 1], help="refinement rounds (DESIGN.md R33)")
    ap.add_argument("--fan", type=int, default=16)
    ap.add_argument("--reverse", action="store_true", help="R35 rounds (reverse neighbours joined)")
    ap.add_argument("--no-exact", action="store_true")
    ap.add_argument("--search-L", type=int, nargs="*", default=[],
                    help="also search each partitioned graph at these L (T=4, 1024 threads, SHARED, w=12/16)")
    ap.add_argument("--nq", type=int, default=2000)
    a = ap.parse_args()
    w = synth.WORKLOADS[a.workload]
    X = synth.base_vectors(w)
    Q = synth.query_vectors(w, a.nq)
    Xd = torch.from_numpy(X).cuda()
    Qd = torch.from_numpy(Q).cuda()
    ti, _ = algas.knn(Xd, Qd, w.k, w.metric)
    ti = ti.cpu().numpy().view(np.uint32)
    sample = np.arange(0, w.n, max(1, w.n // 2000))
    se, _ = algas.knn(Xd, Xd[torch.from_numpy(sample).cuda()], w.knn_degree, w.metric)
    se = se.cpu().numpy().view(np.uint32)  # includes self at column 0 (self_base not applied)
    p = algas.default_params(k=w.k, itopk=64, width=8, offset_beam=1, n_seeds=32, ctas_per_query=1,
                             threads_per_cta=512, seed=3)
    out = {"workload": w.name, "n": w.n, "dim": w.dim, "knn_degree": w.knn_degree, "degree": w.degree}
    if not a.no_exact:
        torch.cuda.synchronize()
        t0 = time.time()
        ge = algas.build_graph(Xd, w.degree, knn_degree=w.knn_degree, metric=w.metric)
        torch.cuda.synchronize()
        out["exact_build_s"] = time.time() - t0
        r = algas.Index(Xd, ge, w.metric).search(Q, params=p)
        out["exact_search_recall"] = float((r["ids"][:, :w.k, None] == ti[:, None, :w.k]).any(2).mean())
        print(json.dumps({"exact_build_s": out["exact_build_s"], "exact_search_recall": out["exact_search_recall"]}),
              flush=True)
    out["partitioned"] = []
    for m in a.clusters:
        for c in a.overlap:
            torch.cuda.synchronize()
            t0 = time.time()
            ids, dd = algas.knn_partitioned(Xd, w.knn_degree, m, c, w.metric)
            torch.cuda.synchronize()
            t_knn = time.time() - t0
            for rounds in a.refine:
                torch.cuda.synchronize()
                t0 = time.time()
                ri, _ = (algas.knn_refine(Xd, ids, dd, fan=a.fan, rounds=rounds, metric=w.metric, reverse=a.reverse)
                          if rounds else (ids, dd))
                torch.cuda.synchronize()
                t_ref = time.time() - t0
                rih = ri.cpu().numpy().view(np.uint32)
                hit = np.mean([len(set(rih[i].tolist()) & set(se[j, 1:].tolist())) / (w.knn_degree - 1)
                               for j, i in enumerate(sample)])
                t0 = time.time()
                gp = algas.build_graph_partitioned(Xd, w.degree, m, c, knn_degree=w.knn_degree, metric=w.metric,
                                                   refine_fan=-a.fan if a.reverse else a.fan, refine_rounds=rounds)
                torch.cuda.synchronize()
                t_build = time.time() - t0
                rp = algas.Index(Xd, gp, w.metric).search(Q, params=p)
                rec = float((rp["ids"][:, :w.k, None] == ti[:, None, :w.k]).any(2).mean())
                curve = []
                idx_p = algas.Index(Xd, gp, w.metric)
                for L in a.search_L:
                    ps = algas.default_params(k=w.k, itopk=L, width=min(L, 12 if L <= 32 else 16), offset_beam=1,
                                              n_seeds=32, ctas_per_query=4, threads_per_cta=1024, slots=32, seed=3,
                                              visited_mode=1)
                    rr = idx_p.search_dynamic(Qd, ps)
                    curve.append([L, float((rr["ids"][:, :w.k, None] == ti[:, None, :w.k]).any(2).mean()),
                                  round(a.nq / (rr["info"].kernel_ms / 1e3))])
                out["partitioned"].append({"clusters": m, "overlap": c, "refine_rounds": rounds, "fan": a.fan,
                                           "reverse": a.reverse,
                                           "knn_s": t_knn, "refine_s": t_ref, "build_s": t_build,
                                           "knn_graph_recall_sample": float(hit), "search_recall": rec,
                                           "search_T4_L_recall_qps": curve})
                print(json.dumps(out["partitioned"][-1]), flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
