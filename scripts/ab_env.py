"""A/B of search-kernel switches at the bench operating points (GPU box):
each variant is a set of environment switches read per call by make_plan
(ALGAS_GATHER_MODE, ALGAS_PREFETCH); same parameters and queries.  Prints
QPS (kernel events, median of 3), device p50, recall and the per-step phase
cycles (thread 0 of each CTA: select / gather+filter / distance / merge).

usage: python scripts/ab_env.py C2 "GM=0" "GM=3" "GM=3,SR=2" ...
       (GM = ALGAS_GATHER_MODE, PF = ALGAS_PREFETCH, SR = stage_rows param)
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_chencyzw025_b200 as algas  # noqa: E402
import synth  # noqa: E402

POINTS = {"C2": [(12, 12, 4, 1024, 1), (64, 16, 1, 1024, 0)],
          "C3": [(64, 16, 4, 512, 1)],
          "C4": [(128, 16, 4, 1024, 1)]}


def recall(found, truth, k):
    return float(np.mean([len(set(f[:k].tolist()) & set(t[:k].tolist())) / k for f, t in zip(found, truth)]))


def main():
    cfg, variants = sys.argv[1], sys.argv[2:]
    w = synth.WORKLOADS[cfg]
    X = torch.from_numpy(synth.base_vectors(w)).cuda()
    Q = torch.from_numpy(synth.query_vectors(w, 4000)).cuda()
    knn, _ = algas.knn(X, X, w.knn_degree, w.metric, self_base=0)
    G = algas.prune(knn, w.degree)
    del knn
    truth = algas.knn(X, Q, w.k, w.metric)[0].cpu().numpy().view(np.uint32)
    idx = algas.Index(X, G, w.metric)
    for L, wd, T, nt, vis in POINTS[cfg]:
        for v in variants:
            kv = dict(x.split("=") for x in v.split(",") if x)
            for key, env in (("GM", "ALGAS_GATHER_MODE"), ("PF", "ALGAS_PREFETCH")):
                if key in kv:
                    os.environ[env] = kv[key]
                else:
                    os.environ.pop(env, None)
            p = algas.default_params(k=w.k, itopk=L, width=wd, offset_beam=1, ctas_per_query=T, threads_per_cta=nt,
                                     slots=32, n_seeds=32, seed=1, visited_mode=vis,
                                     stage_rows=int(kv.get("SR", 0)), hash_bits=int(kv.get("HB", 0)))
            try:
                idx.search_dynamic(Q, p)
            except algas.AlgasError as e:
                print(json.dumps({"cfg": cfg, "variant": v, "L": L, "error": str(e)}), flush=True)
                continue
            res = [idx.search_dynamic(Q, p) for _ in range(3)]
            qps = [Q.shape[0] / (r["info"].kernel_ms / 1e3) for r in res]
            st = res[-1]["stats"]
            it = np.maximum(st["iters"] + T, 1).astype(np.float64)
            lat = (st["t_end_ns"] - st["t_start_ns"]) / 1e3
            print(json.dumps({"cfg": cfg, "variant": v, "lib": os.path.basename(algas.build.LIB), "L": L, "w": wd,
                              "T": T, "threads": nt, "visited": vis, "qps": round(float(np.median(qps))),
                              "p50_us": round(float(np.percentile(lat, 50)), 1),
                              "recall": round(recall(res[-1]["ids"], truth, w.k), 4),
                              "steps_per_cta": round(float((st["iters"] / T).mean()), 2),
                              "evals_per_query": round(float(st["dist_evals"].mean()), 1),
                              "cyc_per_step": {ph: round(float((st["cyc_" + ph] / it).mean())) for ph in
                                               ("select", "gather", "dist", "sort")},
                              "hash_bits": res[-1]["info"].hash_bits, "smem": res[-1]["info"].smem_per_cta}),
                  flush=True)
    for env in ("ALGAS_GATHER_MODE", "ALGAS_PREFETCH"):
        os.environ.pop(env, None)


if __name__ == "__main__":
    main()
