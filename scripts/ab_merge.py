"""A/B of the candidate-update paths at the bench operating points
of C2 / C3 / C4 (GPU box): the fused warp-register bitonic merge (default)
against the CTA-wide rank merge (ALGAS_PREFETCH bit 64 disables the fused
path), same parameters, same queries; QPS (kernel events), device p50,
recall, and how many candidate updates each path served.

usage: python scripts/ab_merge.py C4 [C3 ...]  -> JSON lines on stdout
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

# (L, w, T, threads, visited) operating points per config
POINTS = {"C2": [(12, 12, 4, 1024, 1), (64, 16, 1, 512, 0)],
          "C3": [(64, 16, 4, 512, 1), (128, 16, 2, 512, 0)],
          "C4": [(128, 16, 4, 1024, 1), (128, 16, 4, 512, 1), (256, 16, 2, 512, 0)]}


def recall(found, truth, k):
    return float(np.mean([len(set(f[:k].tolist()) & set(t[:k].tolist())) / k for f, t in zip(found, truth)]))


def main():
    for cfg in sys.argv[1:]:
        w = synth.WORKLOADS[cfg]
        X = torch.from_numpy(synth.base_vectors(w)).cuda()
        Q = torch.from_numpy(synth.query_vectors(w, 4000)).cuda()
        knn, _ = algas.knn(X, X, w.knn_degree, w.metric, self_base=0)
        G = algas.prune(knn, w.degree)
        del knn
        truth = algas.knn(X, Q, w.k, w.metric)[0].cpu().numpy().view(np.uint32)
        idx = algas.Index(X, G, w.metric)
        for L, wd, T, nt, vis in POINTS[cfg]:
            p = algas.default_params(k=w.k, itopk=L, width=wd, offset_beam=1, ctas_per_query=T, threads_per_cta=nt,
                                     slots=32, n_seeds=32, seed=1, visited_mode=vis)
            for name, pf in (("bitonic", None), ("rank", "72")):
                if pf is None:
                    os.environ.pop("ALGAS_PREFETCH", None)
                else:
                    os.environ["ALGAS_PREFETCH"] = pf
                idx.search_dynamic(Q, p)  # warm-up
                res = []
                for _ in range(3):
                    r = idx.search_dynamic(Q, p)
                    res.append(r)
                qps = [Q.shape[0] / (r["info"].kernel_ms / 1e3) for r in res]
                st = res[-1]["stats"]
                lat = (st["t_end_ns"] - st["t_start_ns"]) / 1e3
                print(json.dumps({"cfg": cfg, "L": L, "w": wd, "T": T, "threads": nt, "visited": vis, "merge": name,
                                  "qps": round(float(np.median(qps))), "p50_us": round(float(np.percentile(lat, 50)), 1),
                                  "recall": round(recall(res[-1]["ids"], truth, w.k), 4),
                                  "merges_bitonic": float(st["merges_bitonic"].mean()),
                                  "merges_rank": float(st["merges_rank"].mean()),
                                  "cyc_sort_per_iter": float((st["cyc_sort"] / np.maximum(st["iters"], 1)).mean())}),
                      flush=True)
        os.environ.pop("ALGAS_PREFETCH", None)
        del idx, X, Q, G
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
