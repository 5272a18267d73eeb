"""Generator calibration (GPU box): for a few mixture variants of a workload,
build the kNN(+prune) graph and report recall@k at several L, iteration
spread and distance evaluations, to pick a recipe whose recall curve spans
0.90-0.99 over L in [32, 256] like the real datasets.

usage: python scripts/calibrate.py C2 [n]
"""
import dataclasses
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


def recall(found, truth, k):
    hits = 0
    for f, t in zip(found[:, :k], truth[:, :k]):
        hits += len(set(f.tolist()) & set(t.tolist()))
    return hits / float(truth.shape[0] * k)


def main():
    cfg = sys.argv[1]
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    base = synth.WORKLOADS[cfg]
    variants = json.loads(sys.argv[3]) if len(sys.argv) > 3 else [
        dict(rank=24, noise=0.3), dict(rank=32, noise=0.5), dict(rank=48, noise=0.5, spread=3.0),
        dict(rank=32, noise=1.0, spread=4.0)]
    out = []
    for v in variants:
        w = dataclasses.replace(base, n=n or base.n, **v)
        t0 = time.time()
        X = synth.base_vectors(w)
        Q = synth.query_vectors(w, 2000)
        Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
        knn, _ = algas.knn(Xd, Xd, w.knn_degree, w.metric, self_base=0)
        G = algas.prune(knn, w.degree) if w.prune else knn[:, :w.degree].contiguous()
        ti, _ = algas.knn(Xd, Qd, w.k, w.metric)
        ti = ti.cpu().numpy().view(np.uint32)
        G = G.cpu().numpy().view(np.uint32)
        idx = algas.Index(Xd, G, w.metric)
        res = dict(variant=v, build_s=time.time() - t0, rows=[])
        for L in ([16, 32, 64, 128, 256] if w.k <= 10 else [100, 128, 256, 512]):
            p = algas.default_params(k=w.k, itopk=L, width=4, offset_beam=max(1, L // 4), ctas_per_query=1,
                                     threads_per_cta=64, slots=64, seed=1, hash_bits=14)
            r = idx.search_dynamic(Qd, p)
            it = r["stats"]["iters"].astype(np.float64)
            res["rows"].append(dict(L=L, recall=recall(r["ids"], ti, w.k), iters=it.mean(),
                                    spread=it.max() / it.mean(), evals=float(r["stats"]["dist_evals"].mean())))
        print(json.dumps(res), flush=True)
        out.append(res)
        del idx
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    json.dump(out, open(os.path.join(ROOT, "gpurun_out", f"calibrate_{cfg}.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
