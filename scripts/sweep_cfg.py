"""Recall/QPS sweep of one workload recipe (GPU box), optionally with the
synthetic recipe's noise overridden -- used to calibrate synth/ so each
config is shaped like its dataset.

usage: python scripts/sweep_cfg.py C3 [--noise 0.15] [--n 1000000] [--nq 2000]
"""
import argparse
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg")
    ap.add_argument("--noise", type=float, default=None)
    ap.add_argument("--center-scale", type=float, default=None)
    ap.add_argument("--Ts", default="1,4")
    ap.add_argument("--rank", type=int, default=None)
    ap.add_argument("--n", type=int, default=0)
    ap.add_argument("--nq", type=int, default=2000)
    ap.add_argument("--threads", type=int, default=512)
    a = ap.parse_args()
    w = synth.WORKLOADS[a.cfg]
    if a.noise is not None:
        w = dataclasses.replace(w, noise=a.noise)
    if a.center_scale is not None:
        w = dataclasses.replace(w, center_scale=a.center_scale)
    if a.rank is not None:
        w = dataclasses.replace(w, rank=a.rank)
    n = a.n or w.n
    t0 = time.time()
    X = synth.base_vectors(w, n)
    Q = synth.query_vectors(w, a.nq)
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    knn, _ = algas.knn(Xd, Xd, w.knn_degree, w.metric, self_base=0)
    G = algas.prune(knn, w.degree)
    del knn
    ti, _ = algas.knn(Xd, Qd, w.k, w.metric)
    ti = ti.cpu().numpy().view(np.uint32)
    print(f"{w.name} noise={w.noise} center_scale={w.center_scale} rank={w.rank} n={n}: setup {time.time() - t0:.1f} s", flush=True)
    idx = algas.Index(Xd, G, w.metric)
    for T in (int(x) for x in a.Ts.split(",")):
        vis = 1 if T > 1 else 0
        for L in (32, 64, 128, 256):
            if L < w.k:
                continue
            p = algas.default_params(k=w.k, itopk=L, width=min(16, L), offset_beam=1, ctas_per_query=T,
                                     threads_per_cta=a.threads, slots=32, n_seeds=32, seed=1, visited_mode=vis)
            r = idx.search_dynamic(Qd, p)
            rec = sum(len(set(x.tolist()) & set(y.tolist())) for x, y in zip(r["ids"][:, :w.k], ti[:, :w.k])) / ti[:, :w.k].size
            st = r["stats"]
            print(json.dumps({"T": T, "itopk": L, "recall": round(rec, 4), "qps": round(a.nq / (r["info"].kernel_ms / 1e3)),
                              "steps": float(st["max_iters"].mean()), "evals": float(st["dist_evals"].mean())}), flush=True)


if __name__ == "__main__":
    main()
