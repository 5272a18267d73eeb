"""Workload driver for ncu captures (GPU box): build a BASELINE workload, then
launch the search kernels a bounded number of times with fixed parameters.

usage: ncu ... python scripts/profile_run.py C2 --nq 3000 --itopk 64 --width 4 --threads 256 --ctas 1 --slots 32
       [--batch-kernel] [--reps 2]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_chencyzw025_b200 as algas  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg")
    ap.add_argument("--nq", type=int, default=3000)
    ap.add_argument("--itopk", type=int, default=64)
    ap.add_argument("--width", type=int, default=4)
    ap.add_argument("--offset", type=int, default=-1)
    ap.add_argument("--visited", default="private", choices=["private", "shared"])
    ap.add_argument("--threads", type=int, default=256)
    ap.add_argument("--ctas", type=int, default=1)
    ap.add_argument("--slots", type=int, default=32)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--batch-kernel", action="store_true")
    ap.add_argument("--load", default=None, help="directory with X.npy / G.npy (bench.py's built index)")
    ap.add_argument("--params-json", default=None, help="algas_params fields (overrides the flags)")
    a = ap.parse_args()
    w = synth.WORKLOADS[a.cfg]
    Q = synth.query_vectors(w, a.nq)
    Qd = torch.from_numpy(Q).cuda()
    if a.load:
        Xd = torch.from_numpy(np.load(os.path.join(a.load, "X.npy"))).cuda()
        G = np.load(os.path.join(a.load, "G.npy"))
    else:
        Xd = torch.from_numpy(synth.base_vectors(w)).cuda()
        knn, _ = algas.knn(Xd, Xd, w.knn_degree, w.metric, self_base=0)
        G = algas.prune(knn, w.degree) if w.prune else knn[:, :w.degree].contiguous()
        del knn
    idx = algas.Index(Xd, G, w.metric)
    if a.params_json:
        p = algas.default_params(**json.loads(a.params_json))
    else:
        p = algas.default_params(k=w.k, itopk=a.itopk, width=a.width,
                                 offset_beam=a.offset if a.offset > 0 else max(1, a.itopk // 4),
                                 ctas_per_query=a.ctas, threads_per_cta=a.threads, slots=a.slots, seed=1,
                                 visited_mode=1 if a.visited == "shared" else 0)
    out = []
    for _ in range(a.reps):
        if a.batch_kernel:
            r = idx.search(Qd, params=p)
        else:
            r = idx.search_dynamic(Qd, p)
        st = r["stats"]
        out.append(dict(kernel_ms=r["info"].kernel_ms, parents=float(st["parents"].mean()),
                        dist_evals=float(st["dist_evals"].mean()), iters=float(st["iters"].mean())))
    print(json.dumps(dict(cfg=a.cfg, nq=a.nq, itopk=p.itopk, width=p.width, offset=p.offset_beam,
                          threads=p.threads_per_cta, ctas=p.ctas_per_query,
                          slots=a.slots, runs=out)))


if __name__ == "__main__":
    main()
