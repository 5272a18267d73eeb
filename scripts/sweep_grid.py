"""Operating-point grid sweep (GPU box): for every (T, threads, width, seeds,
visited) the smallest L whose recall@k on a calibration set reaches the
target, then QPS (kernel events, median of 3) / device p50 / p99 on the
measured set.  Prints JSON lines sorted by QPS at the end.

usage: python scripts/sweep_grid.py C2 --T 4,6,8 --threads 512,1024 --width 4,6,8,12 --seeds 8,16,32
"""
import argparse
import itertools
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_chencyzw025_b200 as algas  # noqa: E402
import synth  # noqa: E402

LS = [10, 11, 12, 13, 14, 16, 18, 20, 24, 28, 32, 40, 48, 56, 64, 80, 96, 128, 160, 192, 256, 320, 384, 512]


def recall(found, truth, k):
    return float(np.mean([len(set(f[:k].tolist()) & set(t[:k].tolist())) / k for f, t in zip(found, truth)]))


def main():
    ints = lambda x: [int(v) for v in x.split(",")]  # noqa: E731
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg")
    ap.add_argument("--T", type=ints, default=[4])
    ap.add_argument("--threads", type=ints, default=[1024])
    ap.add_argument("--width", type=ints, default=[8])
    ap.add_argument("--seeds", type=ints, default=[32])
    ap.add_argument("--visited", type=ints, default=[1])
    ap.add_argument("--slots", type=int, default=32)
    ap.add_argument("--target", type=float, default=0.954)
    ap.add_argument("--nq", type=int, default=5000)
    a = ap.parse_args()
    w = synth.WORKLOADS[a.cfg]
    X = torch.from_numpy(synth.base_vectors(w)).cuda()
    Q = torch.from_numpy(synth.query_vectors(w, a.nq)).cuda()
    Qc = torch.from_numpy(synth.query_vectors(w, a.nq, stream=1)).cuda()
    knn, _ = algas.knn(X, X, w.knn_degree, w.metric, self_base=0)
    G = algas.prune(knn, w.degree)
    del knn
    truth = algas.knn(X, Q, w.k, w.metric)[0].cpu().numpy().view(np.uint32)
    tc = algas.knn(X, Qc, w.k, w.metric)[0].cpu().numpy().view(np.uint32)
    idx = algas.Index(X, G, w.metric)
    out = []
    for T, nt, wd, S, vis in itertools.product(a.T, a.threads, a.width, a.seeds, a.visited):
        if T == 1 and vis:
            continue
        for L in LS:
            if L < w.k:
                continue
            p = algas.default_params(k=w.k, itopk=L, width=min(wd, L), offset_beam=1, ctas_per_query=T,
                                     threads_per_cta=nt, slots=a.slots, n_seeds=S, seed=1,
                                     visited_mode=vis if T > 1 else 0)
            try:
                r = idx.search_dynamic(Qc, p)
            except algas.AlgasError as e:
                print(json.dumps({"T": T, "nt": nt, "w": wd, "S": S, "vis": vis, "error": str(e)[:90]}), flush=True)
                break
            if recall(r["ids"], tc, w.k) < a.target:
                continue
            res = [idx.search_dynamic(Q, p) for _ in range(3)]
            st = res[-1]["stats"]
            lat = (st["t_end_ns"] - st["t_start_ns"]) / 1e3
            d = {"T": T, "nt": nt, "w": p.width, "S": S, "vis": vis, "L": L,
                 "qps": round(float(np.median([a.nq / (x["info"].kernel_ms / 1e3) for x in res]))),
                 "recall": round(recall(res[-1]["ids"], truth, w.k), 4),
                 "p50": round(float(np.percentile(lat, 50)), 1), "p99": round(float(np.percentile(lat, 99)), 1),
                 "evals": round(float(st["dist_evals"].mean())), "steps_cta": round(float((st["iters"] / T).mean()), 2),
                 "bps": res[-1]["info"].blocks_per_sm}
            print(json.dumps(d), flush=True)
            out.append(d)
            break
    print("==== sorted by qps")
    for d in sorted(out, key=lambda d: -d["qps"])[:15]:
        print(json.dumps(d))


if __name__ == "__main__":
    main()
