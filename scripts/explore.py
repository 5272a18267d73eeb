"""Parameter exploration on a BASELINE.json workload (GPU box): build the graph,
ground truth, then sweep (L, w, T, threads, slots) and print recall / QPS /
latency / work counters.  Writes gpurun_out/explore_<cfg>.json.

usage: python scripts/explore.py C2 [--nq 10000] [--quick]
"""
import argparse
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
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg")
    ap.add_argument("--nq", type=int, default=10000)
    ap.add_argument("--n", type=int, default=0)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--noprune", action="store_true")
    a = ap.parse_args()
    w = synth.WORKLOADS[a.cfg]
    n = a.n or w.n
    t0 = time.time()
    X = synth.base_vectors(w, n)
    Q = synth.query_vectors(w, a.nq)
    t_gen = time.time() - t0
    Xd = torch.from_numpy(X).cuda()
    Qd = torch.from_numpy(Q).cuda()
    torch.cuda.synchronize()
    t0 = time.time()
    knn_ids, _ = algas.knn(Xd, Xd, w.knn_degree, w.metric, self_base=0)
    torch.cuda.synchronize()
    t_knn = time.time() - t0
    t0 = time.time()
    if w.prune and not a.noprune:
        G = algas.prune(knn_ids, w.degree)
    else:
        G = knn_ids[:, :w.degree].contiguous()
    torch.cuda.synchronize()
    t_prune = time.time() - t0
    t0 = time.time()
    kt = max(w.k, 10)
    ti, td = algas.knn(Xd, Qd, kt, w.metric)
    torch.cuda.synchronize()
    t_gt = time.time() - t0
    ti = ti.cpu().numpy().view(np.uint32) if hasattr(ti, "cpu") else ti
    G = G.cpu().numpy().view(np.uint32) if hasattr(G, "cpu") else G
    print(f"gen {t_gen:.1f}s knn {t_knn:.1f}s prune {t_prune:.1f}s gt {t_gt:.1f}s", flush=True)
    idx = algas.Index(Xd, G, w.metric)
    rows = []
    Ls = [32, 48, 64, 96, 128, 192, 256] if w.k <= 10 else [128, 192, 256, 384, 512]
    grid = []
    for L in Ls:
        for (wd, T, nt) in [(1, 1, 64), (4, 1, 64), (4, 1, 128), (4, 4, 64), (2, 8, 64), (4, 8, 64)]:
            grid.append((L, wd, T, nt))
    if os.environ.get("GRID") == "tune":
        grid = [(64, 4, 1, 256, 1), (64, 8, 1, 256, 1), (64, 16, 1, 256, 1), (56, 8, 2, 256, 1),
                (48, 8, 4, 256, 1), (56, 8, 4, 256, 1), (96, 16, 1, 256, 1), (64, 8, 2, 256, 1)]
    elif os.environ.get("GRID") == "pf":
        grid = [(64, 4, 1, 256, 1), (64, 8, 1, 256, 1), (64, 4, 2, 256, 1), (56, 4, 2, 256, 1), (48, 4, 4, 256, 1),
                (56, 4, 4, 256, 1), (64, 4, 1, 128, 1)]
    elif os.environ.get("GRID") == "nt":
        grid = []
        for nt in (256, 512, 1024):
            for (L, wd, T) in [(64, 8, 1), (56, 7, 2), (48, 6, 4), (64, 4, 1), (64, 16, 1), (56, 8, 4), (96, 8, 1)]:
                grid.append((L, wd, T, nt, 1))
    elif os.environ.get("GRID") == "pf2":
        grid = []
        for pf in (0, 2, 6):
            for (L, wd, T, off) in [(64, 8, 1, 16), (64, 8, 1, 8), (64, 8, 1, 1), (56, 7, 2, 14), (56, 7, 2, 4),
                                    (48, 6, 4, 12), (52, 8, 4, 4)]:
                grid.append((L, wd, T, 256, 1, off, pf))
    elif os.environ.get("GRID") == "wide":
        grid = []
        for nt in (256, 512, 1024):
            for T in (1, 2, 4):
                for wd in (8, 16, 32):
                    for L in (40, 48, 56, 64):
                        grid.append((L, wd, T, nt, 1, 1, 0))
    elif os.environ.get("GRID") == "shared":
        grid = []
        for (L, wd, T, nt) in [(24, 16, 4, 1024), (32, 16, 4, 1024), (24, 16, 4, 512), (40, 8, 4, 512),
                               (40, 16, 2, 1024), (32, 8, 4, 1024), (16, 16, 4, 1024), (24, 8, 4, 1024)]:
            grid.append((L, wd, T, nt, 1, 1, 0))
    elif os.environ.get("GRID") == "pf8":
        grid = []
        for pf in (0, 8):
            for (L, wd, T, nt) in [(12, 8, 4, 512), (12, 8, 4, 1024), (16, 16, 4, 1024), (20, 16, 4, 1024)]:
                grid.append((L, wd, T, nt, 1, 1, pf))
    elif os.environ.get("GRID") == "cs":
        grid = [(64, 4, 1, 256, 1), (64, 4, 1, 256, 4), (64, 8, 1, 256, 4), (64, 8, 1, 256, 8)]
    elif a.quick:
        grid = [(64, 4, 1, 256, 1), (64, 4, 1, 256, 2), (64, 4, 1, 256, 4), (64, 8, 1, 256, 4),
                (64, 4, 2, 256, 2), (48, 4, 2, 256, 2), (48, 4, 4, 256, 1), (64, 8, 1, 256, 2),
                (128, 8, 1, 256, 4), (64, 2, 1, 256, 4)]
    grid = [g if len(g) >= 5 else g + (1,) for g in grid]
    grid = [g if len(g) == 7 else g + (max(1, g[0] // 4), int(os.environ.get("ALGAS_PREFETCH", "0"))) for g in grid]
    for (L, wd, T, nt, cs, off, pf) in grid:
        os.environ["ALGAS_PREFETCH"] = str(pf)
        for slots in ([32] if not a.quick else [32]):
            p = algas.default_params(k=w.k, itopk=L, width=wd, offset_beam=off, ctas_per_query=T,
                                     threads_per_cta=nt, slots=slots, n_seeds=32, seed=1, cluster_size=cs,
                                     visited_mode=int(os.environ.get("VIS", "0")))
            try:
                r = idx.search_dynamic(Qd, p)
            except algas.AlgasError as e:
                print("skip", L, wd, T, nt, slots, e)
                continue
            ms = r["info"].kernel_ms
            st = r["stats"]
            lat = (st["t_end_ns"] - st["t_start_ns"]) / 1e3
            rec = recall(r["ids"], ti, w.k)
            row = dict(L=L, w=wd, T=T, threads=nt, cs=cs, off=off, pf=pf, vis=int(os.environ.get("VIS", "0")),
                       slots=slots, recall=rec, qps=a.nq / (ms / 1e3),
                       kernel_ms=ms, lat_p50_us=float(np.percentile(lat, 50)),
                       lat_p99_us=float(np.percentile(lat, 99)), iters=float(st["iters"].mean() / T),
                       dist_evals=float(st["dist_evals"].mean()), spills=int((st["spills"] > 0).sum()),
                       overflows=int(st["overflows"].sum()), blocks_per_sm=r["info"].blocks_per_sm,
                       smem=r["info"].smem_per_cta,
                       gbps=float(st["dist_evals"].sum() * w.dim * 4 / (ms / 1e3) / 1e9),
                       cyc_per_iter={ph: float(st["cyc_" + ph].sum() / max(1, st["iters"].sum()))
                                     for ph in ("select", "gather", "dist", "sort")})
            rows.append(row)
            print(json.dumps(row), flush=True)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", f"explore_{a.cfg}.json"), "w") as f:
        json.dump(dict(cfg=a.cfg, n=n, nq=a.nq, t_gen=t_gen, t_knn=t_knn, t_prune=t_prune, t_gt=t_gt, rows=rows),
                  f, indent=1)


if __name__ == "__main__":
    main()
