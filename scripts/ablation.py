"""SURVEY §8(f) row f1 on the GPU box: the paper's own ablations on synthetic data.

  * static vs dynamic batching (Fig. 13): the same persistent
    kernel and operating point, fed either one batch of B queries at a time
    (the next batch starts when the slowest query of the previous one is done:
    static batching) or from one queue with B slots (dynamic batching);
    per-query latency = batch start -> batch end (static) or slot pickup ->
    published (dynamic); QPS over the whole query set
  * beam extend on/off (Figs. 16-17): offset_beam = 1 (beam
    from the first step), L/4 (the paper's default), L (off: Alg. 1, one
    parent per step) at equal itopk -- recall, steps, sort share of the step
  * step-count spread (Figs. 1-2): max/mean steps per query
  * query-bubble waste: in static batching, the share of slot time
    a finished query waits for its batch

usage: python scripts/ablation.py C2 [--nq 4000] -> gpurun_out/ablation_<cfg>.json
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
    return sum(len(set(a.tolist()) & set(b.tolist())) for a, b in zip(found[:, :k], truth[:, :k])) / truth[:, :k].size


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg")
    ap.add_argument("--nq", type=int, default=4000)
    ap.add_argument("--batch", type=int, default=32)
    ap.add_argument("--itopk", type=int, default=32)
    ap.add_argument("--width", type=int, default=8)
    ap.add_argument("--ctas", type=int, default=2)
    ap.add_argument("--threads", type=int, default=1024)
    a = ap.parse_args()
    w = synth.WORKLOADS[a.cfg]
    X = synth.base_vectors(w)
    Q = synth.query_vectors(w, a.nq)
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    knn, _ = algas.knn(Xd, Xd, w.knn_degree, w.metric, self_base=0)
    G = algas.prune(knn, w.degree)
    del knn
    ti, _ = algas.knn(Xd, Qd, w.k, w.metric)
    ti = ti.cpu().numpy().view(np.uint32)
    idx = algas.Index(Xd, G, w.metric)
    out = {"workload": w.name, "nq": a.nq, "batch": a.batch}

    def params(L, wd, off, T, vis=1):
        return algas.default_params(k=w.k, itopk=L, width=wd, offset_beam=off, ctas_per_query=T,
                                    threads_per_cta=a.threads if T * a.batch <= 148 else 512, slots=a.batch,
                                    n_seeds=32, seed=1, visited_mode=vis if T > 1 else 0)

    # ---------------- static vs dynamic batching (same kernel, same point)
    p = params(a.itopk, a.width, 1, a.ctas)
    idx.search_dynamic(Qd[:a.batch * 4], p)  # warm-up
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    r = idx.search_dynamic(Qd, p)
    t_dyn = time.perf_counter() - t0
    s = r["stats"]
    lat_dyn = (s["t_end_ns"] - s["t_start_ns"]) / 1e3
    lat_st, busy_st, t_st, ids_st = [], [], 0.0, []
    for b0 in range(0, a.nq, a.batch):
        qb = Qd[b0:b0 + a.batch]
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        rb = idx.search_dynamic(qb, p, tag0=b0)
        dt = time.perf_counter() - t0
        t_st += dt
        sb = rb["stats"]
        t_first = sb["t_start_ns"].min()
        t_last = sb["t_end_ns"].max()
        lat_st.append(np.full(qb.shape[0], (t_last - t_first) / 1e3))   # every query waits for its batch
        busy_st.append((sb["t_end_ns"] - sb["t_start_ns"]) / 1e3)
        ids_st.append(rb["ids"])
    lat_st = np.concatenate(lat_st)
    busy_st = np.concatenate(busy_st)
    bubble = float(np.mean(lat_st - busy_st) / np.mean(busy_st))
    pct = lambda x: {f"p{q}": float(np.percentile(x, q)) for q in (10, 25, 50, 75, 90, 99)}  # noqa: E731
    out["static_vs_dynamic"] = {
        "params": {"itopk": p.itopk, "width": p.width, "ctas_per_query": p.ctas_per_query,
                   "threads_per_cta": p.threads_per_cta, "visited": "shared" if p.visited_mode else "private"},
        "dynamic": {"qps_wall": a.nq / t_dyn, "latency_us": pct(lat_dyn), "recall": recall(r["ids"], ti, w.k)},
        "static": {"qps_wall": a.nq / t_st, "latency_us": pct(lat_st), "recall": recall(np.concatenate(ids_st), ti, w.k),
                   "bubble_share_of_active_latency": bubble,
                   "definition": "batches of B queries, next batch after the slowest query; latency = batch "
                                 "first pickup -> last publish; bubble = mean (batch latency - own busy) / own busy"},
        "sorted_latency_curve_us": {"dynamic": np.sort(lat_dyn)[::max(1, a.nq // 50)].round(1).tolist(),
                                    "static": np.sort(lat_st)[::max(1, a.nq // 50)].round(1).tolist()},
    }
    print(json.dumps(out["static_vs_dynamic"]["dynamic"]), json.dumps(out["static_vs_dynamic"]["static"]), flush=True)

    # ---------------- beam extend on / off at equal itopk, T = 1 and T = ctas
    beam = []
    for T in (1, a.ctas):
        for L in (32, 64):
            for off, wd, name in ((1, a.width, "beam from step 1"), (max(1, L // 4), a.width, "beam after L/4 (paper)"),
                                  (L, 1, "off (Alg. 1, one parent per step)")):
                pb = params(L, wd, off, T)
                rr = idx.search_dynamic(Qd, pb)
                st = rr["stats"]
                cyc = {f: float(st[f].mean()) for f in ("cyc_select", "cyc_gather", "cyc_dist", "cyc_sort")}
                tot = sum(cyc.values())
                lat = (st["t_end_ns"] - st["t_start_ns"]) / 1e3
                beam.append({"T": T, "itopk": L, "offset_beam": off, "width": wd, "mode": name,
                             "recall": recall(rr["ids"], ti, w.k), "qps_kernel": a.nq / (rr["info"].kernel_ms / 1e3),
                             "p50_us": float(np.percentile(lat, 50)), "p99_us": float(np.percentile(lat, 99)),
                             "steps_mean": float(st["max_iters"].mean()),
                             "steps_max_over_mean": float(st["max_iters"].max() / max(1e-9, st["max_iters"].mean())),
                             "dist_evals": float(st["dist_evals"].mean()),
                             "sort_share": cyc["cyc_sort"] / tot if tot else None,
                             "select_share": cyc["cyc_select"] / tot if tot else None})
                print(json.dumps(beam[-1]), flush=True)
    out["beam_extend"] = beam
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", f"ablation_{a.cfg}.json"), "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
