"""Where a C2 query's latency goes (GPU box): per-query step counts of the
mean vs the slowest CTA, pickup -> loop entry, loop end -> publish, and the
per-step phase cycles, at parameter points given on the command line.

usage: python scripts/diag_tail.py C2 "L=12,w=12,T=4,nt=1024,vis=1" "L=12,w=12,T=4,nt=1024,vis=1,S=16" ...
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


def recall(found, truth, k):
    return float(np.mean([len(set(f[:k].tolist()) & set(t[:k].tolist())) / k for f, t in zip(found, truth)]))


def main():
    cfg, variants = sys.argv[1], sys.argv[2:]
    nq = int(os.environ.get("NQ", "4000"))
    w = synth.WORKLOADS[cfg]
    X = torch.from_numpy(synth.base_vectors(w)).cuda()
    Q = torch.from_numpy(synth.query_vectors(w, nq)).cuda()
    knn, _ = algas.knn(X, X, w.knn_degree, w.metric, self_base=0)
    G = algas.prune(knn, w.degree)
    del knn
    truth = algas.knn(X, Q, w.k, w.metric)[0].cpu().numpy().view(np.uint32)
    idx = algas.Index(X, G, w.metric)
    for v in variants:
        kv = dict(x.split("=") for x in v.split(",") if x)
        envs = {"GM": "ALGAS_GATHER_MODE", "PF": "ALGAS_PREFETCH"}
        for key, env in envs.items():
            if key in kv:
                os.environ[env] = kv[key]
            else:
                os.environ.pop(env, None)
        T = int(kv.get("T", 4))
        p = algas.default_params(k=w.k, itopk=int(kv.get("L", 12)), width=int(kv.get("w", 12)),
                                 offset_beam=int(kv.get("off", 1)), ctas_per_query=T,
                                 threads_per_cta=int(kv.get("nt", 1024)), slots=int(kv.get("slots", 32)),
                                 n_seeds=int(kv.get("S", 32)), seed=1, visited_mode=int(kv.get("vis", 1)),
                                 max_iter=int(kv.get("mi", 0)))
        try:
            idx.search_dynamic(Q, p)
        except algas.AlgasError as e:
            print(json.dumps({"variant": v, "error": str(e)}), flush=True)
            continue
        res = [idx.search_dynamic(Q, p) for _ in range(3)]
        qps = [Q.shape[0] / (r["info"].kernel_ms / 1e3) for r in res]
        st = res[-1]["stats"]
        lat = (st["t_end_ns"] - st["t_start_ns"]) / 1e3
        it = np.maximum(st["iters"] + T, 1).astype(np.float64)
        out = {"variant": v, "qps": round(float(np.median(qps))), "recall": round(recall(res[-1]["ids"], truth, w.k), 4),
               "p50": round(float(np.percentile(lat, 50)), 1), "p99": round(float(np.percentile(lat, 99)), 1),
               "steps_mean_cta": round(float((st["iters"] / T).mean()), 2),
               "steps_max_cta": round(float(st["max_iters"].mean()), 2),
               "idle_frac_est": round(float(1 - ((st["iters"] / T) / np.maximum(st["max_iters"], 1)).mean()), 3),
               "us_pickup_to_loop_first": round(float(np.median((st["t_loop_first_ns"] - st["t_start_ns"]) / 1e3)), 2),
               "us_pickup_to_loop_last": round(float(np.median((st["t_loop_last_ns"] - st["t_start_ns"]) / 1e3)), 2),
               "us_loop_end_to_end": round(float(np.median((st["t_end_ns"] - st["t_loop_end_ns"]) / 1e3)), 2),
               "us_per_step_slowest": round(float(np.median((st["t_loop_end_ns"] - st["t_loop_last_ns"]) / 1e3 /
                                                            np.maximum(st["max_iters"], 1))), 2),
               "evals": round(float(st["dist_evals"].mean()), 1),
               "cyc_per_step": {ph: round(float((st["cyc_" + ph] / it).mean())) for ph in
                                ("select", "gather", "dist", "sort")},
               "hist_max_iters": np.bincount(st["max_iters"], minlength=1).tolist()[:30]}
        if os.environ.get("SUBLAP"):  # -DALGAS_SUBLAP=1 build: per-warp gather sub-phases (first pass)
            ws = max(float(st["merges_rank"].astype(np.float64).sum()), 1.0)
            out["sub_id_cyc"] = round(float(st["cyc_select"].astype(np.float64).sum() / ws))
            out["sub_hash_cyc"] = round(float(st["merges_bitonic"].astype(np.float64).sum() / ws))
            out["sub_claim_cyc"] = round(float(st["cap_hits"].astype(np.float64).sum() / ws))
            out["sub_warps_per_step"] = round(ws / max(float(st["iters"].astype(np.float64).sum()), 1.0), 1)
        if os.environ.get("SUBLAP") == "2":  # merge-phase probes (diagnosis build)
            its = max(float(st["iters"].astype(np.float64).sum()), 1.0)
            out["m_entry"] = round(float(st["cyc_select"].astype(np.float64).sum() / its))
            out["m_keyload"] = round(float(st["merges_bitonic"].astype(np.float64).sum() / its))
            out["m_lowerbound"] = round(float(st["cap_hits"].astype(np.float64).sum() / its))
            out["m_loop"] = round(float(st["merges_rank"].astype(np.float64).sum() / its), 1)
        print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
