"""Where does a search_dynamic call spend its time? (GPU box)
usage: ALGAS_TRACE=1 python scripts/probe_call.py C2 itopk width offset ctas threads visited"""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_chencyzw025_b200 as algas  # noqa: E402
import synth  # noqa: E402

w = synth.WORKLOADS[sys.argv[1]]
L, wd, off, T, nt, vis = (int(x) for x in sys.argv[2:8])
X = synth.base_vectors(w)
Q = synth.query_vectors(w, 10000)
Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
knn, _ = algas.knn(Xd, Xd, w.knn_degree, w.metric, self_base=0)
print("knn stats", algas.knn_last_stats(), flush=True)
G = algas.prune(knn, w.degree)
idx = algas.Index(Xd, G, w.metric)
p = algas.default_params(k=w.k, itopk=L, width=wd, offset_beam=off, ctas_per_query=T, threads_per_cta=nt, slots=32,
                         seed=1, visited_mode=vis)
st = torch.cuda.current_stream()
for i in range(6):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    e0.record(st)
    r = idx.search_dynamic(Qd, p, stream=st)
    e1.record(st)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    inf = r["info"]
    print(f"events {e0.elapsed_time(e1):7.2f} ms  python {1e3 * (t1 - t0):7.2f} ms  call {inf.call_ms:7.2f} "
          f"kernel {inf.kernel_ms:7.2f} merge {inf.merge_ms:6.2f}", flush=True)
s = r["stats"]
T = p.ctas_per_query
print("per query (summed over its CTAs): " + "  ".join(
    f"{f}={float(s[f].mean()):.1f}" for f in ("iters", "max_iters", "parents", "dist_evals", "cyc_select", "cyc_gather",
                                              "cyc_dist", "cyc_sort")), flush=True)
lat = (s["t_end_ns"] - s["t_start_ns"]) / 1e3
print(f"latency us p50 {np.percentile(lat, 50):.1f} p99 {np.percentile(lat, 99):.1f}  ctas/query {T}")
