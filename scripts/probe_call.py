"""Where does a search_dynamic call / a query spend its time? (GPU box)

usage: [ALGAS_TRACE=1] python scripts/probe_call.py C2 L,w,off,T,threads,visited[,seeds] [...]
Prints per call: CUDA-event time, host call phases, kernel time; per config:
per-query work counters, phase cycles, and the device-timestamp timeline of a
query (pickup -> CTAs in loop -> loop end -> published)."""
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
X = synth.base_vectors(w)
Q = synth.query_vectors(w, 10000)
Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
knn, _ = algas.knn(Xd, Xd, w.knn_degree, w.metric, self_base=0)
G = algas.prune(knn, w.degree)
del knn
ti, _ = algas.knn(Xd, Qd, w.k, w.metric)
ti = ti.cpu().numpy().view(np.uint32)
idx = algas.Index(Xd, G, w.metric)
st = torch.cuda.current_stream()

for spec in sys.argv[2:]:
    f = [int(x) for x in spec.split(",")]
    L, wd, off, T, nt, vis = f[:6]
    S = f[6] if len(f) > 6 else 32
    p = algas.default_params(k=w.k, itopk=L, width=wd, offset_beam=off, ctas_per_query=T, threads_per_cta=nt,
                             slots=32, seed=1, visited_mode=vis, n_seeds=S)
    print(f"==== L={L} w={wd} off={off} T={T} threads={nt} visited={'shared' if vis else 'private'} seeds={S}",
          flush=True)
    for i in range(4):
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
              f"kernel {inf.kernel_ms:7.2f} merge {inf.merge_ms:6.2f}  grid {inf.grid} bps {inf.blocks_per_sm}",
              flush=True)
    s = r["stats"]
    hits = sum(len(set(a.tolist()) & set(b.tolist())) for a, b in zip(r["ids"][:, :w.k], ti[:, :w.k]))
    print(f"recall {hits / ti[:, :w.k].size:.4f}  qps(kernel) {Q.shape[0] / (inf.kernel_ms / 1e3):.0f}")
    print("per query (summed over its CTAs): " + "  ".join(
        f"{f}={float(s[f].mean()):.1f}" for f in ("iters", "max_iters", "parents", "dist_evals", "cyc_select",
                                                  "cyc_gather", "cyc_dist", "cyc_sort")), flush=True)
    lat = (s["t_end_ns"] - s["t_start_ns"]) / 1e3
    print(f"latency us p50 {np.percentile(lat, 50):.1f} p99 {np.percentile(lat, 99):.1f}")
    ok = s["t_loop_last_ns"] > 0
    for name, a, b in (("pickup -> last CTA search entry", "t_start_ns", "t_entry_last_ns"),
                       ("last search entry -> last in loop", "t_entry_last_ns", "t_loop_last_ns"),
                       ("pickup -> first CTA in loop", "t_start_ns", "t_loop_first_ns"),
                       ("pickup -> last CTA in loop", "t_start_ns", "t_loop_last_ns"),
                       ("last in loop -> last out of loop", "t_loop_last_ns", "t_loop_end_ns"),
                       ("first in -> last out of loop", "t_loop_first_ns", "t_loop_end_ns"),
                       ("last out of loop -> last published", "t_loop_end_ns", "t_end_ns")):
        d = (s[b][ok].astype(np.int64) - s[a][ok].astype(np.int64)) / 1e3
        print(f"  {name:36s} mean {d.mean():7.2f} us  p50 {np.percentile(d, 50):7.2f}  p99 {np.percentile(d, 99):7.2f}")
