"""Pretty-print explore.py JSON lines (stdin)."""
import json
import sys

for l in sys.stdin:
    if not l.startswith("{"):
        print(l.rstrip())
        continue
    r = json.loads(l)
    c = r["cyc_per_iter"]
    print(f"L={r['L']:3d} w={r['w']:2d} T={r['T']} nt={r['threads']:4d} off={r.get('off', '-')!s:>3} pf={r.get('pf', '-')} vis={r.get('vis', 0)} "
          f"rec={r['recall']:.4f} qps={r['qps'] / 1e3:6.1f}k p50={r['lat_p50_us']:6.1f} p99={r['lat_p99_us']:6.1f} "
          f"it={r['iters']:5.1f} ev={r['dist_evals']:6.0f} sel={c['select']:5.0f} gat={c['gather']:5.0f} "
          f"dist={c['dist']:5.0f} sort={c['sort']:5.0f}")
