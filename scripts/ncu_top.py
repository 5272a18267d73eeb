"""Top SASS instructions by warp-stall samples (with the dominant stall
reasons) from `ncu -i X --page source --csv --print-source sass`, plus the
kernel-wide stall breakdown.  usage: ncu_top.py src.csv [N]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = rows[1], rows[2:]
ci = {h: i for i, h in enumerate(hdr)}
S = ci["Warp Stall Sampling (All Samples)"]
f = lambda x: float(x or 0)
tot = sum(f(r[S]) for r in data)
sc = [h for h in hdr if h.startswith("stall_") and "(Not Issued)" not in h]
agg = {h: sum(f(r[ci[h]]) for r in data) for h in sc}
print("total samples", tot, " kernel-wide:",
      ", ".join(f"{h[6:]} {100*v/tot:.1f}%" for h, v in sorted(agg.items(), key=lambda x: -x[1])[:8]))
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
for r in sorted(data, key=lambda r: -f(r[S]))[:N]:
    rs = sorted(((h[6:], f(r[ci[h]])) for h in sc), key=lambda x: -x[1])[:2]
    print(f"{100*f(r[S])/tot:5.1f}% {r[ci['Address']][-5:]:>6} {r[ci['Source']][:70]:70s} "
          + " ".join(f"{n}:{100*v/max(1,f(r[S])):.0f}%" for n, v in rs if v))
