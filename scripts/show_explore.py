import json, sys
d = json.load(open(sys.argv[1]))
for r in d['rows']:
    print(r['L'], r['w'], r['T'], r['threads'], 'cs', r.get('cs', 1), 'rec', round(r['recall'], 4), 'qps', round(r['qps']), 'p50', round(r['lat_p50_us']),
          'p99', round(r['lat_p99_us']), 'it', round(r['iters'], 1), {k: round(v) for k, v in r.get('cyc_per_iter', {}).items()})
